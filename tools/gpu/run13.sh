for i in 1 2; do
for v in "" "MOBIUS_NO_BIAS_ROW=1"; do
env $v timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/ab.json'));print('$v', round(d['value']), {k: round(v) for k, v in d['breakdown_ms'].items() if isinstance(v, float)}, d['clocks']['sm_mhz'])"
done
done
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --micro-batch 64 --microbatches 2 > gpurun_out/ab.json 2>gpurun_out/ab.err
python -c "import json;d=json.load(open('gpurun_out/ab.json'));print('mbs64xM2', round(d['value']), {k: round(v) for k, v in d['breakdown_ms'].items() if isinstance(v, float)}, d['clocks']['sm_mhz'], d['memory'])"
tail -2 gpurun_out/ab.err
