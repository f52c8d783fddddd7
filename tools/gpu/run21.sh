for i in 1 2; do
for v in "X=1" "MOBIUS_GEMM_SPLITK=0" "MOBIUS_NO_BIAS_ROW=1"; do
env $v timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab.json 2>gpurun_out/ab.err
python -c "import json;d=json.load(open('gpurun_out/ab.json'));print('$v', round(d['value']), {k: round(v) for k, v in d['breakdown_ms'].items() if isinstance(v, float)}, d['clocks']['sm_mhz'])" || tail -3 gpurun_out/ab.err
done
done
