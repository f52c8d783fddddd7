timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2_gputest_22.log 2>&1; echo "tests rc=$?"
tail -3 gpurun_out/r2_gputest_22.log; grep -a FAILED gpurun_out/r2_gputest_22.log | head
for i in 1 2; do
for v in "X=1" "MOBIUS_SYNC_UPDATE=1"; do
env $v timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ab.json 2>gpurun_out/ab.err
python -c "import json;d=json.load(open('gpurun_out/ab.json'));print('$v', round(d['value']), round(d['e2e']['value']), round(d['ms_per_step'],1), {k: round(v) for k, v in d['breakdown_ms'].items() if isinstance(v, float)}, d['clocks']['sm_mhz'])" || tail -3 gpurun_out/ab.err
done
done
