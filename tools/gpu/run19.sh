timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2_gputest_19.log 2>&1; echo "tests rc=$?"
tail -3 gpurun_out/r2_gputest_19.log; grep -a FAILED gpurun_out/r2_gputest_19.log | head
for i in 1 2; do
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2_bench_19_$i.json 2> gpurun_out/r2_bench_19_$i.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2_bench_19_$i.json'));print(d['value'],d['e2e']['value'],{k: round(v) for k, v in d['breakdown_ms'].items() if isinstance(v, float)},d['clocks'],d['roofline']['frac'],d['step_roofline']['frac'])"
done
