set -x
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2_gputest_12.log 2>&1; echo "tests rc=$?"
tail -5 gpurun_out/r2_gputest_12.log
grep -a "FAILED" gpurun_out/r2_gputest_12.log | head
grep -a "elementwise worst\|norm-wise" gpurun_out/r2_gputest_12.log | cut -c1-400
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/r2_bench_12.json 2> gpurun_out/r2_bench_12.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2_bench_12.json'));print(d['value'],d['e2e']['value'],d['breakdown_ms'],d['clocks'],d['roofline']['frac'],d['step_roofline']['frac'])"
