set -x
timeout 1800 python -m pytest tests -m gpu -q -s -p no:cacheprovider > gpurun_out/r2_gputest_2.log 2>&1; echo "tests rc=$?"
tail -5 gpurun_out/r2_gputest_2.log
grep -a "elementwise worst\|norm-wise" gpurun_out/r2_gputest_2.log
ELEM_T=32768 timeout 300 python tools/elem_bench.py > gpurun_out/r2_elem_1.log 2>&1; cat gpurun_out/r2_elem_1.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/r2_bench_2.json 2> gpurun_out/r2_bench_2.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2_bench_2.json'));print(d['value'],d['breakdown_ms'],d['clocks'])"
