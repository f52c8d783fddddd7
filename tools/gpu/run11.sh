set -x
for G in 0 16 32 64 128; do echo "group $G"; MOBIUS_FLASH_GROUP=$G timeout 120 python tools/flash_time.py 64 32 1024 25; MOBIUS_FLASH_GROUP=$G timeout 120 python tools/flash_time.py 128 2 2048 40; done
timeout 1500 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_fullsize.py tests/test_gpu_step.py -m gpu -q -x -p no:cacheprovider > gpurun_out/r2_gputest_11.log 2>&1; echo "tests rc=$?"
tail -5 gpurun_out/r2_gputest_11.log
grep -a "elementwise worst\|norm-wise" gpurun_out/r2_gputest_11.log | cut -c1-600
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r2_bench_11.json 2> gpurun_out/r2_bench_11.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2_bench_11.json'));print(d['value'],d['breakdown_ms'],d['clocks'],d['roofline']['frac'])"
MOBIUS_NO_BIAS_ROW=1 MOBIUS_FLASH_GROUP=0 timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2_bench_11_old.json 2> gpurun_out/r2_bench_11_old.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2_bench_11_old.json'));print(d['value'],d['breakdown_ms'],d['clocks'],d['roofline']['frac'])"
