set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q -s -p no:cacheprovider > gpurun_out/r2_gputest_1.log 2>&1; echo "tests rc=$?"
tail -5 gpurun_out/r2_gputest_1.log
grep -a "elementwise worst" gpurun_out/r2_gputest_1.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/r2_bench_1.json 2> gpurun_out/r2_bench_1.err; echo "bench rc=$?"
tail -c 3000 gpurun_out/r2_bench_1.json
