set -x
timeout 1200 python -m pytest tests/test_gpu_step.py tests/test_gpu_multirank.py tests/test_gpu_topology.py -m gpu -q -x -p no:cacheprovider > gpurun_out/r2_gputest_7.log 2>&1; echo "tests rc=$?"
tail -15 gpurun_out/r2_gputest_7.log
timeout 900 python bench.py --steps 3 --warmup 3 --micro-batch 8 --microbatches 4 --arena-cap-gib 2 --no-cpu-baseline > gpurun_out/r2_bench_c2_2g.json 2> gpurun_out/r2_bench_c2_2g.err; echo "c2 rc=$?"
tail -3 gpurun_out/r2_bench_c2_2g.err
python -c "import json;d=json.load(open('gpurun_out/r2_bench_c2_2g.json'));print(d['value'],d['e2e']['value'],d['config']['n_stages'],d['memory'],d['step_roofline']['frac'],d['overlap']['h2d_hidden_frac'],d['swap_in'])"
