set -x
timeout 1200 python -m pytest tests/test_gpu_step.py tests/test_gpu_multirank.py tests/test_gpu_topology.py -m gpu -q -p no:cacheprovider > gpurun_out/r2_gputest_8.log 2>&1; echo "tests rc=$?"
tail -15 gpurun_out/r2_gputest_8.log
for cap in 2 4; do
timeout 900 python bench.py --steps 3 --warmup 3 --micro-batch 8 --microbatches 4 --arena-cap-gib $cap --no-cpu-baseline > gpurun_out/r2_bench_c2_${cap}g.json 2> gpurun_out/r2_bench_c2_${cap}g.err; echo "c2 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2_bench_c2_${cap}g.json'));print(d['value'],d['e2e']['value'],d['config']['n_stages'],d['memory'],d['step_roofline']['frac'],d['overlap']['h2d_hidden_frac'],d['swap_in'])"
done
free -g
nproc
