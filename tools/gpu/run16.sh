timeout 900 python -m pytest tests/test_gpu_multirank.py -m gpu -q -p no:cacheprovider 2>&1 | tail -4
MOBIUS_BENCH_SAME_GPU=1 timeout 900 python bench.py --gpus 2 --steps 2 --warmup 1 --layers 8 --no-cpu-baseline > gpurun_out/r2_bench_2rank_samegpu.json 2> gpurun_out/r2_bench_2rank_samegpu.err; echo "bench2 rc=$?"
tail -3 gpurun_out/r2_bench_2rank_samegpu.err
python -c "import json;d=json.load(open('gpurun_out/r2_bench_2rank_samegpu.json'));print(d['value'],d['n_gpus'],d['config']['prefetch_order'],d['config']['uplink_groups'],d['config']['mapping_contention'])"
