for P in 0 2 4 6 8; do
  echo "poly pairs $P"
  MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FLASH_POLY_PAIRS$P.so timeout 120 python tools/flash_time.py 64 32 1024 25
  MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FLASH_POLY_PAIRS$P.so timeout 120 python tools/flash_time.py 128 2 2048 40
done
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -p no:cacheprovider -k "attention or flash or block" 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -p no:cacheprovider -k "block_full_size" 2>&1 | tail -3
timeout 1500 python bench.py --config 13b --layers 24 --cap-gib 4 --steps 3 --warmup 2 --no-cpu-baseline > gpurun_out/r2_bench_13b_l24.json 2> gpurun_out/r2_bench_13b_l24.err; echo "13b rc=$?"
tail -3 gpurun_out/r2_bench_13b_l24.err
python -c "import json;d=json.load(open('gpurun_out/r2_bench_13b_l24.json'));print(d['value'],d['e2e']['value'],d['config']['n_stages'],d['memory'],d['step_roofline'],d['overlap'],d['swap_in'],d['breakdown_ms'])"
