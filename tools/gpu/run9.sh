for P in 0 2 4 6 8; do
  echo "poly pairs $P"
  MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FLASH_POLY_PAIRS$P.so timeout 120 python tools/flash_time.py 64 32 1024 25
  MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FLASH_POLY_PAIRS$P.so timeout 120 python tools/flash_time.py 128 2 2048 40
done
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -p no:cacheprovider -k "attention or flash or block" 2>&1 | tail -3
