for cp in 2 4 2 4; do echo "BWD CP=$cp"; MOBIUS_FLASH_BWD_CP=$cp timeout 120 python tools/flash_time.py 64 32 1024 25; done
MOBIUS_FLASH_BWD_CP=4 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -p no:cacheprovider -k "attention or block" 2>&1 | tail -3
MOBIUS_FLASH_BWD_CP=2 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -p no:cacheprovider -k "attention or block" 2>&1 | tail -3
