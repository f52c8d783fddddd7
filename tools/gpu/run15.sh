timeout 120 python tools/flash_time.py 64 32 1024 25
timeout 120 python tools/flash_time.py 128 2 2048 40
timeout 120 python tools/flash_time.py 64 32 1024 25
timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -p no:cacheprovider -k "attention or block" 2>&1 | tail -3
