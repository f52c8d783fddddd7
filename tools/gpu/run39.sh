MOBIUS_FLASH_FWD_NB=1 timeout 600 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q -k "attention or flash" 2>&1 | tail -3
for i in 1 2; do python tools/flash_time.py 64 32; MOBIUS_FLASH_FWD_NB=1 python tools/flash_time.py 64 32; done
MOBIUS_FLASH_FWD_NB=1 python tools/flash_time.py 64 8
python tools/flash_time.py 64 8
