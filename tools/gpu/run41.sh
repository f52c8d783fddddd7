export MOBIUS_KT_NOSYNC=1
timeout 900 python -m pytest tests/test_gpu_kernels.py -m gpu -x -q 2>&1 | tail -2
for i in 1 2; do python tools/flash_time.py 64 32; python tools/flash_time.py 128 16; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_HEAD1.so python tools/flash_time.py 64 32;  MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_HEAD1.so python tools/flash_time.py 128 16; done
