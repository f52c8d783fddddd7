export MOBIUS_KT_NOSYNC=1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_block.py -m gpu -x -q 2>&1 | tail -3
for i in 1 2; do python tools/flash_time.py 64 32; python tools/flash_time.py 128 16; python tools/gemm_epi_ab.py 32768 6400 1600 0 2; done
MOBIUS_LIB_PATH=tools/gpu/var/libmobius_r1.so python tools/flash_time.py 128 16
