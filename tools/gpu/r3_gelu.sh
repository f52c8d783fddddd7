export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm or block" 2>&1 | tail -2
python tools/gemm_epi_clock.py
MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_DUMMY0.so python tools/gemm_epi_clock.py
GEMM_T=32768 python tools/gemm_vs_cublas.py
