export MOBIUS_KT_NOSYNC=1 GEMM_T=32768 OURS_ONLY=1
MOBIUS_GEMM_NP=2 timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
echo NP1; python tools/gemm_sustained.py | cut -c1-80
echo NP2; MOBIUS_GEMM_NP=2 python tools/gemm_sustained.py | cut -c1-80
