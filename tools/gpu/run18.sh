for v in 1 0; do echo "SPLITK=$v"; MOBIUS_GEMM_SPLITK=$v GEMM_T=32768 timeout 300 python tools/gemm_vs_cublas.py | grep -E "dW|total"; done
timeout 900 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -p no:cacheprovider -k "gemm or block" 2>&1 | tail -3
