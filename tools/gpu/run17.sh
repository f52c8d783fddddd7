GEMM_T=32768 timeout 300 python tools/gemm_vs_cublas.py
nvidia-smi --query-gpu=clocks.sm,power.draw --format=csv
