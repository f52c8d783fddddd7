export GEMM_T=32768 OURS_ONLY=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
echo default; python tools/gemm_sustained.py | cut -c1-80
for g in 2 3; do echo G$g; MOBIUS_GEMM_GROUP=$g python tools/gemm_sustained.py | cut -c1-80; done
