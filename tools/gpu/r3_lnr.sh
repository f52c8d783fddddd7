export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "layernorm" 2>&1 | tail -1
ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_bwd  "
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:ln_ --csv python tools/elem_bench.py 2>/dev/null | grep -E "ln_param|ln_bwd_fused" | head -4 | cut -c1-40,150-
