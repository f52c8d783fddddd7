export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "layernorm or block" 2>&1 | tail -2
for i in 1 2; do
ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep ln_bwd
MOBIUS_LN_BWD_FUSED=0 ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep ln_bwd
done
