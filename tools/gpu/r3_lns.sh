export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "layernorm or block" 2>&1 | tail -1
MOBIUS_LN_FWD_STAGED=0 python tools/ln_fwd_ident.py /tmp/lnw.npz && MOBIUS_LN_FWD_STAGED=1 python tools/ln_fwd_ident.py /tmp/lns.npz /tmp/lnw.npz
for i in 1 2; do
echo staged; ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_fwd"
echo warp; MOBIUS_LN_FWD_STAGED=0 ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_fwd"
done
