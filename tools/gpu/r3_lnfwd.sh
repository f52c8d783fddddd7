export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "layernorm or block" 2>&1 | tail -1
for i in 1 2; do
echo W1; ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_fwd"
echo nonpersist; MOBIUS_LN_FWD_PERSIST=0 ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_fwd"
for w in 2 4; do echo W$w; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_LN_FWD_WAVES$w.so ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_fwd"; done
done
