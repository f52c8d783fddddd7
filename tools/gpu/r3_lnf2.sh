export MOBIUS_KT_NOSYNC=1
for v in MOBIUS_LNF_CTAS2 MOBIUS_LNF_CTAS3 MOBIUS_LNF_CTAS4; do echo $v; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_$v.so timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "layernorm" 2>&1 | tail -1; done
for i in 1 2; do
for v in MOBIUS_LNF_CTAS2 MOBIUS_LNF_CTAS3 MOBIUS_LNF_CTAS4; do echo $v; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_$v.so ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_bwd  "; done
done
