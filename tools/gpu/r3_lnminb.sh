export MOBIUS_KT_NOSYNC=1
for i in 1 2; do
echo MINB3; ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_fwd"
for m in 4 5; do echo MINB$m; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_LN_FWD_MINB$m.so ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep "ln_fwd"; done
done
