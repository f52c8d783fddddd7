export MOBIUS_KT_NOSYNC=1
for v in MOBIUS_FIN_MEMBAR0_MOBIUS_FIN_EXP1 MOBIUS_FIN_MEMBAR0_MOBIUS_FIN_EXP2 MOBIUS_FIN_MEMBAR0_MOBIUS_FIN_EXP3; do echo $v; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_$v.so python tools/flash_time.py 64 32; done
