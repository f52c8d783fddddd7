export MOBIUS_KT_NOSYNC=1
for i in 1 2; do python tools/flash_time.py 64 32; for n in 2 4 6; do echo BWDPOLY=$n; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FLASH_BWD_POLY_PAIRS$n.so python tools/flash_time.py 64 32; done; done
