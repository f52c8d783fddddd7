export MOBIUS_KT_NOSYNC=1
for i in 1 2; do python tools/flash_time.py 64 32; for v in 1 2 3; do echo POLY$v; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_BWD_POLY$v.so python tools/flash_time.py 64 32; done; done
