export MOBIUS_KT_NOSYNC=1
for i in 1 2; do python tools/flash_time.py 128 16; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FLASH_POLY_PAIRS0.so python tools/flash_time.py 128 16;  MOBIUS_LIB_PATH=tools/gpu/var/libmobius_r1.so python tools/flash_time.py 128 16; done
