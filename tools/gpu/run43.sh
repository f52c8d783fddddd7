export MOBIUS_KT_NOSYNC=1
for i in 1 2; do python tools/flash_time.py 128 16; for c in 5f813c0 01bd9d1; do echo $c; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_AT_${c}1.so python tools/flash_time.py 128 16; done; done
