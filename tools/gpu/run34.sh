for i in 1 2; do
python tools/flash_time.py 64 32
for a in MOBIUS_FWD_KVS2 MOBIUS_FWD_KVS5 MOBIUS_FWD_KVS5_MOBIUS_FWD_ABL7 MOBIUS_FWD_ABL7; do echo $a; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_$a.so python tools/flash_time.py 64 32; done
done
