for i in 1 2; do
python tools/flash_time.py 64 32
for a in 7 15 23 31 8 16; do echo ABL=$a; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FWD_ABL$a.so python tools/flash_time.py 64 32; done
done
