for i in 1 2; do
python tools/flash_time.py 64 32
for a in 1 2 3 4 7; do echo ABL=$a; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FWD_ABL$a.so python tools/flash_time.py 64 32; done
done
