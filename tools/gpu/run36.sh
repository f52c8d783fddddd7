for i in 1 2; do
python tools/flash_time.py 64 32
for a in MOBIUS_FWD_PACKED1 MOBIUS_FWD_PACKED1_MOBIUS_FLASH_POLY_PAIRS4; do echo $a; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_$a.so python tools/flash_time.py 64 32; done
done
bash tools/gpu/run35.sh 2>&1 | grep "blk 0" | sort
