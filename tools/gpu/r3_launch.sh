export MOBIUS_KT_NOSYNC=1
python tools/flash_time.py 64 32 && ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 56 -c 16 --csv python tools/flash_time.py 64 32 > gpurun_out/r3_flash_launch.csv 2>&1; echo rc=$?
