export MOBIUS_KT_NOSYNC=1
python tools/flash_time.py 64 32 1024 25 && \
timeout 600 ncu --set full --import-source on --kernel-name regex:flash_fwd64_kernel -c 1 -o gpurun_out/r3_flash_fwd64_full python tools/flash_time.py 64 32 1024 25 > gpurun_out/r3_flash_fwd_ncu.log 2>&1; echo "ncu rc=$?"
