timeout 600 ncu --set full --import-source on --kernel-name regex:flash_fwd_kernel -c 1 -o gpurun_out/r2_flash_fwd_full python tools/flash_time.py 64 32 1024 25 > gpurun_out/r2_flash_fwd_ncu.log 2>&1; echo "ncu rc=$?"
timeout 600 ncu --set full --import-source on --kernel-name regex:flash_bwd_kernel -c 1 -o gpurun_out/r2_flash_bwd_full python tools/flash_time.py 64 32 1024 25 > gpurun_out/r2_flash_bwd_ncu.log 2>&1; echo "ncu rc=$?"
ls -la gpurun_out/*.ncu-rep
