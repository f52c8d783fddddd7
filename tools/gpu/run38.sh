timeout 600 ncu --set full --clock-control none --import-source on -k regex:flash_fwd -s 1 -c 1 -o gpurun_out/fwd_full python tools/flash_prof.py 2 > gpurun_out/fwdncu.log 2>&1; echo ncu rc=$?
