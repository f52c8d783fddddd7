python tools/elem_ncu.py && \
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --print-units base --csv --log-file gpurun_out/r3_elem_dram.csv python tools/elem_ncu.py > gpurun_out/r3_elem_ncu.log 2>&1; echo "ncu rc=$?"
python tools/elem_dram.py gpurun_out/r3_elem_dram.csv 6550.7 > gpurun_out/r3_elem_dram_summary.csv
