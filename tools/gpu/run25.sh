timeout 900 ncu --clock-control none --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --print-units base --csv --log-file gpurun_out/r2_elem_dram_unlocked.csv python tools/elem_ncu.py > gpurun_out/r2_elem_ncu2.log 2>&1; echo "ncu rc=$?"
python tools/elem_dram.py gpurun_out/r2_elem_dram_unlocked.csv 6553 | grep mobius | tee gpurun_out/r2_elem_dram_unlocked_summary.csv
