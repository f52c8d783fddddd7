set -x
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --print-units base --csv --log-file gpurun_out/r2_elem_dram.csv python tools/elem_ncu.py > gpurun_out/r2_elem_ncu.log 2>&1; echo "ncu rc=$?"
python tools/elem_dram.py gpurun_out/r2_elem_dram.csv 6553 | tee gpurun_out/r2_elem_dram_summary.csv
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/r2_launches_v2.csv python bench.py --steps 1 --warmup 0 --microbatches 2 --no-e2e --no-cpu-baseline > gpurun_out/r2_launches_v2.log 2>&1; echo "ncu2 rc=$?"
python tools/launch_shares.py gpurun_out/r2_launches_v2.csv | head -30
