python bench.py --steps 1 --warmup 0 --microbatches 2 --no-e2e --no-cpu-baseline > gpurun_out/r3_lb2_plain.log 2>&1 && \
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/r3_launches_M2_v4.csv python bench.py --steps 1 --warmup 0 --microbatches 2 --no-e2e --no-cpu-baseline > gpurun_out/r3_lb2_ncu.log 2>&1; echo rc=$?
