set -x
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_kernels.py -m gpu -q -x -p no:cacheprovider -k "arena or ckpt or embedding or colsum or token or poison or failed_create or weight_decay or multistep or tail" > gpurun_out/r2_gputest_3.log 2>&1; echo "tests rc=$?"
tail -30 gpurun_out/r2_gputest_3.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/r2_launches_v1.csv python bench.py --steps 1 --warmup 0 --microbatches 2 --no-e2e --no-cpu-baseline > gpurun_out/r2_launches_v1.log 2>&1; echo "ncu rc=$?"
python tools/launch_shares.py gpurun_out/r2_launches_v1.csv | head -30
