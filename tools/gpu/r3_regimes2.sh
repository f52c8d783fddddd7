timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm or layernorm" 2>&1 | tail -1
python bench.py --config 13b --layers 24 --microbatches 16 --micro-batch 2 --cap-gib 4 --no-e2e --no-cpu-baseline > gpurun_out/r3_13b2.json 2> gpurun_out/r3_13b2.err
python bench.py --no-e2e --no-cpu-baseline > gpurun_out/r3_15b2.json 2> gpurun_out/r3_15b2.err
