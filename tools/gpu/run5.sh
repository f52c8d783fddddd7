MBS=32 timeout 300 python tools/embed_bench.py
MBS=4 timeout 300 python tools/embed_bench.py
timeout 900 python -m pytest tests/test_gpu_kernels.py -m gpu -q -x -p no:cacheprovider -k "embed" 2>&1 | tail -3
