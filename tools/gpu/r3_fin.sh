export MOBIUS_KT_NOSYNC=1
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -2
python tools/flash_time.py 64 32
python tools/flash_time.py 64 32
unset MOBIUS_KT_NOSYNC
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_fullsize.py -q -x 2>&1 | tail -3
