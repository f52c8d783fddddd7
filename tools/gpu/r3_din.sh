export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -1
for i in 1 2; do python tools/flash_time.py 64 32; echo DIN0; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_BWD_DIN0.so python tools/flash_time.py 64 32; done
unset MOBIUS_KT_NOSYNC
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_fullsize.py -q -x 2>&1 | tail -1
