export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention_core" 2>&1 | tail -1
for i in 1 2; do python tools/flash_time.py 64 32; echo OLD; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_OLDCAST1.so python tools/flash_time.py 64 32; done
