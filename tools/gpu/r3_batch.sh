export MOBIUS_KT_NOSYNC=1
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -2
for i in 1 2; do python tools/flash_time.py 64 32; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_FWD_MMA_BATCH0.so python tools/flash_time.py 64 32; done
bash tools/gpu/run46.sh
