export MOBIUS_KT_NOSYNC=1
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -1
MOBIUS_FLASH_BWD_V1=1 MOBIUS_FLASH_FWD_V1=1 timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -1
MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_BWD_QS2_MOBIUS_BWD_SLAB321.so timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -1
for i in 1 2; do python tools/flash_time.py 64 32; for v in MOBIUS_BWD_QS2 MOBIUS_BWD_QS2_MOBIUS_BWD_SLAB321; do echo $v; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_$v.so python tools/flash_time.py 64 32; done; done
