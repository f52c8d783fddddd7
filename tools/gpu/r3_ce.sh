export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_fullsize.py -q -x -k "head or cross or entropy or ce" 2>&1 | tail -1
for i in 1 2; do ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep cross; echo OLD; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_OLDCE1.so ELEM_T=32768 python tools/elem_bench.py 2>&1 | grep cross; done
