export MOBIUS_KT_NOSYNC=1
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -3
python tools/flash_time.py 64 32
python tools/flash_time.py 64 32
MOBIUS_FLASH_FWD_V1=1 python tools/flash_time.py 64 32
python tools/flash_time.py 64 8
bash tools/gpu/run46.sh
