export MOBIUS_KT_NOSYNC=1
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -5
unset MOBIUS_KT_NOSYNC
export MOBIUS_KT_NOSYNC=1
python tools/flash_time.py 64 32
python tools/flash_time.py 64 32
python tools/flash_time.py 128 8 2048 40
bash tools/gpu/run44.sh
