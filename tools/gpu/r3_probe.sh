set -x
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv
./tools/gpu/var/sfu_probe
export MOBIUS_KT_NOSYNC=1
python tools/flash_time.py 64 32
python tools/flash_time.py 128 8 2048 40
bash tools/gpu/run44.sh
