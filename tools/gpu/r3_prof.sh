export MOBIUS_KT_NOSYNC=1
python tools/flash_time.py 64 32
bash tools/gpu/run44.sh
