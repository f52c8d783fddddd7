export MOBIUS_KT_NOSYNC=1
python tools/flash_time.py 64 32
MOBIUS_LIB_PATH=tools/gpu/var/libmobius_MOBIUS_BWD_EXP_EXPERIMENT2.so python tools/flash_time.py 64 32
sed 's/MOBIUS_BWD_PROF1/MOBIUS_BWD_EXP_EXPERIMENT2_MOBIUS_BWD_PROF1/' tools/gpu/run44.sh > /tmp/r44b.sh; bash /tmp/r44b.sh
