export MOBIUS_KT_NOSYNC=1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" 2>&1 | tail -1
for i in 1 2; do python tools/flash_time.py 64 32; MOBIUS_FLASH_FWD_GROUP=0 python tools/flash_time.py 64 32; done
unset MOBIUS_KT_NOSYNC
for i in 1 2; do python bench.py --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['clocks']['sm_mhz'], d['breakdown_ms']['attention'])"; done
