timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm or block" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_fullsize.py -q -x 2>&1 | tail -1
for i in 1 2; do
for e in 1 0; do echo PDL=$e; MOBIUS_PDL=$e python bench.py --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['clocks']['sm_mhz'], d['breakdown_ms']['gemm'])"; done
done
