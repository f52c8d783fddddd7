for i in 1 2; do python bench.py --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['clocks']['sm_mhz'], d['breakdown_ms']['gemm'], d['breakdown_ms']['attention'], d['breakdown_ms']['elementwise'], d['roofline']['frac'])"; done
