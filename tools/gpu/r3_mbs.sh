for cfg in "--microbatches 4 --micro-batch 32" "--microbatches 2 --micro-batch 64" "--microbatches 4 --micro-batch 32" "--microbatches 2 --micro-batch 64"; do
  echo "== $cfg"; python bench.py $cfg --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['clocks']['sm_mhz'], d['memory']['recompute_blocks'], d['breakdown_ms']['gemm'], d['breakdown_ms']['attention'], d['breakdown_ms']['elementwise'])"
done
