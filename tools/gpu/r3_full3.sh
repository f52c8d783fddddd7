timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3
python bench.py > gpurun_out/r3_bench4.json 2> gpurun_out/r3_bench4.err
tail -1 gpurun_out/r3_bench4.json | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['clocks'], d['breakdown_ms'], d['roofline']['frac'], d['e2e']['value'])"
