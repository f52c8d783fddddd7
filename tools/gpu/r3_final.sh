python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3
python bench.py > gpurun_out/r3_bench_final.json 2> gpurun_out/r3_bench_final.err
tail -1 gpurun_out/r3_bench_final.json | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['clocks'], d['breakdown_ms'], d['roofline']['frac'], d['step_roofline']['frac'], d['e2e']['value'], d['gpu_launches'])"
python bench.py --impl reference 2>/dev/null | tail -1 | cut -c1-300
