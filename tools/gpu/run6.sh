set -x
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2_gputest_6.log 2>&1; echo "tests rc=$?"
tail -5 gpurun_out/r2_gputest_6.log
grep -a "FAIL\|Error" gpurun_out/r2_gputest_6.log | head -20
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/r2_bench_6.json 2> gpurun_out/r2_bench_6.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2_bench_6.json'));print(d['value'],d['breakdown_ms'],d['clocks'])"
for cap in 2 4 8; do
timeout 900 python bench.py --steps 3 --warmup 3 --micro-batch 8 --microbatches 4 --arena-cap-gib $cap --no-cpu-baseline > gpurun_out/r2_bench_c2_${cap}g.json 2> gpurun_out/r2_bench_c2_${cap}g.err; echo "c2 $cap rc=$?"
tail -3 gpurun_out/r2_bench_c2_${cap}g.err
python -c "import json;d=json.load(open('gpurun_out/r2_bench_c2_${cap}g.json'));print(d['value'],d['e2e']['value'],d['config']['n_stages'],d['config']['stage_layers'],d['memory'],d['step_roofline'],d['overlap'])"
done
