for i in 1 2; do
for lib in tools/gpu/var/libmobius_r1.so paper_conf_asplos_fengxtwls23_b200/libmobius.so; do
MOBIUS_LIB_PATH=$lib timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab.json 2>gpurun_out/ab.err
python -c "import json;d=json.load(open('gpurun_out/ab.json'));print('$lib'.split('/')[-1], round(d['value']), {k: round(v) for k, v in d['breakdown_ms'].items() if isinstance(v, float)}, d['clocks']['sm_mhz'], d['memory']['recompute_blocks'])" || tail -3 gpurun_out/ab.err
done
done
