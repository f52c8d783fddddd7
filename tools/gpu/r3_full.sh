timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -5
python bench.py > gpurun_out/r3_bench2.json 2> gpurun_out/r3_bench2.err
tail -2 gpurun_out/r3_bench2.err
