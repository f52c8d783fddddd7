MBS=32 timeout 300 python tools/embed_bench.py
MBS=4 timeout 300 python tools/embed_bench.py
