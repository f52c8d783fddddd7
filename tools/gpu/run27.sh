for i in 1 2; do python tools/ln_bench.py; MOBIUS_LN_FLOATROW=1 python tools/ln_bench.py; done
