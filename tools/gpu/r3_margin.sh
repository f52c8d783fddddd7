for m in 2.5 1.5 1.0; do echo MARGIN=$m; MOBIUS_KEEP_MARGIN_GIB=$m python bench.py 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['clocks']['sm_mhz'], d['memory']['recompute_blocks'], d['memory']['arena_GB'], d['e2e']['value'])"; done
