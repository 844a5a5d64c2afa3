cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_variants.py -q -p no:cacheprovider 2>&1 | tail -2
one() { python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e "$@" 2>&1 | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1]); p=d.get('prepared') or {}
print('std', round(d['ms_per_step'],3), d['roofline']['phase_ms_per_step'], '| prep', round(p.get('ms_per_step',0),3), (p.get('phase_ms_per_step') or {}).get('reduce'))"; }
for t in 16384 65536 131072; do echo "REDUCE_THREADS=$t"; GZKP_REDUCE_THREADS=$t one; done
