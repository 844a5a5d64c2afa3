cd $GRAFT_REPO_ROOT
one() { python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e "$@" 2>&1 | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1]); p=d.get('prepared') or {}
print('std', round(d['ms_per_step'],3), 'accum', d['roofline']['phase_ms_per_step']['accumulate'], 'frac', round(d['roofline']['frac'],3), '| prep', round(p.get('ms_per_step',0),3), (p.get('phase_ms_per_step') or {}).get('accumulate'))"; }
for T in 32 64 96 128; do echo "BLS T=$T"; GZKP_ACCUM_THREADS=$T one; done
for T in 32 64 96 128; do echo "BN T=$T"; GZKP_ACCUM_THREADS=$T one --workload bn254_2p20; done
