cd $GRAFT_REPO_ROOT
one() { python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e "$@" 2>&1 | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1]); p=d.get('prepared') or {}
print('std', round(d['ms_per_step'],3), d['roofline']['phase_ms_per_step'], '| prep', p.get('window_bits'), round(p.get('ms_per_step',0),3), p.get('phase_ms_per_step'))"; }
for S in 32 64 96 128 256; do echo "S=$S"; GZKP_SEGMENT=$S one --no-prepared; done
for c in 18 19 20 21 22; do echo "prep c=$c"; GZKP_WINDOW_BITS_PREPARED=$c one; done
for c in 14 15 16; do echo "std c=$c"; GZKP_WINDOW_BITS=$c one --no-prepared; done
