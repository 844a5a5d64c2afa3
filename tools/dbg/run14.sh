cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_field_ec.py -q -p no:cacheprovider -k "field_ops" 2>&1 | tail -2
GZKP_DFP=1 timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_large.py -q -p no:cacheprovider -x -k "bls or config1 or sharding or prepared or weighted" 2>&1 | tail -2
one() { python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e "$@" 2>&1 | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1]); p=d.get('prepared') or {}
print('std', round(d['ms_per_step'],3), 'accum', d['roofline']['phase_ms_per_step']['accumulate'], 'frac', round(d['roofline']['frac'],3), '| prep', round(p.get('ms_per_step',0),3), (p.get('phase_ms_per_step') or {}).get('accumulate'))"; }
echo "DFP=0"; GZKP_DFP=0 one
echo "DFP=1"; GZKP_DFP=1 one
