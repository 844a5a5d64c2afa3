cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_msm.py -q -p no:cacheprovider -x -k "host or prepared or config1" 2>&1 | tail -2
python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-prepared 2>&1 | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1]); print('std', round(d['ms_per_step'],3), 'e2e', d['e2e'])"
