cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 -x > gpurun_out/pytest_gpu.txt 2>&1; tail -5 gpurun_out/pytest_gpu.txt
python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b_lib.txt 2>&1
python -c "
import json
d=json.loads(open('gpurun_out/b_lib.txt').read().strip().split('\n')[-1]); print(d['ms_per_step'], d['value']/1e6, d['roofline']['frac'], d['roofline']['phase_ms_per_step']); print(json.dumps(d['prepared']))
"
for c in 16 18 19 20 21; do GZKP_WINDOW_BITS_PREPARED=$c python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b_c$c.txt 2>&1; python -c "
import json
d=json.loads(open('gpurun_out/b_c$c.txt').read().strip().split('\n')[-1]); p=d['prepared']; print($c, p['ms_per_step'], p['value']/1e6, p['accum_frac_imad_peak'], p['phase_ms_per_step'])
"; done
