cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 -x > gpurun_out/pytest_gpu.txt 2>&1; tail -3 gpurun_out/pytest_gpu.txt
for c in 16 18 20; do GZKP_WINDOW_BITS_PREPARED=$c python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b_c$c.txt 2>&1; python -c "
import json
d=json.loads(open('gpurun_out/b_c$c.txt').read().strip().split('\n')[-1]); p=d['prepared']; print('std', d['ms_per_step'], d['roofline']['phase_ms_per_step']); print($c, p['ms_per_step'], p['value']/1e6, p['accum_frac_imad_peak'], p['phase_ms_per_step'])
"; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_accum -s 2 -c 1 -o gpurun_out/accum_r1 python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/ncu_full.log
