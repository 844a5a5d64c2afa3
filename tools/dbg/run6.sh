cd $GRAFT_REPO_ROOT
for wl in bls12_381_2p22 bn254_2p20 mnt4_753_2p20; do
python bench.py --workload $wl --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b6_$wl.txt 2>&1; python -c "
import json
d=json.loads(open('gpurun_out/b6_$wl.txt').read().strip().split('\n')[-1]); p=d['prepared']; print('$wl std', round(d['ms_per_step'],3), round(d['value']/1e6,2), round(d['roofline']['frac'],3), d['roofline']['phase_ms_per_step']); print('   prep', p['window_bits'], round(p['ms_per_step'],3), round(p['value']/1e6,2), round(p['accum_frac_imad_peak'],3), p['phase_ms_per_step'])
" || tail -5 gpurun_out/b6_$wl.txt; done
