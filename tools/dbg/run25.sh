cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for w in bn254_2p20 mnt4_753_2p20 bls12_381_2p26_sparse bls12_381_2p26; do timeout 900 python bench.py --workload $w --steps 5 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; python -c "
import json,sys; d=json.loads(open('gpurun_out/bench_$w.json').read().strip().split('\n')[-1]); p=d.get('prepared') or {}
print('$w', round(d['ms_per_step'],3), round(d['value']/1e6,1), 'Mpts/s frac', round(d['roofline']['frac'],3), d['roofline']['phase_ms_per_step'], 'prep', round(p.get('ms_per_step',0),3), 'e2e', round((d.get('e2e') or {}).get('ms_per_step',0),2), 'cpu', (d.get('cpu_baseline') or {}).get('value'))" || tail -5 gpurun_out/bench_$w.err; done
