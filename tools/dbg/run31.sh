cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.txt; tail -3 gpurun_out/pytest_gpu.txt; grep FAILED gpurun_out/pytest_gpu.txt | head
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
one() { timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e "$@" 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1]); p=d.get('prepared') or {}
print(round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,2) for k,v in (d['roofline'].get('phase_ms_per_step') or {}).items()}, 'prep', round(p.get('ms_per_step',0),3))"; }
for w in bls12_381_2p22 bls12_381_2p26_sparse bn254_g2_2p20; do echo -n "$w "; one --workload $w; done
for w in bls12_381_ntt_2p24 bn254_ntt_2p22; do echo -n "$w minb3 "; one --workload $w; echo -n "$w minb2 "; GZKP_NTT_MINB=2 one --workload $w; done
