cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.txt; tail -3 gpurun_out/pytest_gpu.txt; grep FAILED gpurun_out/pytest_gpu.txt | head
one() { timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e "$@" 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1]); p=d.get('prepared') or {}
print(round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,2) for k,v in d['roofline']['phase_ms_per_step'].items()}, 'prep', round(p.get('ms_per_step',0),3))"; }
for w in bls12_381_2p22 bn254_2p20 bls12_381_2p26_sparse; do echo -n "$w "; one --workload $w; done
timeout 900 ncu --set full --clock-control none -k regex:"k_scatter|k_digits|k_to_mont" -s 3 -c 3 -o gpurun_out/sort_bls22 python bench.py --workload bls12_381_2p22 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none -k regex:"k_scatter|k_digits|k_to_mont" -s 3 -c 3 -o gpurun_out/sort_sparse2 python bench.py --workload bls12_381_2p26_sparse --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1; echo ncu $?
