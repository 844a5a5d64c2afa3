cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_field_ec.py tests/test_gpu_ntt.py -q -x --timeout 600 -p no:cacheprovider -k "field or ntt_small or multipass" > gpurun_out/pytest_field.txt 2>&1
echo "field exit $?" >> gpurun_out/pytest_field.txt; tail -3 gpurun_out/pytest_field.txt
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.txt; tail -3 gpurun_out/pytest_gpu.txt
for w in bls12_381_2p22 bn254_2p20 bls12_381_ntt_2p24 bn254_ntt_2p22; do timeout 900 python bench.py --workload $w --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; python -c "
import json,sys; d=json.loads(open('gpurun_out/bench_$w.json').read().strip().split('\n')[-1]); p=d.get('prepared') or {}
print('$w', round(d['ms_per_step'],3), round(d['value']/1e6,1), 'M/s frac', round(d['roofline']['frac'],3), d['roofline'].get('phase_ms_per_step'), 'prep', round(p.get('ms_per_step',0),3))" || tail -5 gpurun_out/bench_$w.err; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches_sparse.csv python bench.py --workload bls12_381_2p26_sparse --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1; echo ncu $?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches_mnt4.csv python bench.py --workload mnt4_753_2p20 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1; echo ncu $?
