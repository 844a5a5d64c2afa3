cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ntt.py -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_ntt.txt 2>&1
echo "ntt exit $?" >> gpurun_out/pytest_ntt.txt; tail -3 gpurun_out/pytest_ntt.txt
for w in bls12_381_ntt_2p24 bn254_ntt_2p22 mnt4_753_ntt_2p20; do timeout 600 python bench.py --workload $w --steps 10 > gpurun_out/bench_$w.json 2>&1; python -c "
import json,sys; d=json.loads(open('gpurun_out/bench_$w.json').read().strip().split('\n')[-1]); print('$w', round(d['ms_per_step'],3), round(d['roofline']['frac'],3))"; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ntt_pass -s 6 -c 3 -o gpurun_out/ntt_bls3 python bench.py --workload bls12_381_ntt_2p24 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_ntt.csv python bench.py --workload bls12_381_ntt_2p24 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu2 $?
