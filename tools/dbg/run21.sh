cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ntt.py -q -x --timeout 600 -p no:cacheprovider > gpurun_out/pytest_ntt.txt 2>&1
echo "ntt exit $?" >> gpurun_out/pytest_ntt.txt; tail -30 gpurun_out/pytest_ntt.txt
for w in bls12_381_ntt_2p24 bn254_ntt_2p22 mnt4_753_ntt_2p20; do timeout 600 python bench.py --workload $w --steps 5 --no-cpu-baseline > gpurun_out/bench_$w.json 2>&1; tail -c 1200 gpurun_out/bench_$w.json; echo; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ntt_pass -s 6 -c 3 -o gpurun_out/ntt_bls python bench.py --workload bls12_381_ntt_2p24 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu $?
