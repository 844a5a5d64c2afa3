cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_g2.py -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_g2.txt 2>&1
echo "g2 exit $?" >> gpurun_out/pytest_g2.txt; tail -5 gpurun_out/pytest_g2.txt
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider --deselect tests/test_gpu_g2.py > gpurun_out/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.txt; tail -5 gpurun_out/pytest_gpu.txt
for w in bn254_g2_2p20 bls12_381_g2_2p20; do timeout 600 python bench.py --workload $w --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_$w.json 2>&1; tail -c 1500 gpurun_out/bench_$w.json; echo; done
