#!/bin/bash
# sort iteration: digit/sort tests, default + sparse bench phases, ncu DRAM bytes of the sort kernels
mkdir -p gpurun_out/q
timeout 900 python -m pytest tests/test_gpu_digits.py tests/test_gpu_msm.py -m gpu -q -x -p no:cacheprovider > gpurun_out/q/pytest.txt 2>&1
python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/q/bench_default.json 2> gpurun_out/q/bench_default.err
python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared --workload bls12_381_2p26_sparse > gpurun_out/q/bench_sparse.json 2> gpurun_out/q/bench_sparse.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_bin|k_fine|k_scan|k_to_mont" -c 14 --csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/q/ncu_sort.csv 2> gpurun_out/q/ncu_sort.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_bin|k_fine|k_scan|k_to_mont" -c 14 --csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared --workload bls12_381_2p26_sparse > gpurun_out/q/ncu_sort_sparse.csv 2> gpurun_out/q/ncu_sort_sparse.err
tail -2 gpurun_out/q/pytest.txt
