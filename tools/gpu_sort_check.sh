#!/bin/bash
# new two-level sort: full -m gpu suite, default + sparse 2^26 bench, ncu of the sort kernels
mkdir -p gpurun_out/s
timeout 2400 python -m pytest tests -m gpu -q -x -rfE --timeout 1200 -p no:cacheprovider > gpurun_out/s/pytest_gpu.txt 2>&1
python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/s/bench_default.json 2> gpurun_out/s/bench_default.err
python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --workload bls12_381_2p26_sparse > gpurun_out/s/bench_sparse.json 2> gpurun_out/s/bench_sparse.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_bin|k_fine|k_scan|k_to_mont" -c 40 --csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/s/ncu_sort.csv 2> gpurun_out/s/ncu_sort.err
tail -3 gpurun_out/s/pytest_gpu.txt
