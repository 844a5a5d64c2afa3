#!/bin/bash
mkdir -p gpurun_out/sp
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_to_mont|k_digits|k_scan|k_scatter" -c 6 --csv python bench.py --workload bls12_381_2p26_sparse --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/sp/ncu_sparse.csv 2> gpurun_out/sp/ncu_sparse.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_to_mont|k_digits|k_scan|k_scatter" -c 6 --csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/sp/ncu_dense.csv 2> gpurun_out/sp/ncu_dense.err
