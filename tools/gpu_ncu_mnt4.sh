#!/bin/bash
mkdir -p gpurun_out/n
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_accum" -c 1 -o gpurun_out/n/k_accum_mnt4_753_2p20 python bench.py --workload mnt4_753_2p20 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/n/ncu_mnt4.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_tail" -c 1 -o gpurun_out/n/tail_reduce_bls12_381_2p19 python bench.py --workload bls12_381_2p19 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/n/ncu_tail.log 2>&1
python bench.py --workload mnt4_753_2p17 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/n/bench_mnt4_2p17.json 2> gpurun_out/n/bench_mnt4_2p17.err
python bench.py --workload bls12_381_2p19 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/n/bench_bls_2p19.json 2> gpurun_out/n/bench_bls_2p19.err
ls -la gpurun_out/n
