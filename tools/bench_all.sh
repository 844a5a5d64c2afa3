#!/bin/bash
# Round bench lines: the default (full contract) and every BASELINE workload.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/bench
timeout 300 python bench.py > gpurun_out/bench/default.json 2> gpurun_out/bench/default.err
for w in bn254_2p20 mnt4_753_2p20 bls12_381_2p26_sparse bls12_381_2p19 bn254_g2_2p20 bls12_381_g2_2p20 bls12_381_2p26; do
  timeout 300 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench/$w.json 2> gpurun_out/bench/$w.err
done
timeout 200 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench/reference.json 2> gpurun_out/bench/reference.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/bench/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1
