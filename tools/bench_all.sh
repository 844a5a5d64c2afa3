#!/bin/bash
# Round bench lines: the default (full contract) and every BASELINE workload,
# each with the parity leg (closed-form check of the timed MSM's bytes).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
OUT=${OUT:-gpurun_out/bench}
mkdir -p $OUT
timeout 400 python bench.py > $OUT/default.json 2> $OUT/default.err
for w in bn254_2p10 bn254_2p20 mnt4_753_2p20 mnt4_753_2p17 bls12_381_2p19 bls12_381_2p26_sparse bls12_381_2p26 \
         bn254_g2_2p20 bls12_381_g2_2p20 bls12_381_ntt_2p24 bn254_ntt_2p22 mnt4_753_ntt_2p20; do
  timeout 600 python bench.py --workload $w > $OUT/$w.json 2> $OUT/$w.err
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $OUT/reference.json 2> $OUT/reference.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1
