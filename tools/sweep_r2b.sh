#!/bin/bash
# round-2 sweep: reduction sub-groups (GZKP_REDUCE_GROUPS) and the prepared-path window size
OUT=${OUT:-gpurun_out/sw}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_variants.py -m gpu -q -x -p no:cacheprovider -k "REDUCE" > $OUT/pytest.txt 2>&1
tail -n1 $OUT/pytest.txt
for wl in bls12_381_2p19 mnt4_753_2p17 bls12_381_2p22 mnt4_753_2p20; do
  for R in 1 2 4; do
    GZKP_REDUCE_GROUPS=$R timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > $OUT/${wl}_R$R.json 2>$OUT/${wl}_R$R.err
  done
done
for wl in bls12_381_2p19 bls12_381_2p22 mnt4_753_2p17; do
  for c in 13 14 15 16 17 18; do
    GZKP_WINDOW_BITS_PREPARED=$c timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/${wl}_prep_c$c.json 2>$OUT/${wl}_prep_c$c.err
  done
done
