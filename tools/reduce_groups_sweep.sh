#!/bin/bash
# bucket reduction in R sub-groups with the Horner tail overlapped (GZKP_REDUCE_GROUPS)
OUT=${OUT:-gpurun_out/rg}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_variants.py tests/test_gpu_msm.py -m gpu -q -x -p no:cacheprovider > $OUT/pytest.txt 2>&1
tail -n1 $OUT/pytest.txt
for wl in bls12_381_2p22 bls12_381_2p19 mnt4_753_2p17 mnt4_753_2p20 bn254_2p20; do
  for R in 1 2 3 4 8; do
    GZKP_REDUCE_GROUPS=$R python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > $OUT/${wl}_R$R.json 2>/dev/null
  done
done
