#!/bin/bash
# k_reduce_seg on CoopS groups: parity suites + bench lines (GZKP_SEG_COOP=1 default vs 0)
OUT=${OUT:-gpurun_out/sc}
mkdir -p $OUT
timeout 1500 python -m pytest tests/test_gpu_msm.py tests/test_gpu_g2.py tests/test_gpu_variants.py -m gpu -q -x -rfE -p no:cacheprovider > $OUT/pytest.txt 2>&1
tail -n2 $OUT/pytest.txt
for wl in bls12_381_2p19 bls12_381_2p22 mnt4_753_2p17 mnt4_753_2p20 bls12_381_g2_2p20 bn254_g2_2p20; do
  for K in 1 0; do
    GZKP_SEG_COOP=$K timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/${wl}_sc$K.json 2> $OUT/${wl}_sc$K.err
  done
done
python tools/summ.py $OUT/*.json
