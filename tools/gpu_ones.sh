#!/bin/bash
# scalar-1 points summed apart (k_ones_sum): parity suites + bench lines (GZKP_ONES=1 default vs 0)
OUT=${OUT:-gpurun_out/ones}
mkdir -p $OUT
timeout 1800 python -m pytest tests/test_gpu_msm.py tests/test_gpu_variants.py tests/test_gpu_large.py tests/test_gpu_digits.py tests/test_gpu_dist.py -m gpu -q -x -rfE -p no:cacheprovider > $OUT/pytest.txt 2>&1
tail -n2 $OUT/pytest.txt
for wl in bls12_381_2p26_sparse bls12_381_2p22 bn254_2p20; do
  for K in 1 0; do
    GZKP_ONES=$K timeout 400 python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > $OUT/${wl}_ones$K.json 2> $OUT/${wl}_ones$K.err
  done
done
python tools/summ.py $OUT/*.json
