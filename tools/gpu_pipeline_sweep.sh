#!/bin/bash
mkdir -p gpurun_out/pl
for wl in bls12_381_2p22 bls12_381_2p19; do
  python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/pl/base_$wl.json 2>/dev/null
  GZKP_PIPELINE=1 python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/pl/p1_$wl.json 2>/dev/null
  for low in 2 4 8; do
    GZKP_PIPELINE=2 GZKP_PIPELINE_LOW=$low python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/pl/p2_low${low}_$wl.json 2>/dev/null
  done
done
timeout 900 python -m pytest tests/test_gpu_variants.py tests/test_gpu_msm.py -m gpu -q -x -p no:cacheprovider > gpurun_out/pl/pytest.txt 2>&1
tail -n1 gpurun_out/pl/pytest.txt
