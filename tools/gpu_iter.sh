#!/bin/bash
# iteration check: MSM parity suites + a few bench lines with phases
# usage: bash tools/gpu_iter.sh "tests/test_gpu_msm.py ..." "workload ..."
OUT=${OUT:-gpurun_out/it}
mkdir -p $OUT
timeout 1500 python -m pytest $1 -m gpu -q -x -rfE -p no:cacheprovider > $OUT/pytest.txt 2>&1
tail -n1 $OUT/pytest.txt
for wl in $2; do
  python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > $OUT/$wl.json 2> $OUT/$wl.err
done
