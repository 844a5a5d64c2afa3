#!/bin/bash
# batch-affine levels: parity under GZKP_AFFINE_LEVELS, bench phase sweep
mkdir -p gpurun_out/a
GZKP_AFFINE_LEVELS=3 timeout 900 python -m pytest tests/test_gpu_msm.py -m gpu -q -x -p no:cacheprovider > gpurun_out/a/pytest_msm_L3.txt 2>&1
GZKP_AFFINE_LEVELS=8 timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_large.py -m gpu -q -x -p no:cacheprovider -k "not bench_config" > gpurun_out/a/pytest_msm_L8.txt 2>&1
for L in 0 3 8; do
  GZKP_AFFINE_LEVELS=$L python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/a/bench_L$L.json 2> gpurun_out/a/bench_L$L.err
done
GZKP_AFFINE_LEVELS=6 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:"k_affine|k_accum" -c 7 --csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/a/ncu_affine.csv 2> gpurun_out/a/ncu_affine.err
for f in gpurun_out/a/pytest_*.txt; do tail -n 1 $f; done
