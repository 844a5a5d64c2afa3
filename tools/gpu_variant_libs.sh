#!/bin/bash
# compile-time variants (build.py -D... --out libgzkp_<v>.so) timed against the default library
# usage: bash tools/gpu_variant_libs.sh "v1 v2" "workload1 workload2" [pytest]
mkdir -p gpurun_out/v3
P=paper_conf_asplos_maxsm0k0zsh23_b200
for v in default $1; do
  if [ $v = default ]; then L=$P/libgzkp.so; else L=$P/libgzkp_$v.so; fi
  for wl in $2; do
    GZKP_LIB=$PWD/$L python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/v3/${v}_$wl.json 2> gpurun_out/v3/${v}_$wl.err
  done
  if [ -n "$3" ] && [ $v != default ]; then
    GZKP_LIB=$PWD/$L timeout 600 python -m pytest tests/test_gpu_msm.py tests/test_gpu_field_ec.py -m gpu -q -x -p no:cacheprovider > gpurun_out/v3/pytest_$v.txt 2>&1
    tail -n1 gpurun_out/v3/pytest_$v.txt
  fi
done
