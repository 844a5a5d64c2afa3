#!/bin/bash
# compile-time variants (build.py -D...) timed against the default library
mkdir -p gpurun_out/v2
P=paper_conf_asplos_maxsm0k0zsh23_b200
for v in default coopsos mulsos; do
  if [ $v = default ]; then L=$P/libgzkp.so; else L=$P/libgzkp_$v.so; fi
  for wl in bls12_381_2p19 bls12_381_2p22 mnt4_753_2p17; do
    GZKP_LIB=$PWD/$L python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/v2/${v}_$wl.json 2> gpurun_out/v2/${v}_$wl.err
  done
done
GZKP_LIB=$PWD/$P/libgzkp_mulsos.so timeout 600 python -m pytest tests/test_gpu_msm.py -m gpu -q -x -p no:cacheprovider > gpurun_out/v2/pytest_mulsos.txt 2>&1
GZKP_LIB=$PWD/$P/libgzkp_coopsos.so timeout 600 python -m pytest tests/test_gpu_msm.py -m gpu -q -x -p no:cacheprovider > gpurun_out/v2/pytest_coopsos.txt 2>&1
tail -n1 gpurun_out/v2/pytest_*.txt
