#!/bin/bash
mkdir -p gpurun_out/sc
timeout 900 python -m pytest tests/test_gpu_digits.py tests/test_gpu_msm.py -m gpu -q -x -p no:cacheprovider > gpurun_out/sc/pytest.txt 2>&1
for wl in bls12_381_2p22 bls12_381_2p26_sparse bls12_381_2p19; do
python bench.py --workload $wl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/sc/$wl.json 2>/dev/null
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_to_mont|k_digits|k_scan|k_scatter" -c 7 --csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/sc/ncu_dense.csv 2>/dev/null
tail -n1 gpurun_out/sc/pytest.txt
