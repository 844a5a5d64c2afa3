#!/bin/bash
mkdir -p gpurun_out/c
timeout 900 python -m pytest tests/test_gpu_field_ec.py tests/test_gpu_msm.py -m gpu -q -x -rfE -p no:cacheprovider > gpurun_out/c/pytest.txt 2>&1
python bench.py --workload bls12_381_2p19 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/c/bench_bls_2p19.json 2> gpurun_out/c/bench_bls_2p19.err
python bench.py --workload mnt4_753_2p17 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/c/bench_mnt4_2p17.json 2> gpurun_out/c/bench_mnt4_2p17.err
python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/c/bench_default.json 2> gpurun_out/c/bench_default.err
tail -3 gpurun_out/c/pytest.txt
