#!/bin/bash
# One GPU validation pass: build check, smoke, the -m gpu suite, default bench.
mkdir -p gpurun_out/v
nvidia-smi -L > gpurun_out/v/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/v/smoke.txt 2>&1
timeout 3600 python -m pytest tests -m gpu -q -rfE --timeout 1800 -p no:cacheprovider > gpurun_out/v/pytest_gpu.txt 2>&1
python bench.py --steps 10 --warmup 3 > gpurun_out/v/bench_default.json 2> gpurun_out/v/bench_default.err
tail -3 gpurun_out/v/pytest_gpu.txt
