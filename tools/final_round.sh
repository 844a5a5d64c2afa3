#!/bin/bash
# End-of-round evidence: GPU tests, smoke, every bench line, launch list, k_accum ncu capture.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/bench
timeout 420 python -m pytest tests -m gpu -q --timeout 120 -p no:cacheprovider > gpurun_out/bench/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/bench/pytest_gpu.txt
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/bench/smoke.txt 2>&1
bash tools/bench_all.sh
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_accum -s 2 -c 1 -o gpurun_out/bench/accum python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-prepared > gpurun_out/bench/ncu_accum.log 2>&1
