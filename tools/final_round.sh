#!/bin/bash
# End-of-round evidence: GPU tests, smoke, every bench line, launch list, k_accum ncu capture.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
OUT=${OUT:-gpurun_out/bench}
mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q -rfE --timeout 1500 -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1
OUT=$OUT bash tools/bench_all.sh
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_accum -s 2 -c 1 -o $OUT/accum python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-prepared > $OUT/ncu_accum.log 2>&1
