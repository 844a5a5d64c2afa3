#!/bin/bash
# Accumulation launch-configuration sweep (one bench line per variant).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
W=${1:-bls12_381_2p22}
for v in "" "GZKP_ACCUM_THREADS=64" "GZKP_ACCUM_MINB=3" "GZKP_ACCUM_MINB=3 GZKP_ACCUM_THREADS=64"; do
  echo "== $v" >> gpurun_out/variants.txt
  env $v timeout 300 python bench.py --workload $W --steps 5 --no-cpu-baseline --no-e2e --no-prepared 2>/dev/null \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['roofline']['phase_ms_per_step'])" >> gpurun_out/variants.txt
done
