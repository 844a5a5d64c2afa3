#!/bin/bash
# Window-group pipeline on/off (one bench line per variant).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for W in bls12_381_2p22 bn254_2p20; do
for v in "" "GZKP_PIPELINE=1"; do
  echo "== $W $v" >> gpurun_out/variants.txt
  env $v timeout 300 python bench.py --workload $W --steps 5 --no-cpu-baseline --no-e2e --no-prepared 2>/dev/null \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['roofline']['phase_ms_per_step'])" >> gpurun_out/variants.txt
done
done
