#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for w in bls12_381_2p22 bls12_381_2p19 mnt4_753_2p20; do
for v in "GZKP_REDUCE_CTA=128" "GZKP_REDUCE_CTA=64" "GZKP_REDUCE_CTA=32"; do
  echo "== $w $v" >> gpurun_out/quick.txt
  env $v timeout 150 python bench.py --workload $w --steps 5 --no-cpu-baseline --no-e2e --no-prepared 2>>gpurun_out/quick.err \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d['roofline']['phase_ms_per_step'])" >> gpurun_out/quick.txt
done; done
