#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 420 python -m pytest tests -m gpu -x -q --timeout 120 -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.txt
for w in bls12_381_2p22 bls12_381_2p19 bn254_2p20 mnt4_753_2p20 bls12_381_2p26_sparse; do
for v in "" "GZKP_PIPELINE=2"; do
  echo "== $w $v" >> gpurun_out/quick.txt
  env $v timeout 150 python bench.py --workload $w --steps 5 --no-cpu-baseline --no-e2e --no-prepared 2>>gpurun_out/quick.err \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d['step_ms'], d['roofline']['phase_ms_per_step'])" >> gpurun_out/quick.txt
done; done
