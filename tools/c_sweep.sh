#!/bin/bash
# Window-size sweep: ms per MSM and phase split for c in a range.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for spec in ${SPECS:-"bls12_381_2p19:13,14,15,16,17" "bls12_381_2p22:15,16,17" "bn254_2p20:14,15,16"}; do
  w=${spec%%:*}; cs=${spec#*:}
  for c in ${cs//,/ }; do
    echo "== $w c=$c" >> gpurun_out/csweep.txt
    timeout 150 python bench.py --workload $w --window-bits $c --steps 4 --warmup 2 --no-cpu-baseline --no-e2e --no-prepared 2>>gpurun_out/csweep.err \
      | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],3), d['roofline']['phase_ms_per_step'])" >> gpurun_out/csweep.txt
  done
done
