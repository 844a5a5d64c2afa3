#!/bin/bash
# compute-sanitizer over small MSMs (memcheck, racecheck, synccheck, initcheck),
# then memcheck + racecheck once more with the batch-affine levels on.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
OUT=${OUT:-gpurun_out/san}
mkdir -p $OUT
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_small.py > $OUT/sanitize_$tool.txt 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|SANITIZE_PARITY' $OUT/sanitize_$tool.txt | tr '\n' ' ')"
done
for tool in memcheck racecheck; do
  GZKP_AFFINE_LEVELS=3 timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_small.py > $OUT/sanitize_affine_$tool.txt 2>&1
  echo "affine $tool rc=$? $(grep -E 'ERROR SUMMARY|SANITIZE_PARITY' $OUT/sanitize_affine_$tool.txt | tr '\n' ' ')"
done
