#!/bin/bash
# compute-sanitizer over small MSMs (memcheck, racecheck, synccheck, initcheck).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_small.py > gpurun_out/sanitize_$tool.txt 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|SANITIZE_PARITY' gpurun_out/sanitize_$tool.txt | tr '\n' ' ')"
done
