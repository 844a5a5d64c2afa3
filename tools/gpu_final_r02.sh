#!/bin/bash
# round-2 closing evidence: full GPU suite, smoke, every bench line, launch list,
# k_accum ncu capture, then compute-sanitizer over the small MSMs
OUT=gpurun_out/bench bash tools/final_round.sh
tail -n 3 gpurun_out/bench/pytest_gpu.txt
OUT=gpurun_out/san bash tools/run_sanitizers.sh
echo done
