#!/bin/bash
mkdir -p gpurun_out/m
timeout 1500 python -m pytest tests/test_gpu_msm.py tests/test_gpu_large.py tests/test_gpu_variants.py tests/test_gpu_digits.py -m gpu -q -rfE -p no:cacheprovider -k "not bench_config" > gpurun_out/m/pytest.txt 2>&1
for M in 1 2 3; do
python - > gpurun_out/m/prep_M$M.txt 2>&1 <<PY
import torch, time, numpy as np, sys
sys.path.insert(0, ".")
import paper_conf_asplos_maxsm0k0zsh23_b200 as gz, synth
n = 1 << 22
d = synth.dlogs("bls12_381", n, synth.dlog_seed("bls12_381"))
P = gz.fixed_base_mul("bls12_381", gz.to_device(d))
K = gz.to_device(synth.scalars("bls12_381", n, synth.scalar_seed(3)))
h = gz.PreparedPoints("bls12_381", P, weighted=$M)
for _ in range(3): h.msm(K)
torch.cuda.synchronize()
gz.set_profiling(True); gz.profile_read(reset=True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10): h.msm(K)
e1.record(); torch.cuda.synchronize()
pr = gz.profile_read(reset=True)
print("M=$M", h.info(), "ms", e0.elapsed_time(e1) / 10, {k: round(v / 10, 3) for k, v in pr["phase_ms"].items()})
PY
done
tail -3 gpurun_out/m/pytest.txt
