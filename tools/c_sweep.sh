mkdir -p gpurun_out/cs
for c in 15 16 17 18 19; do
  GZKP_WINDOW_BITS=$c python bench.py --workload bls12_381_2p26 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/cs/u26_c$c.json 2>/dev/null
done
for c in 16 17 18; do
  GZKP_WINDOW_BITS=$c python bench.py --workload bls12_381_2p22 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/cs/u22_c$c.json 2>/dev/null
  GZKP_WINDOW_BITS=$c python bench.py --workload mnt4_753_2p20 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/cs/m20_c$c.json 2>/dev/null
  GZKP_WINDOW_BITS=$c python bench.py --workload bls12_381_2p26_sparse --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-prepared > gpurun_out/cs/s26_c$c.json 2>/dev/null
done
