cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
one() { timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared "$@" 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1])
print(round(d['ms_per_step'],3), {k: round(v,2) for k,v in d['roofline']['phase_ms_per_step'].items()})"; }
for w in bn254_2p20 mnt4_753_2p20 bls12_381_2p22 bls12_381_2p26_sparse; do
  echo "== $w"; echo -n "default  "; one --workload $w
  for ch in 128 256; do echo -n "chunk $ch "; one --workload $w --chunk $ch; done
  echo -n "pipeline "; GZKP_PIPELINE=1 one --workload $w
done
