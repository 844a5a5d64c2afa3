cd $GRAFT_REPO_ROOT
for i in 1 2; do python bench.py --workload bn254_2p20 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared 2>&1 | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().split('\n')[-1]); print(round(d['ms_per_step'],3), d['roofline']['phase_ms_per_step'])"; done
GZKP_PROFILE=0 timeout 300 nsys --version 2>/dev/null
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 60 -c 30 --csv --log-file gpurun_out/launches_bn.csv python bench.py --workload bn254_2p20 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/launches_bn.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
for r in rows[1:30]:
    print(r[ki][:50], r[vi])
PY
