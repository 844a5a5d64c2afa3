cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 -x > gpurun_out/pytest_gpu.txt 2>&1; tail -5 gpurun_out/pytest_gpu.txt
python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b_lib.txt 2>&1
python -c "
import json
for f in ['gpurun_out/b_lib.txt']:
    d=json.loads(open(f).read().strip().split('\n')[-1]); print(f, d['ms_per_step'], d['value']/1e6, d['roofline']['frac'], d['roofline']['phase_ms_per_step'])
"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 30 -c 40 --csv --log-file gpurun_out/launches_r1b.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/launches_r1b.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
for r in rows[1:22]:
    print(r[ki][:50], r[vi])
PY
