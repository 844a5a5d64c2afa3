cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_msm.py -q --timeout 600 -p no:cacheprovider -k "sharded or heavy" > gpurun_out/pytest_sh.txt 2>&1; tail -2 gpurun_out/pytest_sh.txt
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -c 2500 gpurun_out/bench_default.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2>&1; tail -c 400 gpurun_out/bench_reference.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_default.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b_ncu.log 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_accum -s 3 -c 1 -o gpurun_out/k_accum_final python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1; echo ncu $?
