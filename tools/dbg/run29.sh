cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches_sparse2.csv python bench.py --workload bls12_381_2p26_sparse --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none -k regex:"k_scatter|k_digits|k_to_mont" -s 3 -c 3 -o gpurun_out/sort_sparse python bench.py --workload bls12_381_2p26_sparse --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-prepared > /dev/null 2>&1; echo ncu $?
bash tools/dbg/run27.sh
