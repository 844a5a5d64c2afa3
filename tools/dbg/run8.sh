cd $GRAFT_REPO_ROOT
nproc
timeout 900 python bench.py > gpurun_out/bench_default.txt 2> gpurun_out/bench_default.err; echo "rc $?"; tail -c 3000 gpurun_out/bench_default.txt
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref.txt 2> gpurun_out/bench_ref.err; echo "rc $?"; tail -c 1500 gpurun_out/bench_ref.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
