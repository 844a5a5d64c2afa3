cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_variants.py -q -p no:cacheprovider > gpurun_out/variants.txt 2>&1; tail -3 gpurun_out/variants.txt
