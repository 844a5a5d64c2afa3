cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_msm.py tests/test_gpu_large.py -q -p no:cacheprovider --timeout 600 -x 2>&1 | tail -2
bash tools/dbg/run6.sh
