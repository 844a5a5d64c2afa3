cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_msm.py -q -p no:cacheprovider --timeout 600 -x 2>&1 | tail -2
for pl in 0 1; do echo "GZKP_PIPELINE=$pl"; GZKP_PIPELINE=$pl bash tools/dbg/run6.sh; done
