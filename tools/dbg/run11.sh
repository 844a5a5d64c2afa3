cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_msm.py -q -p no:cacheprovider --timeout 600 -x 2>&1 | grep -E "FAILED|Error|assert|^E " | head -20
