cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 600 -k "mnt4" 2>&1 | tail -3
