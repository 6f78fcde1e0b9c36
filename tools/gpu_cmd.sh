cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -x -q -m gpu -k "sep or bench_config" 2>&1 | tail -2
