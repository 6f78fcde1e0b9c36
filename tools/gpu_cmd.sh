cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -x -q -m gpu -k "splitk" 2>&1 | tail -30
HIOS_LIB=$PWD/ab/libhios_head.so timeout 900 python -m pytest tests -x -q -m gpu -k "splitk" 2>&1 | tail -3
