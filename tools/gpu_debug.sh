cd $GRAFT_REPO_ROOT
timeout 300 python tools/debug_case.py 20000 200000 two 2>&1 | tail -30
