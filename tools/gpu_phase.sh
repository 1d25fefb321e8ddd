cd $GRAFT_REPO_ROOT
python tools/phase_timing.py 2>&1 | tail -14
