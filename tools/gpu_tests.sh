cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q --maxfail=20 -p no:cacheprovider "$@" > gpurun_out/pytest_gpu.log 2>&1
tail -30 gpurun_out/pytest_gpu.log
