# tests + smoke + bench on one box; logs under gpurun_out/
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
timeout 1500 python -m pytest tests -m gpu -q --maxfail=20 -p no:cacheprovider > gpurun_out/pytest_gpu_$TAG.log 2>&1
tail -25 gpurun_out/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -3 gpurun_out/smoke_$TAG.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1; tail -3 gpurun_out/bench_$TAG.log
