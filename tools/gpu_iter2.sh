cd $GRAFT_REPO_ROOT
TAG=${1:-x}
timeout 900 python -m pytest tests/test_parity_gpu.py -m gpu -q -k "mpi" --maxfail=5 -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1; tail -2 gpurun_out/pytest_$TAG.log
python tools/phase_timing.py 2>&1 | tail -11
timeout 600 python bench.py --levels mpi --no-cpu-baseline > gpurun_out/bench_$TAG.log 2>&1; tail -1 gpurun_out/bench_$TAG.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('VALUE', d['value']/1e9, 'Gm/s', d['ms_per_step'], 'ms', d['roofline']['frac'])"
