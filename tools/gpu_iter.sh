# quick iteration: MPI parity tests + MPI bench + ncu capture of the FIFO kernel
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
timeout 900 python -m pytest tests/test_parity_gpu.py -m gpu -q -k "mpi" --maxfail=5 -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1; tail -4 gpurun_out/pytest_$TAG.log
timeout 600 python bench.py --levels mpi --no-cpu-baseline > gpurun_out/bench_$TAG.log 2>&1; tail -1 gpurun_out/bench_$TAG.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('VALUE', d['value']/1e9, 'Gm/s', d['ms_per_step'], 'ms', d['roofline']['frac'])"
ncu --set full --clock-control none --import-source on -k regex:k_mpi_fifo -s 3 -c 1 -o gpurun_out/prof_fifo_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi --no-cpu-baseline > gpurun_out/ncu_fifo_$TAG.log 2>&1
tail -2 gpurun_out/ncu_fifo_$TAG.log
