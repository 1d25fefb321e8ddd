cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "wide or multibatch or world2 or contract" 2>&1 | tail -5
nproc; python -c "import os; print(len(os.sched_getaffinity(0)))"
/usr/bin/time -v timeout 900 python bench.py > gpurun_out/bench_r2a.log 2> gpurun_out/bench_r2a.err; tail -3 gpurun_out/bench_r2a.err | head -3; grep "Elapsed" gpurun_out/bench_r2a.err
bash tools/gpu_level_traffic.sh r2a ordered,mpi
