cd $GRAFT_REPO_ROOT
TAG=${1:-x}
ncu --set full --clock-control none --import-source on -k regex:k_mpi_fifo -s 3 -c 1 -o gpurun_out/prof_fifo_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi --no-cpu-baseline > gpurun_out/ncu_fifo_$TAG.log 2>&1
tail -1 gpurun_out/ncu_fifo_$TAG.log
