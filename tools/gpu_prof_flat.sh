cd $GRAFT_REPO_ROOT
TAG=${1:-x}
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_flat_$TAG.csv \
    python bench.py --steps 1 --warmup 3 --levels ordered,unordered --no-cpu-baseline > gpurun_out/ncu_flat_$TAG.log 2>&1
tail -1 gpurun_out/ncu_flat_$TAG.log | cut -c1-200
