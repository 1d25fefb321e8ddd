# launch list of one bench run + ncu --set full of the top kernels; usage: bash tools/gpu_profile_all.sh <tag>
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_mpi_fifo|k_mpi_matrix" -s 6 -c 2 -o gpurun_out/prof_mpi_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi,mpi_matrix --no-cpu-baseline > gpurun_out/ncu_mpi_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_part_scatter|k_bucket_pair|k_part_hist|k_bucket_bounds" -s 20 -c 8 -o gpurun_out/prof_flat_$TAG \
    python bench.py --steps 1 --warmup 3 --levels ordered,unordered --no-cpu-baseline > gpurun_out/ncu_flat_$TAG.log 2>&1
ls gpurun_out | grep $TAG
