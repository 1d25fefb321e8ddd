# usage: bash tools/gpu_profile.sh <tag>
cd $GRAFT_REPO_ROOT
TAG=${1:-r01}
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_bench_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_mpi -s 2 -c 1 -o gpurun_out/prof_mpi_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi --no-cpu-baseline > gpurun_out/ncu_full_mpi_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_part_scatter|k_hash_insert|k_hash_probe|k_pair" -s 8 -c 6 -o gpurun_out/prof_flat_$TAG \
    python bench.py --steps 1 --warmup 3 --levels ordered,unordered --no-cpu-baseline > gpurun_out/ncu_full_flat_$TAG.log 2>&1
ls -la gpurun_out
