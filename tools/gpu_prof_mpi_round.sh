cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
TAG=r01e
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_mpi_fifo" -s 2 -c 1 -o gpurun_out/prof_mpi_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi --no-cpu-baseline > gpurun_out/ncu_mpi_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_mpi_matrix" -s 2 -c 1 -o gpurun_out/prof_mpim_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi_matrix --no-cpu-baseline > gpurun_out/ncu_mpim_$TAG.log 2>&1
ls -la gpurun_out/prof_mpi*_$TAG*
