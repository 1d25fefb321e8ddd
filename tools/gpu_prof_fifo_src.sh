# ncu --set full of k_mpi_fifo on configs[1] + per-source-line export; usage: bash tools/gpu_prof_fifo_src.sh <tag>
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || { tail -20 gpurun_out/build_$TAG.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_mpi_fifo" -s 3 -c 1 -o gpurun_out/prof_fifo_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi --no-cpu-baseline > gpurun_out/ncu_fifo_$TAG.log 2>&1
tail -3 gpurun_out/ncu_fifo_$TAG.log
