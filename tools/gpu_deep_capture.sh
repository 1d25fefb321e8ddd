# configs[4] deep-endpoint launch: ncu --set full capture (k_mpi_fifo_deep counters) + a bench run
# usage: bash tools/gpu_deep_capture.sh <tag>
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || { tail -20 gpurun_out/build_$TAG.log; exit 1; }
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_mpi_fifo" -s 2 -c 1 -o gpurun_out/prof_deep_$TAG \
    python bench.py --steps 1 --warmup 3 --levels mpi_worst --no-cpu-baseline > gpurun_out/ncu_deep_$TAG.log 2>&1
tail -2 gpurun_out/ncu_deep_$TAG.log
timeout 300 python tools/e2e_pipeline.py 2>&1 | head -14 > gpurun_out/e2e_$TAG.log; cat gpurun_out/e2e_$TAG.log
ls gpurun_out | grep $TAG
