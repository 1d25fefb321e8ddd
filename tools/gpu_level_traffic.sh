# ncu DRAM traffic of one step per bench level, inside the engine's timed region
# (NVTX mm_region nested in the level's mm_timed range) -> profiles/level_traffic.json
# usage: bash tools/gpu_level_traffic.sh <tag> [levels]
cd $GRAFT_REPO_ROOT
TAG=${1:-x}
LEVELS=${2:-mpi,mpi_cookies,mpi_matrix,ordered,unordered,unordered_256m,mpi_worst}
mkdir -p gpurun_out
ARGS=""
for L in ${LEVELS//,/ }; do
  timeout 900 ncu --nvtx --nvtx-include "mm_timed:$L/mm_region]" \
      --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/lvl_${L}_$TAG.csv python bench.py --levels $L --steps 1 --warmup 3 --no-cpu-baseline --nvtx \
      > gpurun_out/lvl_${L}_$TAG.log 2>&1
  ARGS="$ARGS $L=gpurun_out/lvl_${L}_$TAG.csv"
done
python tools/level_traffic.py gpurun_out/level_traffic_$TAG.json $ARGS
