# ncu --set full of the bucket kernel + both scatter passes (unordered level); usage: bash tools/gpu_prof_flat_src.sh <tag> [level]
cd $GRAFT_REPO_ROOT
TAG=${1:-x}; LV=${2:-unordered}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1 || { tail -20 gpurun_out/build_$TAG.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_bucket_pair|k_part_scatter|k_part_hist" -s 14 -c 6 -o gpurun_out/prof_flat_$TAG \
    python bench.py --steps 1 --warmup 3 --levels $LV --no-cpu-baseline > gpurun_out/ncu_flat_$TAG.log 2>&1
tail -2 gpurun_out/ncu_flat_$TAG.log
