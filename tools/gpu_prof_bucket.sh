cd $GRAFT_REPO_ROOT
TAG=${1:-x}
ncu --set full --clock-control none --import-source on -k regex:"k_bucket_pair|k_part_scatter" -s 6 -c 6 -o gpurun_out/prof_bucket_$TAG \
    python bench.py --steps 1 --warmup 3 --levels ordered,unordered --no-cpu-baseline > gpurun_out/ncu_bucket_$TAG.log 2>&1
tail -1 gpurun_out/ncu_bucket_$TAG.log
