# build + MPI-level GPU tests, then A/B of configs[1] (MM_AB_DEFINES builds)
# usage: bash tools/gpu_ab_test.sh "<pytest -k expr>" "<defines A>" "<defines B>" ...
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
K="$1"; shift
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_ab.log 2>&1 || { tail -20 gpurun_out/build_ab.log; exit 1; }
if [ -n "$K" ]; then timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "$K" 2>&1 | tail -3; fi
bash tools/gpu_ab_mpi.sh "$@"
