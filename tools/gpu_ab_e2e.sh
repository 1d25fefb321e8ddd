# A/B of the MPI-level host pipeline (e2e, pinned host buffers) via MM_AB_DEFINES builds:
# every build's e2e ms/step per MM_OPT_PIPELINE_CHUNKS value, twice (E2E_MAPPED=1: mapped host outputs)
# usage: bash tools/gpu_ab_e2e.sh "<defines A>" "<defines B>" ...
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
for cfg in "$@"; do
  export MM_AB_DEFINES="$cfg"
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='ab')" > /dev/null 2>&1 || { echo "build fail $cfg"; continue; }
  echo "== $cfg (mapped=${E2E_MAPPED:-0})"
  MM_LIB=$PWD/paper_conf_ipps_klenkfed17_b200/lib/libmm_ab.so E2E_ONLY=1 timeout 600 python tools/e2e_pipeline.py 2>&1 | grep chunks
done
done
