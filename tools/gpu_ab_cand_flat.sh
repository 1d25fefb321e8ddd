# no-wildcard GPU tests through a candidate A/B build (MM_LIB), then level A/B of several builds
# usage: TESTS="<pytest -k>" LEVELS=<levels> bash tools/gpu_ab_cand_flat.sh "<candidate defines>" "<defines A>" ...
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
export MM_AB_DEFINES="$1"; shift
python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='ab')" > /dev/null 2>&1 || { echo "build fail"; exit 1; }
cp paper_conf_ipps_klenkfed17_b200/lib/libmm_ab.so /tmp/libmm_cand.so
MM_LIB=/tmp/libmm_cand.so timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "${TESTS:-unordered or fallback or sharded or back_to_back or smoke}" 2>&1 | tail -2
LEVELS=${LEVELS:-unordered,unordered_256m} bash tools/gpu_ab_levels.sh "$@"
