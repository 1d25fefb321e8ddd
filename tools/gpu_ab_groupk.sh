# A/B of the K threshold below which single-type wildcards use stream_chain
cd $GRAFT_REPO_ROOT
python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True); _build.build_library(variant='timing')" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "mpi" 2>&1 | tail -1
python tools/phase_timing.py 2>&1 | tail -6
for k in 0 32; do
  sed -i "s/^#define MM_GROUP_MIN_K [0-9]*/#define MM_GROUP_MIN_K $k/" paper_conf_ipps_klenkfed17_b200/csrc/k_mpi_fifo.cu
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True)" > /dev/null 2>&1
  for i in 1 2; do timeout 300 python bench.py --levels mpi --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K>$k', round(d['value']/1e9,3), d['roofline']['kernel_ms'])"; done
done
