# A/B of the on-chip MPI kernel (configs[1]) via MM_AB_DEFINES builds
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in "$@"; do
  export MM_AB_DEFINES="$cfg"
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='ab')" > /dev/null 2>&1 || { echo "build fail $cfg"; continue; }
  for i in 1 2; do MM_LIB=$PWD/paper_conf_ipps_klenkfed17_b200/lib/libmm_ab.so timeout 600 python bench.py --levels mpi --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('$cfg', ' '.join('%s %.3f %.4f' % (k, v['value']/1e9, v['roofline']['kernel_ms']) for k, v in d['levels'].items()))"; done
done
