# A/B of nvcc / ptxas flags on configs[1] (MM_AB_FLAGS builds), twice each
# usage: bash tools/gpu_ab_flags.sh "<flags A>" "<flags B>" ...
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in "$@"; do
  export MM_AB_FLAGS="$cfg"
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='ab')" > /dev/null 2>&1 || { echo "build fail $cfg"; continue; }
  grep -A3 "Function properties for _ZN2mm10k_mpi_fifoILi256ELb1ELi1E" paper_conf_ipps_klenkfed17_b200/lib/ptxas_ab.log | grep Used
  for i in 1 2; do MM_LIB=$PWD/paper_conf_ipps_klenkfed17_b200/lib/libmm_ab.so timeout 600 python bench.py --levels mpi,ordered,unordered --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('[$cfg]', ' '.join('%s %.3f' % (k, v['value']/1e9) for k, v in d['levels'].items()))"; done
done
