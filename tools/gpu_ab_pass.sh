# A/B of the partition pass shape (threads x items x min blocks) via variant builds
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in ${CFGS:-"512 8 2"}; do
  set -- ${cfg//_/ }
  export MM_AB_DEFINES="MM_PASS_THREADS=$1 MM_PASS_ITEMS=$2 MM_PASS_MINB=$3"
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(variant='ab')" > /dev/null 2>&1 || { echo "build fail $cfg"; continue; }
  grep -A2 "k_part_pass" paper_conf_ipps_klenkfed17_b200/lib/ptxas_ab.log | grep -i "spill" | head -1
  for i in 1 2; do MM_LIB=$PWD/paper_conf_ipps_klenkfed17_b200/lib/libmm_ab.so timeout 600 python bench.py --levels ordered,unordered --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('thr/items/minb $cfg', ' '.join('%s %.3f %.4f' % (k, v['value']/1e9, v['roofline']['kernel_ms']) for k, v in d['levels'].items()))"; done
done
