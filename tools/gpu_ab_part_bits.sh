# A/B: exact digit-width ballots vs the ten-ballot sentinel scheme in the scatter
cd $GRAFT_REPO_ROOT
F=paper_conf_ipps_klenkfed17_b200/csrc/mm_internal.cuh
for v in 1 0 1 0; do
  sed -i "s/^#define MM_PART_ALWAYS_SENTINEL [0-9]/#define MM_PART_ALWAYS_SENTINEL $v/" $F
  python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True)" > /dev/null 2>&1
  timeout 600 python bench.py --levels ordered,unordered --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('sentinel $v', ' '.join('%s %.3f %.4f' % (k, v['value']/1e9, v['roofline']['kernel_ms']) for k, v in d['levels'].items()))"
done
sed -i "s/^#define MM_PART_ALWAYS_SENTINEL [0-9]/#define MM_PART_ALWAYS_SENTINEL 0/" $F
python -c "from paper_conf_ipps_klenkfed17_b200 import _build; _build.build_library(force=True)" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "ordered or unordered or route or fuzz" 2>&1 | tail -1
