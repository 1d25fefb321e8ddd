# flat-level tests + two bench lines
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for i in 1 2; do timeout 600 python bench.py --levels ordered,unordered --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print(' '.join('%s %.3f %.4f %.4f' % (k, v['value']/1e9, v['ms_per_step'], v['roofline']['kernel_ms']) for k, v in d['levels'].items()))"; done
timeout 300 python tools/kernel_split.py ordered 3 2>&1 | grep -v -i warn | grep -i "k_tm\|hist\|scatter" | head -8
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "ordered or unordered or route or fuzz" 2>&1 | tail -1
