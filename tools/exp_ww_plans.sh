cd $GRAFT_REPO_ROOT
for W in 0 1; do echo "== PCNN_WW=$W"; PCNN_LIB=build/prof/libpcnn_prof.so PCNN_WW=$W timeout 300 python tools/plan_sweep.py 256 conv2 2>&1 | grep -v Warn; done
timeout 300 python bench.py --no-sweep --no-extra --no-cpu-baseline --steps 20 > /tmp/o.json 2>/dev/null
python -c "
import json; d=json.load(open('/tmp/o.json'))
print('release', d['value'], d['ms_per_step'], d['roofline']['frac'], [(l['layer'], round(l['ms']*1000,1), l.get('tile')) for l in d['per_layer'] if l['layer'].startswith('conv')])"
