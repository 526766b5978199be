cd $GRAFT_REPO_ROOT
for rep in 1 2; do for W in 0 1 -1; do
PCNN_LIB=build/prof/libpcnn_prof.so PCNN_WW=$W timeout 300 python bench.py --net vgg16 --no-sweep --no-extra --no-cpu-baseline --steps 10 > /tmp/o.json 2>/dev/null
python -c "
import json; d=json.load(open('/tmp/o.json'))
print('WW=$W', d['value'], d['ms_per_step'], [(l['layer'], round(l['ms']*1000,1), l.get('tile')) for l in d['per_layer'] if l['layer'].startswith('conv')])"
done; done
