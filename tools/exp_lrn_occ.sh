# LRN+pool occupancy A/B (experiments build): 2 CTAs/SM (default) vs 3 (<= 85 registers, 75 KB bands)
cd $GRAFT_REPO_ROOT
for rep in 1 2; do for E in "X=0" "PCNN_LRN_OCC3=1 PCNN_LB_KB=75" "PCNN_LB_KB=75"; do
  env $E PCNN_LIB=build/prof/libpcnn_prof.so timeout 200 python bench.py --no-sweep --no-extra --no-cpu-baseline --steps 20 > /tmp/o.json 2>/dev/null
  python -c "
import json; d=json.load(open('/tmp/o.json'))
pl={l['layer']: l['ms'] for l in d['per_layer']}
print('$E', d['value'], pl['norm1'], pl['norm2'])"
done; done
