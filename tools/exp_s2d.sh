# staging variants A/B (release builds in build/exp): per-pixel vs (pixel, chunk) threads, rows per band
cd $GRAFT_REPO_ROOT
for rep in 1 2; do for T in base n3r3 n3r2 n4r2 n3r4; do
  PCNN_LIB=build/exp/lib_$T.so timeout 200 python bench.py --no-sweep --no-extra --no-cpu-baseline --steps 30 > /tmp/o.json 2>/dev/null
  python -c "
import json; d=json.load(open('/tmp/o.json'))
pl={l['layer']: l['ms'] for l in d['per_layer']}
print('$T', d['value'], d['ms_per_step'], pl['staging+softmax+unstage'], pl['conv1'])"
done; done
