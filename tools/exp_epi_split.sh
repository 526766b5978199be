# conv epilogue A/B (release builds in build/exp): new = this commit, old = HEAD
cd $GRAFT_REPO_ROOT
for rep in 1 2 3; do for T in old new; do
  PCNN_LIB=build/exp/lib_tc_$T.so timeout 200 python bench.py --no-sweep --no-extra --no-cpu-baseline --steps 30 > /tmp/o.json 2>/dev/null
  python -c "
import json; d=json.load(open('/tmp/o.json'))
pl={l['layer']: l['ms'] for l in d['per_layer']}
print('$T', d['value'], d['ms_per_step'], pl['conv1'], pl['conv2'], pl['conv3'], pl['conv4'], pl['conv5'])"
done; done
