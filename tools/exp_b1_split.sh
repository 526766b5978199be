cd $GRAFT_REPO_ROOT
for rep in 1 2; do for S in 0 1; do
  if [ $S = 0 ]; then E=""; else E="PCNN_FORCE_SPLIT=1"; fi
  env $E PCNN_LIB=build/prof/libpcnn_prof.so timeout 200 python bench.py --batch 1 --no-sweep --no-extra --no-cpu-baseline --steps 200 > /tmp/o.json 2>/dev/null
  python -c "
import json; d=json.load(open('/tmp/o.json'))
print('split=$S', d['value'], d['ms_per_step'], d['gpu_launches'])"
done; done
