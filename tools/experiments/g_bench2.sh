# both nets, per-layer, optional env A/B: bash tools/g_bench2.sh "ENV=.. ENV2=.." ...
python __graft_entry__.py > /dev/null 2>&1 || { echo build failed; exit 1; }
pl() { python -c "
import json,sys;d=json.load(open(sys.argv[1]))
print(sys.argv[1], d['value'], 'ms', d['ms_per_step'], 'roof', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])
print('   ' + ' '.join('%s=%s' % (l['layer'], l['ms']) for l in d['per_layer']))" $1; }
mkdir -p gpurun_out/b2
i=0
for envs in "" "$@"; do
  for net in alexnet vgg16; do
    i=$((i+1))
    env $envs timeout 300 python bench.py --net $net --no-sweep --no-cpu-baseline --steps 30 > gpurun_out/b2/$i.json 2> gpurun_out/b2/$i.err
    echo "[$envs] $net"; pl gpurun_out/b2/$i.json || tail -3 gpurun_out/b2/$i.err
  done
done
