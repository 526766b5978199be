# whole-window padded mode: tests, then release-build bench per-layer plans (AlexNet, VGG-16)
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_padded.py tests/test_gpu_parity.py -q -x -p no:cacheprovider 2>&1 | tail -2
for NET in alexnet vgg16; do for rep in 1 2; do
timeout 300 python bench.py --net $NET --no-sweep --no-extra --no-cpu-baseline --steps 20 > /tmp/o.json 2>/dev/null
python -c "
import json; d=json.load(open('/tmp/o.json'))
print('$NET', d['value'], d['ms_per_step'], d['roofline']['frac'], [(l['layer'], round(l['ms']*1000,1), l.get('tile')) for l in d['per_layer'] if l['layer'].startswith('conv')])"
done; done
