python __graft_entry__.py > /dev/null 2>&1
for v in "" PCNN_STAGE_ROWS=1 PCNN_STAGE_ROWS=2 PCNN_STAGE_ROWS=4 PCNN_OLD_STAGE=1; do for net in alexnet vgg16; do
env $v timeout 300 python bench.py --net $net --no-sweep --no-cpu-baseline --steps 30 > /tmp/x.json 2>/dev/null; python -c "
import json;d=json.load(open('/tmp/x.json'));print('[$v] $net', d['value'], [l['ms'] for l in d['per_layer'] if l['layer'].startswith('staging')])"
done; done
