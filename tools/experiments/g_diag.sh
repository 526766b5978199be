# Per-layer diagnostics: unfused conv1, role breakdowns and isolated layer timings.
mkdir -p gpurun_out/diag
python __graft_entry__.py > /dev/null 2>&1
pl() { python -c "
import json,sys;d=json.load(open(sys.argv[1]))
print(sys.argv[1], d['value'], 'ms', d['ms_per_step'], 'clocks', d['clocks'])
[print('  ', l['layer'], l['ms'], l.get('tflops', l.get('gbs')), l.get('tile'), l.get('grid')) for l in d['per_layer']]" $1; }
PCNN_NO_FUSE=1 timeout 300 python bench.py --no-sweep --no-cpu-baseline > gpurun_out/diag/alex_nofuse.json 2>&1; pl gpurun_out/diag/alex_nofuse.json
timeout 300 python bench.py --no-sweep --no-cpu-baseline --steps 200 > gpurun_out/diag/alex.json 2>&1; pl gpurun_out/diag/alex.json
for l in conv1s conv2 conv3 conv5 vgg1_1s+pm vgg1_2+pm vgg2_2+pm vgg5_2 vgg3_2+pm; do
  B=256; case $l in vgg*) B=64;; esac
  timeout 120 python tools/one_layer.py $l $B 20
  timeout 120 python tools/tc_roles.py $l $B
done > gpurun_out/diag/layers.txt 2>&1
cat gpurun_out/diag/layers.txt
for l in norm1pool1 norm2pool2 pool5 stage; do timeout 60 python tools/one_layer.py $l 256 20; done 2>&1 | tee gpurun_out/diag/other.txt
