python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "staging or space_to_depth or alexnet or vgg or cifar" 2>&1 | tail -1
for R in 0 2 3 4 6; do
 for net in alexnet vgg16; do
  echo "== $net rows=$R: $(PCNN_STAGE_ROWS=$R timeout 120 python bench.py --net $net --no-sweep --no-cpu-baseline --steps 20 | python -c "import json,sys; d=json.load(sys.stdin); print(d['value'], [l['ms'] for l in d['per_layer'] if l['layer'].startswith('stag')])")"
 done
done
