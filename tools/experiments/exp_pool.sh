python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for net in vgg16 alexnet; do for v in 0 1; do
  echo "== $net old_pool=$v: $( ( [ $v = 1 ] && export PCNN_OLD_POOL=1; timeout 120 python bench.py --net $net --no-sweep --no-cpu-baseline --steps 30 ) | python -c "import json,sys; d=json.load(sys.stdin); print(d['value'], [(l['layer'],l['ms']) for l in d['per_layer'] if l['layer'].startswith('pool')])")"
done; done
