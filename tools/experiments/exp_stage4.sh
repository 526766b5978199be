python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t4.log 2>&1; echo tests=$?; tail -1 gpurun_out/t4.log
for net in vgg16 alexnet; do for v in 0 1; do
  echo "== $net old_stage=$v: $( ( [ $v = 1 ] && export PCNN_OLD_STAGE=1; timeout 120 python bench.py --net $net --no-sweep --no-cpu-baseline --steps 30 ) | python -c "import json,sys; d=json.load(sys.stdin); print(d['value'], [(l['layer'],l['ms']) for l in d['per_layer'] if l['layer'].startswith('stag') or l['layer']=='conv1_1'])")"
done; done
