python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "staging or space_to_depth or alexnet or cifar" 2>&1 | tail -2
for v in 0 1; do
  echo "== old_stage=$v: $( ( [ $v = 1 ] && export PCNN_OLD_STAGE=1; timeout 120 python bench.py --no-sweep --no-cpu-baseline --steps 20 ) | python -c "import json,sys; d=json.load(sys.stdin); print(d['value'], [l['ms'] for l in d['per_layer'] if l['layer'].startswith('stag')])")"
done
