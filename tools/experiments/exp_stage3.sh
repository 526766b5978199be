python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "staging or space_to_depth or alexnet or cifar" 2>&1 | tail -1
for R in 2 4 6 8; do
  echo "== s2d rows=$R: $(PCNN_S2D_ROWS=$R timeout 120 python bench.py --no-sweep --no-cpu-baseline --steps 20 | python -c "import json,sys; d=json.load(sys.stdin); print(d['value'], [l['ms'] for l in d['per_layer'] if l['layer'].startswith('stag')])")"
done
mkdir -p gpurun_out/ncu; timeout 300 ncu --set full --clock-control none --import-source on -k regex:stage -c 1 -o gpurun_out/ncu/stage_s2d python tools/one_layer.py conv1 256 2 > /dev/null 2>&1
