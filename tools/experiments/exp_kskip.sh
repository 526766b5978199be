python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_padded.py -x -q 2>&1 | tail -1
for v in 0 1; do
  echo "== no_kskip=$v: $(PCNN_NO_KSKIP=$v timeout 120 python bench.py --no-sweep --no-cpu-baseline --steps 30 | python -c "import json,sys; d=json.load(sys.stdin); print(d['value'], d['roofline']['frac'], [(l['layer'],l['ms']) for l in d['per_layer'] if l['layer'] in ('conv1','conv2')])")"
done
