python __graft_entry__.py > gpurun_out/build.log 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "lrn" 2>&1 | tail -2
for L in norm1pool1 norm2pool2; do
  for KB in 100 72 56 40; do
    echo "== $L KB=$KB"; PCNN_LB_KB=$KB timeout 60 python tools/one_layer.py $L 256 20
    echo "== $L KB=$KB cpt3"; PCNN_LRN_CPT=3 PCNN_LB_KB=$KB timeout 60 python tools/one_layer.py $L 256 20
  done
done
