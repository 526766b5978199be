python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "lrn" 2>&1 | tail -1
PCNN_LRN_CPT=3 timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "lrn" 2>&1 | tail -1
for L in norm1pool1 norm2pool2; do
  for cfg in "0 100" "3 100" "3 72" "3 64"; do set -- $cfg
    echo "== $L cpt=$1 kb=$2: $(PCNN_LRN_CPT=$1 PCNN_LB_KB=$2 timeout 60 python tools/one_layer.py $L 256 30 | tail -1)"
  done
done
