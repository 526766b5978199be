python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "lrn or pool or alexnet" 2>&1 | tail -2
for L in norm1pool1 norm2pool2; do
  echo "== $L head: $(PCNN_LIB=build/ab/libpcnn_head.so timeout 60 python tools/one_layer.py $L 256 30 | tail -1)"
  echo "== $L new : $(timeout 60 python tools/one_layer.py $L 256 30 | tail -1)"
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:lrn_reg -c 1 -o gpurun_out/ncu/lrn_reg2 python tools/one_layer.py norm1pool1 256 2 > /dev/null 2>&1
