# A/B: current build vs build/ab/libpcnn_head.so on single-layer shapes
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for spec in "conv1p+pm 256" "conv2p+pm 256" "conv3+pm 256" "conv4+pm 256" "conv5+pm 256" "vgg1_2+pm 64" "vgg2_2+pm 64" "vgg3_2+pm 64" "vgg4_2+pm 64" "vgg5_2+pm 64"; do
  set -- $spec
  echo "== $1 B=$2 head: $(PCNN_LIB=build/ab/libpcnn_head.so timeout 60 python tools/one_layer.py $1 $2 30 | tail -1)"
  echo "== $1 B=$2 new : $(timeout 60 python tools/one_layer.py $1 $2 30 | tail -1)"
  echo "== $1 B=$2 new msub1: $(PCNN_PM_MSUB=1 timeout 60 python tools/one_layer.py $1 $2 30 | tail -1)"
done
