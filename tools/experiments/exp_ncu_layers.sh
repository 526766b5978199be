python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
mkdir -p gpurun_out/ncu
for spec in "vgg1_1s+pm 64" "fc6 256" "stage 256"; do
  set -- $spec
  K=regex:conv_tc; [ "$1" = "stage" ] && K=regex:stage
  timeout 300 ncu --set full --clock-control none --import-source on -k $K -c 1 -o gpurun_out/ncu/${1%+pm}_$2 python tools/one_layer.py $1 $2 2 > gpurun_out/ncu/${1%+pm}.log 2>&1
done
ls -la gpurun_out/ncu
