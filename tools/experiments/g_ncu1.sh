mkdir -p gpurun_out/ncu1
python __graft_entry__.py > /dev/null 2>&1
for l in vgg1_2+pm vgg1_1s+pm; do
  n=$(echo $l | tr '+' '_')
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:conv_tc -c 1 -o /tmp/$n python tools/one_layer.py $l 64 2 > /dev/null 2>&1
  python tools/ncu_hot.py /tmp/$n.ncu-rep 40 > gpurun_out/ncu1/hot_$n.txt 2>&1
  python tools/ncu_summary.py /tmp/$n.ncu-rep > gpurun_out/ncu1/sum_$n.csv 2>&1
  ncu -i /tmp/$n.ncu-rep --page details > gpurun_out/ncu1/details_$n.txt 2>&1
  ncu -i /tmp/$n.ncu-rep --page source --csv > gpurun_out/ncu1/src_$n.csv 2>&1
done
