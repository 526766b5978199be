python __graft_entry__.py > /dev/null
mkdir -p gpurun_out/g2
timeout 300 python tools/pm_check.py
PCNN_NO_PM=1 timeout 300 python tools/pm_check.py bf16
for sk in 0 3 7; do echo "skip $sk"; PCNN_TC_SKIP=$sk timeout 120 python tools/one_layer.py vgg1_1s 64; done
timeout 300 ncu --set full --import-source on --clock-control none -k regex:conv_tc -c 1 -o /tmp/v11 python tools/one_layer.py vgg1_1s 64 1 > /dev/null 2>&1
python tools/ncu_hot.py /tmp/v11.ncu-rep 45 > gpurun_out/g2/hot_vgg11.txt 2>&1
ncu -i /tmp/v11.ncu-rep --page details --section WarpStateStats --section MemoryWorkloadAnalysis > gpurun_out/g2/details_vgg11.txt 2>&1
