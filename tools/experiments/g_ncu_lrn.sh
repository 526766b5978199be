mkdir -p gpurun_out/ncu_lrn
python __graft_entry__.py > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:lrn_band -c 1 -o /tmp/lrn python tools/one_layer.py norm1pool1 256 2 > /dev/null 2>&1
ncu -i /tmp/lrn.ncu-rep --page details > gpurun_out/ncu_lrn/details.txt 2>&1
python tools/ncu_hot.py /tmp/lrn.ncu-rep 30 > gpurun_out/ncu_lrn/hot.txt 2>&1
ncu -i /tmp/lrn.ncu-rep --page raw --csv > gpurun_out/ncu_lrn/raw.csv 2>&1
