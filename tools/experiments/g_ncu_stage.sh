mkdir -p gpurun_out/ncu_stage
python __graft_entry__.py > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:stage_gather3 -c 1 -o /tmp/st python bench.py --steps 1 --warmup 3 --no-sweep --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/st.ncu-rep --page details > gpurun_out/ncu_stage/details.txt 2>&1
python tools/ncu_hot.py /tmp/st.ncu-rep 30 > gpurun_out/ncu_stage/hot.txt 2>&1
