cd $GRAFT_REPO_ROOT
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:conv_tc -s 6 -c 12 python tools/rank_probe.py 256 64 2>&1 | grep -E "conv_tc|duration|tensor|tile" | head -40
timeout -s KILL 900 python tools/tune_demo.py 256 > gpurun_out/tune_demo_r02_b256.json 2> gpurun_out/tune_demo.err; echo "tune rc=$?"
