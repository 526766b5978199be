cd $GRAFT_REPO_ROOT
python tools/fc_probe.py bf16 > gpurun_out/fc_probe7.json 2>&1
timeout 900 python -m pytest tests/test_gpu_fc.py tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/gputest_e.log 2>&1
echo "pytest rc=$?" >> gpurun_out/gputest_e.log
FC_BATCHES=1,256 ncu --set full --clock-control none -k regex:fc_tc -s 3 -c 6 -o gpurun_out/fc_prof7 python tools/fc_probe.py bf16 > /dev/null 2>&1
tail -4 gpurun_out/gputest_e.log
