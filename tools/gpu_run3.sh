cd $GRAFT_REPO_ROOT
python tools/fc_probe.py bf16 > gpurun_out/fc_probe.json 2>&1
timeout 900 python -m pytest tests/test_gpu_fc.py -q -x -p no:cacheprovider > gpurun_out/gputest_c.log 2>&1
echo "pytest rc=$?" >> gpurun_out/gputest_c.log
ncu --set full --clock-control none -k regex:fc_tc -s 6 -c 3 -o gpurun_out/fc_prof python tools/fc_probe.py bf16 > /dev/null 2>&1
tail -5 gpurun_out/gputest_c.log
cat gpurun_out/fc_probe.json
