cd $GRAFT_REPO_ROOT
FC_BATCHES=256 ncu --set full --clock-control none -k regex:fc_tc -s 3 -c 3 -o gpurun_out/fc_prof256 python tools/fc_probe.py bf16 > /dev/null 2>&1
echo done
