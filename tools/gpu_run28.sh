cd $GRAFT_REPO_ROOT
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:conv_tc -s 8 -c 1 -o gpurun_out/stage2_prof python tools/rank_probe.py 256 64 > /dev/null 2>&1
echo done
