cd $GRAFT_REPO_ROOT
ncu --set full --clock-control none --import-source on -k regex:"lrn_reg|stage_s2d4" -s 6 -c 3 -o gpurun_out/lrn_prof python bench.py --minimal --steps 3 --warmup 3 > /dev/null 2>&1
echo done
