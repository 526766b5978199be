# The round-2 profile captures (one B200; run under gpurun, then
# `python tools/summarize_profiles.py r02` here).  Launch lists cover only the
# timed steps of `bench.py --minimal` (warm-up launches skipped with -s).
cd $GRAFT_REPO_ROOT
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_alexnet_b256_r02.csv python bench.py --minimal --steps 20 --warmup 5 > /dev/null 2>&1
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_alexnet_b1_r02.csv python bench.py --minimal --steps 20 --warmup 5 --batch 1 > /dev/null 2>&1
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 90 -c 200 --csv --log-file gpurun_out/launches_vgg16_b64_r02.csv python bench.py --minimal --steps 5 --warmup 3 --net vgg16 > /dev/null 2>&1
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:"conv_tc|fc_tc" -s 10 -c 8 -o gpurun_out/full_alexnet_b256_r02 python bench.py --minimal --steps 1 --warmup 3 > /dev/null 2>&1
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:"lrn_reg|stage_s2d4|pool_direct|softmax" -s 15 -c 5 -o gpurun_out/full_alexnet_b256_other_r02 python bench.py --minimal --steps 1 --warmup 3 > /dev/null 2>&1
