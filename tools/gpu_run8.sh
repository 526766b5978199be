cd $GRAFT_REPO_ROOT
timeout 600 python bench.py > gpurun_out/bench_f.json 2> gpurun_out/bench_f.err
echo "bench rc=$?"
# launch list of exactly the B=256 timed region: 5 warm-up + 20 timed steps, skip the warm-up launches
ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_alexnet_b256.csv python bench.py --minimal --steps 20 --warmup 5 > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_alexnet_b1.csv python bench.py --minimal --steps 20 --warmup 5 --batch 1 > /dev/null 2>&1
echo done
