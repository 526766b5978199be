cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python bench.py > gpurun_out/bench_r02a.json 2> gpurun_out/bench_r02a.err; echo "bench rc=$?"
timeout -s KILL 600 python -m pytest tests/test_gpu_planted.py -q -p no:cacheprovider 2>&1 | grep -E "^E |passed|failed" | head
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_alexnet_b256_r02.csv python bench.py --minimal --steps 20 --warmup 5 > /dev/null 2>&1
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_alexnet_b1_r02.csv python bench.py --minimal --steps 20 --warmup 5 --batch 1 > /dev/null 2>&1
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 90 -c 200 --csv --log-file gpurun_out/launches_vgg16_b64_r02.csv python bench.py --minimal --steps 5 --warmup 3 --net vgg16 > /dev/null 2>&1
timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:"conv_tc|fc_tc" -s 10 -c 8 -o gpurun_out/full_alexnet_b256_r02 python bench.py --minimal --steps 1 --warmup 3 > /dev/null 2>&1
echo done
