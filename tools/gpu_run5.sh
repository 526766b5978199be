cd $GRAFT_REPO_ROOT
python tools/fc_probe.py bf16 > gpurun_out/fc_probe5.json 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x -k "not (planted and vgg16)" -p no:cacheprovider > gputest_d.log 2>&1
echo "pytest rc=$?" >> gputest_d.log; cp gputest_d.log gpurun_out/
timeout 600 python bench.py --no-extra --no-cpu-baseline > gpurun_out/bench_d.json 2> gpurun_out/bench_d.err
echo "bench rc=$?"
tail -15 gpurun_out/gputest_d.log
