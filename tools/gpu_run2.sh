cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_fc.py tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/gputest_b.log 2>&1
echo "pytest rc=$?" >> gpurun_out/gputest_b.log
timeout 600 python bench.py --no-extra --no-cpu-baseline > gpurun_out/bench_b.json 2> gpurun_out/bench_b.err
echo "bench rc=$?"
tail -15 gpurun_out/gputest_b.log
