cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1500 python -m pytest tests -m gpu -q -k "not (planted and vgg16)" -p no:cacheprovider > gpurun_out/gputest_a.log 2>&1
echo "pytest rc=$?" >> gpurun_out/gputest_a.log
timeout 600 python bench.py > gpurun_out/bench_a.json 2> gpurun_out/bench_a.err
echo "bench rc=$?"
tail -5 gpurun_out/gputest_a.log
