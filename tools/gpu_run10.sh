cd $GRAFT_REPO_ROOT
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/gputest_full.log 2>&1
echo "pytest rc=$?" >> gpurun_out/gputest_full.log
tail -30 gpurun_out/gputest_full.log
