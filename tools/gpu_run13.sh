cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "lrn or alexnet or fused" 2>&1 | tail -3
ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_b256_h.csv python bench.py --minimal --steps 20 --warmup 5 > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_b256_h.csv b256 2>/dev/null | head -14
