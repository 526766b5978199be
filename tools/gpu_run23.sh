cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "stag or alexnet or space" 2>&1 | grep -E "^E |passed|failed" | head -5
timeout -s KILL 120 python tools/ab_flags.py 256 0 | python -c "import json,sys; d=json.load(sys.stdin)['0']; print(d['ms_per_step'])"
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:stage -s 5 -c 3 python tools/ab_flags.py 256 0 2>&1 | grep -E "duration" | head -3
