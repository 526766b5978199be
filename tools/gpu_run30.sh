cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_padded.py tests/test_gpu_budget_rank.py -q -x -p no:cacheprovider 2>&1 | grep -E "^E |passed|failed" | head -5
timeout -s KILL 120 python tools/ab_flags.py 256 0 | python -c "import json,sys; d=json.load(sys.stdin)['0']; print(d['ms_per_step'], d['layers'])"
timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:conv_tc -s 6 -c 6 python tools/rank_probe.py 256 64 2>&1 | grep -E "duration" | head -6
timeout -s KILL 300 python bench.py --net vgg16 --no-sweep --no-extra --no-cpu-baseline --steps 20 | python -c "import json,sys; d=json.load(sys.stdin); print(d['value'], d['ms_per_step'], d['roofline']['frac'], [(l['layer'], l['ms']) for l in d['per_layer'][:6]])"
