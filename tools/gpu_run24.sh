cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python -m pytest tests/test_gpu_padded.py tests/test_gpu_parity.py tests/test_gpu_budget_rank.py -q -x -p no:cacheprovider 2>&1 | grep -E "^E |passed|failed" | head -5
for b in 1 8 64 256; do timeout -s KILL 120 python tools/ab_flags.py $b 0 | python -c "import json,sys; d=json.load(sys.stdin)['0']; print($b, d['ms_per_step'], d['launches'], d['layers'])"; done
