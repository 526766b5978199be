cd $GRAFT_REPO_ROOT
python tools/dbg_round.py 2>&1 | tail -12
timeout 900 python -m pytest tests/test_gpu_padded.py tests/test_gpu_perforation.py tests/test_gpu_rounding.py tests/test_gpu_budget_rank.py tests/test_gpu_fc.py -q -p no:cacheprovider 2>&1 | tail -12
