cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_padded.py tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "lrn or fused or pool" 2>&1 | grep -E "^E |Error|passed|failed" | head -20
python tools/ab_flags.py 256 0 8
