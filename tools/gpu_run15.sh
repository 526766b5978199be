cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_padded.py tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "lrn or fused or pool" 2>&1 | tail -3
python tools/ab_flags.py 256 0 8
python tools/ab_flags.py 1 0 8 | python -c "import json,sys; d=json.load(sys.stdin); print({k:v['ms_per_step'] for k,v in d.items()})"
