cd $GRAFT_REPO_ROOT
timeout -s KILL 120 python tools/ab_flags.py 2 0 | python -c "import json,sys; d=json.load(sys.stdin)['0']; print('b2 ok', d['ms_per_step'])"
timeout -s KILL 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "not planted" 2>&1 | grep -E "^E |passed|failed|Error" | head -20
timeout -s KILL 120 python tools/ab_flags.py 256 0 | python -c "import json,sys; d=json.load(sys.stdin)['0']; print(d['ms_per_step'], d['layers'])"
timeout -s KILL 120 python tools/ab_flags.py 64 0 | python -c "import json,sys; d=json.load(sys.stdin)['0']; print(d['ms_per_step'])"
