# wide (64-column) bf16 TMA-store boxes: parity + per-role breakdown + A/B
timeout -s KILL 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
timeout -s KILL 120 python tools/tc_roles.py vgg1_1s 64
timeout -s KILL 120 python tools/tc_roles.py rank2 256
timeout -s KILL 300 python tools/rank_plans.py
timeout -s KILL 300 python bench.py --steps 20 --warmup 5 --minimal 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'])"
timeout -s KILL 300 python bench.py --net vgg16 --steps 10 --warmup 3 --minimal 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d[\"value\"], d[\"ms_per_step\"], d[\"roofline\"][\"frac\"])"
