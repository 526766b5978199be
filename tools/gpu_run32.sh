timeout -s KILL 120 python tools/tc_roles.py vgg1_1s 64
timeout -s KILL 120 python tools/tc_roles.py rank2 256
timeout -s KILL 120 python tools/tc_roles.py conv1p 256
timeout -s KILL 300 python tools/rank_plans.py
timeout -s KILL 300 python tools/ab_flags.py 256 0 2>&1 | tail -20
