timeout -s KILL 120 python tools/tc_roles.py vgg1_1s 64
timeout -s KILL 120 python tools/tc_roles.py rank2 256
timeout -s KILL 120 python tools/tc_roles.py conv1p 256
timeout -s KILL 120 python tools/tc_roles.py vgg1_2 64
