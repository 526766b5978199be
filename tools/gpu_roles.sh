set -x
python tools/tc_roles.py vgg1_1s 64
python tools/tc_roles.py rank2 256
python tools/tc_roles.py rank2+pm 256
python tools/tc_roles.py conv3 256
python tools/tc_roles.py vgg1_2 64
