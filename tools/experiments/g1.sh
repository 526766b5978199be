nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/usp tools/umma_shift_probe.cu 2>/dev/null; timeout 60 /tmp/usp
python __graft_entry__.py > /dev/null
timeout 300 python tools/pm_check.py
PCNN_NO_PM=1 timeout 300 python tools/pm_check.py bf16
for l in vgg1_1s vgg1_2; do timeout 120 python tools/tc_roles.py $l 64; timeout 120 python tools/one_layer.py $l 64; done
