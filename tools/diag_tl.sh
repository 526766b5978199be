for L in conv3+pm conv2p+pm conv1p conv4+pm; do for B in 1 256; do timeout 120 python tools/tc_roles.py $L $B 2>&1 | grep -v Traceback | tail -3; done; done
