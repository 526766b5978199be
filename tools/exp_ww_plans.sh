cd $GRAFT_REPO_ROOT
for W in 0 1; do echo "== PCNN_WW=$W"; PCNN_LIB=build/prof/libpcnn_prof.so PCNN_WW=$W timeout 300 python tools/plan_sweep.py 256 conv1 conv2 conv3 conv4 conv5 2>&1 | grep -v Warn; done
