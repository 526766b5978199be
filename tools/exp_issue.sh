# conv2 (padded mode, B=256): time with TMA loads / MMAs skipped (experiments build,
# PCNN_TC_SKIP bit 1 = A loads, 2 = B loads, 4 = MMAs) -- the issue-loop floor
cd $GRAFT_REPO_ROOT
for S in 0 4 3 7; do
  PCNN_LIB=build/prof/libpcnn_prof.so PCNN_TC_SKIP=$S timeout 120 python tools/one_layer.py conv2p+pm 256 20 2>&1 | tail -2 | sed "s/^/skip=$S /"
  PCNN_LIB=build/prof/libpcnn_prof.so PCNN_TC_SKIP=$S timeout 120 python tools/one_layer.py conv3+pm 256 20 2>&1 | tail -2 | sed "s/^/skip=$S /"
done
