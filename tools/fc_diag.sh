for S in 0 2 4 8 16; do for L in fc6 fc7 fc8; do
  if [ $S = 0 ]; then timeout 120 python tools/fc_diag.py $L 1 256 2>&1 | tail -2; else PCNN_FC_SPLIT=$S timeout 120 python tools/fc_diag.py $L 1 256 2>&1 | tail -2; fi
done; done
