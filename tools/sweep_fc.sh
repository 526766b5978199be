# Split-K / CTA-pair sweep of the AlexNet FC GEMMs at B=256 in isolation
# (tools/one_layer.py: layer events only), against the planner's own choice.
for L in fc6 fc7; do
  echo "== $L planner"; timeout 60 python tools/one_layer.py $L 256 30
  for cg in 1 2; do
    sps="1 2 3 4 6 8 9 12 16"; [ $L = fc7 ] && sps="1 2 4 8 16"   # splits that divide the K-blocks
    for sp in $sps; do
      printf "cg=%s split=%s: " $cg $sp
      PCNN_FORCE_CG=$cg PCNN_FORCE_SPLIT=$sp timeout 60 python tools/one_layer.py $L 256 30 2>&1 | tail -1
    done
  done
done
