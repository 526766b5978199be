# role isolation: PCNN_TC_SKIP (1 no A loads, 2 no B loads, 4 no MMAs) x PCNN_FORCE_CG
python __graft_entry__.py > /dev/null 2>&1 || { echo build failed; exit 1; }
for lb in "$@"; do
  l=${lb%%:*}; B=${lb#*:}; [ "$B" = "$lb" ] && B=256
  for cg in 1 2; do for sk in 0 3 4 7; do
    echo "== $l B=$B cg=$cg skip=$sk"
    PCNN_FORCE_CG=$cg PCNN_TC_SKIP=$sk timeout 120 python tools/tc_roles.py $l $B | grep -E "plan|per CTA"
  done; done
done
