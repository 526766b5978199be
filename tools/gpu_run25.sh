cd $GRAFT_REPO_ROOT
export PCNN_LIB=$GRAFT_REPO_ROOT/build/prof/libpcnn_prof.so
for cfg in "" "PCNN_FC_SPLIT=8" "PCNN_FC_SPLIT=4" "PCNN_FC_SPLIT=2"; do
  echo "== $cfg"
  env $cfg FC_BATCHES=1,64,256 timeout -s KILL 120 python tools/fc_probe.py bf16 | python -c "
import json,sys
d=json.load(sys.stdin)
for B,v in d.items(): print(B, ' '.join('%s %s(%s)'%(k,x['us'],x['plan']) for k,x in v.items()))
"
done
