# usage: bash tools/g_layers.sh OUTDIR layer[:B] ...   -- isolated layer timings + role breakdowns
out=$1; shift
mkdir -p gpurun_out/$out
python __graft_entry__.py > /dev/null 2>&1 || { echo build failed; exit 1; }
for lb in "$@"; do
  l=${lb%%:*}; B=${lb#*:}; [ "$B" = "$lb" ] && B=256
  timeout 120 python tools/one_layer.py $l $B 20
  timeout 120 python tools/tc_roles.py $l $B | tail -6
done 2>&1 | tee gpurun_out/$out/layers.txt
