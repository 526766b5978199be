python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
for L in fc6 fc7; do
  echo "== $L auto: $(timeout 60 python tools/one_layer.py $L 256 30 | tail -1)"
  for CG in 1 2; do for BN in 128 256; do for SP in 1 2 3 4 6 8 9 12 16; do
    r=$(PCNN_FORCE_CG=$CG PCNN_FORCE_BN=$BN PCNN_FORCE_SPLIT=$SP timeout 60 python tools/one_layer.py $L 256 30 2>&1 | tail -1)
    echo "$L cg=$CG bn=$BN sp=$SP: $r"
  done; done; done
done
for R in 1 2 3 4 6 8; do echo "== stage rows $R"; PCNN_STAGE_ROWS=$R timeout 120 python bench.py --no-sweep --no-cpu-baseline --steps 20 | python -c "import json,sys; d=json.load(sys.stdin); print(d['value'], [l for l in d['per_layer'] if l['layer'].startswith('stag')])"; done
