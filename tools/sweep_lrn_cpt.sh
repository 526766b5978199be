# lrn_reg_kernel chunks per lane: default (6 for norm1's 96 channels, 8 for norm2) vs 3
# (PCNN_LRN_CPT=3: 80 registers, no stack), with band budgets that let 3 CTAs share an SM.
mkdir -p gpurun_out/sweep
run() {
  env "$@" timeout 120 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-sweep \
    > gpurun_out/sweep/out.json 2> gpurun_out/sweep/err.log
  python - "$*" <<'PY'
import json, sys
d = json.load(open("gpurun_out/sweep/out.json"))
pl = {l["layer"]: l["ms"] for l in d["per_layer"]}
print(sys.argv[1], d["value"], "norm1", pl.get("norm1"), "norm2", pl.get("norm2"))
PY
}
run X=0
run PCNN_LRN_CPT=3
run PCNN_LRN_CPT=3 PCNN_LB_KB=75
run PCNN_LRN_CPT=3 PCNN_LB_KB=60
