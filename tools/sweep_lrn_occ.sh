# lrn_reg_kernel occupancy experiment on the AlexNet B=256 bench step:
# default (<= 128 regs -> 2 CTAs / SM) vs PCNN_LRN_OCC3=1 (__launch_bounds__(256, 3):
# 80 regs, 3 CTAs / SM when the band fits 1/3 of shared memory), with band budgets.
mkdir -p gpurun_out/sweep
run() {
  env "$@" timeout 120 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-sweep \
    > gpurun_out/sweep/out.json 2> gpurun_out/sweep/err.log
  python - "$*" <<'EOF'
import json, sys
d = json.load(open("gpurun_out/sweep/out.json"))
pl = {l["layer"]: l["ms"] for l in d["per_layer"]}
print(sys.argv[1], d["value"], "norm1", pl.get("norm1"), "norm2", pl.get("norm2"),
      "stage+", pl.get("staging+softmax+unstage"))
EOF
}
run X=0
run PCNN_LRN_OCC3=1
run PCNN_LRN_OCC3=1 PCNN_LB_KB=75
run PCNN_LRN_OCC3=1 PCNN_LB_KB=60
run X=0
