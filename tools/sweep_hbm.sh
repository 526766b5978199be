# Sweep the band sizes of the two HBM-bound AlexNet kernels (input staging
# stage_s2d4_kernel: PCNN_S2D_ROWS staged rows per band; LRN+pool
# lrn_reg_kernel: PCNN_LB_KB shared-memory budget per band) on the AlexNet
# B=256 bench step, not under a profiler.  Prints one line per setting.
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
for r in 1 3 4 6; do run PCNN_S2D_ROWS=$r; done
for kb in 32 48 64 80 150; do run PCNN_LB_KB=$kb; done
