# VGG-16 B=64: conv1_1 (1x1 GEMM over the staged 27(->32)-channel im2col, N = 64) under
# planner overrides; prints conv1_1 / conv1_2 ms and img/s of the whole step.
mkdir -p gpurun_out/sweep
run() {
  env "$@" timeout 150 python bench.py --net vgg16 --steps 20 --warmup 4 --no-cpu-baseline --no-sweep \
    > gpurun_out/sweep/v.json 2> gpurun_out/sweep/v.err
  python - "$*" <<'PY'
import json, sys
d = json.load(open("gpurun_out/sweep/v.json"))
pl = {l["layer"]: l for l in d["per_layer"]}
c = pl["conv1_1"]
print(sys.argv[1], d["value"], "conv1_1", c["ms"], c["tile"], "conv1_2", pl["conv1_2"]["ms"], "stage+", pl["staging+softmax+unstage"]["ms"])
PY
}
run X=0
run PCNN_NO_TMA_STORE=1
run PCNN_FORCE_CG=1
run PCNN_FORCE_CG=2
run PCNN_PM_MSUB=1
