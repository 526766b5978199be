"""Per-layer A/B of the conv plan overrides (pcnn_set_layer_plan: CTA group,
M sub-tiles) on the AlexNet step: CUDA-event per-layer ms for each plan.
    python tools/plan_sweep.py [batch] [layer names ...]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_hpca_songhcl17_b200 import pcnn

B = int(sys.argv[1]) if len(sys.argv) > 1 else 256
names = sys.argv[2:] or ["conv2", "conv3", "conv4", "conv5"]
net = synth.alexnet()
w, b = synth.net_params(net)
x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
idx = {L.get("name"): i for i, L in enumerate(net["layers"])}
n = pcnn.Net(net, w, b, B, "bf16")
out = torch.empty((B, 1000), device="cuda")


def run(li):
    n.set_layer_timing(True)
    for _ in range(3):
        n.infer(x, out)
    n.read_layer_timing()
    for _ in range(10):
        n.infer(x, out)
    ms, k = n.read_layer_timing()
    n.set_layer_timing(False)
    q = n.query_layer(li, B)
    return ms[li] / k, q


for name in names:
    li = idx[name]
    for cg, ms_ in [(0, 0), (2, 1), (2, 2), (1, 1), (1, 2)]:  # (0, 0): the planner's choice
        try:
            n.set_layer_plan(li, cg, ms_)
        except Exception as e:
            print(name, cg, ms_, "unsupported", e)
            continue
        t, q = run(li)
        print("%s plan(cg=%d, msub=%d): %.1f us  tile %dx%d grid %d util %.3f" % (
            name, cg, ms_, t * 1e3, q["tile_m"], q["tile_n"], q["grid"], q.get("util", 0)))
    n.set_layer_plan(li, 0, 0)
