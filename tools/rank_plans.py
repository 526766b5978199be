"""A/B of tile plans (pcnn_set_layer_plan) for AlexNet conv2's rank-r variant
and for VGG-16 conv1_1, per-layer ms from live events."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402


def layer_ms(n, x, layer, reps=10):
    for _ in range(3):
        n.infer(x)
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(reps):
        n.infer(x)
    n.set_layer_timing(False)
    ms, k = n.read_layer_timing()
    return round(ms[layer] / k * 1000, 1)


res = {}
net = synth.alexnet()
w, b = synth.net_params(net)
x = torch.from_numpy(synth.images(0, 256, net["in_shape"])).cuda()
for cg, ms in [(0, 0), (1, 1), (1, 2), (2, 1), (2, 2)]:
    n = pcnn.Net(net, w, b, 256, "bf16")
    n.set_variant(3, "rank", 64)
    n.set_layer_plan(3, cg, ms)
    res["alexnet_conv2_r64_cg%d_ms%d" % (cg, ms)] = [layer_ms(n, x, 3), n.query_layer(3, 256)["tile_m"], n.query_layer(3, 256)["tile_n"]]
    n.close()
net = synth.vgg16()
w, b = synth.net_params(net)
x = torch.from_numpy(synth.images(0, 64, net["in_shape"])).cuda()
for cg, ms in [(0, 0), (1, 1), (1, 2), (2, 1), (2, 2)]:
    n = pcnn.Net(net, w, b, 64, "bf16")
    n.set_layer_plan(0, cg, ms)
    res["vgg_conv1_1_cg%d_ms%d" % (cg, ms)] = [layer_ms(n, x, 0), n.query_layer(0, 64)["tile_m"], n.query_layer(0, 64)["tile_n"]]
    n.close()
print(json.dumps(res, indent=1))
