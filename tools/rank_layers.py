"""Per-layer ms (live events) of exact vs rank-r two-stage convs:
AlexNet B=256 conv2..conv5 and VGG-16 B=64 conv3_2 / conv4_2 / conv5_2."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402


def layer_ms(n, x, reps=10):
    for _ in range(3):
        n.infer(x)
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(reps):
        n.infer(x)
    n.set_layer_timing(False)
    ms, k = n.read_layer_timing()
    return [round(v / k * 1000, 1) for v in ms]


res = {}
for netname, B, cases in (("alexnet", 256, {3: (32, 64), 6: (64, 128, 192), 7: (48, 96), 8: (32, 64)}),
                          ("vgg16", 64, {7: (64, 128), 11: (128, 256), 15: (128, 256)})):
    net = getattr(synth, netname)()
    w, b = synth.net_params(net)
    x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
    n = pcnn.Net(net, w, b, B, "bf16")
    base = layer_ms(n, x)
    n.close()
    for li, ranks in cases.items():
        row = {"exact": base[li]}
        for r in ranks:
            n = pcnn.Net(net, w, b, B, "bf16")
            n.set_variant(li, "rank", r)
            row["r%d" % r] = layer_ms(n, x)[li]
            n.close()
        res["%s_L%d" % (netname, li)] = row
print(json.dumps(res, indent=1))
