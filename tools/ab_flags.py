"""A/B of pcnn_net_desc.flags on the AlexNet step: graph-replay ms per step and
per-layer ms (live events) for each flag value given on the command line.

    python tools/ab_flags.py [batch] [flags ...]      e.g.  256 0 8
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 256
flag_list = [int(f) for f in sys.argv[2:]] or [0]
net = synth.alexnet()
w, b = synth.net_params(net)
x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
res = {}
for fl in flag_list:
    n = pcnn.Net(net, w, b, B, "bf16", flags=fl)
    out = torch.empty((B, 1000), device="cuda")
    for _ in range(5):
        n.infer(x, out)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(30):
        n.infer(x, out)
    e1.record()
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(10):
        n.infer(x, out)
    n.set_layer_timing(False)
    ms, k = n.read_layer_timing()
    res[fl] = {"ms_per_step": round(e0.elapsed_time(e1) / 30, 4),
               "launches": n.last_launch_count(),
               "layers": {L.get("name"): round(ms[i] / k, 4) for i, L in enumerate(net["layers"])}}
    n.close()
print(json.dumps(res, indent=1))
