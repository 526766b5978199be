"""Time the AlexNet FC layers alone (fc6 -> fc7 -> fc8 net) at several batches
through the C ABI, per-layer CUDA events; prints the FC plans."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402

net = dict(name="fc678", in_shape=(256, 6, 6), layers=[
    dict(kind="fc", out=4096, in_f=9216, relu=True, name="fc6"),
    dict(kind="fc", out=4096, in_f=4096, relu=True, name="fc7"),
    dict(kind="fc", out=1000, in_f=4096, relu=False, name="fc8")])
w, b = synth.net_params(net)
prec = sys.argv[1] if len(sys.argv) > 1 else "bf16"
out = {}
BATCHES = [int(v) for v in os.environ.get("FC_BATCHES", "1,16,64,128,256").split(",")]
for B in BATCHES:
    n = pcnn.Net(net, w, b, max_batch=B, precision=prec)
    x = torch.from_numpy(synth.images(0, B, net["in_shape"], lo=0, hi=2)).cuda()
    for _ in range(3):
        n.infer(x)
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(20):
        n.infer(x)
    n.set_layer_timing(False)
    ms, k = n.read_layer_timing()
    infos = [n.query_layer(i, B) for i in range(3)]
    out[B] = {L["name"]: {"us": round(ms[i] / k * 1000, 2),
                          "gbs": round(infos[i]["bytes"] / (ms[i] / k / 1000) / 1e9, 0),
                          "plan": "%dx%d grid %d split %d" % (infos[i]["tile_m"], infos[i]["tile_n"],
                                                              infos[i]["grid"], infos[i]["splits"])}
              for i, L in enumerate(net["layers"])}
    n.close()
print(json.dumps(out, indent=1))
