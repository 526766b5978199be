"""Per-launch view of AlexNet with conv2 at rank r (two-stage variant): run a
few passes so an ncu launch list can time stage 1 and stage 2 separately, and
print the plans of both stages."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 256
r = int(sys.argv[2]) if len(sys.argv) > 2 else 64
net = synth.alexnet()
w, b = synth.net_params(net)
n = pcnn.Net(net, w, b, B, "bf16")
n.set_variant(3, "rank", r)
x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
for _ in range(6):
    n.infer(x)
torch.cuda.synchronize()
print(n.query_layer(3, B))
