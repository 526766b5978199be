import os, sys
sys.path.insert(0, os.getcwd())
import torch, synth
from paper_conf_hpca_songhcl17_b200 import pcnn
net = synth.alexnet(); w, b = synth.net_params(net)
B = 256
x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
n = pcnn.Net(net, w, b, B, "bf16")
n.set_variant(3, "rank", int(sys.argv[1]))
for _ in range(3): n.infer(x)
torch.cuda.synchronize()
for st in ("r1", "r2"):
    pass
print(n.query_layer(3, B))
