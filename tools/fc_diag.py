"""FC kernel timeline at B=1 / 256 (prof build) + cluster occupancy:
    python tools/fc_diag.py [fc6|fc7] [batch ...]"""
import ctypes, os, sys
os.environ["PCNN_TC_PROFILE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_songhcl17_b200 import build as _b
os.environ["PCNN_LIB"] = _b.build(prof=True)
import torch
import synth
from paper_conf_hpca_songhcl17_b200 import pcnn
from tools.one_layer import make_net

lib = pcnn.library()
lib.pcnn_debug_fc_profile.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_ulonglong)]
out = (ctypes.c_ulonglong * 16)()
name = sys.argv[1] if len(sys.argv) > 1 else "fc6"
for B in [int(b) for b in sys.argv[2:]] or [1, 256]:
    shape, net, li = make_net(name)
    w, b = synth.net_params(net)
    n = pcnn.Net(net, w, b, B, "bf16")
    x = torch.from_numpy(synth.images(0, B, shape, lo=-1, hi=1)).cuda()
    n.infer(x); torch.cuda.synchronize()
    lib.pcnn_debug_fc_profile(1, out)
    n.infer(x)
    lib.pcnn_debug_fc_profile(1, out)
    c = list(out)
    k = max(c[6], 1)
    M = (1 << 64) - 1
    info = n.query_layer(li, B)
    print("%s B=%d splits %d grid %d: per CTA from PDL wait (us): entry->wait %.2f, acc ready %.2f, "
          "partial stored %.2f, peers met %.2f, reduced %.2f, exit %.2f; first wait -> last exit %.2f, "
          "span %.2f" % (name, B, info["splits"], info["grid"], c[0] / k / 1e3, c[1] / k / 1e3,
                         c[2] / k / 1e3, c[3] / k / 1e3, c[4] / k / 1e3, c[5] / k / 1e3,
                         (c[8] - (M - c[9])) / 1e3, (c[8] - (M - c[7])) / 1e3))
    n.close()
