"""Per-role barrier-wait breakdown of the tcgen05 kernel for one layer shape.
    python tools/tc_roles.py conv3 [batch]      (sets PCNN_TC_PROFILE=1)
Counters are summed over CTAs; divided by CTAs they give the average cycles
per CTA each role spent blocked."""
import ctypes, os, sys
os.environ["PCNN_TC_PROFILE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_songhcl17_b200 import build as _b   # counters need the -DPCNN_TC_PROF=1 build
os.environ["PCNN_LIB"] = _b.build(prof=True)
import torch
import synth
from paper_conf_hpca_songhcl17_b200 import pcnn
from tools.one_layer import make_net

name = sys.argv[1]
B = int(sys.argv[2]) if len(sys.argv) > 2 else 256
shape, net, li = make_net(name)
w, b = synth.net_params(net)
n = pcnn.Net(net, w, b, B, "bf16")
x = torch.from_numpy(synth.images(0, B, shape, lo=-1, hi=1)).cuda()
lib = pcnn.library()
lib.pcnn_debug_tc_profile.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_ulonglong)]
out = (ctypes.c_ulonglong * 32)()
n.infer(x); torch.cuda.synchronize()
lib.pcnn_debug_tc_profile(1, out)
for _ in range(1):
    n.infer(x)
lib.pcnn_debug_tc_profile(1, out)
c = list(out)
ctas = max(c[7], 1)
life = c[4] / ctas
print("%s B=%d plan %s" % (name, B, {k: v for k, v in n.query_layer(li, B).items() if k in ("tile_m", "tile_n", "grid", "splits", "tiles")}))
print("  per CTA: lifetime %.0f cyc, K-blocks %.1f (%.0f cyc/kb)" % (life, c[5] / ctas, life / max(c[5] / ctas, 1)))
for i, lab in [(0, "producer wait EMPTY"), (1, "MMA wait FULL"), (2, "MMA wait TEMPTY"), (3, "epi wait TFULL"), (6, "epi busy")]:
    print("  %-22s %5.1f%%" % (lab, 100.0 * c[i] / ctas / life))
if c[11]:
    print("  epilogue TMA-store chunks (warp 2): %.1f per CTA; per chunk: compute %.0f cyc, "
          "box wait %.0f, st.shared %.0f, fence %.0f, issue %.0f cyc" % (c[11] / ctas, c[8] / c[11], c[9] / c[11], c[10] / c[11], c[12] / c[11], c[13] / c[11]))

if c[20]:
    M = (1 << 64) - 1
    k = c[20]
    span = (c[22] - (M - c[21])) / 1e3
    print("  timeline (us, per CTA from its PDL wait): setup+wait %.2f, first accumulator %.2f, "
          "epilogue done %.2f, exit %.2f; launch span %.2f us, wait release spread %.2f us, "
          "first wait -> last exit %.2f us (one launch)" % (
              c[16] / k / 1e3, c[17] / k / 1e3, c[18] / k / 1e3, c[19] / k / 1e3, span,
              (c[24] - (M - c[23])) / 1e3, (c[22] - (M - c[23])) / 1e3))
