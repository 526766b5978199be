"""End-to-end breakdown (experiments build): pinned H2D bandwidth, and
pcnn_infer_host_u8 at B=256 with 1 / 2 / 4 chunks (PCNN_H2D_CHUNKS)."""
import os, subprocess, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if len(sys.argv) > 1:
    import torch, synth
    from paper_conf_hpca_songhcl17_b200 import pcnn
    net = synth.alexnet(); w, b = synth.net_params(net); B = 256
    n = pcnn.Net(net, w, b, B, "bf16")
    px = torch.from_numpy(synth.pixels(0, B, net["in_shape"])).pin_memory()
    oh = torch.empty((B, 1000)).pin_memory(); ph = torch.empty((B, 1000)).pin_memory(); hh = torch.empty((B,)).pin_memory()
    for _ in range(3): n.infer_host_u8(px, oh, mean=[128.0] * 3, probs=ph, entropy=hh)
    t0 = time.perf_counter()
    for _ in range(20): n.infer_host_u8(px, oh, mean=[128.0] * 3, probs=ph, entropy=hh)
    dt = (time.perf_counter() - t0) / 20
    print("chunks=%s  %.3f ms/step  %.1fk img/s" % (os.environ.get("PCNN_H2D_CHUNKS"), dt * 1e3, B / dt / 1e3))
    sys.exit(0)
import torch
x = torch.empty(40 << 20, dtype=torch.uint8).pin_memory(); d = torch.empty_like(x, device="cuda")
for _ in range(3): d.copy_(x, non_blocking=True)
torch.cuda.synchronize(); t0 = time.perf_counter()
for _ in range(10): d.copy_(x, non_blocking=True)
torch.cuda.synchronize(); print("pinned H2D %.1f GB/s" % (10 * x.numel() / (time.perf_counter() - t0) / 1e9))
from paper_conf_hpca_songhcl17_b200 import build as _b
lib = _b.build(prof=True)
for k in ["1", "2", "4"]:
    r = subprocess.run([sys.executable, __file__, "x"], env=dict(os.environ, PCNN_LIB=lib, PCNN_H2D_CHUNKS=k), capture_output=True, text=True)
    print(r.stdout.strip(), r.stderr[-300:])
