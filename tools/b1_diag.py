"""Small-batch diagnosis: graph-replayed chain of trivial kernels (launch floor)
and per-layer CTA lifetimes of the tcgen05 conv at B=1 (prof build)."""
import os, sys, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
x = torch.zeros(16, device="cuda")
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
with torch.cuda.stream(s):
    for _ in range(3):
        x.add_(1)
    torch.cuda.synchronize()
    with torch.cuda.graph(g):
        for _ in range(13):
            x.add_(1)
torch.cuda.synchronize()
for _ in range(10):
    g.replay()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(100):
    g.replay()
e1.record()
torch.cuda.synchronize()
print("13 trivial kernels per graph replay: %.2f us per replay" % (e0.elapsed_time(e1) * 10))
for name in ["conv3+pm", "conv2p+pm", "conv1p", "fc6", "fc7"]:
    r = subprocess.run([sys.executable, "tools/tc_roles.py", name, "1"], capture_output=True, text=True)
    print(name, r.stdout.strip()[-900:], r.stderr.strip()[-300:])
    r = subprocess.run([sys.executable, "tools/one_layer.py", name, "1", "50"], capture_output=True, text=True)
    print(name, r.stdout.strip()[-600:], r.stderr.strip()[-300:])
