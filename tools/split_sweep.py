"""Small-batch split-K sweep of the padded-mode conv layers (experiments
build, PCNN_FORCE_SPLIT): one layer between identity pools, CUDA-event time of
the conv (+ its reduction launch) per split count.
    python tools/split_sweep.py [batch]"""
import os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_hpca_songhcl17_b200 import build as _b
lib = _b.build(prof=True)
B = sys.argv[1] if len(sys.argv) > 1 else "1"
for L in ["conv2p+pm", "conv3+pm", "conv4+pm", "conv5+pm"]:
    for S in ["0", "1", "2", "3", "4", "6", "12"]:
        env = dict(os.environ, PCNN_LIB=lib)
        if S != "0":
            env["PCNN_FORCE_SPLIT"] = S
        r = subprocess.run([sys.executable, "tools/one_layer.py", L, B, "50"], env=env,
                           capture_output=True, text=True)
        lines = [l for l in r.stdout.splitlines() if "per layer" in l or "tile" in l]
        print(L, "split", S or "plan", " | ".join(l.strip() for l in lines)[-260:], r.stderr[-200:])
