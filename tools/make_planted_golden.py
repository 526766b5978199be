"""Write tests/golden/planted_<net>_fc7.npz: the FP64 oracle's fc7 features of
the planted-class prototypes (SURVEY.md §8(d) planted set).

Calls only oracle/ and synth/ (the seeded generators); the CUDA path is not
involved.  The planted-class tests build fc8 from these features, so the
expensive VGG-16 prototype pass (≈10 min of FP64 CPU work) runs once here
instead of in every GPU test session.

    python tools/make_planted_golden.py vgg16 [n_classes]
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from oracle import oracle  # noqa: E402


def main():
    name = sys.argv[1]
    n_classes = int(sys.argv[2]) if len(sys.argv) > 2 else 100
    net = synth.get_net(name)
    w, b = synth.net_params(net)
    protos = synth.prototypes(n_classes, net["in_shape"])
    _, outs = oracle.run_net(net, w, b, protos, return_all=True)
    feats = np.asarray(outs[-2], dtype=np.float64)        # fc7 output [n, 4096]
    path = os.path.join(ROOT, "tests", "golden", "planted_%s_fc7.npz" % name)
    np.savez_compressed(path, feats=feats, n_classes=n_classes, seed_w=synth.WEIGHT_SEED,
                        seed_x=synth.IMAGE_SEED)
    print(path, feats.shape)


if __name__ == "__main__":
    main()
