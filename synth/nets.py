"""Layer lists of the networks the paper evaluates (plain data, no arithmetic).

* AlexNet: PAPER.md P:53 (§II.A, Fig. 1) names "five convolutional layers, three
  max-pooling layers" plus classifiers; the models are Caffe-trained and
  Table IV's per-group GEMM shapes (CONV2 128x729, CONV5 128x169)
  fix Caffe's grouped ``bvlc_alexnet`` (groups 1,2,1,2,2).  ReLU / LRN follow
  that Caffe model (readings R2-R3).
* VGG-16: the VGGNet of P:14 / Table III (configuration D of [4]).
* CIFAR-quick-shaped single conv layer: BASELINE.json configs[0].

A layer is a dict.  Keys:
  kind   : "conv" | "lrn" | "maxpool" | "avgpool" | "fc"
  conv   : out, k, stride, pad, groups, relu, in_c (input channels)
  fc     : out, in_f (flattened input features, C*H*W of the input), relu
  lrn    : size, alpha, beta, k
  pool   : k, stride
Every weight shape is written out (``in_c`` / ``in_f``) so that no shape
arithmetic lives in this shared module.
"""


def _conv(out, k, in_c, stride=1, pad=0, groups=1, relu=True, name=None):
    return dict(kind="conv", out=out, k=k, stride=stride, pad=pad,
                groups=groups, relu=relu, in_c=in_c, name=name)


def _fc(out, in_f, relu=True, name=None):
    return dict(kind="fc", out=out, in_f=in_f, relu=relu, name=name)


def _lrn(name=None):
    # Caffe bvlc_alexnet norm1/norm2: local_size 5, alpha 1e-4, beta 0.75, k 1
    return dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0, name=name)


def _maxpool(k, stride, name=None):
    return dict(kind="maxpool", k=k, stride=stride, name=name)


def alexnet():
    """Caffe bvlc_alexnet: 227x227x3 input, 1000 classes."""
    layers = [
        _conv(96, 11, 3, stride=4, name="conv1"),
        _lrn("norm1"),
        _maxpool(3, 2, "pool1"),
        _conv(256, 5, 96, pad=2, groups=2, name="conv2"),
        _lrn("norm2"),
        _maxpool(3, 2, "pool2"),
        _conv(384, 3, 256, pad=1, name="conv3"),
        _conv(384, 3, 384, pad=1, groups=2, name="conv4"),
        _conv(256, 3, 384, pad=1, groups=2, name="conv5"),
        _maxpool(3, 2, "pool5"),
        _fc(4096, 256 * 6 * 6, name="fc6"),
        _fc(4096, 4096, name="fc7"),
        _fc(1000, 4096, relu=False, name="fc8"),
    ]
    return dict(name="alexnet", in_shape=(3, 227, 227), layers=layers)


def vgg16():
    """VGG-16 (configuration D): 224x224x3 input, 1000 classes."""
    layers = []
    c_in = 3
    for stage, (width, reps) in enumerate([(64, 2), (128, 2), (256, 3),
                                           (512, 3), (512, 3)], start=1):
        for i in range(1, reps + 1):
            layers.append(_conv(width, 3, c_in, pad=1,
                                name=f"conv{stage}_{i}"))
            c_in = width
        layers.append(_maxpool(2, 2, f"pool{stage}"))
    layers += [
        _fc(4096, 512 * 7 * 7, name="fc6"),
        _fc(4096, 4096, name="fc7"),
        _fc(1000, 4096, relu=False, name="fc8"),
    ]
    return dict(name="vgg16", in_shape=(3, 224, 224), layers=layers)


def cifar_quick():
    """BASELINE.json configs[0]: 3x32x32, 16 filters 5x5 pad 2 + ReLU + 2x2 maxpool."""
    layers = [
        _conv(16, 5, 3, pad=2, name="conv1"),
        _maxpool(2, 2, "pool1"),
    ]
    return dict(name="cifar_quick", in_shape=(3, 32, 32), layers=layers)


NETS = {"alexnet": alexnet, "vgg16": vgg16, "cifar_quick": cifar_quick}


def get_net(name):
    return NETS[name]()


def weight_shapes(net):
    """(weight shape, bias shape) per layer; None for weightless layers.

    conv: OIHW = (out, in_c/groups, k, k); fc: (out, in_f).  Read straight
    from the layer dicts (no arithmetic beyond the group split).
    """
    out = []
    for L in net["layers"]:
        if L["kind"] == "conv":
            out.append(((L["out"], L["in_c"] // L["groups"], L["k"], L["k"]),
                        (L["out"],)))
        elif L["kind"] == "fc":
            out.append(((L["out"], L["in_f"]), (L["out"],)))
        else:
            out.append(None)
    return out
