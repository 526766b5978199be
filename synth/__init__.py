"""Seeded synthetic workloads shared by the oracle side and the CUDA side.

This package holds NO arithmetic of the method (no convolution, pooling, LRN,
FC or softmax, and no output-size formulas).  It only defines

* the layer lists of the paper's networks (AlexNet [1] and VGG-16 [4], the nets
  of PAPER.md P:53 / P:122, Caffe ``bvlc_alexnet`` reading per SURVEY.md D2/D3),
  as plain dictionaries with every weight shape written out, and
* a counter-based random number generator (splitmix64 of (seed, tensor id,
  element index)) plus the value distributions of the DESIGN.md input recipe.

Both ``oracle/`` and ``paper_conf_hpca_songhcl17_b200/`` consume these plain
arrays; neither imports the other.
"""
from .rng import (counter_u64, uniform, normal, round_to_bf16, images, pixels,
                  he_weights, biases, net_params, IMAGE_TENSOR_ID,
                  WEIGHT_SEED, IMAGE_SEED, prototypes, planted_images)
from .nets import NETS, alexnet, vgg16, cifar_quick, weight_shapes, get_net

__all__ = [
    "counter_u64", "uniform", "normal", "round_to_bf16", "images", "pixels", "he_weights",
    "biases", "net_params", "IMAGE_TENSOR_ID", "WEIGHT_SEED", "IMAGE_SEED",
    "NETS", "alexnet", "vgg16", "cifar_quick", "weight_shapes", "get_net",
    "prototypes", "planted_images",
]
