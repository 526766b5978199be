"""Counter-based RNG and value distributions.

Every value is a pure function of (seed, tensor_id, element index):
    z   = seed * G1 + tensor_id * G2 + (index + 1) * G3      (mod 2**64)
    u64 = splitmix64_finalize(z)
so any rank or shard can regenerate any image of a batch from its global
index, and the oracle side and the CUDA side see bit-identical inputs.

All generated floats are rounded to BF16-representable FP32 values
(round-to-nearest-even), so the FP32-SIMT, TF32 and BF16 paths all start from
identical operands.
"""
import numpy as np

G1 = np.uint64(0x9E3779B97F4A7C15)
G2 = np.uint64(0xD1B54A32D192ED03)
G3 = np.uint64(0xBF58476D1CE4E5B9)
M1 = np.uint64(0xBF58476D1CE4E5B9)
M2 = np.uint64(0x94D049BB133111EB)

WEIGHT_SEED = 17          # seed 17 for weights
IMAGE_SEED = 18           # seed 18 for images
IMAGE_TENSOR_ID = 1000    # tensor id of the image stream
BIAS_TENSOR_OFFSET = 500  # bias of layer i uses tensor id i + 500


def counter_u64(seed, tensor_id, index):
    """splitmix64 finaliser of the counter; ``index`` is an int64/uint64 array."""
    idx = np.asarray(index, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = (np.uint64(seed) * G1 + np.uint64(tensor_id) * G2
             + (idx + np.uint64(1)) * G3)
        z = (z ^ (z >> np.uint64(30))) * M1
        z = (z ^ (z >> np.uint64(27))) * M2
        z = z ^ (z >> np.uint64(31))
    return z


def _u01(seed, tensor_id, index):
    """Uniform in [0, 1) with 53 random bits."""
    return (counter_u64(seed, tensor_id, index) >> np.uint64(11)).astype(
        np.float64) * (1.0 / 9007199254740992.0)


def uniform(seed, tensor_id, start, count, lo, hi):
    idx = np.arange(start, start + count, dtype=np.uint64)
    return lo + (hi - lo) * _u01(seed, tensor_id, idx)


def normal(seed, tensor_id, start, count, std=1.0):
    """Box-Muller on counters 2i, 2i+1 (so element i depends only on i)."""
    i = np.arange(start, start + count, dtype=np.uint64)
    u1 = _u01(seed, tensor_id, np.uint64(2) * i)
    u2 = _u01(seed, tensor_id, np.uint64(2) * i + np.uint64(1))
    u1 = np.maximum(u1, 1e-300)
    return std * np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)


def round_to_bf16(a):
    """Round float64/float32 values to the nearest BF16 value (ties to even),
    returned as float32."""
    f = np.ascontiguousarray(np.asarray(a, dtype=np.float32))
    u = f.view(np.uint32).astype(np.uint64)
    lsb = (u >> np.uint64(16)) & np.uint64(1)
    u = (u + np.uint64(0x7FFF) + lsb) & np.uint64(0xFFFF0000)
    return u.astype(np.uint32).view(np.float32).reshape(f.shape)


def images(n_start, count, shape, seed=IMAGE_SEED, lo=-128.0, hi=128.0, bf16=True):
    """Images [count, C, H, W] float32 (BF16-representable), U[lo, hi).

    Image ``n`` (global index) uses counters n*C*H*W ... (n+1)*C*H*W-1, so a
    shard can regenerate its images without any exchange.  The range
    ±128 is Caffe's mean-subtracted pixel scale (keeps LRN active, c3)."""
    per = int(np.prod(shape))
    v = uniform(seed, IMAGE_TENSOR_ID, n_start * per, count * per, lo, hi)
    if not bf16:      # full FP32 values (exercises the CUDA path's own rounding)
        return v.astype(np.float32).reshape((count,) + tuple(shape))
    return round_to_bf16(v).reshape((count,) + tuple(shape))


def pixels(n_start, count, shape, seed=IMAGE_SEED):
    """8-bit images [count, C, H, W] uint8, uniform over 0..255: the pixels'
    native format (pcnn_infer_host_u8).  Same counters as ``images``, so
    ``pixels - 128`` is an integer-valued image on Caffe's ±128 scale."""
    per = int(np.prod(shape))
    v = uniform(seed, IMAGE_TENSOR_ID, n_start * per, count * per, 0.0, 256.0)
    return np.minimum(np.floor(v), 255).astype(np.uint8).reshape((count,) + tuple(shape))


def he_weights(shape, fan_in, layer_index, seed=WEIGHT_SEED, bf16=True):
    """He-normal N(0, 2/fan_in), BF16-representable float32 (bf16=False: full
    FP32 values)."""
    n = int(np.prod(shape))
    v = normal(seed, layer_index, 0, n, std=np.sqrt(2.0 / fan_in))
    if not bf16:
        return v.astype(np.float32).reshape(shape)
    return round_to_bf16(v).reshape(shape)


def biases(count, layer_index, seed=WEIGHT_SEED, lo=-0.1, hi=0.1, bf16=True):
    v = uniform(seed, layer_index + BIAS_TENSOR_OFFSET, 0, count, lo, hi)
    return round_to_bf16(v) if bf16 else v.astype(np.float32)


def net_params(net, seed=WEIGHT_SEED, bf16=True):
    """(weights, biases) lists aligned with net['layers'] (None for weightless).
    bf16=False draws full FP32 values, so the CUDA path's own operand rounding
    (BF16 RNE / TF32 RNA) is exercised."""
    from .nets import weight_shapes
    ws, bs = [], []
    for i, shp in enumerate(weight_shapes(net)):
        if shp is None:
            ws.append(None)
            bs.append(None)
            continue
        wshape, bshape = shp
        fan_in = int(np.prod(wshape[1:]))
        ws.append(he_weights(wshape, fan_in, i, seed, bf16))
        bs.append(biases(bshape[0], i, seed, bf16=bf16))
    return ws, bs


PROTO_TENSOR_ID = 1 << 20        # planted-class prototypes
NOISE_TENSOR_ID = (1 << 20) + 1


def prototypes(count, shape, seed=IMAGE_SEED, block=16):
    """Planted-class prototypes [count, C, H, W]: a
    block x block piecewise-constant low-frequency field at U[-128, 128) per
    channel plus U[-32, 32) texture.  Pure generation, no method arithmetic."""
    C, H, W = shape
    bh, bw = (H + block - 1) // block, (W + block - 1) // block
    out = np.empty((count, C, H, W), dtype=np.float32)
    for k in range(count):
        coarse = uniform(seed, PROTO_TENSOR_ID, k * C * bh * bw, C * bh * bw,
                         -128.0, 128.0).reshape(C, bh, bw)
        field = np.repeat(np.repeat(coarse, block, axis=1), block, axis=2)[:, :H, :W]
        tex = uniform(seed, PROTO_TENSOR_ID + 2, k * C * H * W, C * H * W,
                      -32.0, 32.0).reshape(C, H, W)
        out[k] = field + tex
    return round_to_bf16(out)


def planted_images(n_start, count, shape, n_classes, seed=IMAGE_SEED):
    """Images of the planted-class set: image n is prototype (n mod n_classes)
    plus N(0, sigma^2) noise, sigma = U[0.02, 0.08) x 128 per image; returns
    (images [count, C, H, W], labels [count])."""
    per = int(np.prod(shape))
    labels = (np.arange(n_start, n_start + count) % n_classes).astype(np.int64)
    protos = prototypes(n_classes, shape, seed)
    sig = uniform(seed, NOISE_TENSOR_ID + 1, n_start, count, 0.02 * 128, 0.08 * 128)
    noise = normal(seed, NOISE_TENSOR_ID, n_start * per, count * per).reshape((count,) + tuple(shape))
    x = protos[labels] + noise * sig[:, None, None, None].astype(np.float32)
    return round_to_bf16(x), labels
