"""Thin ctypes binding of libpcnn.so (include/pcnn.h) -- argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels.  There is no
CPU fallback: if libpcnn.so is missing this module raises ImportError.
Torch is used only for device memory and streams (tensors are passed by
pointer).  Names follow the C ABI: create_net / set_variant / set_sm_budget /
infer / query_layer ...
"""
import ctypes
import os

PKG = os.path.dirname(os.path.abspath(__file__))
# PCNN_LIB: A/B experiments against another build of the same library
LIB_PATH = os.environ.get("PCNN_LIB") or os.path.join(PKG, "libpcnn.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        "libpcnn.so not built (%s); run `python -m paper_conf_hpca_songhcl17_b200.build`"
        " -- there is no CPU fallback" % LIB_PATH)

_lib = ctypes.CDLL(LIB_PATH)

# enums (mirror include/pcnn.h)
OK = 0
CONV, LRN, MAXPOOL, AVGPOOL, FC = 0, 1, 2, 3, 4
FP32_SIMT, TF32, BF16 = 0, 1, 2
VARIANT_EXACT, VARIANT_RANK = 0, 1
# pcnn_net_flag (layout choices of pcnn_create_net)
FLAG_NO_SPACE_TO_DEPTH = 1
FLAG_NO_PADDED_LAYOUT = 2
FLAG_NO_LRN_POOL_FUSION = 4
FLAG_CONV_LRN_EPILOGUE = 8
FLAG_PER_ROW_WINDOWS = 64
FLAG_NARROW_SLABS = 16
FLAG_PERFORATION_IM2COL = 32
PRECISIONS = {"fp32": FP32_SIMT, "fp32_simt": FP32_SIMT, "tf32": TF32, "bf16": BF16}
_KINDS = {"conv": CONV, "lrn": LRN, "maxpool": MAXPOOL, "avgpool": AVGPOOL, "fc": FC}


class LayerDesc(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("out_channels", ctypes.c_int),
                ("kernel", ctypes.c_int), ("stride", ctypes.c_int),
                ("pad", ctypes.c_int), ("groups", ctypes.c_int),
                ("relu", ctypes.c_int), ("lrn_alpha", ctypes.c_float),
                ("lrn_beta", ctypes.c_float), ("lrn_k", ctypes.c_float)]


class NetDesc(ctypes.Structure):
    _fields_ = [("in_channels", ctypes.c_int), ("in_height", ctypes.c_int),
                ("in_width", ctypes.c_int), ("max_batch", ctypes.c_int),
                ("precision", ctypes.c_int), ("device", ctypes.c_int),
                ("flags", ctypes.c_int)]


class LayerInfo(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("in_c", ctypes.c_int), ("in_h", ctypes.c_int),
                ("in_w", ctypes.c_int), ("out_c", ctypes.c_int), ("out_h", ctypes.c_int),
                ("out_w", ctypes.c_int), ("groups", ctypes.c_int),
                ("gemm_m", ctypes.c_longlong), ("gemm_n", ctypes.c_int),
                ("gemm_k", ctypes.c_int), ("flops", ctypes.c_double),
                ("flops_exact", ctypes.c_double), ("bytes", ctypes.c_double),
                ("variant", ctypes.c_int), ("rank", ctypes.c_int), ("n_sms", ctypes.c_int),
                ("tlp", ctypes.c_int), ("engine", ctypes.c_int), ("tile_m", ctypes.c_int),
                ("tile_n", ctypes.c_int), ("tiles", ctypes.c_longlong), ("grid", ctypes.c_int),
                ("util", ctypes.c_double), ("rec", ctypes.c_double), ("splits", ctypes.c_int),
                ("a_mode", ctypes.c_int), ("halo_in", ctypes.c_int), ("halo_out", ctypes.c_int),
                ("cta_group", ctypes.c_int), ("t_unit_us", ctypes.c_double),
                ("whole_window", ctypes.c_int)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class BudgetPlan(ctypes.Structure):
    _fields_ = [("grid_size", ctypes.c_longlong), ("opt_tlp", ctypes.c_int),
                ("n_invocations", ctypes.c_int), ("opt_sm", ctypes.c_int),
                ("cta_group", ctypes.c_int), ("t_model_us", ctypes.c_double),
                ("t_launch_us", ctypes.c_double), ("t_unit_us", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_P = ctypes.c_void_p
_FP = ctypes.POINTER(ctypes.c_float)
_lib.pcnn_create_net.argtypes = [ctypes.POINTER(NetDesc), ctypes.POINTER(LayerDesc),
                                 ctypes.c_int, ctypes.POINTER(_FP), ctypes.POINTER(_FP),
                                 ctypes.POINTER(_P)]
_lib.pcnn_destroy_net.argtypes = [_P]
_lib.pcnn_set_variant.argtypes = [_P, ctypes.c_int, ctypes.c_int, ctypes.c_int]
_lib.pcnn_set_variant_factors.argtypes = [_P, ctypes.c_int, ctypes.c_int, _FP, _FP]
_lib.pcnn_set_sm_budget.argtypes = [_P, ctypes.c_int, ctypes.c_int, ctypes.c_int]
_lib.pcnn_set_layer_plan.argtypes = [_P, ctypes.c_int, ctypes.c_int, ctypes.c_int]
_lib.pcnn_set_perforation.argtypes = [_P, ctypes.c_int, ctypes.c_int, ctypes.c_int]
_lib.pcnn_infer.argtypes = [_P, _P, ctypes.c_int, _P, _P, _P, _P]
_lib.pcnn_infer_host.argtypes = [_P, _P, ctypes.c_int, _P, _P, _P, _P]
_lib.pcnn_infer_host_u8.argtypes = [_P, _P, _P, ctypes.c_float, ctypes.c_int, _P, _P, _P, _P]
_lib.pcnn_output_size.argtypes = [_P, ctypes.POINTER(ctypes.c_int)]
_lib.pcnn_num_layers.argtypes = [_P, ctypes.POINTER(ctypes.c_int)]
_lib.pcnn_query_layer.argtypes = [_P, ctypes.c_int, ctypes.c_int, ctypes.POINTER(LayerInfo)]
_lib.pcnn_plan_budget.argtypes = [_P, ctypes.c_int, ctypes.c_int, ctypes.POINTER(BudgetPlan)]
_lib.pcnn_model_layer_time.argtypes = [_P, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                       ctypes.POINTER(ctypes.c_double)]
_lib.pcnn_describe_net.argtypes = [ctypes.POINTER(NetDesc), ctypes.POINTER(LayerDesc),
                                   ctypes.c_int, ctypes.c_int, ctypes.POINTER(LayerInfo)]
_lib.pcnn_profile_layers.argtypes = [_P, _P, ctypes.c_int, _P, ctypes.c_int, _FP, _FP, _P]
_lib.pcnn_set_layer_timing.argtypes = [_P, ctypes.c_int]
_lib.pcnn_read_layer_timing.argtypes = [_P, _FP, ctypes.POINTER(ctypes.c_int)]
_lib.pcnn_last_launch_count.argtypes = [_P, ctypes.POINTER(ctypes.c_int)]
_lib.pcnn_enable_sm_census.argtypes = [_P, ctypes.c_int]
_lib.pcnn_get_sm_census.argtypes = [_P, ctypes.c_int, ctypes.POINTER(ctypes.c_uint)]
_lib.pcnn_device_sm_count.argtypes = [ctypes.c_int]
_lib.pcnn_device_sm_count.restype = ctypes.c_int
_lib.pcnn_version.restype = ctypes.c_char_p
_lib.pcnn_status_string.argtypes = [ctypes.c_int]
_lib.pcnn_status_string.restype = ctypes.c_char_p
_lib.pcnn_last_error_message.restype = ctypes.c_char_p
for _f in ("pcnn_create_net", "pcnn_destroy_net", "pcnn_set_variant",
           "pcnn_set_variant_factors", "pcnn_set_sm_budget", "pcnn_set_layer_plan",
           "pcnn_set_perforation", "pcnn_infer", "pcnn_infer_host", "pcnn_infer_host_u8", "pcnn_output_size", "pcnn_num_layers", "pcnn_query_layer", "pcnn_plan_budget",
           "pcnn_model_layer_time", "pcnn_describe_net", "pcnn_profile_layers", "pcnn_enable_sm_census",
           "pcnn_get_sm_census", "pcnn_set_layer_timing", "pcnn_read_layer_timing",
           "pcnn_last_launch_count"):
    getattr(_lib, _f).restype = ctypes.c_int

EXPORTED = ["pcnn_create_net", "pcnn_destroy_net", "pcnn_set_variant",
            "pcnn_set_variant_factors", "pcnn_set_sm_budget", "pcnn_set_layer_plan",
            "pcnn_set_perforation", "pcnn_infer", "pcnn_infer_host", "pcnn_infer_host_u8", "pcnn_output_size", "pcnn_num_layers", "pcnn_query_layer", "pcnn_plan_budget",
            "pcnn_model_layer_time", "pcnn_describe_net", "pcnn_profile_layers", "pcnn_enable_sm_census",
            "pcnn_get_sm_census", "pcnn_set_layer_timing", "pcnn_read_layer_timing",
            "pcnn_last_launch_count", "pcnn_device_sm_count", "pcnn_version",
            "pcnn_status_string", "pcnn_last_error_message"]


class PcnnError(RuntimeError):
    def __init__(self, status, what):
        msg = "%s: %s (%s)" % (what, _lib.pcnn_status_string(status).decode(),
                               _lib.pcnn_last_error_message().decode())
        super().__init__(msg)
        self.status = status


def _check(st, what):
    if st != OK:
        raise PcnnError(st, what)


def library():
    return _lib


def version():
    return _lib.pcnn_version().decode()


def device_sm_count(device=0):
    return _lib.pcnn_device_sm_count(device)


def layer_descs(layers):
    """synth-style layer dicts -> ctypes LayerDesc array (marshalling)."""
    arr = (LayerDesc * len(layers))()
    for i, L in enumerate(layers):
        d = arr[i]
        d.kind = _KINDS[L["kind"]]
        if L["kind"] == "conv":
            d.out_channels, d.kernel, d.stride = L["out"], L["k"], L.get("stride", 1)
            d.pad, d.groups, d.relu = L.get("pad", 0), L.get("groups", 1), int(L.get("relu", True))
        elif L["kind"] == "fc":
            d.out_channels, d.relu, d.groups = L["out"], int(L.get("relu", True)), 1
        elif L["kind"] == "lrn":
            d.kernel = L["size"]
            d.lrn_alpha, d.lrn_beta, d.lrn_k = L["alpha"], L["beta"], L["k"]
        else:
            d.kernel, d.stride = L["k"], L["stride"]
    return arr


def net_desc(in_shape, max_batch, precision, device=0, flags=0):
    c, h, w = in_shape
    p = PRECISIONS[precision] if isinstance(precision, str) else int(precision)
    return NetDesc(c, h, w, max_batch, p, device, int(flags))


def describe_net(net, batch=1, precision="bf16"):
    """Host-only shape / FLOP / byte inference (no GPU needed)."""
    layers = layer_descs(net["layers"])
    nd = net_desc(net["in_shape"], max(batch, 1), precision)
    infos = (LayerInfo * len(net["layers"]))()
    _check(_lib.pcnn_describe_net(ctypes.byref(nd), layers, len(net["layers"]), batch,
                                  infos), "pcnn_describe_net")
    return [i.as_dict() for i in infos]


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream_ptr(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


class Net:
    """A built network (pcnn_create_net) on one device."""

    def __init__(self, net, weights, biases, max_batch, precision="bf16", device=0, flags=0):
        import numpy as np
        self.spec = net
        self.n_layers = len(net["layers"])
        self.precision = precision
        self.device = device
        layers = layer_descs(net["layers"])
        nd = net_desc(net["in_shape"], max_batch, precision, device, flags)
        keep = []
        wp = (_FP * self.n_layers)()
        bp = (_FP * self.n_layers)()
        for i in range(self.n_layers):
            if weights[i] is not None:
                w = np.ascontiguousarray(weights[i], dtype=np.float32)
                keep.append(w)
                wp[i] = w.ctypes.data_as(_FP)
            if biases is not None and biases[i] is not None:
                b = np.ascontiguousarray(biases[i], dtype=np.float32)
                keep.append(b)
                bp[i] = b.ctypes.data_as(_FP)
        h = ctypes.c_void_p()
        _check(_lib.pcnn_create_net(ctypes.byref(nd), layers, self.n_layers, wp, bp,
                                    ctypes.byref(h)), "pcnn_create_net")
        self._h = h
        n = ctypes.c_int()
        _check(_lib.pcnn_output_size(h, ctypes.byref(n)), "pcnn_output_size")
        self.out_elems = n.value
        self.max_batch = max_batch

    def close(self):
        if getattr(self, "_h", None):
            _lib.pcnn_destroy_net(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_variant(self, layer, variant, rank=0):
        v = {"exact": VARIANT_EXACT, "rank": VARIANT_RANK}.get(variant, variant)
        _check(_lib.pcnn_set_variant(self._h, layer, int(v), int(rank)), "pcnn_set_variant")

    def set_variant_factors(self, layer, rank, A, B):
        import numpy as np
        A = np.ascontiguousarray(A, dtype=np.float32)
        B = np.ascontiguousarray(B, dtype=np.float32)
        _check(_lib.pcnn_set_variant_factors(self._h, layer, rank, A.ctypes.data_as(_FP),
                                             B.ctypes.data_as(_FP)), "pcnn_set_variant_factors")

    def set_layer_plan(self, layer, cta_group=0, m_sub=0):
        _check(_lib.pcnn_set_layer_plan(self._h, layer, cta_group, m_sub), "pcnn_set_layer_plan")

    def set_perforation(self, layer, sh, sw):
        _check(_lib.pcnn_set_perforation(self._h, layer, sh, sw), "pcnn_set_perforation")

    def set_sm_budget(self, layer, n_sms, ctas_per_sm=0):
        _check(_lib.pcnn_set_sm_budget(self._h, layer, n_sms, ctas_per_sm), "pcnn_set_sm_budget")

    def infer(self, images, out=None, probs=None, entropy=None, stream=None):
        """images: cuda fp32 [B,C,H,W]; returns (out, probs, entropy) cuda tensors.
        Pass probs=True / entropy=True to allocate them."""
        import torch
        B = images.shape[0]
        if out is None:
            out = torch.empty((B, self.out_elems), device=images.device, dtype=torch.float32)
        if probs is True:
            probs = torch.empty_like(out)
        if entropy is True:
            entropy = torch.empty((B,), device=images.device, dtype=torch.float32)
        probs = probs if probs is not None and probs is not False else None
        entropy = entropy if entropy is not None and entropy is not False else None
        _check(_lib.pcnn_infer(self._h, _ptr(images), B, _ptr(out), _ptr(probs),
                               _ptr(entropy), _stream_ptr(stream)), "pcnn_infer")
        return out, probs, entropy

    def infer_host(self, images, out, probs=None, entropy=None, stream=None):
        """images / out / probs / entropy: CPU fp32 tensors (pinned for speed)."""
        B = images.shape[0]
        _check(_lib.pcnn_infer_host(self._h, _ptr(images), B, _ptr(out), _ptr(probs),
                                    _ptr(entropy), _stream_ptr(stream)), "pcnn_infer_host")
        return out

    def infer_host_u8(self, pixels, out, mean=None, scale=1.0, probs=None, entropy=None,
                      stream=None):
        """pixels: CPU uint8 tensor [B][C][H][W] (pinned for speed); the network
        input is (pixel - mean[c]) * scale, converted on the device."""
        B = pixels.shape[0]
        m = None
        if mean is not None:
            m = (ctypes.c_float * len(mean))(*[float(v) for v in mean])
        _check(_lib.pcnn_infer_host_u8(self._h, _ptr(pixels), m, ctypes.c_float(scale), B,
                                       _ptr(out), _ptr(probs), _ptr(entropy),
                                       _stream_ptr(stream)), "pcnn_infer_host_u8")
        return out

    def query_layer(self, layer, batch):
        info = LayerInfo()
        _check(_lib.pcnn_query_layer(self._h, layer, batch, ctypes.byref(info)),
               "pcnn_query_layer")
        return info.as_dict()

    def plan_budget(self, layer, batch):
        """eqs. 8 / 11 / 12 for one layer (see pcnn_plan_budget)."""
        bp = BudgetPlan()
        _check(_lib.pcnn_plan_budget(self._h, layer, batch, ctypes.byref(bp)),
               "pcnn_plan_budget")
        return bp.as_dict()

    def model_layer_time(self, layer, batch, n_sms=0):
        """eq. 12 (NEXT-3): modelled latency in us of one layer on n_sms SMs."""
        t = ctypes.c_double()
        _check(_lib.pcnn_model_layer_time(self._h, layer, batch, n_sms, ctypes.byref(t)),
               "pcnn_model_layer_time")
        return t.value

    def apply_opt_budgets(self, batch):
        """Give every GEMM layer its eq. 11 optSM x optTLP budget;
        returns the plans."""
        plans = [self.plan_budget(i, batch) for i in range(self.n_layers)]
        for i, p in enumerate(plans):
            if p["grid_size"] > 0:
                self.set_sm_budget(i, p["opt_sm"], 0)
        return plans

    def profile_layers(self, images, reps=5, out=None, stream=None):
        import torch
        B = images.shape[0]
        if out is None:
            out = torch.empty((B, self.out_elems), device=images.device, dtype=torch.float32)
        ms = (ctypes.c_float * self.n_layers)()
        tot = ctypes.c_float()
        _check(_lib.pcnn_profile_layers(self._h, _ptr(images), B, _ptr(out), reps, ms,
                                        ctypes.byref(tot), _stream_ptr(stream)),
               "pcnn_profile_layers")
        return list(ms), tot.value

    def set_layer_timing(self, enable=True):
        _check(_lib.pcnn_set_layer_timing(self._h, int(enable)), "pcnn_set_layer_timing")

    def read_layer_timing(self):
        """(per-layer ms summed over the recorded infers, number of infers)."""
        ms = (ctypes.c_float * self.n_layers)()
        n = ctypes.c_int()
        _check(_lib.pcnn_read_layer_timing(self._h, ms, ctypes.byref(n)),
               "pcnn_read_layer_timing")
        return list(ms), n.value

    def last_launch_count(self):
        n = ctypes.c_int()
        _check(_lib.pcnn_last_launch_count(self._h, ctypes.byref(n)), "pcnn_last_launch_count")
        return n.value

    def enable_sm_census(self, enable=True):
        _check(_lib.pcnn_enable_sm_census(self._h, int(enable)), "pcnn_enable_sm_census")

    def sm_census(self, layer):
        m = (ctypes.c_uint * 8)()
        _check(_lib.pcnn_get_sm_census(self._h, layer, m), "pcnn_get_sm_census")
        return sorted(w * 32 + b for w in range(8) for b in range(32) if (m[w] >> b) & 1)
