"""B200-native (sm_100a) P-CNN batched-inference hot path.

The product is the C-ABI library libpcnn.so (include/pcnn.h); ``pcnn`` is its
thin ctypes binding.  Import ``paper_conf_hpca_songhcl17_b200.pcnn`` to use it
(it raises ImportError if the library has not been built).
"""
__all__ = ["pcnn", "build"]
