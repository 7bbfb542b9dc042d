"""B200-native TeMCO: fused reduced-skip inference over Tucker-2 / CP
decomposed CNNs behind the C ABI of include/temco.h.

`Plan` (temco.py) is a thin ctypes binding of libtemco.so; building the
library: `python -m paper_conf_icpp_songljkj0024_b200.build`.  Accessing any
binding name without the library raises ImportError (no CPU fallback); the
lazy import only lets `build` run before the library exists.
"""
_BINDING = {"Plan", "TemcoError", "library_path", "exported_symbols", "EXPORTS", "F32", "BF16", "FLAG_NO_DEVICE",
            "FLAG_NO_SKIPOPT", "FLAG_NO_FUSION", "FLAG_CUDA_GRAPH", "FLAG_SIMT_ONLY", "FLAG_OVERHEAD_ALWAYS",
            "FLAG_OVERHEAD_NEVER", "FLAG_MMA_SMALL", "FLAG_MMA_CAT", "FLAG_PAPER_SCHEDULE", "FLAG_NO_CSE",
            "FLAG_NO_RESCHEDULE", "FLAG_CSE_BOUND"}


def __getattr__(name):
    if name in _BINDING:
        from . import temco
        return getattr(temco, name)
    raise AttributeError(name)
