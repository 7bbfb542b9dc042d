"""Thin ctypes binding of libtemco.so (include/temco.h): argument marshalling
only -- every step of the inference path runs in the library's kernels.

There is no CPU fallback: if libtemco.so is missing, importing this module
raises.  PyTorch is used by callers only for device memory and streams.
"""
from __future__ import annotations

import ctypes as C
import json
import os

import numpy as np

_LIB_PATH = os.environ.get("TEMCO_LIB") or os.path.join(os.path.dirname(os.path.abspath(__file__)), "libtemco.so")
if not os.path.exists(_LIB_PATH):
    raise ImportError(f"{_LIB_PATH} is missing: build it with `python -m paper_conf_icpp_songljkj0024_b200.build` "
                      "(there is no CPU fallback)")
_lib = C.CDLL(_LIB_PATH)

OPS = {"input": 0, "conv": 1, "bn": 2, "relu": 3, "silu": 4, "add": 5, "concat": 6, "maxpool": 7,
       "avgpool": 8, "gap": 9, "linear": 10, "conv_transpose": 11}
F32, BF16 = 0, 1
FLAG_NO_DEVICE = 1 << 0
FLAG_NO_SKIPOPT = 1 << 1
FLAG_NO_FUSION = 1 << 2
FLAG_CUDA_GRAPH = 1 << 3
FLAG_SIMT_ONLY = 1 << 4
FLAG_OVERHEAD_ALWAYS = 1 << 5
FLAG_OVERHEAD_NEVER = 1 << 6
FLAG_MMA_SMALL = 1 << 7
FLAG_MMA_CAT = 1 << 8
FLAG_PAPER_SCHEDULE = 1 << 9   # without the round-2 schedule extensions R34-R38
FLAG_NO_CSE = 1 << 10          # no merged-fconv CSE (R37)
FLAG_NO_RESCHEDULE = 1 << 11   # keep S's order (no R38)
FLAG_CSE_BOUND = 1 << 12       # R37 keeps merges with peak <= the unfused peak

EXPORTS = ["temco_plan_create", "temco_run", "temco_run_host", "temco_run_host_async", "temco_peak_internal_bytes", "temco_output_shape",
           "temco_plan_describe", "temco_run_profiled", "temco_debug_step_output", "temco_debug_step_tensor",
           "temco_plan_destroy",
           "temco_status_string", "temco_last_error"]

_fp = C.POINTER(C.c_float)


class _Layer(C.Structure):
    _fields_ = [("op", C.c_int32), ("n_inputs", C.c_int32), ("inputs", C.POINTER(C.c_int32)),
                ("out_channels", C.c_int32), ("kernel", C.c_int32), ("stride", C.c_int32), ("pad", C.c_int32),
                ("groups", C.c_int32), ("weight", _fp), ("bias", _fp), ("bn_gamma", _fp), ("bn_beta", _fp),
                ("bn_mean", _fp), ("bn_var", _fp), ("bn_eps", C.c_float)]


class _Decomp(C.Structure):
    _fields_ = [("layer", C.c_int32), ("kind", C.c_int32), ("rank_in", C.c_int32), ("rank_out", C.c_int32),
                ("first", _fp), ("core", _fp), ("core2", _fp), ("last", _fp), ("rank_mid", C.c_int32)]


class _Edge(C.Structure):
    _fields_ = [("src", C.c_int32), ("dst", C.c_int32)]


class _Config(C.Structure):
    _fields_ = [("batch", C.c_int32), ("height", C.c_int32), ("width", C.c_int32), ("channels", C.c_int32),
                ("dtype", C.c_int32), ("distance_threshold", C.c_int32), ("flags", C.c_int32)]


_lib.temco_plan_create.argtypes = [C.POINTER(_Layer), C.c_int32, C.POINTER(_Decomp), C.c_int32, C.POINTER(_Edge),
                                   C.c_int32, C.POINTER(_Config), C.POINTER(C.c_void_p)]
_lib.temco_run.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
_lib.temco_run_host.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
_lib.temco_run_host_async.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
_lib.temco_run_profiled.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, _fp, C.c_int32]
_lib.temco_peak_internal_bytes.argtypes = [C.c_void_p, C.c_int32, C.POINTER(C.c_int64)]
_lib.temco_debug_step_output.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_int32, C.c_void_p,
                                         C.c_int64, C.POINTER(C.c_int64)]
_lib.temco_debug_step_tensor.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_int32, C.c_int32,
                                         C.c_void_p, C.c_int64, C.POINTER(C.c_int64)]
_lib.temco_output_shape.argtypes = [C.c_void_p, C.POINTER(C.c_int64), C.POINTER(C.c_int32)]
_lib.temco_plan_describe.argtypes = [C.c_void_p, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)]
_lib.temco_plan_destroy.argtypes = [C.c_void_p]
_lib.temco_status_string.argtypes = [C.c_int]
_lib.temco_status_string.restype = C.c_char_p
_lib.temco_last_error.restype = C.c_char_p
for _f in ["temco_plan_create", "temco_run", "temco_run_host", "temco_run_host_async", "temco_run_profiled", "temco_peak_internal_bytes",
           "temco_output_shape", "temco_plan_describe", "temco_debug_step_output", "temco_debug_step_tensor",
           "temco_plan_destroy"]:
    getattr(_lib, _f).restype = C.c_int


class TemcoError(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        super().__init__(f"{where}: {_lib.temco_status_string(status).decode()} "
                         f"({status}): {_lib.temco_last_error().decode()}")


def _check(st, where):
    if st != 0:
        raise TemcoError(st, where)


def _f32(a):
    if a is None:
        return None
    return np.ascontiguousarray(np.asarray(a, dtype=np.float32))


def _ptr(a):
    return a.ctypes.data_as(_fp) if a is not None else None


def library_path():
    return _LIB_PATH


def exported_symbols():
    return [s for s in EXPORTS if hasattr(_lib, s)]


def _stream_handle(stream):
    if stream is None:
        import torch
        return C.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return C.c_void_p(stream)
    return C.c_void_p(stream.cuda_stream)


class Plan:
    """A TeMCO plan built from a `workloads.Model`-shaped graph description
    (layers, decomps, batch/height/width/channels, dtype)."""

    def __init__(self, model, flags: int = 0, distance_threshold: int = 1, skip_edges=None):
        keep = []
        layers = (_Layer * len(model.layers))()
        for i, l in enumerate(model.layers):
            ins = np.asarray(l.inputs, dtype=np.int32)
            keep.append(ins)
            L = layers[i]
            L.op = OPS[l.op]
            L.n_inputs = len(l.inputs)
            L.inputs = ins.ctypes.data_as(C.POINTER(C.c_int32)) if len(l.inputs) else None
            L.out_channels = int(l.out_channels or 0)
            L.kernel, L.stride, L.pad, L.groups = int(l.kernel), int(l.stride), int(l.pad), int(l.groups)
            decomposed = i in model.decomps
            for name, arr in (("weight", None if decomposed else l.weight), ("bias", l.bias),
                              ("bn_gamma", l.bn_gamma), ("bn_beta", l.bn_beta),
                              ("bn_mean", l.bn_mean), ("bn_var", l.bn_var)):
                a = _f32(arr)
                keep.append(a)
                setattr(L, name, _ptr(a))
            L.bn_eps = float(l.bn_eps)
        decs = (_Decomp * max(1, len(model.decomps)))()
        for j, (li, d) in enumerate(sorted(model.decomps.items())):
            D = decs[j]
            D.layer, D.kind = li, {"tucker2": 1, "cp": 2, "tt": 3}[d.kind]
            D.rank_in, D.rank_out = d.rank_in, d.rank_out
            D.rank_mid = getattr(d, "rank_mid", 0)
            for name in ("first", "core", "core2", "last"):
                a = _f32(getattr(d, name))
                keep.append(a)
                setattr(D, name, _ptr(a))
        if skip_edges is None:
            skip_edges = [(s, dd) for dd, l in enumerate(model.layers) for s in l.inputs if dd - s > 1]
        edges = (_Edge * max(1, len(skip_edges)))()
        for j, (s, dd) in enumerate(skip_edges):
            edges[j].src, edges[j].dst = s, dd
        self.dtype = model.dtype
        cfg = _Config(model.batch, model.height, model.width, model.channels,
                      BF16 if model.dtype == "bf16" else F32, distance_threshold, flags)
        h = C.c_void_p()
        _check(_lib.temco_plan_create(layers, len(model.layers), decs, len(model.decomps), edges, len(skip_edges),
                                      C.byref(cfg), C.byref(h)), "temco_plan_create")
        self._h = h
        self.batch = model.batch
        self.input_shape = (model.batch, model.height, model.width, model.channels)

    # -- queries ---------------------------------------------------------------
    def peak_internal_bytes(self, which: int = 0) -> int:
        v = C.c_int64()
        _check(_lib.temco_peak_internal_bytes(self._h, which, C.byref(v)), "temco_peak_internal_bytes")
        return v.value

    def output_shape(self):
        dims = (C.c_int64 * 4)()
        nd = C.c_int32()
        _check(_lib.temco_output_shape(self._h, dims, C.byref(nd)), "temco_output_shape")
        return tuple(dims[i] for i in range(nd.value))

    def describe(self) -> dict:
        need = C.c_size_t()
        _check(_lib.temco_plan_describe(self._h, None, 0, C.byref(need)), "temco_plan_describe")
        buf = C.create_string_buffer(need.value)
        _check(_lib.temco_plan_describe(self._h, buf, need.value, C.byref(need)), "temco_plan_describe")
        return json.loads(buf.value.decode())

    # -- execution (device pointers: torch CUDA tensors or raw ints) -----------
    def run(self, x, y, stream=None):
        xp = x if isinstance(x, int) else x.data_ptr()
        yp = y if isinstance(y, int) else y.data_ptr()
        _check(_lib.temco_run(self._h, C.c_void_p(xp), C.c_void_p(yp), _stream_handle(stream)), "temco_run")

    def run_host(self, x_host, y_host, stream=None):
        """x_host / y_host: CPU tensors or numpy arrays (pinned for async DMA)."""
        xp = x_host.data_ptr() if hasattr(x_host, "data_ptr") else x_host.ctypes.data
        yp = y_host.data_ptr() if hasattr(y_host, "data_ptr") else y_host.ctypes.data
        _check(_lib.temco_run_host(self._h, C.c_void_p(xp), C.c_void_p(yp), _stream_handle(stream)),
               "temco_run_host")

    def run_host_async(self, x_host, y_host, stream=None):
        """Pipelined host-buffer run (temco_run_host_async): returns before the
        work completes; synchronise `stream` before reading y_host."""
        xp = x_host.data_ptr() if hasattr(x_host, "data_ptr") else x_host.ctypes.data
        yp = y_host.data_ptr() if hasattr(y_host, "data_ptr") else y_host.ctypes.data
        _check(_lib.temco_run_host_async(self._h, C.c_void_p(xp), C.c_void_p(yp), _stream_handle(stream)),
               "temco_run_host_async")

    def run_profiled(self, x, y, stream=None):
        n = len(self.describe()["steps"])
        ms = (C.c_float * n)()
        _check(_lib.temco_run_profiled(self._h, C.c_void_p(x.data_ptr()), C.c_void_p(y.data_ptr()),
                                       _stream_handle(stream), ms, n), "temco_run_profiled")
        return list(ms)

    def step_output(self, x, y, step, stream=None, which=0):
        """Run schedule steps 0..step and return that step's output tensor `which` (0: the
        step's tensor; 1..: a merged group's further reduce outputs) as raw bytes (NHWC,
        plan dtype; fp32 for the graph output) -- a verification hook."""
        nb = C.c_int64(0)
        xs, ys = C.c_void_p(x.data_ptr()), C.c_void_p(y.data_ptr())
        _check(_lib.temco_debug_step_tensor(self._h, xs, ys, _stream_handle(stream), step, which, None, 0,
                                            C.byref(nb)), "temco_debug_step_tensor")
        buf = np.empty(nb.value, np.uint8)
        _check(_lib.temco_debug_step_tensor(self._h, xs, ys, _stream_handle(stream), step, which,
                                            buf.ctypes.data_as(C.c_void_p), nb.value, C.byref(nb)),
               "temco_debug_step_tensor")
        return buf

    def close(self):
        if getattr(self, "_h", None):
            _lib.temco_plan_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
