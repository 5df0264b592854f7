"""ctypes binding of libspp (include/spp.h) — argument marshalling only.

Every step of the hot path runs in libspp's sm_100a kernels; PyTorch supplies
device memory, streams and process groups.  There is no CPU fallback: if
``libspp.so`` is missing or the device is not an sm_100 GPU, calls raise.
Function names mirror the C ABI.
"""
from __future__ import annotations

import ctypes as C
import os
from pathlib import Path
from typing import Sequence

import numpy as np

_PKG = Path(__file__).resolve().parent
# SPP_LIB may point at an experimental build variant (scripts/variants.py)
LIB_PATH = Path(os.environ["SPP_LIB"]) if os.environ.get("SPP_LIB") else _PKG / "libspp.so"

SPP_OK, SPP_ERR_INVALID_ARG, SPP_ERR_BUFFER_TOO_SMALL, SPP_ERR_CORRUPT, SPP_ERR_UNSUPPORTED, SPP_ERR_CUDA = range(6)
SPP_FMT_COSMO, SPP_FMT_DEEPCAM = 1, 2
SPP_OUT_F16, SPP_OUT_F32, SPP_OUT_I16 = 1, 2, 3
FMT = {"cosmo": SPP_FMT_COSMO, "deepcam": SPP_FMT_DEEPCAM}
OUT = {"f16": SPP_OUT_F16, "f32": SPP_OUT_F32, "i16": SPP_OUT_I16}

# every symbol include/spp.h declares (checked by tests/test_host.py)
EXPORTS = (
    "spp_cosmo_max_encoded_size", "spp_encode_cosmo", "spp_deepcam_max_encoded_size", "spp_encode_deepcam",
    "spp_encode_deepcam_ex", "spp_encode_cosmo_ex",
    "spp_stream_info", "spp_decode_opts_init", "spp_decode_workspace_size", "spp_decoded_sample_bytes",
    "spp_decode_batch", "spp_decode_launches", "spp_pipeline_create", "spp_pipeline_destroy", "spp_decode_host",
    "spp_pipeline_last_launches", "spp_status_string", "spp_version",
    "spp_label_max_encoded_size", "spp_encode_label_mask", "spp_encode_label_vector", "spp_decode_labels",
)
SPP_LABEL_MASK, SPP_LABEL_VECTOR = 1, 2
LABEL_KIND = {"mask": SPP_LABEL_MASK, "vector": SPP_LABEL_VECTOR}


class SppError(RuntimeError):
    def __init__(self, code: int, what: str):
        super().__init__(f"{what}: {spp_status_string(code)} ({code})")
        self.code = code


class spp_cosmo_params(C.Structure):
    _fields_ = [("localize", C.c_int), ("escape_keys", C.c_int)]


class spp_deepcam_params(C.Structure):
    _fields_ = [("lookahead", C.c_int), ("repeat_min", C.c_int), ("rel_err", C.c_float), ("err_budget", C.c_int),
                ("raw16", C.c_int), ("raw_segments", C.c_int), ("repeat_tol", C.c_void_p),
                ("max_abs_err", C.c_void_p)]


class spp_decode_opts(C.Structure):
    _fields_ = [("out", C.c_int), ("transform", C.c_int), ("shift", C.c_void_p), ("scale", C.c_void_p),
                ("status", C.c_void_p), ("src_bytes", C.c_void_p), ("workspace", C.c_void_p),
                ("workspace_size", C.c_size_t), ("C", C.c_int), ("D", C.c_int), ("H", C.c_int), ("W", C.c_int),
                ("timing_events", C.c_void_p), ("escape_keys", C.c_int), ("raw_segments", C.c_int)]


_lib = None


def load() -> C.CDLL:
    """Load the in-tree libspp.so (built by __graft_entry__.build()); fail loudly."""
    global _lib
    if _lib is not None:
        return _lib
    if not LIB_PATH.exists():
        raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                          "(there is no CPU fallback)")
    L = C.CDLL(str(LIB_PATH))
    P, I, SZ, I64 = C.c_void_p, C.c_int, C.c_size_t, C.c_int64
    sig = {
        "spp_cosmo_max_encoded_size": ([I, I, I, I], SZ),
        "spp_encode_cosmo": ([P, I, I, I, I, P, SZ, C.POINTER(SZ)], I),
        "spp_encode_cosmo_ex": ([P, I, I, I, I, C.POINTER(spp_cosmo_params), P, SZ, C.POINTER(SZ)], I),
        "spp_deepcam_max_encoded_size": ([I, I, I], SZ),
        "spp_encode_deepcam": ([P, I, I, I, P, SZ, C.POINTER(SZ)], I),
        "spp_encode_deepcam_ex": ([P, I, I, I, C.POINTER(spp_deepcam_params), P, SZ, C.POINTER(SZ)], I),
        "spp_stream_info": ([I, P, SZ, C.POINTER(I64)], I),
        "spp_decode_opts_init": ([C.POINTER(spp_decode_opts), I, I, I, I, I], None),
        "spp_decode_workspace_size": ([I, I, C.POINTER(spp_decode_opts)], SZ),
        "spp_decoded_sample_bytes": ([I, C.POINTER(spp_decode_opts)], SZ),
        "spp_decode_batch": ([I, P, I, P, C.POINTER(spp_decode_opts), P], I),
        "spp_decode_launches": ([I], I),
        "spp_pipeline_create": ([C.POINTER(P), I, C.POINTER(spp_decode_opts), SZ, I, I], I),
        "spp_pipeline_destroy": ([P], None),
        "spp_decode_host": ([P, P, P, I, P, C.POINTER(spp_decode_opts), P], I),
        "spp_pipeline_last_launches": ([P], I),
        "spp_status_string": ([I], C.c_char_p),
        "spp_label_max_encoded_size": ([I, I, I], SZ),
        "spp_encode_label_mask": ([P, I, I, P, SZ, C.POINTER(SZ)], I),
        "spp_encode_label_vector": ([P, I, P, SZ, C.POINTER(SZ)], I),
        "spp_decode_labels": ([I, P, P, I, P, I, I, P, P], I),
        "spp_version": ([], C.c_char_p),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    _lib = L
    return L


def _check(rc: int, what: str):
    if rc != SPP_OK:
        raise SppError(rc, what)


def spp_status_string(code: int) -> str:
    return load().spp_status_string(int(code)).decode()


def spp_version() -> str:
    return load().spp_version().decode()


# ---------------------------------------------------------------- host encoders
def spp_cosmo_max_encoded_size(Cc: int, D: int, H: int, W: int) -> int:
    return int(load().spp_cosmo_max_encoded_size(Cc, D, H, W))


def spp_encode_cosmo(counts: np.ndarray, localize: bool = False, escape: bool = False) -> np.ndarray:
    """int16 [4, D, H, W] counts -> encoded uint8 stream (FORMAT.md 1); with
    `localize` through spp_encode_cosmo_ex (FORMAT.md 1.4 localized tables)."""
    a = np.ascontiguousarray(counts, dtype=np.int16)
    if a.ndim != 4:
        raise ValueError("counts must be [4, D, H, W]")
    Cc, D, H, W = a.shape
    cap = spp_cosmo_max_encoded_size(Cc, D, H, W)
    dst = np.empty(max(cap, 64), dtype=np.uint8)
    size = C.c_size_t(0)
    if localize or escape:
        prm = spp_cosmo_params(int(localize), int(escape))
        _check(load().spp_encode_cosmo_ex(a.ctypes.data, Cc, D, H, W, C.byref(prm), dst.ctypes.data, dst.size,
                                          C.byref(size)), "spp_encode_cosmo_ex")
    else:
        _check(load().spp_encode_cosmo(a.ctypes.data, Cc, D, H, W, dst.ctypes.data, dst.size, C.byref(size)),
               "spp_encode_cosmo")
    return dst[: size.value].copy()


def spp_deepcam_max_encoded_size(Cc: int, H: int, W: int) -> int:
    return int(load().spp_deepcam_max_encoded_size(Cc, H, W))


def spp_encode_deepcam(x: np.ndarray, lookahead: int = 0, repeat_min: int = 0, rel_err: float = 0.0,
                       err_budget: int = 0, raw16: bool = False, raw_segments: bool = False, repeat_tol=None,
                       max_abs_err=None) -> np.ndarray:
    """fp32 [C, H, W] -> encoded uint8 stream (FORMAT.md 2); nonzero knobs go
    through spp_encode_deepcam_ex (0 = the FORMAT.md 2.4 default; err_budget
    > 0 = the FORMAT.md 2.5 error budget at relative error rel_err;
    repeat_tol / max_abs_err = the FORMAT.md 2.8 per-channel fp32[C] REPEAT
    tolerance and absolute error bound)."""
    a = np.ascontiguousarray(x, dtype=np.float32)
    if a.ndim != 3:
        raise ValueError("x must be [C, H, W]")
    Cc, H, W = a.shape
    cap = spp_deepcam_max_encoded_size(Cc, H, W)
    dst = np.empty(max(cap, 64), dtype=np.uint8)
    size = C.c_size_t(0)
    rt = None if repeat_tol is None else np.ascontiguousarray(repeat_tol, dtype=np.float32)
    me = None if max_abs_err is None else np.ascontiguousarray(max_abs_err, dtype=np.float32)
    for arr in (rt, me):
        if arr is not None and arr.shape != (Cc,):
            raise ValueError("per-channel knobs are fp32[C]")
    if lookahead or repeat_min or rel_err or err_budget or raw16 or raw_segments or rt is not None or me is not None:
        prm = spp_deepcam_params(int(lookahead), int(repeat_min), float(rel_err), int(err_budget), int(bool(raw16)),
                                 int(bool(raw_segments)), None if rt is None else rt.ctypes.data,
                                 None if me is None else me.ctypes.data)
        _check(load().spp_encode_deepcam_ex(a.ctypes.data, Cc, H, W, C.byref(prm), dst.ctypes.data, dst.size,
                                            C.byref(size)), "spp_encode_deepcam_ex")
    else:
        _check(load().spp_encode_deepcam(a.ctypes.data, Cc, H, W, dst.ctypes.data, dst.size, C.byref(size)),
               "spp_encode_deepcam")
    return dst[: size.value].copy()


def spp_stream_info(fmt: str, buf: np.ndarray):
    b = np.ascontiguousarray(buf, dtype=np.uint8)
    info = (C.c_int64 * 4)()
    _check(load().spp_stream_info(FMT[fmt], b.ctypes.data, b.size, info), "spp_stream_info")
    return tuple(int(v) for v in info)


# ---------------------------------------------------------------- device decode
def spp_decode_opts_init(fmt: str, Cc: int, D: int, H: int, W: int, out: str = "f16",
                         transform: int | None = None) -> spp_decode_opts:
    o = spp_decode_opts()
    load().spp_decode_opts_init(C.byref(o), FMT[fmt], Cc, D, H, W)
    o.out = OUT[out]
    if transform is not None:
        o.transform = int(transform)
    return o


def spp_decode_workspace_size(fmt: str, n: int, opts: spp_decode_opts) -> int:
    return int(load().spp_decode_workspace_size(FMT[fmt], n, C.byref(opts)))


def spp_decoded_sample_bytes(fmt: str, opts: spp_decode_opts) -> int:
    return int(load().spp_decoded_sample_bytes(FMT[fmt], C.byref(opts)))


def spp_decode_launches(fmt: str) -> int:
    return int(load().spp_decode_launches(FMT[fmt]))


def spp_decode_batch(fmt: str, d_src_ptrs: int, n: int, d_dst: int, opts: spp_decode_opts, stream: int = 0):
    """Raw call: d_src_ptrs = device address of n device pointers; d_dst = device address."""
    _check(load().spp_decode_batch(FMT[fmt], d_src_ptrs, n, d_dst, C.byref(opts), stream), "spp_decode_batch")


def spp_pipeline_create(fmt: str, opts: spp_decode_opts, slot_bytes: int, nslots: int, max_chunk: int) -> int:
    h = C.c_void_p()
    _check(load().spp_pipeline_create(C.byref(h), FMT[fmt], C.byref(opts), slot_bytes, nslots, max_chunk),
           "spp_pipeline_create")
    return h.value


def spp_pipeline_destroy(handle: int):
    load().spp_pipeline_destroy(handle)


def spp_decode_host(handle: int, h_ptrs: Sequence[int], sizes: Sequence[int], d_dst: int, opts: spp_decode_opts,
                    stream: int = 0):
    n = len(h_ptrs)
    ptrs = (C.c_void_p * n)(*h_ptrs)
    sz = (C.c_size_t * n)(*sizes)
    _check(load().spp_decode_host(handle, ptrs, sz, n, d_dst, C.byref(opts), stream), "spp_decode_host")


def spp_pipeline_last_launches(handle: int) -> int:
    return int(load().spp_pipeline_last_launches(handle))


# ---------------------------------------------------------------- labels (FORMAT.md 3)
def spp_label_max_encoded_size(kind: str, H: int, W: int) -> int:
    return int(load().spp_label_max_encoded_size(LABEL_KIND[kind], H, W))


def spp_encode_label_mask(mask: np.ndarray) -> np.ndarray:
    """u8 [H, W] class mask -> lossless label stream (FORMAT.md 3)."""
    a = np.ascontiguousarray(mask, dtype=np.uint8)
    if a.ndim != 2:
        raise ValueError("mask must be [H, W]")
    H, W = a.shape
    dst = np.empty(max(spp_label_max_encoded_size("mask", H, W), 32), dtype=np.uint8)
    size = C.c_size_t(0)
    _check(load().spp_encode_label_mask(a.ctypes.data, H, W, dst.ctypes.data, dst.size, C.byref(size)),
           "spp_encode_label_mask")
    return dst[: size.value].copy()


def spp_encode_label_vector(v: np.ndarray) -> np.ndarray:
    """fp32 [n] -> lossless label stream (FORMAT.md 3, binary32 verbatim)."""
    a = np.ascontiguousarray(v, dtype=np.float32).ravel()
    dst = np.empty(max(spp_label_max_encoded_size("vector", 1, a.size), 32), dtype=np.uint8)
    size = C.c_size_t(0)
    _check(load().spp_encode_label_vector(a.ctypes.data, a.size, dst.ctypes.data, dst.size, C.byref(size)),
           "spp_encode_label_vector")
    return dst[: size.value].copy()


def spp_decode_labels(kind: str, d_src_ptrs: int, n: int, d_dst: int, H: int, W: int, status: int = 0,
                      src_bytes: int = 0, stream: int = 0):
    """Raw call: device pointer table of n label streams -> u8 [n][H][W] (mask) or fp32 [n][W] (vector)."""
    _check(load().spp_decode_labels(LABEL_KIND[kind], d_src_ptrs, src_bytes or None, n, d_dst, H, W, status or None,
                                    stream), "spp_decode_labels")
