"""CPU oracle for the decode+preprocess hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product (``paper_conf_ipps_ibrahimo22_b200``) never imports it, and the two
share no code.  The arithmetic lives in ``spp_oracle.c`` (plain C, single
thread, ``-O2 -ffp-contract=off``, no FTZ/DAZ); this module only marshals numpy
arrays through ctypes.  Every function cites the FORMAT.md / PAPER.md passage
it follows in ``spp_oracle.c``; the pins are ``tests/test_oracle_pins.py``.
"""
from __future__ import annotations

import ctypes as C
import subprocess
from pathlib import Path

import numpy as np

_HERE = Path(__file__).resolve().parent
SRC = _HERE / "spp_oracle.c"
LIB = _HERE / "liboracle.so"
CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11", "-Wall", "-Wextra",
          "-shared", "-fPIC"]

OUT = {"f16": 1, "f32": 2, "i16": 3}
_DT = {"f16": np.float16, "f32": np.float32, "i16": np.int16}
ERR = {0: "ok", 1: "invalid argument", 2: "buffer too small", 3: "corrupt stream"}


class OracleError(RuntimeError):
    def __init__(self, rc: int, what: str):
        super().__init__(f"{what}: {ERR.get(rc, rc)}")
        self.rc = rc


def build(force: bool = False) -> Path:
    """Compile the oracle with gcc (building the checker is not using it)."""
    if force or not LIB.exists() or LIB.stat().st_mtime < SRC.stat().st_mtime:
        tmp = LIB.with_suffix(".so.tmp")
        subprocess.run(["gcc", *CFLAGS, "-o", str(tmp), str(SRC), "-lm"], check=True)
        tmp.replace(LIB)
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(str(LIB))
        P, I, I64, SZ = C.c_void_p, C.c_int, C.c_int64, C.c_size_t
        L.orc_f32_to_f16.argtypes = [C.c_float]; L.orc_f32_to_f16.restype = C.c_uint16
        L.orc_f32_to_f16_array.argtypes = [P, I64, P]; L.orc_f32_to_f16_array.restype = None
        L.orc_cosmo_f32.argtypes = [I]; L.orc_cosmo_f32.restype = C.c_float
        L.orc_cosmo_direct.argtypes = [P, I64, I, I, P]; L.orc_cosmo_direct.restype = I
        L.orc_cosmo_max_encoded_size.argtypes = [I, I, I]; L.orc_cosmo_max_encoded_size.restype = SZ
        L.orc_cosmo_encode.argtypes = [P, I, I, I, P, SZ, C.POINTER(SZ)]; L.orc_cosmo_encode.restype = I
        L.orc_cosmo_encode_ex.argtypes = [P, I, I, I, I, P, SZ, C.POINTER(SZ)]; L.orc_cosmo_encode_ex.restype = I
        L.orc_cosmo_decode.argtypes = [P, SZ, I, I, P, I, I, I, I]; L.orc_cosmo_decode.restype = I
        L.orc_deepcam_code.argtypes = [I]; L.orc_deepcam_code.restype = I
        L.orc_deepcam_decode_line.argtypes = [P, SZ, I, P]; L.orc_deepcam_decode_line.restype = I
        L.orc_deepcam_decode.argtypes = [P, SZ, P, P, I, P, I, I, I]; L.orc_deepcam_decode.restype = I
        L.orc_deepcam_max_encoded_size.argtypes = [I, I, I]; L.orc_deepcam_max_encoded_size.restype = SZ
        L.orc_deepcam_encode.argtypes = [P, I, I, I, P, SZ, C.POINTER(SZ)]; L.orc_deepcam_encode.restype = I
        L.orc_deepcam_encode_a.argtypes = [P, I, I, I, I, P, SZ, C.POINTER(SZ)]; L.orc_deepcam_encode_a.restype = I
        L.orc_deepcam_encode_p.argtypes = [P, I, I, I, I, I, I, P, SZ, C.POINTER(SZ)]
        L.orc_deepcam_encode_p.restype = I
        L.orc_deepcam_encode_q.argtypes = [P, I, I, I, I, I, I, C.c_float, I, P, SZ, C.POINTER(SZ)]
        L.orc_deepcam_encode_q.restype = I
        L.orc_deepcam_encode_r.argtypes = [P, I, I, I, I, I, I, C.c_float, I, I, P, SZ, C.POINTER(SZ)]
        L.orc_deepcam_encode_r.restype = I
        L.orc_deepcam_encode_s.argtypes = [P, I, I, I, I, I, I, C.c_float, I, I, I, P, SZ, C.POINTER(SZ)]
        L.orc_deepcam_encode_s.restype = I
        L.orc_deepcam_encode_t.argtypes = [P, I, I, I, I, I, I, C.c_float, I, I, I, P, P, P, SZ, C.POINTER(SZ)]
        L.orc_deepcam_encode_t.restype = I
        L.orc_label_max_encoded_size.argtypes = [I, I, I]; L.orc_label_max_encoded_size.restype = SZ
        L.orc_label_encode_mask.argtypes = [P, I, I, P, SZ, C.POINTER(SZ)]; L.orc_label_encode_mask.restype = I
        L.orc_label_encode_vector.argtypes = [P, I, P, SZ, C.POINTER(SZ)]; L.orc_label_encode_vector.restype = I
        L.orc_label_decode.argtypes = [P, SZ, I, I, I, P]; L.orc_label_decode.restype = I
        L.orc_f16_to_f32.argtypes = [C.c_uint16]; L.orc_f16_to_f32.restype = C.c_float
        L.orc_deepcam_align.argtypes = [I]; L.orc_deepcam_align.restype = I
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _check(rc: int, what: str):
    if rc != 0:
        raise OracleError(rc, what)


def f32_to_f16(x) -> np.ndarray:
    """RNE binary32 -> binary16 bit patterns (uint16)."""
    a = np.ascontiguousarray(x, dtype=np.float32)
    out = np.empty(a.shape, dtype=np.uint16)
    lib().orc_f32_to_f16_array(_p(a), a.size, _p(out))
    return out


def cosmo_f32(count: int) -> float:
    return float(np.float32(lib().orc_cosmo_f32(int(count))))


def cosmo_transform_table() -> np.ndarray:
    """fp32 RN(ln(1+c)) for every c in [0, 32767]."""
    return np.array([lib().orc_cosmo_f32(c) for c in range(32768)], dtype=np.float32)


def cosmo_direct(counts: np.ndarray, transform: int = 1, out: str = "f16") -> np.ndarray:
    a = np.ascontiguousarray(counts, dtype=np.int16)
    o = np.empty(a.shape, dtype=_DT[out])
    _check(lib().orc_cosmo_direct(_p(a), a.size, transform, OUT[out], _p(o)), "cosmo_direct")
    return o


def cosmo_encode(counts: np.ndarray, localize: bool = False, escape: bool = False) -> np.ndarray:
    """FORMAT.md 1.3 encoder; `localize` selects the 1.4 localized-table
    policy, `escape` the 1.5 escaped 1-byte keys."""
    a = np.ascontiguousarray(counts, dtype=np.int16)
    assert a.ndim == 4 and a.shape[0] == 4
    _, D, H, W = a.shape
    cap = lib().orc_cosmo_max_encoded_size(D, H, W)
    dst = np.zeros(cap, dtype=np.uint8)
    size = C.c_size_t(0)
    _check(lib().orc_cosmo_encode_ex(_p(a), D, H, W, int(localize) | (2 if escape else 0), _p(dst), cap,
                                     C.byref(size)),
           "cosmo_encode")
    return dst[: size.value].copy()


def cosmo_decode(stream: np.ndarray, shape, transform: int = 1, out: str = "f16") -> np.ndarray:
    s = np.ascontiguousarray(stream, dtype=np.uint8)
    Cc, D, H, W = shape
    o = np.empty((Cc, D, H, W), dtype=_DT[out])
    _check(lib().orc_cosmo_decode(_p(s), s.size, transform, OUT[out], _p(o), Cc, D, H, W), "cosmo_decode")
    return o


def deepcam_code(b: int) -> int:
    return int(lib().orc_deepcam_code(int(b)))


def f16_to_f32(h: int) -> float:
    return float(lib().orc_f16_to_f32(int(h)))


def deepcam_encode(x: np.ndarray, align: int | None = None, lookahead: int = 64, repeat_min: int = 16,
                   rel_err: float = 0.1, err_budget: int = 0, raw16: bool = False,
                   raw_segments: bool = False, repeat_tol=None, max_abs_err=None) -> np.ndarray:
    """FORMAT.md 2.4 encoder; `align` overrides the default alignment rule,
    `lookahead` / `repeat_min` the policy knobs (defaults 64 / 16);
    `err_budget` > 0 applies the FORMAT.md 2.5 error budget (a SEG line with
    that many values above `rel_err` relative error is written RAW);
    `repeat_tol` / `max_abs_err` (fp32[C] or None) the FORMAT.md 2.8 per-channel
    REPEAT tolerance and absolute error bound."""
    a = np.ascontiguousarray(x, dtype=np.float32)
    assert a.ndim == 3
    Cc, H, W = a.shape
    cap = lib().orc_deepcam_max_encoded_size(Cc, H, W)
    dst = np.zeros(cap, dtype=np.uint8)
    size = C.c_size_t(0)
    A = lib().orc_deepcam_align(W) if align is None else int(align)
    rt = None if repeat_tol is None else np.ascontiguousarray(repeat_tol, dtype=np.float32)
    me = None if max_abs_err is None else np.ascontiguousarray(max_abs_err, dtype=np.float32)
    assert rt is None or rt.shape == (Cc,)
    assert me is None or me.shape == (Cc,)
    _check(lib().orc_deepcam_encode_t(_p(a), Cc, H, W, A, int(lookahead), int(repeat_min), float(rel_err),
                                      int(err_budget), int(bool(raw16)), int(bool(raw_segments)),
                                      None if rt is None else _p(rt), None if me is None else _p(me), _p(dst), cap,
                                      C.byref(size)), "deepcam_encode")
    return dst[: size.value].copy()


def deepcam_decode_line(stream: np.ndarray, line: int, W: int) -> np.ndarray:
    s = np.ascontiguousarray(stream, dtype=np.uint8)
    o = np.empty(W, dtype=np.float32)
    _check(lib().orc_deepcam_decode_line(_p(s), s.size, int(line), _p(o)), "deepcam_decode_line")
    return o


def deepcam_decode(stream: np.ndarray, shape, shift=None, scale=None, out: str = "f16") -> np.ndarray:
    s = np.ascontiguousarray(stream, dtype=np.uint8)
    Cc, H, W = shape
    o = np.empty((Cc, H, W), dtype=_DT[out])
    sh = None if shift is None else np.ascontiguousarray(shift, dtype=np.float32)
    sc = None if scale is None else np.ascontiguousarray(scale, dtype=np.float32)
    _check(lib().orc_deepcam_decode(_p(s), s.size, None if sh is None else _p(sh),
                                    None if sc is None else _p(sc), OUT[out], _p(o), Cc, H, W),
           "deepcam_decode")
    return o


# ---------------------------------------------------------------- labels (FORMAT.md 3)
def label_encode_mask(m: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(m, dtype=np.uint8)
    assert a.ndim == 2
    H, W = a.shape
    cap = lib().orc_label_max_encoded_size(1, H, W)
    dst = np.zeros(cap, dtype=np.uint8)
    size = C.c_size_t(0)
    _check(lib().orc_label_encode_mask(_p(a), H, W, _p(dst), cap, C.byref(size)), "label_encode_mask")
    return dst[: size.value].copy()


def label_encode_vector(v: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(v, dtype=np.float32).ravel()
    cap = lib().orc_label_max_encoded_size(2, 1, a.size)
    dst = np.zeros(cap, dtype=np.uint8)
    size = C.c_size_t(0)
    _check(lib().orc_label_encode_vector(_p(a), a.size, _p(dst), cap, C.byref(size)), "label_encode_vector")
    return dst[: size.value].copy()


def label_decode(stream: np.ndarray, kind: int, H: int, W: int) -> np.ndarray:
    s = np.ascontiguousarray(stream, dtype=np.uint8)
    o = np.empty((H, W), dtype=np.uint8) if kind == 1 else np.empty(W, dtype=np.float32)
    _check(lib().orc_label_decode(_p(s), s.size, int(kind), int(H), int(W), _p(o)), "label_decode")
    return o
