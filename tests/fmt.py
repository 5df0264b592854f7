"""Test-side readers of the FORMAT.md byte layouts (struct unpacking only).

These parse headers/tables so tests can check encoder output against brute
force (set cardinalities, orderings); they hold no decode arithmetic.
"""
import struct

import numpy as np


def cosmo_header(b: np.ndarray):
    raw = bytes(b[:64])
    magic, ver, flags, C, D, H, W, nU, T, U_off, slab_off, total = struct.unpack_from(
        "<IHHHHHHIIQQQ", raw, 0)
    U = np.frombuffer(bytes(b[U_off:U_off + 2 * nU]), dtype="<i2")
    slabs = []
    for t in range(T):
        z0, z1, G, kw, lut_off, keys_off = struct.unpack_from("<IIIB3xQQ", bytes(b[slab_off + 32 * t: slab_off + 32 * t + 32]), 0)
        slabs.append(dict(z0=z0, z1=z1, G=G, kw=kw, lut_off=lut_off, keys_off=keys_off))
    return dict(magic=magic, ver=ver, C=C, D=D, H=H, W=W, nU=nU, T=T, U=U, slabs=slabs,
                U_off=U_off, slab_off=slab_off, total=total)


def cosmo_lut(b, slab):
    G = slab["G"]
    return np.frombuffer(bytes(b[slab["lut_off"]:slab["lut_off"] + 8 * G]), dtype="<u2").reshape(G, 4)


def cosmo_keys(b, slab, Nt):
    kw = slab["kw"]
    if kw == 0:
        return np.zeros(Nt, dtype=np.int64)
    if kw == 8:
        return np.frombuffer(bytes(b[slab["keys_off"]:slab["keys_off"] + 8 * Nt]), dtype="<u2").reshape(4, Nt)
    dt = "<u1" if kw == 1 else "<u2"
    return np.frombuffer(bytes(b[slab["keys_off"]:slab["keys_off"] + kw * Nt]), dtype=dt).astype(np.int64)


def deepcam_header(b: np.ndarray):
    raw = bytes(b[:64])
    magic, ver, flags, C, H, W, A, L, res, dir_off, payload_off, total = struct.unpack_from(
        "<IHHHHHHIIQQQ", raw, 0)
    d = np.frombuffer(bytes(b[dir_off:dir_off + 4 * (L + 1)]), dtype="<u4")
    return dict(magic=magic, ver=ver, C=C, H=H, W=W, A=A, L=L, dir=d, dir_off=dir_off,
                payload_off=payload_off, total=total)


def deepcam_line(b, hdr, l):
    a, e = int(hdr["dir"][l]), int(hdr["dir"][l + 1])
    p = bytes(b[hdr["payload_off"] + a: hdr["payload_off"] + e])
    if p[0] in (0, 2):                 # RAW (fp32) / RAW16 (FORMAT.md 2.6)
        return dict(mode=int(p[0]), size=len(p))
    nseg = struct.unpack_from("<H", p, 2)[0]
    segs = []
    for s in range(nseg):
        ln, kind, eb = struct.unpack_from("<HBB", p, 4 + 4 * s)
        h = struct.unpack_from("<f", p, 4 + 4 * nseg + 4 * s)[0]
        segs.append(dict(len=ln, kind=kind, emin_b=eb, emin=eb - 150, head=np.float32(h)))
    return dict(mode=int(p[0]), size=len(p), nseg=nseg, segs=segs, delta=p[4 + 8 * nseg:])


def build_seg_line(W, segs, deltas, mode=1):
    """Assemble one SEG line payload by hand (FORMAT.md 2.1).  segs: list of
    (len, kind, emin_b, head_f32); deltas: the delta-area bytes (DIFF codes;
    with mode 3 also the binary32 values of RAW segments, FORMAT.md 2.7)."""
    n = len(segs)
    out = bytearray(struct.pack("<BBH", mode, 0, n))
    for ln, kind, eb, _ in segs:
        out += struct.pack("<HBB", ln, kind, eb)
    for _, _, _, h in segs:
        out += struct.pack("<f", float(np.float32(h)))
    out += bytes(deltas)
    out += b"\0" * ((-len(out)) % 16)
    return bytes(out)


def build_raw_line(x):
    out = bytearray(b"\0" * 16)
    out += np.asarray(x, dtype="<f4").tobytes()
    out += b"\0" * ((-len(out)) % 16)
    return bytes(out)


def build_deepcam_stream(C, H, W, lines, A=1):
    """Assemble a whole DeepCAM stream from per-line payloads (FORMAT.md 2.1);
    A is the declared segment alignment."""
    L = C * H
    assert len(lines) == L
    dir_off = 64
    payload_off = dir_off + 4 * (L + 1)
    payload_off += (-payload_off) % 16
    offs = [0]
    for ln in lines:
        offs.append(offs[-1] + len(ln))
    total = payload_off + offs[-1]
    hdr = struct.pack("<IHHHHHHIIQQQ", 0x44505053, 1, 0, C, H, W, A, L, 0, dir_off, payload_off, total)
    hdr += b"\0" * 16
    body = bytearray(hdr)
    body += np.asarray(offs, dtype="<u4").tobytes()
    body += b"\0" * (payload_off - len(body))
    for ln in lines:
        body += ln
    return np.frombuffer(bytes(body), dtype=np.uint8).copy()


def label_header(b: np.ndarray):
    """FORMAT.md 3 label stream header and (kind 1) row directory."""
    raw = bytes(b[:32])
    magic, ver, kind, H, W, _res, total = struct.unpack_from("<IHHHHIQ", raw, 0)
    d = dict(magic=magic, ver=ver, kind=kind, H=H, W=W, total=total)
    if kind == 1:
        d["dir"] = np.frombuffer(bytes(b[32:32 + 4 * (H + 1)]), dtype="<u4")
        d["payload_off"] = 32 + ((4 * (H + 1) + 15) // 16) * 16
    return d


def label_row(b, hdr, y):
    a, e = int(hdr["dir"][y]), int(hdr["dir"][y + 1])
    p = bytes(b[hdr["payload_off"] + a: hdr["payload_off"] + e])
    if p[0] == 0:
        return dict(mode=0, size=len(p))
    nrun = struct.unpack_from("<H", p, 2)[0]
    lens = np.frombuffer(p[4:4 + 2 * nrun], dtype="<u2")
    vals = np.frombuffer(p[4 + 2 * nrun:4 + 3 * nrun], dtype=np.uint8)
    return dict(mode=1, size=len(p), nrun=nrun, lens=lens, vals=vals)
