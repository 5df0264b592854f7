"""Pins of the CPU oracle to things other than itself (no GPU needed).

Each test names what fixes the expected value: IEEE-754 exact arithmetic
(Fractions), a library routine (numpy float16 conversion, mpmath), brute force
over sets on tiny inputs, closed forms from the paper, or special cases.
PAPER.md lines are cited as P:<n>; readings S<n> are listed in DESIGN.md.
"""
import json
import struct
from fractions import Fraction
from pathlib import Path

import mpmath
import numpy as np
import pytest

from tests import exact, fmt

GOLDEN = Path(__file__).parent / "golden"


# --------------------------------------------------------------------------
# binary32 -> binary16 RNE (FORMAT.md 1.2 / 2.3 emission; P:110 FP16 samples)
# pinned against numpy's conversion (library routine)

def test_f16_conversion_matches_numpy(orc):
    rng = np.random.default_rng(7)
    bits = rng.integers(0, 2**32, size=400_000, dtype=np.uint64).astype(np.uint32)
    # every half value, its neighbours' midpoints and +-1 binary32 ulp around them
    h = np.arange(0, 0x7C00, dtype=np.uint16).view(np.float16).astype(np.float32)
    mids = ((h[:-1].astype(np.float64) + h[1:].astype(np.float64)) / 2).astype(np.float32)
    extra = np.concatenate([h, mids, np.nextafter(mids, np.float32(np.inf)),
                            np.nextafter(mids, np.float32(0)), np.float32([65504, 65519.99, 65520, 7e4, 1e-8,
                                                                           2**-25, 2**-24, 3 * 2**-26, np.inf])])
    x = np.concatenate([bits.view(np.float32), extra, -extra])
    got = orc.f32_to_f16(x)
    with np.errstate(over="ignore"):
        ref = x.astype(np.float16).view(np.uint16)
    nan = np.isnan(x)
    assert np.array_equal(got[~nan], ref[~nan])
    assert np.all(np.isnan(got[nan].view(np.float16)))


# --------------------------------------------------------------------------
# CosmoFlow transform: RN_f32(ln(1+c)) (readings S1/S2), exhaustive vs mpmath

def _mp_f32_log1p(c: int) -> np.float32:
    with mpmath.workprec(200):
        v = mpmath.log1p(c)
        m, e = mpmath.mpf(v).man_exp
        q = Fraction(int(m)) * (Fraction(2) ** int(e)) if e >= 0 else Fraction(int(m), 2 ** (-int(e)))
    return exact.to_f32(q), q


def test_cosmo_transform_exhaustive_mpmath(orc):
    table = orc.cosmo_transform_table()
    bad = []
    for c in range(32768):
        ref, _ = _mp_f32_log1p(c)
        if table[c].view(np.uint32) != ref.view(np.uint32):
            bad.append(c)
    assert bad == []
    # fp16 = RNE_f16(the fp32 value) ("casting to FP16")
    f16 = orc.f32_to_f16(table).view(np.float16)
    for c in (0, 1, 2, 100, 558, 10363, 15316, 32767):
        assert f16[c] == exact.to_f16(Fraction(float(table[c])))


def test_cosmo_fp16_double_rounding_cases(orc):
    """Reading S2: fp16 is rounded from the fp32 value.  At these counts that
    differs from rounding the exact logarithm directly (documented cases)."""
    found = []
    table = orc.cosmo_transform_table()
    f16 = orc.f32_to_f16(table).view(np.float16)
    for c in range(32768):
        _, q = _mp_f32_log1p(c)
        if exact.to_f16(q) != f16[c]:
            found.append(c)
    golden = json.loads((GOLDEN / "cosmo_fp16_double_rounding.json").read_text())
    assert found == golden["counts"]


def test_cosmo_direct_special_values(orc):
    x = np.array([0, 1, 2, 3, 32767], dtype=np.int16)
    f32 = orc.cosmo_direct(x, 1, "f32")
    assert f32[0] == 0.0 and f32.view(np.uint32)[0] == 0          # ln(1) = +0 exactly
    assert f32[1] == np.float32(np.log(2.0))                      # RN(ln 2)
    assert orc.cosmo_direct(x, 0, "i16").tolist() == x.tolist()   # identity
    assert orc.cosmo_direct(x, 0, "f32").tolist() == [0, 1, 2, 3, 32767]
    with pytest.raises(orc.OracleError):
        orc.cosmo_direct(np.array([-1], dtype=np.int16), 1, "f32")   # reading S7


# --------------------------------------------------------------------------
# CosmoFlow LUT format: brute force over sets on tiny volumes

def _tiny_volumes():
    rng = np.random.default_rng(11)
    vols = []
    for n in (1, 2, 3, 4, 8):
        vols.append(rng.integers(0, 5, size=(4, n, n, n)).astype(np.int16))      # few values
        vols.append((rng.pareto(1.5, size=(4, n, n, n)) * 3).astype(np.int16))  # power-law
    vols.append(np.zeros((4, 5, 3, 2), dtype=np.int16))                         # all equal -> kw 0
    vols.append(np.full((4, 6, 4, 4), 7, dtype=np.int16))
    v = rng.integers(0, 3, size=(1, 6, 5, 7)).astype(np.int16)
    vols.append(np.concatenate([v, v + 1, v * 2, v], axis=0))                   # fully coupled
    vols.append(np.arange(4 * 4 * 4 * 4, dtype=np.int16).reshape(4, 4, 4, 4))   # all distinct
    return vols


@pytest.mark.parametrize("vi", range(14))
def test_cosmo_encoder_bruteforce_tiny(orc, vi):
    x = _tiny_volumes()[vi]
    b = orc.cosmo_encode(x)
    h = fmt.cosmo_header(b)
    _, D, H, W = x.shape
    N = D * H * W
    assert h["magic"] == 0x43505053 and h["ver"] == 1 and (h["C"], h["D"], h["H"], h["W"]) == (4, D, H, W)
    assert h["total"] == b.size and b.size % 16 == 0
    # |U| = |set of values|, U ascending
    assert h["U"].tolist() == sorted(set(x.ravel().tolist()))
    Uidx = {v: i for i, v in enumerate(h["U"].tolist())}
    flat = x.reshape(4, N)
    assert h["T"] == 1  # tiny volumes never need a split
    s = h["slabs"][0]
    tuples = [tuple(Uidx[int(flat[c, v])] for c in range(4)) for v in range(N)]
    G = len(set(tuples))
    if s["kw"] == 8:
        assert 8 * G + (0 if G == 1 else (1 if G <= 256 else 2)) * N >= 8 * N
        raw = fmt.cosmo_keys(b, s, N)
        assert [tuple(int(raw[c, v]) for c in range(4)) for v in range(N)] == tuples
    else:
        assert s["G"] == G
        assert s["kw"] == (0 if G == 1 else (1 if G <= 256 else 2))
        lut = [tuple(int(t) for t in row) for row in fmt.cosmo_lut(b, s)]
        assert sorted(lut) == sorted(set(tuples))
        freq = {t: tuples.count(t) for t in set(tuples)}
        assert lut == sorted(set(tuples), key=lambda t: (-freq[t], t))   # FORMAT.md 1.3 step 4
        keys = fmt.cosmo_keys(b, s, N)
        assert [lut[int(k)] for k in keys] == tuples
    # lossless round trip against the plain definition
    for out in ("f32", "f16"):
        dec = orc.cosmo_decode(b, x.shape, 1, out)
        ref = orc.cosmo_direct(x, 1, out)
        assert dec.tobytes() == ref.tobytes()
    assert np.array_equal(orc.cosmo_decode(b, x.shape, 0, "i16"), x)


def test_cosmo_slab_split_and_raw_escape(orc):
    rng = np.random.default_rng(5)
    # ~2 x 65536 distinct groups over 8 planes of 128x128, coupled enough that a
    # half-volume fits 16-bit keys: split into slabs, each kw = 2
    D, H, W = 8, 128, 128
    N = D * H * W
    base = rng.integers(0, 150000, size=N)  # group id per voxel
    g = np.array([base % 7, (base // 7) % 11, (base // 77) % 13, (base // 1001) % 151], dtype=np.int16)
    # confine ids per half so each half has <= 65536 groups
    half = N // 2
    ids = np.concatenate([rng.integers(0, 60000, size=half), rng.integers(60000, 120000, size=half)])
    g = np.array([ids % 7, (ids // 7) % 11, (ids // 77) % 13, (ids // 1001) % 151], dtype=np.int16).reshape(4, D, H, W)
    b = orc.cosmo_encode(g)
    h = fmt.cosmo_header(b)
    assert h["T"] >= 2
    assert [(s["z0"], s["z1"]) for s in h["slabs"]][0][0] == 0 and h["slabs"][-1]["z1"] == D
    for s in h["slabs"]:
        assert s["kw"] in (2, 8) and s["G"] <= 65536
    assert np.array_equal(orc.cosmo_decode(b, g.shape, 0, "i16"), g)
    # dense independent volume: LUT would not save space -> RAW escape (kw 8)
    y = rng.integers(0, 200, size=(4, 2, 64, 64)).astype(np.int16)
    hb = orc.cosmo_encode(y)
    hh = fmt.cosmo_header(hb)
    assert all(s["kw"] == 8 and s["G"] == 0 for s in hh["slabs"])
    assert orc.cosmo_decode(hb, y.shape, 1, "f32").tobytes() == orc.cosmo_direct(y, 1, "f32").tobytes()


def _localized_volumes():
    """Tiny volumes whose groups are local in z ("localized lookup
    tables"): per-block palettes, a constant block, a dense random block,
    odd depths (unequal halves)."""
    rng = np.random.default_rng(11)
    vols = []
    for D, H, W, blk, pal in [(8, 8, 8, 2, 100), (8, 16, 16, 4, 200), (7, 8, 8, 1, 45), (6, 12, 12, 3, 150),
                              (16, 8, 8, 2, 90), (8, 16, 16, 8, 300)]:
        planes = []
        for z0 in range(0, D, blk):
            n = min(blk, D - z0) * H * W
            base = 1000 * (z0 // blk)
            gid = base + rng.integers(0, pal, size=n)
            planes.append(np.array([gid % 97, gid % 89, gid // 89, gid % 13], dtype=np.int16)
                          .reshape(4, min(blk, D - z0), H, W))
        vols.append(np.concatenate(planes, axis=1))
    v = vols[1].copy()
    v[:, :2] = 5                                                     # a constant slab (kw 0)
    v[:, 6:] = rng.integers(0, 3000, size=(4, 2, 16, 16))            # dense: RAW escape
    vols.append(v)
    vols.append(rng.integers(0, 3, size=(4, 5, 4, 4)).astype(np.int16))
    return vols


def _dyadic_partitions(z0, z1):
    yield [(z0, z1)]
    if z1 - z0 > 1:
        mid = z0 + (z1 - z0) // 2
        for a in _dyadic_partitions(z0, mid):
            for b in _dyadic_partitions(mid, z1):
                yield a + b


@pytest.mark.parametrize("vi", range(8))
def test_cosmo_localized_tables_bruteforce(orc, vi):
    """FORMAT.md 1.4: the localized stream is the
    byte-smallest of ALL dyadic z-partitions, each slab laid out by FORMAT.md
    1.1/1.3 (sizes counted here from brute-force group sets), never larger
    than the default policy, and decodes losslessly."""
    x = _localized_volumes()[vi]
    _, D, H, W = x.shape
    up16 = lambda v: (v + 15) // 16 * 16
    plane = H * W
    flat = x.reshape(4, D * plane)
    Uidx = {v: i for i, v in enumerate(sorted(set(x.ravel().tolist())))}
    tup = [tuple(Uidx[int(flat[c, v])] for c in range(4)) for v in range(D * plane)]

    def slab_layout(z0, z1):
        Nt = (z1 - z0) * plane
        G = len(set(tup[z0 * plane: z1 * plane]))
        kw = 0 if G == 1 else (1 if G <= 256 else 2)
        if G > 65536 or 8 * G + kw * Nt >= 8 * Nt:
            return 32 + up16(8 * Nt), 8
        return 32 + up16(8 * G) + (up16(kw * Nt) if kw else 0), kw

    head = 64 + up16(2 * len(Uidx))
    costs = {tuple(p): sum(slab_layout(*r)[0] for r in p) for p in _dyadic_partitions(0, D)}
    best = min(costs.values())
    b = orc.cosmo_encode(x, localize=True)
    h = fmt.cosmo_header(b)
    part = tuple((s["z0"], s["z1"]) for s in h["slabs"])
    assert b.size == h["total"] == head + best
    assert costs[part] == best
    # the whole slab is kept when splitting does not strictly save bytes
    assert not (len(part) > 1 and costs[((0, D),)] == best)
    for s in h["slabs"]:
        assert s["kw"] == slab_layout(s["z0"], s["z1"])[1]
    assert b.size <= orc.cosmo_encode(x).size
    assert np.array_equal(orc.cosmo_decode(b, x.shape, 0, "i16"), x)
    assert orc.cosmo_decode(b, x.shape, 1, "f16").tobytes() == orc.cosmo_direct(x, 1, "f16").tobytes()


def test_cosmo_localized_tables_take_one_byte_keys(orc):
    """Sparse paper-like volume (few hundred groups overall, < 256 per 16-plane
    slab): localized slabs take 1-byte keys and the stream shrinks ~2x."""
    from synth import gen_cosmo
    x = gen_cosmo(3001, "sparse")
    a, b = orc.cosmo_encode(x), orc.cosmo_encode(x, localize=True)
    ha, hb = fmt.cosmo_header(a), fmt.cosmo_header(b)
    assert ha["T"] == 1 and ha["slabs"][0]["kw"] == 2
    assert hb["T"] > 1 and all(s["kw"] in (0, 1) for s in hb["slabs"])
    assert b.size < 0.55 * a.size
    assert np.array_equal(orc.cosmo_decode(b, x.shape, 0, "i16"), x)


@pytest.mark.parametrize("vi", [0, 1, 3, 5, 6])
def test_cosmo_escaped_keys_layout_bruteforce(orc, vi):
    """FORMAT.md 1.5 escaped keys, pinned by brute force: on volumes with more
    than 256 groups the slab's keys are the frequency ranks of FORMAT.md 1.3
    step 4; ranks < 255 sit in the low bytes, the rest (low byte 255) in the
    escape list in voxel order, eidx[b] counts the escapes before block b; the
    layout is chosen only when smaller than 2-byte keys; decoding is lossless."""
    rng = np.random.default_rng(20 + vi)
    D, H, W = (8, 16, 16) if vi < 5 else (6, 16, 24)      # 2304 voxels: a partial last block
    n = D * H * W
    # a hot set of ~100 groups and a uniform tail (vi 6: mostly tail, so 2-byte keys win)
    hot_frac = 0.15 if vi == 6 else 0.5 + 0.08 * vi
    tail = 1000 if vi == 6 else 3000
    gid = np.where(rng.random(n) < hot_frac, rng.integers(0, 100, size=n), rng.integers(100, 100 + tail, size=n))
    x = np.array([gid % 31, gid // 31, (gid * 7) % 13, gid % 5], dtype=np.int16).reshape(4, D, H, W)
    b = orc.cosmo_encode(x, escape=True)
    h = fmt.cosmo_header(b)
    assert h["T"] == 1
    s = h["slabs"][0]
    Uidx = {v: i for i, v in enumerate(h["U"].tolist())}
    flat = x.reshape(4, n)
    tuples = [tuple(Uidx[int(flat[c, v])] for c in range(4)) for v in range(n)]
    freq = {t: tuples.count(t) for t in set(tuples)}
    order = sorted(freq, key=lambda t: (-freq[t], t))
    rank = {t: i for i, t in enumerate(order)}
    keys = [rank[t] for t in tuples]
    up16 = lambda v: (v + 15) // 16 * 16
    nb = (n + 255) // 256
    n_esc = sum(k >= 255 for k in keys)
    esc_bytes = up16(4 * (nb + 1)) + up16(n) + up16(2 * n_esc)
    assert len(order) > 256
    if esc_bytes < up16(2 * n):
        assert s["kw"] == 3
        raw = bytes(b[s["keys_off"]:])
        eidx = np.frombuffer(raw[:4 * (nb + 1)], dtype="<u4")
        low = np.frombuffer(raw[up16(4 * (nb + 1)):][:n], dtype=np.uint8)
        esc = np.frombuffer(raw[up16(4 * (nb + 1)) + up16(n):][:2 * n_esc], dtype="<u2")
        assert low.tolist() == [min(k, 255) for k in keys]
        assert esc.tolist() == [k for k in keys if k >= 255]
        assert eidx.tolist() == [sum(k >= 255 for k in keys[:256 * i]) for i in range(nb)] + [n_esc]
        lut = [tuple(int(t) for t in row) for row in fmt.cosmo_lut(b, s)]
        assert lut == order
    else:
        assert s["kw"] == 2
    assert np.array_equal(orc.cosmo_decode(b, x.shape, 0, "i16"), x)
    assert orc.cosmo_decode(b, x.shape, 1, "f16").tobytes() == orc.cosmo_direct(x, 1, "f16").tobytes()
    # a wrong block count is corruption
    if s["kw"] == 3 and nb > 1:
        bad = b.copy()
        o = s["keys_off"] + 4
        bad[o:o + 4] = np.frombuffer(np.uint32(int(np.frombuffer(bytes(b[o:o + 4]), "<u4")[0]) + 1).tobytes(), np.uint8)
        with pytest.raises(Exception):
            orc.cosmo_decode(bad, x.shape, 0, "i16")


def test_cosmo_escaped_keys_paper_ratio(orc):
    """On the paper-shaped generator the escaped layout beats gzip's ~5x
     where the paper's 2-byte keys give ~3.7x; lossless."""
    from synth import gen_cosmo
    x = gen_cosmo(1001)
    a, b = orc.cosmo_encode(x), orc.cosmo_encode(x, escape=True)
    assert 3.6 < x.nbytes / a.size < 3.8 and x.nbytes / b.size > 5.0
    assert fmt.cosmo_header(b)["slabs"][0]["kw"] == 3
    assert np.array_equal(orc.cosmo_decode(b, x.shape, 0, "i16"), x)


def test_cosmo_size_closed_form_and_paper_ratio(orc):
    """P:98 'compression factor of roughly 4x' vs gzip 5x; P:219 gzip files are
    'roughly 75%' of ours.  Layout size = 64 + up16(2|U|) + 32 + up16(8G) + 2N."""
    paper = json.loads((GOLDEN / "paper_numbers.json").read_text())
    up16 = lambda v: (v + 15) // 16 * 16
    N = 128 ** 3
    G, nU = paper["cosmo_example_groups"]["value"], paper["cosmo_example_unique_values"]["value"]
    size = 64 + up16(2 * nU) + 32 + up16(8 * G) + 2 * N
    ratio = 4 * N * 2 / size
    assert 3.6 < ratio < 4.0                                   # "roughly 4x"
    assert 0.70 < ratio / paper["gzip_ratio"]["value"] < 0.80   # "roughly 75%"
    # the oracle's encoder produces exactly the closed-form size
    rng = np.random.default_rng(3)
    D = H = W = 16
    n = D * H * W
    gid = rng.integers(0, 300, size=n)
    gid[:300] = np.arange(300)          # every group present: G = 300 -> kw = 2
    vol = np.array([gid % 5, gid % 7, gid // 5, gid // 7], dtype=np.int16).reshape(4, D, H, W)
    b = orc.cosmo_encode(vol)
    h = fmt.cosmo_header(b)
    nU2 = len(set(vol.ravel().tolist()))
    assert h["slabs"][0]["G"] == 300 and h["slabs"][0]["kw"] == 2
    assert b.size == 64 + up16(2 * nU2) + 32 + up16(8 * 300) + up16(2 * n)


def test_cosmo_paper_shaped_sample(orc):
    """Generator 'paper' preset lands near the paper's example (Fig. 5):
    hundreds of unique values, tens of thousands of 4-groups, 2-byte keys."""
    from synth import gen_cosmo
    x = gen_cosmo(1001)
    b = orc.cosmo_encode(x)
    h = fmt.cosmo_header(b)
    assert 300 <= h["nU"] <= 1500
    assert h["T"] == 1 and 10_000 <= h["slabs"][0]["G"] <= 65_536 and h["slabs"][0]["kw"] == 2
    assert 3.4 < x.nbytes / b.size < 4.2
    assert orc.cosmo_decode(b, x.shape, 1, "f16").tobytes() == orc.cosmo_direct(x, 1, "f16").tobytes()


def test_cosmo_decoder_rejects_corruption(orc):
    x = _tiny_volumes()[6]
    b = orc.cosmo_encode(x)
    for off, val in ((0, 0x00), (4, 0x02), (20, 0x00), (8, 0x03)):
        c = b.copy(); c[off] = val
        with pytest.raises(orc.OracleError):
            orc.cosmo_decode(c, x.shape, 1, "f32")
    with pytest.raises(orc.OracleError):
        orc.cosmo_decode(b[:48], x.shape, 1, "f32")


# --------------------------------------------------------------------------
# DeepCAM 8-bit delta code (1 sign bit, 3 exponent bits, 4 mantissa bits)

def test_delta_code_table_characterisation(orc):
    codes = [orc.deepcam_code(b) for b in range(256)]
    mags = codes[:128]
    # sign bit: b and b^0x80 decode to opposite values
    assert all(codes[b] == -codes[b ^ 0x80] for b in range(256))
    # magnitudes strictly increase with the 7-bit exponent|mantissa field
    assert all(mags[i] < mags[i + 1] for i in range(127))
    # a float with 4 stored mantissa bits (5 significant with the hidden bit):
    # the magnitude set is exactly the integers <= 31*64 with <= 5 significant bits
    def five_bits(n):
        if n < 32:
            return True
        s = n >> (n.bit_length() - 5)
        return n == s << (n.bit_length() - 5)
    assert set(mags) == {n for n in range(0, 31 * 64 + 1) if five_bits(n)}
    assert len(set(mags)) == 128 and max(mags) == 1984 and mags[0] == 0
    # 3-bit exponent field groups magnitudes into 8 classes (E=0 is the linear range)
    for E in range(8):
        grp = mags[16 * E:16 * E + 16]
        steps = {grp[i + 1] - grp[i] for i in range(15)}
        assert steps == {1 if E <= 1 else 2 ** (E - 1)}


# --------------------------------------------------------------------------
# DeepCAM reconstruction: exact rational arithmetic on hand-built lines

def _expected_line(W, segs, deltas, code):
    """Exact value of FORMAT.md 2.3 using Fractions, rounded RNE to fp32."""
    out, pos, dp = [], 0, 0
    for ln, kind, eb, h in segs:
        h = np.float32(h)
        if kind == 0:
            out += [h] * ln
        else:
            S = 0
            out.append(h)
            for j in range(1, ln):
                S += code[deltas[dp]]
                dp += 1
                v = exact.to_f32(exact.frac(h) + S * Fraction(2) ** (eb - 150))
                if v == 0:
                    v = np.float32(0.0)      # exact sum zero: RN gives +0 (h = -0 with S = 0 too)
                out.append(v)
        pos += ln
    assert pos == W
    return np.array(out, dtype=np.float32)


def _random_segs(rng, W, code):
    segs, deltas, pos = [], [], 0
    while pos < W:
        ln = int(min(W - pos, rng.integers(1, 24)))
        kind = int(rng.random() < 0.8)
        eb = int(rng.choice([1, 2, 20, 100, 130, 140, 147, 148, 150, 160, 200, 246]))
        hk = rng.integers(0, 6)
        h = [0.0, -0.0, 1.0, float(rng.standard_normal() * 10.0 ** rng.integers(-40, 38)),
             float(np.float32(2.0 ** -140)), float(rng.standard_normal())][hk]
        segs.append((ln, kind, eb, np.float32(h)))
        if kind == 1:
            deltas += [int(v) for v in rng.integers(0, 256, size=ln - 1)]
        pos += ln
    return segs, deltas


def test_deepcam_reconstruction_exact_rational(orc):
    rng = np.random.default_rng(1234)
    code = [orc.deepcam_code(b) for b in range(256)]
    n_sub = 0
    for trial in range(300):
        W = int(rng.integers(1, 40))
        segs, deltas = _random_segs(rng, W, code)
        line = fmt.build_seg_line(W, segs, deltas)
        stream = fmt.build_deepcam_stream(1, 1, W, [line])
        got = orc.deepcam_decode_line(stream, 0, W)
        with np.errstate(over="ignore"):
            want = _expected_line(W, segs, deltas, code)
        same = (got.view(np.uint32) == want.view(np.uint32))
        assert same.all(), (trial, np.nonzero(~same))
        n_sub += int(np.sum((np.abs(want) < np.float32(2.0 ** -126)) & (want != 0)))
    assert n_sub > 0   # subnormal reconstructions were exercised (no FTZ)


def test_deepcam_raw_and_repeat_lines(orc):
    W = 20
    x = np.array([np.nan, np.inf, -np.inf, -0.0, 1e-45, 3.4e38] + [1.5] * 14, dtype=np.float32)
    raw = fmt.build_raw_line(x)
    rep = fmt.build_seg_line(W, [(W, 0, 0, np.float32(-0.0))], [])
    s = fmt.build_deepcam_stream(1, 2, W, [raw, rep])
    a = orc.deepcam_decode_line(s, 0, W)
    assert np.array_equal(a.view(np.uint32), x.view(np.uint32))        # RAW is verbatim
    r = orc.deepcam_decode_line(s, 1, W)
    assert np.all(r.view(np.uint32) == np.float32(-0.0).view(np.uint32))  # REPEAT keeps -0.0


def test_deepcam_normalisation_all_raw_matches_numpy(orc):
    """P8: with every line RAW the output is numpy's two-rounding fp32 formula
    then the library fp16 cast (reading S18)."""
    rng = np.random.default_rng(9)
    C, H, W = 3, 4, 24
    x = (rng.standard_normal((C, H, W)) * 1e3).astype(np.float32)
    x[0, 0, 0] = np.nan
    lines = [fmt.build_raw_line(x[c, y]) for c in range(C) for y in range(H)]
    s = fmt.build_deepcam_stream(C, H, W, lines)
    shift = np.float32([1.5, -250.0, 3e3])
    scale = np.float32([0.5, 1.0 / 3.0, 1e-3])
    ref32 = ((x - shift[:, None, None]).astype(np.float32) * scale[:, None, None]).astype(np.float32)
    got32 = orc.deepcam_decode(s, (C, H, W), shift, scale, "f32")
    nan = np.isnan(ref32)
    assert np.array_equal(got32[~nan].view(np.uint32), ref32[~nan].view(np.uint32)) and np.isnan(got32[nan]).all()
    got16 = orc.deepcam_decode(s, (C, H, W), shift, scale, "f16")
    ref16 = ref32.astype(np.float16)
    assert np.array_equal(got16[~nan].view(np.uint16), ref16[~nan].view(np.uint16))
    # no shift/scale: fp32 output is x-hat itself
    assert np.array_equal(orc.deepcam_decode(s, (C, H, W), out="f32")[~nan].view(np.uint32), x[~nan].view(np.uint32))


# --------------------------------------------------------------------------
# DeepCAM encoder: per-value error bound (reading S19) and the paper statistic

def _check_bound(x_line, xh_line, seg_info):
    """|x̂_j - x_j| <= ½ulp(x̂_j) + ½ulp(x̂_{j-1}) + max(1/2, |t|/32)·2^emin (exact)."""
    pos = 0
    for s in seg_info:
        ln = s["len"]
        if s["kind"] == 0:
            assert all(xh_line[pos + j].view(np.uint32) == x_line[pos + j].view(np.uint32) for j in range(ln))
        else:
            assert xh_line[pos].view(np.uint32) == x_line[pos].view(np.uint32)  # head exact
            u = Fraction(2) ** s["emin"]
            for j in range(1, ln):
                p = pos + j
                t = (exact.frac(x_line[p]) - exact.frac(xh_line[p - 1])) / u
                bound = exact.ulp32(xh_line[p]) / 2 + exact.ulp32(xh_line[p - 1]) / 2 + max(Fraction(1, 2), abs(t) / 32) * u
                assert abs(exact.frac(xh_line[p]) - exact.frac(x_line[p])) <= bound, (p, t)
        pos += ln


def test_deepcam_encoder_error_bound_and_roundtrip(orc):
    rng = np.random.default_rng(21)
    C, H, W = 2, 6, 300
    x = np.cumsum(rng.standard_normal((C, H, W)) * 0.01, axis=2).astype(np.float32) + 250.0
    x[1] = np.where(rng.random((H, W)) < 0.9, 0.0, rng.random((H, W)) * 1e-6).astype(np.float32)  # sparse
    x[0, 3, 100:140] = 7.0                              # a repeat run
    x[0, 5, 200] = np.inf                               # forces RAW
    b = orc.deepcam_encode(x)
    h = fmt.deepcam_header(b)
    assert h["L"] == C * H and b.size == h["total"]
    for c in range(C):
        for y in range(H):
            l = c * H + y
            xh = orc.deepcam_decode_line(b, l, W)
            info = fmt.deepcam_line(b, h, l)
            if info["mode"] == 0:
                assert np.array_equal(xh.view(np.uint32), x[c, y].view(np.uint32))
            else:
                assert sum(s["len"] for s in info["segs"]) == W
                _check_bound(x[c, y], xh, info["segs"])
    assert fmt.deepcam_line(b, h, 5)["mode"] == 0
    assert any(s["kind"] == 0 for s in fmt.deepcam_line(b, h, 3)["segs"])


def test_deepcam_paper_statistic(orc):
    """roughly 3% of values with more than 10% error, mostly near
    zero.  Soft acceptance on the paper-shaped generator (reading S19)."""
    from synth import gen_deepcam
    x = gen_deepcam(2001, H=192)
    b = orc.deepcam_encode(x)
    xh = orc.deepcam_decode(b, x.shape, out="f32")
    rel = np.abs(xh.astype(np.float64) - x) / np.maximum(np.abs(x.astype(np.float64)), 1e-300)
    rel[(x == 0) & (xh == 0)] = 0.0
    frac_bad = float((rel > 0.1).mean())
    assert frac_bad <= 0.035
    # large errors are near zero: their |x| is far below each channel's scale
    bad = rel > 0.1
    scale = np.abs(x).reshape(x.shape[0], -1).max(axis=1)[:, None, None]
    assert np.median((np.abs(x) / scale)[bad]) < 0.05
    assert x.nbytes / b.size > 3.0                     # it compresses


@pytest.mark.parametrize("rel,budget", [(0.1, 1), (0.1, 8), (0.1, 64), (0.01, 16)])
def test_deepcam_error_budget(orc, rel, budget):
    """FORMAT.md 2.5 (P:82 abrupt areas kept uncompressed, P:86 the "> 10%
    error" statistic): exactly the lines whose default SEG encoding has
    `budget` or more values with |x̂ - x| > rel |x| (counted here with numpy
    on the oracle's decode) become RAW, and no other line changes."""
    from synth import gen_deepcam
    x = gen_deepcam(2004, H=24)
    C, H, W = x.shape
    b0 = orc.deepcam_encode(x)
    b1 = orc.deepcam_encode(x, rel_err=rel, err_budget=budget)
    h0, h1 = fmt.deepcam_header(b0), fmt.deepcam_header(b1)
    x64 = x.astype(np.float64)
    switched = 0
    for l in range(C * H):
        c, y = divmod(l, H)
        i0, i1 = fmt.deepcam_line(b0, h0, l), fmt.deepcam_line(b1, h1, l)
        xh0 = orc.deepcam_decode_line(b0, l, W).astype(np.float64)
        nbad = int((np.abs(xh0 - x64[c, y]) > np.float64(np.float32(rel)) * np.abs(x64[c, y])).sum())
        if i0["mode"] == 1 and nbad >= budget:
            assert i1["mode"] == 0                                          # kept uncompressed
            assert np.array_equal(orc.deepcam_decode_line(b1, l, W).view(np.uint32), x[c, y].view(np.uint32))
            switched += 1
        else:
            assert i1 == i0                                                 # untouched
    assert switched > 0 and b1.size > b0.size
    # the statistic falls: values above 10% error in the budgeted stream
    xh1 = orc.deepcam_decode(b1, x.shape, out="f32").astype(np.float64)
    xh0 = orc.deepcam_decode(b0, x.shape, out="f32").astype(np.float64)
    bad1 = (np.abs(xh1 - x64) > 0.1 * np.abs(x64)).mean()
    bad0 = (np.abs(xh0 - x64) > 0.1 * np.abs(x64)).mean()
    assert bad1 < bad0
    if rel == 0.1:
        assert bad1 <= budget / W + 1e-12                                   # per-line cap holds on average


def test_f16_to_f32_exhaustive(orc):
    """FORMAT.md 2.6 widening: all 65,536 binary16 patterns against numpy."""
    h = np.arange(65536, dtype=np.uint16)
    want = h.view(np.float16).astype(np.float32)
    got = np.array([orc.f16_to_f32(int(v)) for v in h], dtype=np.float32)
    nan = np.isnan(want)
    assert np.array_equal(np.isnan(got), nan)
    assert np.array_equal(got[~nan].view(np.uint32), want[~nan].view(np.uint32))


@pytest.mark.parametrize("budget", [1, 16])
def test_deepcam_raw16_lines(orc, budget):
    """FORMAT.md 2.6: with raw16, exactly the budget's RAW lines whose values
    all round to finite binary16 within rel_err (checked with numpy) become
    RAW16 and decode to numpy's float16 rounding; nothing else changes."""
    from synth import gen_deepcam
    x = gen_deepcam(2008, H=24)
    C, H, W = x.shape
    b0 = orc.deepcam_encode(x, err_budget=budget)
    b1 = orc.deepcam_encode(x, err_budget=budget, raw16=True)
    h0, h1 = fmt.deepcam_header(b0), fmt.deepcam_header(b1)
    n16 = 0
    for l in range(C * H):
        c, y = divmod(l, H)
        i0, i1 = fmt.deepcam_line(b0, h0, l), fmt.deepcam_line(b1, h1, l)
        xs = x[c, y]
        with np.errstate(over="ignore"):
            r16 = xs.astype(np.float16).astype(np.float32)
        ok16 = bool(np.all(np.isfinite(xs)) and np.all(np.isfinite(r16)) and
                    np.all(np.abs(r16.astype(np.float64) - xs) <= np.float64(np.float32(0.1)) * np.abs(xs.astype(np.float64))))
        seg_budget = i0["mode"] == 0 and fmt.deepcam_line(orc.deepcam_encode(x[c:c + 1, y:y + 1]),
                                                           fmt.deepcam_header(orc.deepcam_encode(x[c:c + 1, y:y + 1])),
                                                           0)["mode"] == 1
        if seg_budget and ok16:
            assert i1["mode"] == 2 and i1["size"] == (16 + 2 * W + 15) // 16 * 16
            assert np.array_equal(orc.deepcam_decode_line(b1, l, W).view(np.uint32), r16.view(np.uint32))
            n16 += 1
        else:
            assert i1 == i0
    assert n16 > 0 and b1.size < b0.size


def _raw_segment_line(rng, W, A):
    """(mode-3 line, the same line with each RAW segment replaced by a REPEAT
    of 0, the RAW segments as (start, values)) -- FORMAT.md 2.7."""
    segs3, segs1, d3, d1, raws, pos = [], [], bytearray(), bytearray(), [], 0
    while pos < W:
        ln = min(W - pos, A * int(rng.integers(1, 4)))
        kind = int(rng.integers(0, 3))
        h = np.float32(rng.standard_normal() * 10.0 ** rng.integers(-3, 4))
        if kind == 2:
            v = (rng.standard_normal(ln) * 10.0 ** rng.integers(-30, 30)).astype(np.float32)
            v[rng.integers(0, ln)] = np.float32(2.0 ** -140)
            segs3.append((ln, 2, 0, v[0]))
            d3 += v.astype("<f4").tobytes()
            segs1.append((ln, 0, 0, np.float32(0.0)))
            raws.append((pos, v))
        else:
            eb = int(rng.integers(100, 160))
            segs3.append((ln, kind, eb, h))
            segs1.append((ln, kind, eb, h))
            if kind == 1:
                codes = bytes(int(c) for c in rng.integers(0, 256, size=ln - 1))
                d3 += codes
                d1 += codes
        pos += ln
    return fmt.build_seg_line(W, segs3, d3, mode=3), fmt.build_seg_line(W, segs1, d1), raws


@pytest.mark.parametrize("W,A", [(64, 8), (37, 1), (1152, 36)])
def test_deepcam_raw_segments_decode(orc, W, A):
    """FORMAT.md 2.7 lines (SEG with RAW segments): a RAW segment's positions
    are its stored binary32 values, and every other position decodes exactly
    as in the same line with that segment made a REPEAT (segments decode
    independently), which pins the 4-bytes-per-value delta-area layout."""
    rng = np.random.default_rng(W)
    for _ in range(8):
        l3, l1, raws = _raw_segment_line(rng, W, A)
        b3 = fmt.build_deepcam_stream(1, 1, W, [l3], A=A)
        b1 = fmt.build_deepcam_stream(1, 1, W, [l1], A=A)
        x3, x1 = orc.deepcam_decode_line(b3, 0, W), orc.deepcam_decode_line(b1, 0, W)
        mask = np.ones(W, bool)
        for st, v in raws:
            assert np.array_equal(x3[st:st + len(v)].view(np.uint32), v.view(np.uint32))
            mask[st:st + len(v)] = False
        assert np.array_equal(x3[mask].view(np.uint32), x1[mask].view(np.uint32))
    # RAW segments are not allowed in mode-1 lines
    l3, _, raws = _raw_segment_line(np.random.default_rng(1), W, A)
    while not raws:
        l3, _, raws = _raw_segment_line(np.random.default_rng(len(l3)), W, A)
    bad = bytearray(l3)
    bad[0] = 1
    with pytest.raises(Exception):
        orc.deepcam_decode_line(fmt.build_deepcam_stream(1, 1, W, [bytes(bad)], A=A), 0, W)


@pytest.mark.parametrize("budget", [1, 8])
def test_deepcam_raw_segment_policy(orc, budget):
    """FORMAT.md 2.7 policy, checked with numpy on the oracle's own decodes: a
    line over the budget becomes a mode-3 line whose RAW segments are exactly
    the runs of A-blocks holding a value above 10% error in its default (2.4)
    encoding, those values are exact, and the line is within the budget."""
    from synth import gen_deepcam
    x = gen_deepcam(2012, H=16)
    C, H, W = x.shape
    A = 36
    b0 = orc.deepcam_encode(x)
    b3 = orc.deepcam_encode(x, err_budget=budget, raw_segments=True)
    h0, h3 = fmt.deepcam_header(b0), fmt.deepcam_header(b3)
    rel = np.float64(np.float32(0.1))
    n3 = 0
    for l in range(C * H):
        c, y = divmod(l, H)
        xs = x[c, y].astype(np.float64)
        i0, i3 = fmt.deepcam_line(b0, h0, l), fmt.deepcam_line(b3, h3, l)
        xh0 = orc.deepcam_decode_line(b0, l, W).astype(np.float64)
        flags = np.abs(xh0 - xs) > rel * np.abs(xs)
        if i0["mode"] != 1 or flags.sum() < budget:
            assert i3 == i0
            continue
        if i3["mode"] != 3:                       # the RAW-segment line was not smaller / within budget
            assert i3["mode"] == 0
            continue
        n3 += 1
        blk = flags.reshape(-1, A).any(axis=1)
        raw_runs, pos = [], 0
        for sg in i3["segs"]:
            if sg["kind"] == 2:
                raw_runs.append((pos, pos + sg["len"]))
            pos += sg["len"]
        want, b = [], 0
        while b < len(blk):
            if blk[b]:
                e = b
                while e < len(blk) and blk[e]:
                    e += 1
                want.append((b * A, e * A))
                b = e
            else:
                b += 1
        assert raw_runs == want
        xh3 = orc.deepcam_decode_line(b3, l, W)
        for s0, e0 in raw_runs:
            assert np.array_equal(xh3[s0:e0].view(np.uint32), x[c, y, s0:e0].view(np.uint32))
        assert (np.abs(xh3.astype(np.float64) - xs) > rel * np.abs(xs)).sum() < budget
    assert n3 > 0 and b3.size < orc.deepcam_encode(x, err_budget=budget).size


def test_deepcam_special_shapes(orc):
    for (C, H, W) in ((1, 1, 1), (1, 3, 2), (2, 2, 17), (1, 1, 16)):
        x = np.random.default_rng(C * 100 + W).standard_normal((C, H, W)).astype(np.float32)
        b = orc.deepcam_encode(x)
        xh = orc.deepcam_decode(b, (C, H, W), out="f32")
        assert xh.shape == (C, H, W) and np.isfinite(xh).all()
    x = np.full((1, 2, 64), 3.25, dtype=np.float32)          # constant lines -> REPEAT, exact
    b = orc.deepcam_encode(x)
    info = fmt.deepcam_line(b, fmt.deepcam_header(b), 0)
    assert info["mode"] == 1 and info["nseg"] == 1 and info["segs"][0]["kind"] == 0
    assert np.array_equal(orc.deepcam_decode(b, x.shape, out="f32"), x)


def test_deepcam_decoder_rejects_corruption(orc):
    W = 8
    good = fmt.build_seg_line(W, [(4, 1, 140, 1.0), (4, 0, 0, 2.0)], [1, 2, 3])
    bad_len = fmt.build_seg_line(W, [(4, 1, 140, 1.0), (5, 0, 0, 2.0)], [1, 2, 3])
    bad_kind = fmt.build_seg_line(W, [(4, 3, 140, 1.0), (4, 0, 0, 2.0)], [1, 2, 3])
    bad_emin = fmt.build_seg_line(W, [(4, 1, 0, 1.0), (4, 0, 0, 2.0)], [1, 2, 3])
    orc.deepcam_decode_line(fmt.build_deepcam_stream(1, 1, W, [good]), 0, W)
    for ln in (bad_len, bad_kind, bad_emin):
        with pytest.raises(orc.OracleError):
            orc.deepcam_decode_line(fmt.build_deepcam_stream(1, 1, W, [ln]), 0, W)


def test_deepcam_segment_alignment(orc):
    """FORMAT.md 2.1/2.4: the encoder aligns segment starts to A (36 when
    W = 1152, 8 when W % 8 == 0, else 1) and decoders reject violations."""
    rng = np.random.default_rng(33)
    for W, A in ((384, 8), (1152, 36), (64, 8), (200, 8), (37, 1)):
        x = np.cumsum(rng.standard_normal((1, 6, W)) * 0.05, axis=2).astype(np.float32)
        x[0, 1, W // 3: W // 3 + 40] = 2.5                  # a run
        x[0, 2, W // 2] += 1e4                              # an abrupt jump (forces a split)
        x[0, 3] = np.where(rng.random(W) < 0.7, 0.0, rng.random(W) * 1e-6)
        b = orc.deepcam_encode(x)
        h = fmt.deepcam_header(b)
        assert h["A"] == A
        for l in range(6):
            info = fmt.deepcam_line(b, h, l)
            xh = orc.deepcam_decode_line(b, l, W)
            if info["mode"] == 1:
                starts = np.cumsum([0] + [s["len"] for s in info["segs"]])[:-1]
                assert all(int(st) % A == 0 for st in starts)
                _check_bound(x[0, l], xh, info["segs"])
            else:
                assert np.array_equal(xh.view(np.uint32), x[0, l].view(np.uint32))
    # a declared alignment the segments violate is corrupt; A must divide W
    W = 16
    line = fmt.build_seg_line(W, [(4, 1, 140, 1.0), (12, 0, 0, 2.0)], [1, 2, 3])
    orc.deepcam_decode_line(fmt.build_deepcam_stream(1, 1, W, [line], A=4), 0, W)
    with pytest.raises(orc.OracleError):
        orc.deepcam_decode_line(fmt.build_deepcam_stream(1, 1, W, [line], A=8), 0, W)
    with pytest.raises(orc.OracleError):
        orc.deepcam_decode_line(fmt.build_deepcam_stream(1, 1, W, [line], A=3), 0, W)
    with pytest.raises(orc.OracleError):
        orc.deepcam_decode_line(fmt.build_deepcam_stream(1, 1, W, [line], A=0), 0, W)


# --------------------------------------------------------------------------
# FORMAT.md 2.8: per-channel REPEAT tolerance ("all neighbouring values
# are similar", reading S15) and absolute error bound

def _repeat_bound_ok(x_line, xh_line, segs, tau):
    """Every REPEAT position within tau of x, the head x at the segment start;
    DIFF positions obey the S19 bound (_check_bound)."""
    pos = 0
    for s in segs:
        ln = s["len"]
        if s["kind"] == 0:
            assert s["head"].view(np.uint32) == x_line[pos].view(np.uint32)
            assert np.all(xh_line[pos:pos + ln].view(np.uint32) == x_line[pos].view(np.uint32))
            assert np.all(np.abs(x_line[pos:pos + ln].astype(np.float64) - np.float64(x_line[pos])) <= tau)
        else:
            _check_bound(x_line[pos:pos + ln], xh_line[pos:pos + ln], [s])
        pos += ln


def test_deepcam_repeat_tolerance_closed_forms(orc):
    """A line of c + noise with |noise| <= tau/2 is ONE REPEAT segment of its
    first value at tolerance tau and not at tau = 0; two noisy plateaus meeting
    at an aligned position are two REPEAT segments whose heads are the plateau
    starts; a plateau meeting at an unaligned position ends on the previous
    aligned position (FORMAT.md 2.4 alignment) and the rest is DIFF/REPEAT."""
    rng = np.random.default_rng(28)
    W = 1152
    tau = np.float32(0.01)
    noisy = lambda c, n: (np.float64(c) + rng.uniform(-0.005, 0.005, n)).astype(np.float32)
    flat = noisy(5.0, W)
    steps = np.concatenate([noisy(10.0, 576), noisy(20.0, 576)])          # 576 = 16 * 36
    off = np.concatenate([noisy(10.0, 500), noisy(20.0, 652)])            # 500 is not a multiple of 36
    x = np.stack([flat, steps, off])[None]
    b0 = orc.deepcam_encode(x)
    b1 = orc.deepcam_encode(x, repeat_tol=np.float32([tau]))
    h0, h1 = fmt.deepcam_header(b0), fmt.deepcam_header(b1)
    assert all(s["kind"] == 1 for s in fmt.deepcam_line(b0, h0, 0)["segs"])     # tau = 0: no identical run
    l0 = fmt.deepcam_line(b1, h1, 0)
    assert l0["nseg"] == 1 and l0["segs"][0]["kind"] == 0 and l0["segs"][0]["head"] == flat[0]
    l1 = fmt.deepcam_line(b1, h1, 1)
    assert [(s["len"], s["kind"]) for s in l1["segs"]] == [(576, 0), (576, 0)]
    assert l1["segs"][1]["head"] == steps[576]
    l2 = fmt.deepcam_line(b1, h1, 2)
    assert (l2["segs"][0]["len"], l2["segs"][0]["kind"]) == (468, 0)        # floor(500 / 36) * 36
    for l in range(3):
        _repeat_bound_ok(x[0, l], orc.deepcam_decode_line(b1, l, W), fmt.deepcam_line(b1, h1, l)["segs"], float(tau))
    assert b1.size < b0.size


def test_deepcam_repeat_tolerance_zero_is_default_and_bound(orc):
    """tau = eps = 0 on every channel writes the default stream byte for byte;
    with per-channel tau > 0 every REPEAT value is within its channel's tau and
    every DIFF value obeys the S19 bound (checked exactly)."""
    from synth import deepcam_stats, gen_deepcam
    x = gen_deepcam(2005, H=12, W=288)
    C, H, W = x.shape
    b0 = orc.deepcam_encode(x)
    z = np.zeros(C, np.float32)
    assert np.array_equal(orc.deepcam_encode(x, repeat_tol=z, max_abs_err=z), b0)
    _, rstd = deepcam_stats(x)
    tau = (0.05 / rstd).astype(np.float32)
    b = orc.deepcam_encode(x, repeat_tol=tau)
    h = fmt.deepcam_header(b)
    nrep = 0
    for l in range(C * H):
        c, y = divmod(l, H)
        info = fmt.deepcam_line(b, h, l)
        xh = orc.deepcam_decode_line(b, l, W)
        if info["mode"] == 0:
            assert np.array_equal(xh.view(np.uint32), x[c, y].view(np.uint32))
            continue
        nrep += sum(s["kind"] == 0 for s in info["segs"])
        _repeat_bound_ok(x[c, y], xh, info["segs"], float(tau[c]))
    assert nrep > 0 and b.size < b0.size


@pytest.mark.parametrize("raw16,rawseg", [(False, False), (True, False), (False, True)])
def test_deepcam_absolute_bound(orc, raw16, rawseg):
    """max_abs_err: exactly the lines whose default SEG encoding has a value with
    |x̂ - x| > eps_c (counted with numpy on the oracle's decode) are kept
    uncompressed (RAW, RAW16 when its binary16 values are within both bounds,
    or RAW segments), every other line is untouched, and every decoded value of
    the final stream is within eps_c (exact, binary64)."""
    from synth import deepcam_stats, gen_deepcam
    x = gen_deepcam(2006, H=16, W=288)
    C, H, W = x.shape
    _, rstd = deepcam_stats(x)
    eps = (0.002 / rstd).astype(np.float32)
    eps[3] = 0.0                                                # a channel without a bound
    b0 = orc.deepcam_encode(x)
    b1 = orc.deepcam_encode(x, max_abs_err=eps, raw16=raw16, raw_segments=rawseg)
    h0, h1 = fmt.deepcam_header(b0), fmt.deepcam_header(b1)
    x64 = x.astype(np.float64)
    switched = 0
    for l in range(C * H):
        c, y = divmod(l, H)
        i0, i1 = fmt.deepcam_line(b0, h0, l), fmt.deepcam_line(b1, h1, l)
        xh0 = orc.deepcam_decode_line(b0, l, W).astype(np.float64)
        over = eps[c] > 0 and bool((np.abs(xh0 - x64[c, y]) > np.float64(eps[c])).any())
        if i0["mode"] == 1 and over:
            assert i1["mode"] in ((0, 2, 3) if (raw16 or rawseg) else (0,))
            if not raw16:
                assert i1["mode"] != 2
            if not rawseg:
                assert i1["mode"] != 3
            switched += 1
        else:
            assert i1 == i0
        xh1 = orc.deepcam_decode_line(b1, l, W).astype(np.float64)
        if eps[c] > 0:
            assert np.all(np.abs(xh1 - x64[c, y]) <= np.float64(eps[c]))
    assert switched > 0


# --------------------------------------------------------------------------
# Labels (FORMAT.md 3): lossless coding.  Pinned by the identity
# (decode(encode(m)) == m) and by brute-force run-length sets from numpy.

def _runs(row):
    """maximal runs of equal values (numpy brute force)"""
    cut = np.flatnonzero(np.diff(row.astype(np.int16))) + 1
    starts = np.concatenate([[0], cut])
    ends = np.concatenate([cut, [row.size]])
    return (ends - starts), row[starts]


def _masks():
    from synth import gen_deepcam_labels
    rng = np.random.default_rng(31)
    alt = np.zeros((2, 64), np.uint8)
    alt[:, 1::2] = 1
    one_change = np.zeros((3, 1152), np.uint8)
    one_change[:, 700:] = 255
    return [gen_deepcam_labels(1), gen_deepcam_labels(2, H=64, W=256),
            rng.integers(0, 256, (5, 37), dtype=np.uint8), np.zeros((4, 9), np.uint8),
            np.full((1, 1), 7, np.uint8), alt, one_change, rng.integers(0, 3, (6, 7), dtype=np.uint8)]


@pytest.mark.parametrize("mi", range(8))
def test_label_mask_lossless_and_layout(orc, mi):
    m = _masks()[mi]
    H, W = m.shape
    b = orc.label_encode_mask(m)
    assert np.array_equal(orc.label_decode(b, 1, H, W), m)                 # lossless
    h = fmt.label_header(b)
    assert (h["magic"], h["ver"], h["kind"], h["H"], h["W"]) == (0x4C505053, 1, 1, H, W)
    assert h["total"] == b.size and b.size % 16 == 0
    up16 = lambda v: (v + 15) // 16 * 16
    for y in range(H):
        lens, vals = _runs(m[y])
        r = fmt.label_row(b, h, y)
        run_size, raw_size = up16(4 + 3 * lens.size), up16(16 + W)
        assert r["mode"] == (1 if run_size < raw_size else 0)
        assert r["size"] == min(run_size, raw_size)
        if r["mode"] == 1:
            assert r["nrun"] == lens.size and np.array_equal(r["lens"], lens) and np.array_equal(r["vals"], vals)


def test_label_vector_bitexact(orc):
    v = np.float32([0.3, -0.0, np.inf, 1e-42, -7.5])
    v = np.concatenate([v, np.frombuffer(np.uint32([0x7FC12345]).tobytes(), np.float32)])   # NaN payload
    b = orc.label_encode_vector(v)
    h = fmt.label_header(b)
    assert (h["kind"], h["H"], h["W"], h["total"]) == (2, 1, v.size, 32 + 32)
    assert np.array_equal(orc.label_decode(b, 2, 1, v.size).view(np.uint32), v.view(np.uint32))


def test_label_decoder_rejects_corruption(orc):
    m = _masks()[1]
    b = orc.label_encode_mask(m)
    h = fmt.label_header(b)
    bad = [b.copy() for _ in range(4)]
    bad[0][0] ^= 1                                                  # magic
    bad[1][6] = 2                                                   # kind
    row = h["payload_off"] + int(h["dir"][0])
    bad[2][row + 4] ^= 0x7F                                          # first run length: sum != W
    bad[3][row] = 5                                                 # unknown row mode
    for c in bad:
        with pytest.raises(RuntimeError):
            orc.label_decode(c, 1, *m.shape)


# --------------------------------------------------------------------------
# FORMAT.md 2.4 encoder POLICY, characterised independently of the oracle's
# code: for every segment the oracle wrote, numpy / brute force recompute what
# 2.4 prescribes (identical runs, the emin rule, the nearest code over all 256
# bytes, where the segment must end) from the text of FORMAT.md alone.

_MAG = np.array([(b & 15) if (b >> 4) & 7 == 0 else (16 + (b & 15)) << (((b >> 4) & 7) - 1) for b in range(128)],
                dtype=np.float64)


def _nearest_code(t):
    """2.4: the code value nearest to t, ties toward the smaller magnitude (brute force over all codes)."""
    vals = np.concatenate([_MAG, -_MAG[1:]])          # every distinct code value
    d = np.abs(vals - t)
    best = d.min()
    cand = vals[d == best]
    return cand[np.argmin(np.abs(cand))]


def _policy_check_line(x, A, segs, deltas, lookahead=64, repeat_min=16, stats=None):
    W = x.size
    stats = {} if stats is None else stats
    bits = x.view(np.uint32)

    def rep(i):
        r = 1
        while i + r < W and bits[i + r] == bits[i]:
            r += 1
        return r if i + r == W else (r // A) * A

    def simulate(i, emin, jmax):
        """closed loop from head i at emin; returns (positions coded, overflow position or None, codes)"""
        h = x[i]
        unit = np.float32(2.0 ** emin)
        S, prev, codes = 0, h, []
        for j in range(i + 1, jmax):
            if j % A == 0 and rep(j) >= repeat_min:
                return j, None, codes
            t = (np.float64(x[j]) - np.float64(prev)) / 2.0 ** emin
            if abs(t) > 1984.5:
                return j, j, codes
            k = _nearest_code(t)
            if abs(S + k) > 1983 * 1984:
                return j, j, codes
            S += int(k)
            prev = np.float32(h + np.float32(S) * unit)      # the product is exact: one rounding
            codes.append(k)
        return jmax, None, codes

    pos, dp = 0, 0
    for s in segs:
        i, ln = pos, s["len"]
        assert i % A == 0 and s["head"].view(np.uint32) == bits[i]
        if rep(i) >= repeat_min:
            assert s["kind"] == 0 and ln == rep(i)
        else:
            assert s["kind"] == 1
            m = np.max(np.abs(np.diff(x[i:min(i + lookahead, W)].astype(np.float64))), initial=0.0)
            e0 = -149 if m == 0 else int(min(96, max(-149, np.ceil(np.log2(m / 1984.0)))))
            if m > 0 and 2.0 ** (e0 - 1) * 1984.0 >= m:           # exact ceil of log2 (no float fuzz)
                e0 -= 1
            e = s["emin"]
            assert e >= e0
            for e_low in range(e0, e):                            # a lower emin overflows within A positions
                _, ov, _ = simulate(i, e_low, W)
                assert ov is not None and (ov // A) * A == i
            end, ov, codes = simulate(i, e, W)
            if ov is None:
                assert ln == end - i                              # stopped at W or at a REPEAT start
                stats["stop"] = stats.get("stop", 0) + 1
            else:
                assert ln == (ov // A) * A - i and ln > 0         # overflow: cut at the aligned position
                stats["overflow"] = stats.get("overflow", 0) + 1
            stats["emin_raised"] = stats.get("emin_raised", 0) + (e > e0)
            got = [(-1 if b & 0x80 else 1) * _MAG[b & 127] for b in deltas[dp:dp + ln - 1]]
            assert got == [float(c) for c in codes[:ln - 1]]
            dp += ln - 1
        pos += ln
    assert pos == W


@pytest.mark.parametrize("W,seed", [(64, 1), (37, 2), (1152, 3), (256, 4)])
def test_deepcam_encoder_policy_characterisation(orc, W, seed):
    """Lines with smooth stretches, noise, abrupt jumps (forcing overflow splits
    and emin increments), identical runs at aligned and unaligned positions,
    subnormal and huge magnitudes; every SEG line's segmentation, emin and codes
    match FORMAT.md 2.4 recomputed from scratch."""
    rng = np.random.default_rng(seed)
    C, H = 1, 12
    x = np.empty((C, H, W), np.float32)
    t = np.linspace(0, 6, W)
    for y in range(H):
        base = np.sin(t * (1 + y % 3)) * 10.0 ** (y % 5 - 2) + rng.standard_normal(W) * 10.0 ** (y % 4 - 4)
        if y % 3 == 0:
            base[W // 3: W // 3 + 20] = base[W // 3]                # identical run (unaligned start)
        if y % 4 == 1:
            base[2 * W // 3:] += 1e4                                 # abrupt jump
        if y == 7:
            base = base * 1e-40                                      # subnormal range
        x[0, y] = base.astype(np.float32)
    # closed-loop overflow inside the first A positions at the window's emin (Δ = 1950
    # quantises to 1920, then Δ = 1984 gives t = 2014 > 1984.5): 2.4 raises emin
    x[0, 2, :] = np.float32(3934 + 1000 * np.arange(W) - 2000)
    x[0, 2, :3] = np.float32([0, 1950, 3934])
    A = orc.lib().orc_deepcam_align(W)
    b = orc.deepcam_encode(x)
    h = fmt.deepcam_header(b)
    checked, stats = 0, {}
    for l in range(C * H):
        info = fmt.deepcam_line(b, h, l)
        if info["mode"] != 1:
            continue
        _policy_check_line(x[0, l], A, info["segs"], info["delta"], stats=stats)
        checked += 1
    assert checked >= H // 2
    assert stats.get("stop", 0) > 0, stats
    if A > 1:
        assert stats.get("emin_raised", 0) > 0, stats               # (with A = 1 2.4 never raises emin)
    if W >= 256:
        assert stats.get("overflow", 0) > 0, stats                   # overflow splits exercised
