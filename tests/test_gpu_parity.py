"""GPU parity: libspp's sm_100a kernels vs the CPU oracle, element by element.

Tolerances (BASELINE.json north_star): decoded integer data bit-exact; fp32
within 2 ulp; fp16 within 1 ulp.  By construction (readings S2, S13,
S18) the expected difference is 0 ulp, so these tests demand bit equality
(NaN positions must match; NaN payloads are not compared).
"""
import numpy as np
import pytest

from tests import fmt

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_ibrahimo22_b200 import build
    build.build()
    return torch.device("cuda:0")


def _to_dev(buf: np.ndarray):
    t = torch.empty(int(buf.size) + 15, dtype=torch.uint8, device="cuda")
    t = t[: buf.size]  # torch allocations are 512-B aligned; slicing from 0 keeps alignment
    t.copy_(torch.from_numpy(np.ascontiguousarray(buf)))
    return t


def _same_bits(got: np.ndarray, want: np.ndarray):
    assert got.shape == want.shape and got.dtype == want.dtype
    if got.dtype.kind == "f":
        gn, wn = np.isnan(got), np.isnan(want)
        assert np.array_equal(gn, wn)
        iv = got.view(np.uint16 if got.itemsize == 2 else np.uint32)
        jv = want.view(np.uint16 if got.itemsize == 2 else np.uint32)
        bad = (iv != jv) & ~gn
        assert not bad.any(), f"{int(bad.sum())} mismatches, first at {np.argwhere(bad)[:3].tolist()}"
    else:
        assert np.array_equal(got, want)


def _decode(fmt_name, bufs, dims, out="f16", transform=None, shift=None, scale=None, escape_keys=False,
            raw_segments=False):
    from paper_conf_ipps_ibrahimo22_b200 import Decoder
    dec = Decoder(fmt_name, dims, out=out, transform=transform, escape_keys=escape_keys, raw_segments=raw_segments)
    if shift is not None or scale is not None:
        dec.set_normalisation(shift, scale)
    srcs = [_to_dev(b) for b in bufs]
    res = dec.decode(srcs)
    torch.cuda.synchronize()
    status = int(dec.status.item())
    return res.cpu().numpy(), status


# ------------------------------------------------------------------ CosmoFlow
def test_cosmo_c1_paper_sample_all_outputs(dev, orc):
    """C1: one paper-shaped 4x128^3 sample; fp16 / fp32 / identity int16."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_cosmo(1001)
    b = spp.spp_encode_cosmo(x)
    for out, tr in (("f16", 1), ("f32", 1), ("i16", 0), ("f32", 0), ("f16", 0)):
        got, st = _decode("cosmo", [b], x.shape, out=out, transform=tr)
        assert st == 0
        _same_bits(got[0], orc.cosmo_direct(x, tr, out))


def test_cosmo_transform_table_exhaustive(dev, orc):
    """Every count 0..32767 through the GPU's fp64 log1p -> fp32 (and fp16)."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    vals = np.arange(32768, dtype=np.int16)
    x = np.stack([vals, vals[::-1], np.roll(vals, 7), vals]).reshape(4, 32, 32, 32).copy()
    b = spp.spp_encode_cosmo(x)
    for out in ("f32", "f16"):
        got, st = _decode("cosmo", [b], x.shape, out=out)
        assert st == 0
        _same_bits(got[0], orc.cosmo_direct(x, 1, out))


@pytest.mark.parametrize("preset,n", [("sparse", 64), ("verysparse", 64), ("dense", 64), ("unit", 48),
                                      ("independent", 32), ("coupled", 40)])
def test_cosmo_presets_key_widths_and_slabs(dev, orc, preset, n):
    """C5 sweep shapes: kw = 1 / 2, z-slab split and the RAW escape."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_cosmo(3001, preset, n=n)
    b = spp.spp_encode_cosmo(x)
    got, st = _decode("cosmo", [b], x.shape, out="f16")
    assert st == 0
    _same_bits(got[0], orc.cosmo_direct(x, 1, "f16"))


def test_cosmo_edge_shapes_and_broadcast(dev, orc):
    """Degenerate cases: all-zero volume (kw = 0 broadcast), 1-voxel volume,
    odd shapes (scalar path), a slab split on a tiny volume."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    rng = np.random.default_rng(3)
    cases = [np.zeros((4, 16, 16, 16), dtype=np.int16), np.full((4, 1, 1, 1), 5, dtype=np.int16),
             rng.integers(0, 30, size=(4, 5, 7, 3)).astype(np.int16),
             rng.integers(0, 4, size=(4, 3, 3, 3)).astype(np.int16),
             rng.integers(0, 2000, size=(4, 4, 64, 64)).astype(np.int16)]   # G > 0.75 N -> RAW escape
    for x in cases:
        b = spp.spp_encode_cosmo(x)
        for out in ("f32", "f16"):
            got, st = _decode("cosmo", [b], x.shape, out=out)
            assert st == 0
            _same_bits(got[0], orc.cosmo_direct(x, 1, out))
        got, st = _decode("cosmo", [b], x.shape, out="i16", transform=0)
        assert st == 0 and np.array_equal(got[0], x)


def test_cosmo_localized_tables(dev, orc):
    """FORMAT.md 1.4 localized tables (spp_encode_cosmo_ex): many slabs with
    1-byte keys, mixed kw 0 / 1 / 8 in one stream, a batch mixing both
    policies; every output bit-exact to the plain definition."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    rng = np.random.default_rng(12)
    xs = [gen_cosmo(3001, "sparse"), gen_cosmo(3005, "unit", n=64)]
    v = gen_cosmo(3006, "sparse", n=64)
    v[:, :16] = 3                                                    # constant slab -> kw 0
    v[:, 48:] = rng.integers(0, 3000, size=(4, 16, 64, 64))          # dense slab -> RAW escape
    xs.append(v)
    for x in xs:
        b = spp.spp_encode_cosmo(x, localize=True)
        assert fmt.cosmo_header(b)["T"] > 1 or x.shape[1] < 128
        for out, tr in (("f16", 1), ("f32", 1), ("i16", 0)):
            got, st = _decode("cosmo", [b], x.shape, out=out, transform=tr)
            assert st == 0
            _same_bits(got[0], orc.cosmo_direct(x, tr, out))
    kws = {s["kw"] for s in fmt.cosmo_header(spp.spp_encode_cosmo(xs[2], localize=True))["slabs"]}
    assert {0, 1, 8} <= kws
    x0 = xs[0]
    bufs = [spp.spp_encode_cosmo(x0, localize=True), spp.spp_encode_cosmo(x0)] * 3
    got, st = _decode("cosmo", bufs, x0.shape, out="f16")
    assert st == 0
    want = orc.cosmo_direct(x0, 1, "f16")
    for g in got:
        _same_bits(g, want)


def test_cosmo_escaped_keys(dev, orc):
    """FORMAT.md 1.5 escaped 1-byte keys decode bit-exactly with
    opts.escape_keys = 1 (the staging kernel; its scalar path when a plane is
    not a multiple of the 256-voxel escape block): paper sample, 4x256^3
    multi-table, localized + escaped volume, a 48x40-plane volume, a batch
    mixing formats; all outputs.  Without the flag the vector kernel reports
    SPP_ERR_UNSUPPORTED for such samples."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    cases = [(gen_cosmo(1001), False), (gen_cosmo(1002, n=256), False), (gen_cosmo(3005, "unit", n=64), True),
             (np.ascontiguousarray(gen_cosmo(1003, n=64)[:, :, :48, :40]), False)]
    for x, loc in cases:
        b = spp.spp_encode_cosmo(x, localize=loc, escape=True)
        assert any(s["kw"] == 3 for s in fmt.cosmo_header(b)["slabs"])
        for out, tr in (("f16", 1), ("i16", 0), ("f32", 1)):
            got, st = _decode("cosmo", [b], x.shape, out=out, transform=tr, escape_keys=True)
            assert st == 0
            _same_bits(got[0], orc.cosmo_direct(x, tr, out))
        _, st = _decode("cosmo", [b], x.shape, out="f16", escape_keys=False)
        assert st == 4                                          # SPP_ERR_UNSUPPORTED, sample 0
    x = gen_cosmo(1004)
    bufs = [spp.spp_encode_cosmo(x, escape=True), spp.spp_encode_cosmo(x), spp.spp_encode_cosmo(x, escape=True)]
    got, st = _decode("cosmo", bufs, x.shape, out="f16", escape_keys=True)
    assert st == 0
    want = orc.cosmo_direct(x, 1, "f16")
    for g in got:
        _same_bits(g, want)


def test_cosmo_escaped_keys_edge_layouts(dev, orc):
    """Escaped-key slabs whose tiles hold more escapes than a key stage can
    stage (escapes clustered in z: the global-memory path of the staging
    kernel), and a slab whose last 256-voxel block is partial (scalar path)."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    rng = np.random.default_rng(31)
    vols = []
    n = 32 * 32 * 32                                  # 22 planes of 100 hot groups, 10 of a 3000-group tail
    gid = np.concatenate([rng.integers(0, 100, size=22 * 1024), rng.integers(100, 3100, size=10 * 1024)])
    vols.append(np.array([gid % 31, gid // 31, (gid * 7) % 13, gid % 5], dtype=np.int16).reshape(4, 32, 32, 32))
    n = 5 * 12 * 20                                   # 1200 voxels: 4 full blocks and a partial one
    gid = np.where(rng.random(n) < 0.6, rng.integers(0, 100, size=n), rng.integers(100, 3100, size=n))
    vols.append(np.array([gid % 31, gid // 31, (gid * 7) % 13, gid % 5], dtype=np.int16).reshape(4, 5, 12, 20))
    for x in vols:
        b = spp.spp_encode_cosmo(x, escape=True)
        assert fmt.cosmo_header(b)["slabs"][0]["kw"] == 3
        for out, tr in (("f16", 1), ("i16", 0)):
            got, st = _decode("cosmo", [b, b], x.shape, out=out, transform=tr, escape_keys=True)
            assert st == 0
            want = orc.cosmo_direct(x, tr, out)
            _same_bits(got[0], want)
            _same_bits(got[1], want)


def test_cosmo_escaped_keys_corruption(dev):
    """A wrong escape-block index is reported (status), on both kernels."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_cosmo(1001, n=64)
    b = spp.spp_encode_cosmo(x, escape=True)
    s = fmt.cosmo_header(b)["slabs"][0]
    assert s["kw"] == 3
    bad = b.copy()
    o = s["keys_off"] + 4 * 40
    v = int(np.frombuffer(bytes(bad[o:o + 4]), "<u4")[0]) + 3
    bad[o:o + 4] = np.frombuffer(np.uint32(v).tobytes(), np.uint8)
    _, st = _decode("cosmo", [b, bad], x.shape, out="f16", escape_keys=True)
    assert st == (1 << 8 | 3)                                   # SPP_ERR_CORRUPT, sample 1
    y = np.ascontiguousarray(x[:, :, :48, :40])                 # scalar path of the staging kernel
    by = spp.spp_encode_cosmo(y, escape=True)
    sy = fmt.cosmo_header(by)["slabs"][0]
    bady = by.copy()
    o = sy["keys_off"] + 4 * 20
    bady[o:o + 4] = np.frombuffer(np.uint32(int(np.frombuffer(bytes(by[o:o + 4]), "<u4")[0]) + 3).tobytes(), np.uint8)
    _, st = _decode("cosmo", [by, bady], y.shape, out="f16", escape_keys=True)
    assert st == (1 << 8 | 3)


def test_cosmo_oracle_encoded_stream(dev, orc):
    """The GPU decodes a stream written by the oracle's own encoder."""
    from synth import gen_cosmo
    x = gen_cosmo(1002, n=64)
    b = orc.cosmo_encode(x)
    got, st = _decode("cosmo", [b], x.shape, out="f32")
    assert st == 0
    _same_bits(got[0], orc.cosmo_decode(b, x.shape, 1, "f32"))


def test_cosmo_c2_launch_configuration(dev, orc):
    """C2 at full size (n = 512, the bench's launch configuration): every
    output sample equals the oracle's plain definition of its source."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    pool = [gen_cosmo(1001 + i) for i in range(3)]
    bufs = [_to_dev(spp.spp_encode_cosmo(x)) for x in pool]
    want = [torch.from_numpy(orc.cosmo_direct(x, 1, "f16").view(np.int16)).to(dev) for x in pool]
    n = 512
    dec = Decoder("cosmo", (4, 128, 128, 128))
    out = dec.decode([bufs[i % 3] for i in range(n)])
    torch.cuda.synchronize()
    assert int(dec.status.item()) == 0
    o16 = out.view(torch.int16)
    for i in range(n):
        assert torch.equal(o16[i], want[i % 3]), i


def test_cosmo_256_multi_lut(dev, orc):
    """a 4x256^3 paper-preset volume (8x the paper's sample)
    needs several z-slab lookup tables ("multiple LUTs"); also a
    non-cubic 4x96x256x128 volume.  Both decoded bit-exactly, fp16 and fp32."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_cosmo(1001, n=256)
    b = spp.spp_encode_cosmo(x)
    nU, T, G, kw = spp.spp_stream_info("cosmo", b)
    assert T > 1 and kw == 2                           # multiple tables, 2-byte keys
    for out in ("f16", "f32"):
        got, st = _decode("cosmo", [b], x.shape, out=out)
        assert st == 0
        _same_bits(got[0], orc.cosmo_direct(x, 1, out))
    y = np.ascontiguousarray(x[:, :96, :, ::2])
    b2 = spp.spp_encode_cosmo(y)
    got, st = _decode("cosmo", [b2, b2], y.shape, out="f16")
    assert st == 0
    want = orc.cosmo_direct(y, 1, "f16")
    _same_bits(got[0], want)
    _same_bits(got[1], want)


def test_cosmo_512_full_simulation_volume(dev, orc):
    """The paper's full 512^3 simulation histogram (before the 128^3
    decomposition; "for larger than 128^3 decompositions, multiple lookup
    tables are required"): 4x512^3 counts (1 GiB) built from 64
    offset copies of a paper-shaped 128^3 sample, so groups do not repeat
    across tiles.  Identity output equals the input counts bit for bit over
    the whole volume; fp16 ln(1+c) equals the oracle's plain definition on
    every voxel of sampled planes."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    base = gen_cosmo(1001)
    off = np.arange(64, dtype=np.int16).reshape(4, 4, 4)
    x = np.empty((4, 512, 512, 512), dtype=np.int16)
    for tz in range(4):
        for ty in range(4):
            for tx in range(4):
                x[:, tz * 128:(tz + 1) * 128, ty * 128:(ty + 1) * 128, tx * 128:(tx + 1) * 128] = \
                    base + 7 * off[tz, ty, tx]
    b = spp.spp_encode_cosmo(x)
    nU, T, G, kw = spp.spp_stream_info("cosmo", b)
    assert T > 1
    got, st = _decode("cosmo", [b], x.shape, out="i16", transform=0)
    assert st == 0 and np.array_equal(got[0], x)
    del got
    got, st = _decode("cosmo", [b], x.shape, out="f16")
    assert st == 0
    for z in (0, 127, 128, 255, 300, 511):
        plane = np.ascontiguousarray(x[:, z:z + 1])
        _same_bits(got[0][:, z:z + 1], orc.cosmo_direct(plane, 1, "f16"))


def test_cosmo_corruption_detected(dev):
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_cosmo(1005, n=32)
    b = spp.spp_encode_cosmo(x)
    h = fmt.cosmo_header(b)
    bad_magic = b.copy(); bad_magic[0] ^= 0xFF
    bad_key = b.copy()
    s0 = h["slabs"][0]
    if s0["kw"] == 2:
        bad_key[s0["keys_off"]:s0["keys_off"] + 2] = 0xFF   # key 65535 >= G
    bad_lut = b.copy(); bad_lut[s0["lut_off"]:s0["lut_off"] + 2] = 0xFF  # U index >= nU
    for i, bb in enumerate((bad_magic, bad_key, bad_lut)):
        _, st = _decode("cosmo", [b, bb], x.shape, out="f16")
        assert st & 0xFF == 3 and st >> 8 == 1, (i, st)


def test_cosmo_raw_slabs_full_size(dev, orc):
    """RAW-escape slabs (FORMAT.md 1.1, kw = 8) at the paper's 4x128^3 size,
    in a batch that mixes them with key slabs of the same and other samples
    (the per-sample shared output table and the hot prefix share one region):
    an all-RAW dense sample (lambda = 64) in both policies, a sparse sample with
    a dense RAW band, and the paper preset; fp16, fp32 and int16 bit-exact, and
    an index >= |U| in a RAW plane is reported as corrupt on its sample."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import spp
    rng = np.random.default_rng(77)
    dense = gen_cosmo(3101, lam=64.0, rho_c=0.0)
    band = gen_cosmo(3102, "sparse")
    band[:, 40:72] = rng.integers(0, 3000, size=(4, 32, 128, 128))
    paper = gen_cosmo(3103)
    xs = [dense, band, paper, dense]
    bufs = [spp.spp_encode_cosmo(dense), spp.spp_encode_cosmo(band), spp.spp_encode_cosmo(paper),
            spp.spp_encode_cosmo(dense, localize=True)]
    kws = [{s["kw"] for s in fmt.cosmo_header(b)["slabs"]} for b in bufs]
    assert kws[0] == {8} and 8 in kws[1] and kws[1] - {8} and kws[3] == {8}
    for out, tr in (("f16", 1), ("f32", 1), ("i16", 0)):
        got, st = _decode("cosmo", bufs, dense.shape, out=out, transform=tr)
        assert st == 0
        for g, x in zip(got, xs):
            _same_bits(g, orc.cosmo_direct(x, tr, out))
    h = fmt.cosmo_header(bufs[1])
    rs = [s for s in h["slabs"] if s["kw"] == 8][0]
    bad = bufs[1].copy()
    nvox = (rs["z1"] - rs["z0"]) * 128 * 128
    o = rs["keys_off"] + 2 * (2 * nvox + 12345)  # plane 2 of the slab
    bad[o:o + 2] = 0xFF
    _, st = _decode("cosmo", [bufs[0], bufs[2], bad], dense.shape, out="f16")
    assert st & 0xFF == 3 and st >> 8 == 2, st


# ------------------------------------------------------------------ DeepCAM
def _dc_ref(orc, b, shape, shift, scale, out):
    return orc.deepcam_decode(b, shape, shift, scale, out)


def test_deepcam_c3_paper_sample(dev, orc):
    """C3: one 16x768x1152 sample, per-channel normalisation, fp16 and fp32."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_deepcam(2001)
    mean, rstd = deepcam_stats(x)
    b = spp.spp_encode_deepcam(x)
    for out in ("f16", "f32"):
        got, st = _decode("deepcam", [b], x.shape, out=out, shift=mean, scale=rstd)
        assert st == 0
        _same_bits(got[0], _dc_ref(orc, b, x.shape, mean, rstd, out))
    got, st = _decode("deepcam", [b], x.shape, out="f32")     # x-hat itself
    assert st == 0
    _same_bits(got[0], _dc_ref(orc, b, x.shape, None, None, "f32"))


@pytest.mark.parametrize("budget", [1, 16])
def test_deepcam_error_budget_streams(dev, orc, budget):
    """FORMAT.md 2.5 error-budget streams (many RAW lines interleaved with SEG
    lines) on the full-size C3 shape: bit-exact, and RAW lines are x itself."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_deepcam(2006)
    mean, rstd = deepcam_stats(x)
    b = spp.spp_encode_deepcam(x, err_budget=budget)
    raw, seg, _, _ = spp.spp_stream_info("deepcam", b)
    assert raw > 100 and seg > 100
    got, st = _decode("deepcam", [b, spp.spp_encode_deepcam(x)], x.shape, out="f16", shift=mean, scale=rstd)
    assert st == 0
    _same_bits(got[0], _dc_ref(orc, b, x.shape, mean, rstd, "f16"))
    got, st = _decode("deepcam", [b], x.shape, out="f32")
    assert st == 0
    _same_bits(got[0], _dc_ref(orc, b, x.shape, None, None, "f32"))


@pytest.mark.parametrize("budget", [1, 16])
def test_deepcam_raw16_streams(dev, orc, budget):
    """FORMAT.md 2.6 RAW16 lines (error budget + raw16) on the full C3 shape,
    mixed with SEG and fp32 RAW lines: bit-exact, fp16 / fp32 / x-hat."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_deepcam(2009)
    mean, rstd = deepcam_stats(x)
    b = spp.spp_encode_deepcam(x, err_budget=budget, raw16=True)
    h = fmt.deepcam_header(b)
    modes = {fmt.deepcam_line(b, h, l)["mode"] for l in range(0, h["L"], 5)}
    assert {1, 2} <= modes
    for out, sh, sc in (("f16", mean, rstd), ("f32", mean, rstd), ("f32", None, None)):
        got, st = _decode("deepcam", [b, b], x.shape, out=out, shift=sh, scale=sc)
        assert st == 0
        want = _dc_ref(orc, b, x.shape, sh, sc, out)
        _same_bits(got[0], want)
        _same_bits(got[1], want)


@pytest.mark.parametrize("rs", [False, True])
@pytest.mark.parametrize("budget,raw16", [(1, False), (4, True)])
def test_deepcam_raw_segment_streams(dev, orc, budget, raw16, rs):
    """FORMAT.md 2.7 streams from the encoder (error budget + RAW segments) on
    the full C3 shape: mode-3 lines among SEG (and RAW16) lines, bit-exact."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_deepcam(2013)
    mean, rstd = deepcam_stats(x)
    b = spp.spp_encode_deepcam(x, err_budget=budget, raw16=raw16, raw_segments=True)
    h = fmt.deepcam_header(b)
    assert 3 in {fmt.deepcam_line(b, h, l)["mode"] for l in range(0, h["L"], 3)}
    for out, sh, sc in (("f16", mean, rstd), ("f32", None, None)):
        got, st = _decode("deepcam", [b, b], x.shape, out=out, shift=sh, scale=sc, raw_segments=rs)
        assert st == 0
        want = _dc_ref(orc, b, x.shape, sh, sc, out)
        _same_bits(got[0], want)
        _same_bits(got[1], want)


@pytest.mark.parametrize("W", [37, 64])
def test_deepcam_raw16_narrow_lines(dev, orc, W):
    """RAW16, RAW and SEG lines on the scalar (W = 37) and 8-wide (W = 64)
    decode paths, normalised fp16 / fp32."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_deepcam(2010, H=16, W=W)
    mean, rstd = deepcam_stats(x)
    b = spp.spp_encode_deepcam(x, err_budget=1, raw16=True)
    h = fmt.deepcam_header(b)
    assert {0, 1, 2} <= {fmt.deepcam_line(b, h, l)["mode"] for l in range(h["L"])}
    for out in ("f16", "f32"):
        got, st = _decode("deepcam", [b], x.shape, out=out, shift=mean, scale=rstd)
        assert st == 0
        _same_bits(got[0], _dc_ref(orc, b, x.shape, mean, rstd, out))


def test_deepcam_oracle_encoded_stream(dev, orc):
    from synth import gen_deepcam
    x = gen_deepcam(2002, H=64)
    b = orc.deepcam_encode(x)
    got, st = _decode("deepcam", [b], x.shape, out="f32")
    assert st == 0
    _same_bits(got[0], _dc_ref(orc, b, x.shape, None, None, "f32"))


def _random_line(rng, W, kinds=(0, 1), seglen=(1, 40)):
    segs, deltas, pos = [], [], 0
    while pos < W:
        ln = int(min(W - pos, rng.integers(*seglen)))
        kind = int(rng.choice(kinds))
        eb = int(rng.choice([1, 2, 60, 120, 140, 147, 148, 149, 170, 246]))
        h = np.float32(rng.choice([0.0, -0.0, 1.0, rng.standard_normal() * 10.0 ** rng.integers(-40, 30),
                                   2.0 ** -140]))
        segs.append((ln, kind, eb, h))
        if kind == 1:
            deltas += [int(v) for v in rng.integers(0, 256, size=ln - 1)]
        pos += ln
    return fmt.build_seg_line(W, segs, deltas)


@pytest.mark.parametrize("W", [1, 7, 8, 17, 64, 256, 264, 1152])
def test_deepcam_handbuilt_lines(dev, orc, W):
    """Hand-built SEG/RAW lines: short segments (several per lane: general
    path), REPEAT of -0.0, subnormal and large-exponent scales, heads at every
    lane offset, NaN/Inf RAW lines, W not a multiple of 8 (scalar path)."""
    rng = np.random.default_rng(W)
    C, H = 2, 24
    lines = []
    for l in range(C * H):
        r = l % 6
        if r == 0:
            v = rng.standard_normal(W).astype(np.float32)
            v[rng.integers(0, W)] = np.nan
            v[rng.integers(0, W)] = -np.inf
            lines.append(fmt.build_raw_line(v))
        elif r == 1:
            lines.append(fmt.build_seg_line(W, [(W, 0, 0, np.float32(-0.0))], []))
        elif r == 2:
            lines.append(_random_line(rng, W, seglen=(1, 4)))
        elif r == 3:
            lines.append(_random_line(rng, W, kinds=(1,), seglen=(W, W + 1)))
        else:
            lines.append(_random_line(rng, W))
    b = fmt.build_deepcam_stream(C, H, W, lines)
    shift = np.float32([0.5, -3.0])
    scale = np.float32([2.0, 1e-3])
    for out in ("f32", "f16"):
        got, st = _decode("deepcam", [b], (C, H, W), out=out, shift=shift, scale=scale)
        assert st == 0
        _same_bits(got[0], _dc_ref(orc, b, (C, H, W), shift, scale, out))
    got, st = _decode("deepcam", [b], (C, H, W), out="f32")
    _same_bits(got[0], _dc_ref(orc, b, (C, H, W), None, None, "f32"))


@pytest.mark.parametrize("W,A,rs", [(64, 8, False), (37, 1, True), (1152, 36, False), (1152, 36, True)])
def test_deepcam_raw_segment_lines(dev, orc, W, A, rs):
    """FORMAT.md 2.7 lines (SEG with RAW segments: KD's general line path, or
    the one-pass path with opts.raw_segments at W = 1152) mixed with plain SEG
    and RAW lines: bit-exact, normalised and x-hat."""
    from tests.test_oracle_pins import _raw_segment_line
    rng = np.random.default_rng(100 + W)
    C, H = 2, 12
    lines = []
    for l in range(C * H):
        if l % 4 == 3:
            lines.append(fmt.build_raw_line(rng.standard_normal(W).astype(np.float32)))
        else:
            lines.append(_raw_segment_line(rng, W, A)[l % 4 == 2])
    b = fmt.build_deepcam_stream(C, H, W, lines, A=A)
    shift, scale = np.float32([0.5, -3.0]), np.float32([2.0, 1e-3])
    for out, sh, sc in (("f16", shift, scale), ("f32", shift, scale), ("f32", None, None)):
        got, st = _decode("deepcam", [b, b], (C, H, W), out=out, shift=sh, scale=sc, raw_segments=rs)
        assert st == 0
        want = _dc_ref(orc, b, (C, H, W), sh, sc, out)
        _same_bits(got[0], want)
        _same_bits(got[1], want)


_EB_EDGES = [1, 2, 3, 4, 5, 6, 7, 60, 120, 147, 148, 149, 170, 200, 246]


def _random_aligned_line(rng, W, A, nseg_max, kinds=(0, 1)):
    """SEG line whose segments start on multiples of A (FORMAT.md 2.1, S14):
    lengths are multiples of A except the last, which ends at W."""
    segs, deltas, pos = [], [], 0
    nblk = (W + A - 1) // A
    while pos < W:
        left = nblk - pos // A
        k = 1 if nseg_max >= nblk else int(rng.integers(1, max(2, min(left, 2 * nblk // nseg_max + 1)) + 1))
        ln = min(W - pos, k * A)
        if len(segs) == nseg_max - 1:
            ln = W - pos
        kind = int(rng.choice(kinds))
        eb = int(rng.choice(_EB_EDGES))
        h = np.float32(rng.choice([0.0, -0.0, 1.0, rng.standard_normal() * 10.0 ** rng.integers(-40, 30),
                                   2.0 ** -140, -3.0e38]))
        segs.append((ln, kind, eb, h))
        if kind == 1:
            deltas += [int(v) for v in rng.integers(0, 256, size=ln - 1)]
        pos += ln
    return fmt.build_seg_line(W, segs, deltas)


@pytest.mark.parametrize("nseg_max", [1, 4, 16, 32])
def test_deepcam_handbuilt_aligned_lines(dev, orc, nseg_max):
    """W = 1152 with segment alignment A = 36: the one-pass path (a segment
    starts on a 36-value lane block, so 1..32 segments per line; 32 = every
    lane its own segment); emin_b on both sides of the subnormal-multiplier bound
    (< 6) and of the former large-exponent split (148); REPEAT of signed zero;
    heads at every lane block; RAW lines interleaved."""
    W, A, C, H = 1152, 36, 2, 20
    rng = np.random.default_rng(1000 + nseg_max)
    lines = []
    for l in range(C * H):
        if l % 7 == 6:
            lines.append(fmt.build_raw_line(rng.standard_normal(W).astype(np.float32)))
        else:
            lines.append(_random_aligned_line(rng, W, A, nseg_max))
    b = fmt.build_deepcam_stream(C, H, W, lines, A=A)
    shift = np.float32([0.25, -7.0])
    scale = np.float32([4.0, 3e-2])
    for out in ("f16", "f32"):
        got, st = _decode("deepcam", [b], (C, H, W), out=out, shift=shift, scale=scale)
        assert st == 0
        _same_bits(got[0], _dc_ref(orc, b, (C, H, W), shift, scale, out))
    got, st = _decode("deepcam", [b], (C, H, W), out="f32")
    _same_bits(got[0], _dc_ref(orc, b, (C, H, W), None, None, "f32"))


@pytest.mark.parametrize("W,A", [(1152, 36), (64, 8), (17, 1)])
def test_deepcam_signed_zero_codes(dev, orc, W, A):
    """FORMAT.md 2.3: S_j is an integer prefix (code 0x80 is 0), so after a
    head h = -0.0 every zero-sum position decodes to RN(-0 + 0) = +0 while
    the head itself stays -0; REPEAT of -0 stays -0 everywhere.  Covers the
    one-pass (A = 36), aligned (A = 8) and general (A = 1) line paths."""
    C, H = 1, 6
    half = (W // 2) // A * A or W
    lines = [
        fmt.build_seg_line(W, [(W, 1, 100, np.float32(-0.0))], [0x80] * (W - 1)),
        fmt.build_seg_line(W, [(W, 1, 3, np.float32(-0.0))], ([0x80, 0x00, 0x81, 0x01] * W)[:W - 1]),
        fmt.build_seg_line(W, [(W, 1, 200, np.float32(0.0))], [0x80] * (W - 1)),
        fmt.build_seg_line(W, [(W, 0, 0, np.float32(-0.0))], []),
        fmt.build_seg_line(W, [(half, 1, 5, np.float32(-0.0)), (W - half, 1, 150, np.float32(-0.0))]
                           if half < W else [(W, 1, 5, np.float32(-0.0))],
                           [0x80] * (W - (2 if half < W else 1))),
        fmt.build_seg_line(W, [(half, 0, 0, np.float32(-0.0)), (W - half, 1, 7, np.float32(-0.0))]
                           if half < W else [(W, 0, 0, np.float32(-0.0))],
                           [0x80] * (W - half - 1) if half < W else []),
    ]
    b = fmt.build_deepcam_stream(C, H, W, lines, A=A)
    want = _dc_ref(orc, b, (C, H, W), None, None, "f32")
    # the definition: only heads and REPEAT positions keep -0
    assert np.signbit(want[0, 0, 0]) and not np.signbit(want[0, 0, 1:]).any()
    assert np.signbit(want[0, 3]).all()
    for out in ("f32", "f16"):
        got, st = _decode("deepcam", [b], (C, H, W), out=out)
        assert st == 0
        _same_bits(got[0], _dc_ref(orc, b, (C, H, W), None, None, out))


def test_deepcam_batch_order_independence(dev, orc):
    """P13: decoding samples alone, in a batch, or in another order gives the
    same bytes per sample."""
    from synth import gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import spp
    xs = [gen_deepcam(2010 + i, H=96) for i in range(3)]
    bs = [spp.spp_encode_deepcam(x) for x in xs]
    batch, st = _decode("deepcam", bs, xs[0].shape, out="f16")
    assert st == 0
    rev, _ = _decode("deepcam", bs[::-1], xs[0].shape, out="f16")
    for i in range(3):
        alone, _ = _decode("deepcam", [bs[i]], xs[0].shape, out="f16")
        assert np.array_equal(alone[0].view(np.uint16), batch[i].view(np.uint16))
        assert np.array_equal(rev[2 - i].view(np.uint16), batch[i].view(np.uint16))
        _same_bits(batch[i], _dc_ref(orc, bs[i], xs[0].shape, None, None, "f16"))


def test_deepcam_c4_launch_configuration(dev, orc):
    """C4 at full size (n = 2048 samples -> fp16, the bench's launch
    configuration): every output sample equals the oracle decode of its
    source."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    pool = [gen_deepcam(2001 + i) for i in range(2)]
    mean, rstd = deepcam_stats(pool[0])
    bufs = [_to_dev(spp.spp_encode_deepcam(x)) for x in pool]
    want = [torch.from_numpy(orc.deepcam_decode(spp.spp_encode_deepcam(x), x.shape, mean, rstd, "f16")
                             .view(np.int16)).to(dev) for x in pool]
    n = 2048
    dec = Decoder("deepcam", (16, 768, 1152))
    dec.set_normalisation(mean, rstd)
    out = dec.decode([bufs[i % 2] for i in range(n)])
    torch.cuda.synchronize()
    assert int(dec.status.item()) == 0
    o16 = out.view(torch.int16)
    for i in range(n):
        assert torch.equal(o16[i], want[i % 2]), i
    del out, o16


@pytest.mark.parametrize("rs", [False, True])
def test_deepcam_raw16_lines_w1152(dev, orc, rs):
    """FORMAT.md 2.6 RAW16 lines at W = 1152 among SEG lines (one-pass instance
    with rs, else the general line path): bit-exact, normalised and x-hat; a
    RAW16 line shorter than 16 + 2 W bytes is reported."""
    W, C, H = 1152, 2, 6
    rng = np.random.default_rng(7)
    h16 = rng.integers(0, 1 << 16, size=(C * H, W), dtype=np.uint16)
    h16[:, ::5] = 0x7C00 | (h16[:, ::5] & 0x8000)          # infinities
    h16[:, 1::7] &= 0x83FF                                  # subnormals and zeros
    h16[(h16 & 0x7C00) == 0x7C00] &= 0xFC00                 # no NaN patterns (the encoder never writes them)
    lines = []
    for l in range(C * H):
        if l % 3 == 1:
            lines.append(fmt.build_seg_line(W, [(W, 1, 140, 1.0)], [1] * (W - 1)))
        else:
            lines.append(bytes([2]) + b"\0" * 15 + h16[l].astype("<u2").tobytes())
    b = fmt.build_deepcam_stream(C, H, W, lines, A=36)
    shift, scale = np.float32([0.5, -3.0]), np.float32([2.0, 1e-3])
    for out, sh, sc in (("f16", shift, scale), ("f32", shift, scale), ("f32", None, None)):
        got, st = _decode("deepcam", [b, b], (C, H, W), out=out, shift=sh, scale=sc, raw_segments=rs)
        assert st == 0
        want = _dc_ref(orc, b, (C, H, W), sh, sc, out)
        _same_bits(got[0], want)
        _same_bits(got[1], want)
    short = bytes([2]) + b"\0" * 15 + b"\0" * (2 * W - 16)
    bad = fmt.build_deepcam_stream(C, H, W, lines[:-1] + [short], A=36)
    _, st = _decode("deepcam", [b, bad], (C, H, W), out="f16", raw_segments=rs)
    assert st == (3 | (1 << 8))


@pytest.mark.parametrize("rs", [False, True])
def test_deepcam_raw_segment_onepass_corruption(dev, rs):
    """W = 1152, A = 36 (one-pass path with rs): a RAW segment (kind 2) in a mode-1
    line, and a RAW segment whose 4 len bytes run past the line, are reported
    as corrupt on the sample that holds them (FORMAT.md 2.7)."""
    W, A = 1152, 36
    v = np.arange(A, dtype=np.float32)
    good = fmt.build_seg_line(W, [(A, 2, 0, v[0]), (W - A, 0, 0, 1.0)], v.astype("<f4").tobytes(), mode=3)
    in_mode1 = fmt.build_seg_line(W, [(A, 2, 0, v[0]), (W - A, 0, 0, 1.0)], v.astype("<f4").tobytes(), mode=1)
    too_long = fmt.build_seg_line(W, [(W - A, 2, 0, v[0]), (A, 0, 0, 1.0)], v.astype("<f4").tobytes(), mode=3)
    ok = fmt.build_deepcam_stream(1, 2, W, [good, good], A=A)
    for bad in (in_mode1, too_long):
        b = fmt.build_deepcam_stream(1, 2, W, [good, bad], A=A)
        _, st = _decode("deepcam", [ok, b], (1, 2, W), out="f16", raw_segments=rs)
        assert st == (3 | (1 << 8))
    got, st = _decode("deepcam", [ok], (1, 2, W), out="f32", raw_segments=rs)
    assert st == 0
    want = np.concatenate([v, np.ones(W - A, np.float32)])
    _same_bits(got[0, 0, 0], want)
    _same_bits(got[0, 0, 1], want)


def test_deepcam_corruption_detected(dev):
    W = 64
    good = fmt.build_seg_line(W, [(W, 1, 140, 1.0)], [1] * (W - 1))
    bad_sum = fmt.build_seg_line(W, [(W - 1, 1, 140, 1.0)], [1] * (W - 2))
    bad_kind = fmt.build_seg_line(W, [(W, 5, 140, 1.0)], [1] * (W - 1))
    for bad in (bad_sum, bad_kind):
        b = fmt.build_deepcam_stream(1, 2, W, [good, bad])
        _, st = _decode("deepcam", [b, b], (1, 2, W), out="f16")
        assert st & 0xFF == 3
    b = fmt.build_deepcam_stream(1, 2, W, [good, good])
    c = b.copy(); c[0] = 0
    _, st = _decode("deepcam", [b, c], (1, 2, W), out="f16")
    assert st == (3 | (1 << 8))
    # a RAW16 line (FORMAT.md 2.6) shorter than 16 + 2 W bytes, and an unknown line mode
    short16 = bytes([2]) + b"\0" * 15 + b"\0" * (2 * W - 16)
    mode9 = bytes([9]) + b"\0" * 15 + b"\0" * (2 * W)
    for bad in (short16, mode9):
        b = fmt.build_deepcam_stream(1, 2, W, [good, bad])
        _, st = _decode("deepcam", [b, b], (1, 2, W), out="f16")
        assert st & 0xFF == 3


def test_deepcam_mixed_line_modes_batch(dev, orc):
    """One batch mixing streams of every line mode the encoders write: the
    default SEG stream, an error-budget stream (fp32 RAW lines), a RAW16
    stream, a knob-tuned stream; every output bit-exact."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_deepcam(2011, H=96)
    mean, rstd = deepcam_stats(x)
    bufs = [spp.spp_encode_deepcam(x), spp.spp_encode_deepcam(x, err_budget=4),
            spp.spp_encode_deepcam(x, err_budget=4, raw16=True), spp.spp_encode_deepcam(x, lookahead=8, repeat_min=4)]
    got, st = _decode("deepcam", bufs, x.shape, out="f16", shift=mean, scale=rstd)
    assert st == 0
    for g, b in zip(got, bufs):
        _same_bits(g, _dc_ref(orc, b, x.shape, mean, rstd, "f16"))


# ------------------------------------------------------------------ streamed (b.4 + b.5)
@pytest.mark.parametrize("fmt_name", ["cosmo", "deepcam"])
def test_host_pipeline_matches_device_decode(dev, fmt_name):
    from synth import gen_cosmo, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, HostPipeline, spp
    if fmt_name == "cosmo":
        xs = [gen_cosmo(1001 + i, n=64) for i in range(5)]
        bs = [spp.spp_encode_cosmo(x) for x in xs]
    else:
        xs = [gen_deepcam(2001 + i, H=64) for i in range(5)]
        bs = [spp.spp_encode_deepcam(x) for x in xs]
    dims = xs[0].shape
    host = [torch.from_numpy(b).pin_memory() for b in bs] * 3
    dec = Decoder(fmt_name, dims)
    ref = dec.decode([_to_dev(b) for b in bs])
    pipe = HostPipeline(dec, slot_bytes=2 * max(b.size for b in bs) + 64, nslots=3, max_chunk=2)
    out = dec.alloc_out(len(host))
    pipe.decode(host, out)
    torch.cuda.synchronize()
    assert int(dec.status.item()) == 0
    for i in range(len(host)):
        assert torch.equal(out[i].view(torch.int16), ref[i % 5].view(torch.int16))
    assert pipe.launches() == 2 * ((len(host) + 1) // 2)
    pipe.close()


@pytest.mark.parametrize("fmt_name", ["cosmo", "deepcam"])
def test_host_pipeline_coalesced_runs(dev, fmt_name):
    """spp_decode_host copies samples that lie back to back in host memory as
    one transfer: a packed pinned pool (runs that break at the pool wrap and
    at chunk and slot boundaries) decodes exactly like the device path."""
    from synth import gen_cosmo, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, HostPipeline, spp
    if fmt_name == "cosmo":
        bs = [spp.spp_encode_cosmo(gen_cosmo(1101 + i, n=48)) for i in range(4)]
        dims = (4, 48, 48, 48)
    else:
        bs = [spp.spp_encode_deepcam(gen_deepcam(2101 + i, H=40)) for i in range(4)]
        dims = (16, 40, 1152)
    offs = np.concatenate([[0], np.cumsum([b.size for b in bs])]).astype(np.int64)
    packed = torch.empty(int(offs[-1]), dtype=torch.uint8).pin_memory()
    for i, b in enumerate(bs):
        packed[int(offs[i]):int(offs[i + 1])].copy_(torch.from_numpy(b))
    views = [packed[int(offs[i]):int(offs[i + 1])] for i in range(4)]
    order = [0, 1, 2, 3, 0, 1, 3, 2, 2, 3, 0, 1, 2]
    host = [views[i] for i in order]
    dec = Decoder(fmt_name, dims)
    ref = dec.decode([_to_dev(b) for b in bs])
    for max_chunk, slot in ((3, 3 * max(b.size for b in bs)), (8, 2 * max(b.size for b in bs) + 64)):
        pipe = HostPipeline(dec, slot_bytes=slot, nslots=2, max_chunk=max_chunk)
        out = dec.alloc_out(len(host))
        pipe.decode(host, out)
        torch.cuda.synchronize()
        assert int(dec.status.item()) == 0
        for j, i in enumerate(order):
            assert torch.equal(out[j].view(torch.int16), ref[i].view(torch.int16)), (max_chunk, j)
        pipe.close()


@pytest.mark.parametrize("rs", [False, True])
def test_deepcam_tolerance_streams(dev, orc, rs):
    """FORMAT.md 2.8 streams (per-channel REPEAT tolerance and absolute bound,
    alone and with RAW16 lines / RAW segments): decoded bit-exact on both W = 1152
    KD instances; every value of a bounded channel within its bound."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import spp
    x = gen_deepcam(2013, H=48)
    mean, rstd = deepcam_stats(x)
    tau, eps = (0.02 / rstd).astype(np.float32), (0.005 / rstd).astype(np.float32)
    bufs = [spp.spp_encode_deepcam(x, repeat_tol=tau), spp.spp_encode_deepcam(x, max_abs_err=eps),
            spp.spp_encode_deepcam(x, repeat_tol=tau, max_abs_err=eps, raw16=True, err_budget=8),
            spp.spp_encode_deepcam(x, repeat_tol=tau, max_abs_err=eps, raw_segments=True, err_budget=8)]
    got, st = _decode("deepcam", bufs, x.shape, out="f16", shift=mean, scale=rstd, raw_segments=rs)
    assert st == 0
    for g, b in zip(got, bufs):
        _same_bits(g, _dc_ref(orc, b, x.shape, mean, rstd, "f16"))
    got, st = _decode("deepcam", bufs, x.shape, out="f32", raw_segments=rs)
    assert st == 0
    for k, (g, b) in enumerate(zip(got, bufs)):
        _same_bits(g, _dc_ref(orc, b, x.shape, None, None, "f32"))
        if k >= 1:
            assert np.all(np.abs(g.astype(np.float64) - x) <= eps[:, None, None].astype(np.float64))
