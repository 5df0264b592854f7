"""GPU parity at the limits of the format: every
FORMAT-legal DeepCAM line decodes on the GPU, bit-exact against the oracle,
whatever its length or width; stream-supplied offsets that would wrap a 64-bit
addition are reported as corrupt; streamed decodes on different streams and
loader CUDA graphs stay correct when buffers change.

FORMAT.md 2.1 bounds a line only by u16 fields (W <= 65535, nseg <= W): a SEG
line at A = 1 with one segment per position (9,220 B at W = 1152), or a mode-3
line with hundreds of short RAW segments (FORMAT.md 2.7), is longer than KD's
shared-memory ring and takes the global-memory line path; W > 8192 takes it
for every line.
"""
import struct

import numpy as np
import pytest

from tests import fmt
from tests.test_gpu_parity import _dc_ref, _decode, _same_bits, _to_dev

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_ibrahimo22_b200 import build
    build.build()
    return torch.device("cuda:0")


def _one_per_position_line(rng, W, mode):
    """A SEG line (A = 1) with W segments of length 1 (nseg = W, the FORMAT.md
    maximum): REPEAT, DIFF (no delta byte) and, in mode 3, RAW segments."""
    kinds = (0, 1, 2) if mode == 3 else (0, 1)
    segs, deltas = [], bytearray()
    for p in range(W):
        k = int(rng.choice(kinds))
        v = np.float32(rng.standard_normal() * 10.0 ** rng.integers(-30, 30))
        if k == 2:
            segs.append((1, 2, 0, v))
            deltas += np.float32(v).astype("<f4").tobytes()
        else:
            segs.append((1, k, int(rng.integers(1, 247)) if k == 1 else 0, v))
    return fmt.build_seg_line(W, segs, deltas, mode=mode)


def _many_short_raw_segments_line(rng, W):
    """mode 3: alternating short RAW and DIFF segments, several hundred in all."""
    segs, deltas, pos = [], bytearray(), 0
    while pos < W:
        ln = int(min(W - pos, rng.integers(1, 4)))
        if len(segs) % 2 == 0:
            v = (rng.standard_normal(ln) * 10.0 ** rng.integers(-20, 20)).astype(np.float32)
            segs.append((ln, 2, 0, v[0]))
            deltas += v.astype("<f4").tobytes()
        else:
            segs.append((ln, 1, int(rng.integers(100, 160)), np.float32(rng.standard_normal())))
            deltas += bytes(int(c) for c in rng.integers(0, 256, size=ln - 1))
        pos += ln
    return fmt.build_seg_line(W, segs, deltas, mode=3)


@pytest.mark.parametrize("rs", [False, True])
def test_deepcam_lines_longer_than_the_ring(dev, orc, rs):
    """W = 1152: lines of 1,152 segments (9,220 B and more) and mode-3 lines with
    hundreds of short RAW segments, mixed with ordinary lines; f16/f32 normalised
    and x-hat, bit-exact.  Run on both W = 1152 instances (rs = opts.raw_segments)."""
    W, C, H = 1152, 2, 8
    rng = np.random.default_rng(77)
    lines = []
    for l in range(C * H):
        r = l % 4
        if r == 0:
            lines.append(_one_per_position_line(rng, W, 1))
        elif r == 1:
            lines.append(_one_per_position_line(rng, W, 3))
        elif r == 2:
            lines.append(_many_short_raw_segments_line(rng, W))
        else:
            lines.append(fmt.build_raw_line(rng.standard_normal(W).astype(np.float32)))
    sizes = [len(x) for x in lines]
    assert max(sizes) > 9000 and sum(s > 6176 for s in sizes) >= C * H // 2   # beyond the 3-slot ring
    b = fmt.build_deepcam_stream(C, H, W, lines, A=1)
    shift, scale = np.float32([0.5, -3.0]), np.float32([2.0, 1e-3])
    for out, sh, sc in (("f16", shift, scale), ("f32", shift, scale), ("f32", None, None)):
        got, st = _decode("deepcam", [b, b], (C, H, W), out=out, shift=sh, scale=sc, raw_segments=rs)
        assert st == 0
        want = _dc_ref(orc, b, (C, H, W), sh, sc, out)
        _same_bits(got[0], want)
        _same_bits(got[1], want)


@pytest.mark.parametrize("W,run", [(8192, 7800), (8192, 4200), (12000, 4200)])
def test_deepcam_mode3_raw_segment_far_into_a_wide_line(dev, orc, W, run):
    """a RAW segment starting after position ~4096 of a wide
    mode-3 line (its byte base a = db - 4*start does not fit 16 bits).  The
    library's own encoder writes it: a constant run then abrupt values, error
    budget 1 with RAW segments.  W = 8192 with a 7,800-value run keeps the line
    in shared memory (general path); a 4,200-value run makes it longer than the
    ring (global path); W = 12000 is beyond the shared tables."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    rng = np.random.default_rng(5)
    x = np.empty((1, 4, W), dtype=np.float32)
    for y in range(4):
        x[0, y, :run] = np.float32(1.5 + y)
        x[0, y, run:] = (rng.standard_normal(W - run) * 10.0 ** rng.integers(-3, 3, W - run)).astype(np.float32)
    b = spp.spp_encode_deepcam(x, err_budget=1, raw_segments=True)
    hdr = fmt.deepcam_header(b)
    lines = [fmt.deepcam_line(b, hdr, l) for l in range(4)]
    assert all(ln["mode"] == 3 and ln["segs"][-1]["kind"] == 2 for ln in lines)
    if run == 7800:
        assert max(ln["size"] for ln in lines) < 6000      # fits KD's ring: the shared-memory path
    for out in ("f32", "f16"):
        got, st = _decode("deepcam", [b], x.shape, out=out)
        assert st == 0
        _same_bits(got[0], _dc_ref(orc, b, x.shape, None, None, out))
    # error budget 1: no value above 10% relative error (RAW segments exact)
    got, _ = _decode("deepcam", [b], x.shape, out="f32")
    assert np.all(np.abs(got[0].astype(np.float64) - x) <= 0.1 * np.abs(x.astype(np.float64)))


@pytest.mark.parametrize("W", [8200, 20000, 65535])
def test_deepcam_wide_lines_encoder_streams(dev, orc, W):
    """W beyond the shared tables (every line on the global path), up to the u16
    maximum: encoder streams (smooth, noisy, constant and non-finite lines),
    normalised fp16 and x-hat fp32, bit-exact."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    rng = np.random.default_rng(W)
    C, H = 2, 3
    t = np.linspace(0, 20, W)
    x = np.empty((C, H, W), dtype=np.float32)
    for c in range(C):
        for y in range(H):
            x[c, y] = (np.sin(t * (1 + y)) * 100 + rng.standard_normal(W) * (0.01 if y == 1 else 1.0)).astype(np.float32)
    x[0, 2, :] = np.float32(7.0)
    x[1, 1, W // 3] = np.inf
    b = spp.spp_encode_deepcam(x)
    shift, scale = np.float32([1.0, -2.0]), np.float32([0.01, 3.0])
    got, st = _decode("deepcam", [b], x.shape, out="f16", shift=shift, scale=scale)
    assert st == 0
    _same_bits(got[0], _dc_ref(orc, b, x.shape, shift, scale, "f16"))
    got, st = _decode("deepcam", [b], x.shape, out="f32")
    assert st == 0
    _same_bits(got[0], _dc_ref(orc, b, x.shape, None, None, "f32"))


def test_deepcam_offsets_that_would_wrap(dev):
    """a header whose dir_off + 4 (L + 1) wraps 2^64 is corrupt."""
    W = 64
    good = fmt.build_seg_line(W, [(W, 1, 140, 1.0)], [1] * (W - 1))
    b = fmt.build_deepcam_stream(1, 2, W, [good, good])
    for field, val in ((24, 2 ** 64 - 4 * 3), (24, 2 ** 64 - 4), (32, 2 ** 64 - 16)):
        c = b.copy()
        c[field:field + 8] = np.frombuffer(struct.pack("<Q", val), dtype=np.uint8)
        _, st = _decode("deepcam", [b, c], (1, 2, W), out="f16")
        assert st == (3 | (1 << 8)), (field, val, st)


def test_cosmo_offsets_that_would_wrap(dev):
    """U_off, slab_off, lut_off or keys_off near 2^64 (so that
    offset + length wraps) is corrupt, not an out-of-bounds read."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import gen_cosmo
    x = gen_cosmo(1001, n=16)
    b = spp.spp_encode_cosmo(x)
    hdr = fmt.cosmo_header(b)
    Nt = 16 * 16 * 16
    s0 = hdr["slab_off"]
    cases = [(24, 2 ** 64 - 2), (32, 2 ** 64 - 32), (s0 + 16, 2 ** 64 - 16),
             (s0 + 24, 2 ** 64 - 2 * Nt + 16)]
    for off, val in cases:
        c = b.copy()
        c[off:off + 8] = np.frombuffer(struct.pack("<Q", val % 2 ** 64), dtype=np.uint8)
        _, st = _decode("cosmo", [b, c], x.shape, out="f16")
        assert st & 0xFF == 3 and st >> 8 == 1, (off, val, st)


def test_host_pipeline_two_streams_back_to_back(dev):
    """two spp_decode_host calls on one pipeline, on different
    streams, enqueued back to back: the second waits for the first (shared
    workspace), both outputs equal the device-resident decode."""
    from synth import gen_cosmo
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, HostPipeline, spp
    xs = [gen_cosmo(4100 + i, n=64) for i in range(8)]
    bufs = [spp.spp_encode_cosmo(x) for x in xs]
    dec = Decoder("cosmo", xs[0].shape, out="f16")
    want = dec.decode([_to_dev(b) for b in bufs]).cpu()
    host = [torch.from_numpy(b).pin_memory() for b in bufs]
    pipe = HostPipeline(dec, slot_bytes=max(b.size for b in bufs) * 2 + 4096, nslots=2, max_chunk=2)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    for _ in range(3):
        o1, o2 = dec.alloc_out(4), dec.alloc_out(4)
        pipe.decode(host[:4], o1, stream=s1)
        pipe.decode(host[4:], o2, stream=s2)
        torch.cuda.synchronize()
        dec.check_status()
        assert torch.equal(o1.cpu(), want[:4]) and torch.equal(o2.cpu(), want[4:])
    pipe.close()


def test_loader_graphs_follow_decoder_buffers(dev, orc):
    """CUDA graphs captured by the loader hold the decoder's
    normalisation pointers; after set_normalisation the next pass must use the
    new constants (graphs dropped and re-captured), bit-exact vs the oracle."""
    from synth import gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    from paper_conf_ipps_ibrahimo22_b200.loader import DecodeLoader, EncodedShard, EpochSampler
    xs = [gen_deepcam(2300 + i, H=16) for i in range(4)]
    bufs = [spp.spp_encode_deepcam(x) for x in xs]
    dec = Decoder("deepcam", xs[0].shape, out="f16")
    shard = EncodedShard(bufs, device_resident=True)
    loader = DecodeLoader(dec, shard, batch_size=2, sampler=EpochSampler(4, shuffle=False), cuda_graph=True)
    for k, (sh, sc) in enumerate(((np.zeros(16, np.float32), np.ones(16, np.float32)),
                                  (np.full(16, 3.0, np.float32), np.full(16, 0.25, np.float32)))):
        dec.set_normalisation(sh, sc)
        for _ in range(2):   # second pass replays the captured graphs
            for batch, idx in loader:
                got = batch.cpu().numpy()
                for j, i in enumerate(idx):
                    _same_bits(got[j], orc.deepcam_decode(bufs[int(i)], xs[0].shape, sh, sc, "f16"))


def test_host_pipeline_selects_extended_mode_instance(dev, orc):
    """a stream with RAW-segment / RAW16 lines decoded through
    spp_decode_host with opts.raw_segments = 0 (the caller forgot the flag): the
    pipeline reads the header flags (FORMAT.md 2.1 bit 0) and picks the one-pass
    instance itself; the result is bit-exact either way."""
    from synth import deepcam_stats, gen_deepcam
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, HostPipeline, spp
    xs = [gen_deepcam(2600 + i, H=32) for i in range(3)]
    bufs = [spp.spp_encode_deepcam(x, err_budget=1, raw_segments=True, raw16=True) for x in xs]
    assert all(int(b[6]) & 1 for b in bufs)
    mean, rstd = deepcam_stats(xs[0])
    dec = Decoder("deepcam", xs[0].shape)            # raw_segments left at 0
    dec.set_normalisation(mean, rstd)
    pipe = HostPipeline(dec, slot_bytes=max(b.size for b in bufs) * 2 + 4096, nslots=2, max_chunk=2)
    out = dec.alloc_out(3)
    pipe.decode([torch.from_numpy(b).pin_memory() for b in bufs], out)
    torch.cuda.synchronize()
    dec.check_status()
    pipe.close()
    for g, b in zip(out.cpu().numpy(), bufs):
        _same_bits(g, _dc_ref(orc, b, xs[0].shape, mean, rstd, "f16"))
