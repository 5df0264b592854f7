"""GPU decode of the lossless label streams (FORMAT.md 3; "For
both applications, we use lossless compression of the labels") against the
identity (the masks / vectors themselves) and the oracle's decoder, bit for
bit; corrupt streams reported; labels delivered with their samples by the
loader (the paper's DALI pipeline role)."""
import struct

import numpy as np
import pytest

from tests import fmt
from tests.test_gpu_parity import _to_dev

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_ibrahimo22_b200 import build
    build.build()
    return torch.device("cuda:0")


def _decode(kind, bufs, dims, src_bytes=False):
    from paper_conf_ipps_ibrahimo22_b200 import LabelDecoder
    d = LabelDecoder(kind, dims)
    srcs = [_to_dev(b) for b in bufs]
    sb = torch.tensor([b.size for b in bufs], dtype=torch.int64, device="cuda") if src_bytes else None
    out = d.decode(srcs, src_bytes=sb)
    torch.cuda.synchronize()
    return out.cpu().numpy(), int(d.status.item())


def _runs_mask(rng, H, W):
    """Row y has exactly min(y + 1, W) maximal runs (cut points drawn at random,
    neighbouring runs of different classes): 1..H runs, across the 32-run
    limit of the staged path."""
    m = np.empty((H, W), np.uint8)
    for y in range(H):
        k = min(y + 1, W)
        cuts = np.sort(rng.choice(np.arange(1, W), size=k - 1, replace=False)) if k > 1 else np.array([], int)
        bounds = np.concatenate([[0], cuts, [W]])
        v = int(rng.integers(0, 256))
        for r in range(k):
            m[y, bounds[r]:bounds[r + 1]] = v
            v = (v + 1 + int(rng.integers(0, 255))) % 256
    return m


@pytest.mark.parametrize("H,W", [(768, 1152), (5, 37), (3, 2100), (1, 1), (4, 1024), (40, 1152), (40, 2048),
                                 (36, 16), (40, 1040), (34, 48), (7, 128), (33, 1152), (19, 2304)])
def test_label_masks_lossless(dev, orc, H, W):
    """Paper-shaped DeepCAM masks (cyclone discs, river bands), random masks
    (verbatim rows), constant masks, W not a multiple of 16, W over the 1,024-
    position chunk; rows of exactly 1..40 runs (the staged path takes <= 32 runs
    with W % 16 == 0 and W <= 2048: 1152, 2048, 16, 1040 with a partial last
    lane, 48; 2304 takes the general path; row pairs -- 2 rows of <= 16 runs,
    one half-warp per row (4-row groups of <= 8 runs with SPP_KL_QUADS) -- when
    W % 128 == 0 and W <= 1152: 1152, 1024, 128, odd H); mixed in one batch,
    bit-exact vs the masks and the oracle."""
    from synth import gen_deepcam_labels
    from paper_conf_ipps_ibrahimo22_b200 import spp
    rng = np.random.default_rng(H * 7 + W)
    masks = [gen_deepcam_labels(5000 + i, H=H, W=W) for i in range(6)]
    masks += [rng.integers(0, 256, (H, W), dtype=np.uint8), np.full((H, W), 2, np.uint8),
              (rng.random((H, W)) < 0.5).astype(np.uint8), _runs_mask(rng, H, W)]
    bufs = [spp.spp_encode_label_mask(m) for m in masks]
    for b, m in zip(bufs, masks):
        assert np.array_equal(orc.label_decode(b, 1, H, W), m)
    for sb in (False, True):
        got, st = _decode("mask", bufs, (H, W), src_bytes=sb)
        assert st == 0
        assert np.array_equal(got, np.stack(masks))


def test_label_vectors_bitexact(dev, orc):
    from synth import gen_cosmo_labels
    from paper_conf_ipps_ibrahimo22_b200 import spp
    vs = [gen_cosmo_labels(i) for i in range(63)]
    vs.append(np.frombuffer(np.uint32([0x7FC12345, 0x80000000, 0x00000001, 0x7F800000]).tobytes(), np.float32))
    bufs = [spp.spp_encode_label_vector(v) for v in vs]
    got, st = _decode("vector", bufs, (4,))
    assert st == 0
    assert np.array_equal(got.view(np.uint32), np.stack(vs).view(np.uint32))
    for b, v in zip(bufs, vs):
        assert np.array_equal(orc.label_decode(b, 2, 1, 4).view(np.uint32), v.view(np.uint32))


def test_label_corruption_detected(dev):
    from synth import gen_deepcam_labels
    from paper_conf_ipps_ibrahimo22_b200 import spp
    m = gen_deepcam_labels(9, H=32, W=256)
    good = spp.spp_encode_label_mask(m)
    h = fmt.label_header(good)
    row = h["payload_off"] + int(h["dir"][3])
    bad = [good.copy() for _ in range(5)]
    bad[0][6] = 2                                           # kind
    bad[1][10:12] = np.frombuffer(struct.pack("<H", 255), np.uint8)  # W
    bad[2][row + 4] ^= 0x40                                  # a run length: sum != W
    bad[3][row] = 7                                         # row mode
    bad[4] = good[: good.size // 2].copy()                  # truncated (caught by src_bytes)
    for i, c in enumerate(bad):
        _, st = _decode("mask", [good, c, good], (32, 256), src_bytes=True)
        assert st == (3 | (1 << 8)), (i, st)


def test_label_row_pairs_corruption_and_neighbours(dev):
    """Row pairs (W % 128 == 0: 2 rows of <= 16 runs, else one row per warp;
    4-row groups of <= 8 runs first with SPP_KL_QUADS): a corrupt run length
    in any row of a group is reported on its sample and the other samples of
    the batch decode bit-exactly; rows of 8/9 and 16/17 runs side by side (a
    group falls back to a smaller one when a row has too many runs)."""
    from synth import gen_deepcam_labels
    from paper_conf_ipps_ibrahimo22_b200 import spp
    rng = np.random.default_rng(42)
    H, W = 24, 1152
    m16 = _runs_mask(rng, 40, W)[14:14 + H]  # rows of 15..38 runs: pairs of <= 16 and > 16 runs mixed
    m8 = _runs_mask(rng, 40, W)[np.r_[0:8, 8:12, 4:12, 0:4]]  # rows of 1..12 runs: quads, pairs around 8/9
    masks = [gen_deepcam_labels(71, H=H, W=W), m16, gen_deepcam_labels(72, H=H, W=W), m8]
    bufs = [spp.spp_encode_label_mask(m) for m in masks]
    got, st = _decode("mask", bufs, (H, W), src_bytes=True)
    assert st == 0 and np.array_equal(got, np.stack(masks))
    for y in (0, 1, 2, 3, 6, 7, H - 1):
        bad = bufs[0].copy()
        h = fmt.label_header(bad)
        row = h["payload_off"] + int(h["dir"][y])
        assert bad[row] == 1  # a RUN row
        bad[row + 4] ^= 0x01  # its first run length: the lengths no longer sum to W
        got, st = _decode("mask", [bufs[2], bad, bufs[1]], (H, W), src_bytes=True)
        assert st == (3 | (1 << 8)), (y, st)
        assert np.array_equal(got[0], masks[2]) and np.array_equal(got[2], masks[1])


def test_label_masks_large_launch(dev):
    """A launch writing more than 64 MB of masks (96 paper-shaped 768 x 1152
    masks: the row stores take the L2 evict_first policy) decodes
    bit-exactly, like the small launches above."""
    from synth import gen_deepcam_labels
    from paper_conf_ipps_ibrahimo22_b200 import spp
    masks = [gen_deepcam_labels(6100 + i) for i in range(4)]
    bufs = [spp.spp_encode_label_mask(m) for m in masks]
    n = 96
    assert n * 768 * 1152 > 64 << 20
    got, st = _decode("mask", [bufs[i % 4] for i in range(n)], (768, 1152), src_bytes=True)
    assert st == 0
    for i in range(n):
        assert np.array_equal(got[i], masks[i % 4]), i


@pytest.mark.parametrize("source", ["device", "host"])
def test_loader_delivers_labels(dev, orc, source):
    """DecodeLoader with labels: every batch's decoded samples AND labels match
    the oracle / the original masks for the sampled indices (DeepCAM masks);
    CosmoFlow parameter vectors on the host-source path."""
    from synth import gen_cosmo, gen_cosmo_labels, gen_deepcam, gen_deepcam_labels, deepcam_stats
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, LabelDecoder, spp
    from paper_conf_ipps_ibrahimo22_b200.loader import DecodeLoader, EncodedShard, EpochSampler
    if source == "device":
        xs = [gen_deepcam(2400 + i, H=16) for i in range(6)]
        ms = [gen_deepcam_labels(2400 + i, H=16) for i in range(6)]
        bufs = [spp.spp_encode_deepcam(x) for x in xs]
        mean, rstd = deepcam_stats(xs[0])
        dec = Decoder("deepcam", xs[0].shape)
        dec.set_normalisation(mean, rstd)
        lab = (LabelDecoder("mask", ms[0].shape), EncodedShard([spp.spp_encode_label_mask(m) for m in ms],
                                                               device_resident=True))
        want = lambda i: orc.deepcam_decode(bufs[i], xs[0].shape, mean, rstd, "f16")
    else:
        xs = [gen_cosmo(2500 + i, n=32) for i in range(6)]
        ms = [gen_cosmo_labels(2500 + i) for i in range(6)]
        bufs = [spp.spp_encode_cosmo(x) for x in xs]
        dec = Decoder("cosmo", xs[0].shape)
        lab = (LabelDecoder("vector", (4,)), EncodedShard([spp.spp_encode_label_vector(v) for v in ms],
                                                          device_resident=True))
        want = lambda i: orc.cosmo_direct(xs[i], 1, "f16")
    shard = EncodedShard(bufs, device_resident=(source == "device"))
    loader = DecodeLoader(dec, shard, batch_size=2, sampler=EpochSampler(6, seed=3), source=source, labels=lab)
    seen = 0
    for _ in range(2):
        for batch, labels, idx in loader:
            got, gl = batch.cpu().numpy(), labels.cpu().numpy()
            for j, i in enumerate(idx):
                assert np.array_equal(got[j].view(np.uint16), want(int(i)).view(np.uint16))
                assert np.array_equal(gl[j].view(np.uint8 if source == "device" else np.uint32),
                                      ms[int(i)].view(np.uint8 if source == "device" else np.uint32))
                seen += 1
    assert seen == 12
    loader.close()
