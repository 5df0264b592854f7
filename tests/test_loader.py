"""Loader integration: the sampler and shard packing on CPU,
and on the GPU that every batch the loader yields is bit-identical to the
oracle's decode of the sampled indices (device source with CUDA-graph replay,
and host source streamed through spp_decode_host), in the permuted order."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")


# ------------------------------------------------------------------ CPU: host logic
def test_sampler_partitions_each_epoch():
    from paper_conf_ipps_ibrahimo22_b200.loader import EpochSampler
    n, world = 23, 3
    for epoch in range(3):
        parts = [EpochSampler(n, r, world, seed=7).indices(epoch) for r in range(world)]
        assert len({len(p) for p in parts}) == 1 and len(parts[0]) == n // world
        allidx = np.concatenate(parts)
        assert len(set(allidx.tolist())) == len(allidx)          # disjoint
        assert set(allidx.tolist()) <= set(range(n))
    a = EpochSampler(n, 0, 1, seed=7)
    assert sorted(a.indices(0).tolist()) == list(range(n))          # world 1: a permutation
    assert not np.array_equal(a.indices(0), a.indices(1))           # reshuffled per epoch
    assert np.array_equal(a.indices(2), EpochSampler(n, 0, 1, seed=7).indices(2))  # deterministic
    assert np.array_equal(EpochSampler(n, 0, 1, shuffle=False).indices(5), np.arange(n))


def test_sampler_batches():
    from paper_conf_ipps_ibrahimo22_b200.loader import EpochSampler
    s = EpochSampler(10, 0, 1, seed=1)
    b = s.batches(0, 4)
    assert [len(x) for x in b] == [4, 4]
    assert [len(x) for x in s.batches(0, 4, drop_last=False)] == [4, 4, 2]
    assert np.array_equal(np.concatenate(s.batches(0, 4, drop_last=False)), s.indices(0))
    with pytest.raises(ValueError):
        EpochSampler(2, 0, 3)


def test_shard_packing():
    from paper_conf_ipps_ibrahimo22_b200.loader import EncodedShard
    rng = np.random.default_rng(0)
    bufs = [rng.integers(0, 256, size=64 + 16 * int(k), dtype=np.uint8) for k in rng.integers(0, 40, size=7)]
    sh = EncodedShard(bufs, pin=False)
    assert len(sh) == 7 and sh.nbytes == sum(b.size for b in bufs)
    assert all(int(o) % 256 == 0 for o in sh.offsets)
    for i, b in enumerate(bufs):
        assert np.array_equal(sh.host_view(i).numpy(), b)
    with pytest.raises(ValueError):
        EncodedShard([np.zeros(65, np.uint8)], pin=False)


# ------------------------------------------------------------------ GPU: parity of every batch
def _setup(fmt_name, n_samples):
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import deepcam_stats, gen_cosmo, gen_deepcam
    if fmt_name == "cosmo":
        xs = [gen_cosmo(4100 + i, n=16) for i in range(n_samples)]
        return xs, [spp.spp_encode_cosmo(x) for x in xs], xs[0].shape, None
    if fmt_name == "cosmo_escaped":  # FORMAT.md 1.5 streams (32^3: more than 256 groups)
        xs = [gen_cosmo(4100 + i, n=32) for i in range(n_samples)]
        return xs, [spp.spp_encode_cosmo(x, escape=True) for x in xs], xs[0].shape, None
    xs = [gen_deepcam(4200 + i, H=8, W=1152) for i in range(n_samples)]
    return xs, [spp.spp_encode_deepcam(x) for x in xs], xs[0].shape, deepcam_stats(xs[0])


@pytest.mark.gpu
@pytest.mark.parametrize("fmt_name", ["cosmo", "deepcam", "cosmo_escaped"])
@pytest.mark.parametrize("source,graph", [("device", True), ("device", False), ("host", False)])
def test_loader_batches_match_oracle(fmt_name, source, graph, orc):
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_ibrahimo22_b200 import Decoder
    from paper_conf_ipps_ibrahimo22_b200.loader import DecodeLoader, EncodedShard, EpochSampler
    xs, bufs, dims, stats = _setup(fmt_name, 11)
    want = [orc.cosmo_direct(x, 1, "f16") if fmt_name.startswith("cosmo")
            else orc.deepcam_decode(b, dims, stats[0], stats[1], "f16") for x, b in zip(xs, bufs)]
    dec = Decoder(fmt_name.split("_")[0], dims, out="f16", escape_keys=fmt_name == "cosmo_escaped")
    if fmt_name == "cosmo_escaped":
        from tests import fmt
        assert all(fmt.cosmo_header(b)["slabs"][0]["kw"] == 3 for b in bufs)
    if stats is not None:
        dec.set_normalisation(stats[0], stats[1])
    shard = EncodedShard(bufs, device_resident=(source == "device"))
    sampler = EpochSampler(len(bufs), seed=3)
    ld = DecodeLoader(dec, shard, batch_size=3, sampler=sampler, source=source, depth=2, cuda_graph=graph,
                      chunk=2)
    seen = []
    for epoch in range(2):
        order = []
        for batch, idx in ld:
            # consumer-side work on the batch (on the current stream), then compare
            got = batch.float().cpu().numpy()
            for j, i in enumerate(idx):
                w = want[int(i)].astype(np.float32)
                nan = np.isnan(w)
                assert np.array_equal(np.isnan(got[j]), nan)
                assert np.array_equal(got[j][~nan], w[~nan]), f"epoch {epoch} sample {i}"
            order.extend(int(i) for i in idx)
        assert len(order) == 9 and len(set(order)) == 9
        seen.append(order)
    assert seen[0] != seen[1]                      # epoch reshuffle
    assert ld.launches > 0
    ld.close()


@pytest.mark.gpu
def test_loader_overlaps_consumer_work(orc):
    """A slow consumer (matmuls on the current stream) must see correct
    batches: the ring slot is not overwritten while its batch is in use."""
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_ibrahimo22_b200 import Decoder
    from paper_conf_ipps_ibrahimo22_b200.loader import DecodeLoader, EncodedShard, EpochSampler
    xs, bufs, dims, _ = _setup("cosmo", 8)
    want = [orc.cosmo_direct(x, 1, "f16") for x in xs]
    dec = Decoder("cosmo", dims, out="f16")
    ld = DecodeLoader(dec, EncodedShard(bufs, device_resident=True), 2, EpochSampler(8, seed=5), depth=3)
    a = torch.randn(2048, 2048, device="cuda")
    sums = []
    for batch, idx in ld:
        for _ in range(20):
            a = torch.tanh(a @ a * 1e-3)           # keep the consumer stream busy
        sums.append((batch.float().sum(dim=(1, 2, 3, 4)), idx))
    torch.cuda.synchronize()
    for s, idx in sums:
        for j, i in enumerate(idx):
            assert float(s[j]) == pytest.approx(float(want[int(i)].astype(np.float32).sum()), rel=1e-5)
