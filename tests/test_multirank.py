"""World-size-2 gloo tests of the multi-rank host logic (no GPU): sharding is a
partition, the MAX reduction of elapsed time, and shard invariance of the
decoded outputs (P13, PAPER.md P:84 per-line/per-sample independence) with the
oracle standing in for the device decode."""
import hashlib
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ipps_ibrahimo22_b200.shard import aggregate_throughput, max_over_ranks, shard_indices
        from paper_conf_ipps_ibrahimo22_b200 import spp
        from synth import gen_cosmo
        idx = shard_indices(6, rank, world)
        hashes = {}
        for i in idx:
            x = gen_cosmo(500 + i, n=16)
            b = spp.spp_encode_cosmo(x)
            out = oracle.cosmo_decode(b, x.shape, 1, "f16")
            hashes[i] = hashlib.sha256(out.tobytes()).hexdigest()
        t = max_over_ranks(0.5 + rank, dist)
        gathered = [None] * world
        dist.all_gather_object(gathered, hashes)
        q.put((rank, idx, t, gathered, aggregate_throughput(len(idx), world, 1, t)))
    finally:
        dist.destroy_process_group()


def test_two_rank_sharding_and_timing():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + (os.getpid() % 1000)
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    (r0, idx0, t0, g0, v0), (r1, idx1, t1, g1, v1) = res
    assert sorted(idx0 + idx1) == list(range(6)) and not set(idx0) & set(idx1)
    assert t0 == t1 == 1.5                        # MAX over ranks
    assert v0 == v1 == 2 * 3 / 1.5
    merged = {**g0[0], **g0[1]}
    # single-process reference for the same six samples
    import oracle
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import gen_cosmo
    for i in range(6):
        x = gen_cosmo(500 + i, n=16)
        out = oracle.cosmo_decode(spp.spp_encode_cosmo(x), x.shape, 1, "f16")
        assert merged[i] == __import__("hashlib").sha256(out.tobytes()).hexdigest()


def _gpu_worker(rank, world, port, q):
    """Rank `rank` decodes ITS shard of a 6-sample CosmoFlow set and a 4-sample
    DeepCAM set on the GPU through the real data plane (libspp kernels), and
    publishes per-sample output hashes via all_gather_object."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
        from paper_conf_ipps_ibrahimo22_b200.shard import shard_indices
        from synth import deepcam_stats, gen_cosmo, gen_deepcam
        hashes = {}
        ci = shard_indices(6, rank, world)
        xs = [gen_cosmo(600 + i, n=32) for i in ci]
        dec = Decoder("cosmo", (4, 32, 32, 32))
        out = dec.decode([torch.from_numpy(spp.spp_encode_cosmo(x)).cuda() for x in xs]).cpu().numpy()
        dec.check_status()
        for j, i in enumerate(ci):
            hashes[("cosmo", i)] = hashlib.sha256(out[j].tobytes()).hexdigest()
        di = shard_indices(4, rank, world)
        ys = [gen_deepcam(700 + i, H=16) for i in di]
        mean, rstd = deepcam_stats(gen_deepcam(700, H=16))
        dd = Decoder("deepcam", (16, 16, 1152))
        dd.set_normalisation(mean, rstd)
        outd = dd.decode([torch.from_numpy(spp.spp_encode_deepcam(y)).cuda() for y in ys]).cpu().numpy()
        dd.check_status()
        for j, i in enumerate(di):
            hashes[("deepcam", i)] = hashlib.sha256(outd[j].tobytes()).hexdigest()
        gathered = [None] * world
        dist.all_gather_object(gathered, hashes)
        q.put((rank, gathered))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
def test_two_rank_gpu_shard_invariance():
    """P13 (PAPER.md P:84 per-sample independence) on the real data plane: two
    ranks (gloo, sharing this GPU) each decode their shard with libspp; the union
    of their per-sample output hashes equals one process decoding every sample
    as one batch."""
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    from synth import deepcam_stats, gen_cosmo, gen_deepcam
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 30500 + (os.getpid() % 1000)
    procs = [ctx.Process(target=_gpu_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(2)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    merged = {**res[0][1][0], **res[0][1][1]}
    assert len(merged) == 10
    xs = [gen_cosmo(600 + i, n=32) for i in range(6)]
    out = Decoder("cosmo", (4, 32, 32, 32)).decode([torch.from_numpy(spp.spp_encode_cosmo(x)).cuda() for x in xs])
    ys = [gen_deepcam(700 + i, H=16) for i in range(4)]
    mean, rstd = deepcam_stats(ys[0])
    dd = Decoder("deepcam", (16, 16, 1152))
    dd.set_normalisation(mean, rstd)
    outd = dd.decode([torch.from_numpy(spp.spp_encode_deepcam(y)).cuda() for y in ys])
    for i in range(6):
        assert merged[("cosmo", i)] == hashlib.sha256(out[i].cpu().numpy().tobytes()).hexdigest()
    for i in range(4):
        assert merged[("deepcam", i)] == hashlib.sha256(outd[i].cpu().numpy().tobytes()).hexdigest()
