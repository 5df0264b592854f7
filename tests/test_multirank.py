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
