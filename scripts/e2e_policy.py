#!/usr/bin/env python
"""Streamed (pinned host -> PCIe -> decode) vs HBM-resident throughput of the
two CosmoFlow encoder policies (FORMAT.md 1.3 default, 1.4 localized tables)
on chosen generator presets.  In streamed mode the host->device link bounds
the rate, so the policy with fewer bytes per sample decodes
more samples per second even when its resident decode is slower.

usage (GPU): python scripts/e2e_policy.py [--batch 256] > profiles/r01_e2e_policy.json
"""
from __future__ import annotations

import argparse
import json
import sys
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))


def main():
    import torch

    import oracle
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, HostPipeline, spp
    from synth import gen_cosmo

    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=256)
    ap.add_argument("--pool", type=int, default=4)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--chunk", type=int, default=16)
    a = ap.parse_args()
    dims = (4, 128, 128, 128)
    presets = [("sparse lam0.05 rho0.7", dict(lam=0.05, rho_c=0.7)), ("sparse lam0.05 rho0.0", dict(lam=0.05, rho_c=0.0)),
               ("paper lam2 rho0.7", dict(lam=2.0, rho_c=0.7))]
    rows = []
    for name, kw in presets:
        xs = [gen_cosmo(3001 + i, "paper", **kw) for i in range(a.pool)]
        for policy in ("default", "localized"):
            bufs = [spp.spp_encode_cosmo(x, localize=policy == "localized") for x in xs]
            sizes = [b.size for b in bufs]
            dec = Decoder("cosmo", dims)
            out = dec.alloc_out(a.batch)
            # resident: one device buffer per sample of the batch
            dsrc = [torch.from_numpy(bufs[i % a.pool]).cuda() for i in range(a.batch)]
            for _ in range(2):
                dec.decode(dsrc, out=out)
            torch.cuda.synchronize()
            dec.check_status()
            ok = bool(np.array_equal(out[0].cpu().numpy().view(np.uint16),
                                     oracle.cosmo_direct(xs[0], 1, "f16").view(np.uint16)))
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record()
            for _ in range(a.steps):
                dec.decode(dsrc, out=out)
            e.record()
            torch.cuda.synchronize()
            t_res = s.elapsed_time(e) / 1e3 / a.steps
            del dsrc
            # streamed: the pool packed back to back in pinned memory
            offs = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int64)
            host_all = torch.empty(int(offs[-1]), dtype=torch.uint8).pin_memory()
            for i, b in enumerate(bufs):
                host_all[int(offs[i]): int(offs[i + 1])].copy_(torch.from_numpy(b))
            host = [host_all[int(offs[i]): int(offs[i + 1])] for i in range(a.pool)]
            srcs = [host[i % a.pool] for i in range(a.batch)]
            pipe = HostPipeline(dec, slot_bytes=max(sizes) * a.chunk + 4096, nslots=3, max_chunk=a.chunk)
            pipe.decode(srcs, out)
            torch.cuda.synchronize()
            s.record()
            for _ in range(a.steps):
                pipe.decode(srcs, out)
            e.record()
            torch.cuda.synchronize()
            t_e2e = s.elapsed_time(e) / 1e3 / a.steps
            dec.check_status()
            ok = ok and bool(np.array_equal(out[a.batch - 1].cpu().numpy().view(np.uint16),
                                            oracle.cosmo_direct(xs[(a.batch - 1) % a.pool], 1, "f16").view(np.uint16)))
            pipe.close()
            in_b = sum(sizes[i % a.pool] for i in range(a.batch))
            rows.append({"preset": name, "policy": policy, "bytes_per_sample": in_b / a.batch,
                         "ratio": 2 * 4 * 128 ** 3 / (in_b / a.batch),
                         "resident_samples_per_s": a.batch / t_res, "e2e_samples_per_s": a.batch / t_e2e,
                         "e2e_h2d_GBps": in_b / t_e2e / 1e9, "parity": ok})
            print(json.dumps(rows[-1]), file=sys.stderr, flush=True)
            del out, host_all
            torch.cuda.empty_cache()
    print(json.dumps({"what": "CosmoFlow encoder policies: resident vs streamed (pinned H2D) decode, fp16 out",
                      "batch": a.batch, "pool": a.pool, "chunk": a.chunk, "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
