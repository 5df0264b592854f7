#!/usr/bin/env python
"""Decode throughput of larger CosmoFlow decompositions (
PAPER.md P:96 512^3 simulation histograms, "for larger than 128^3
decompositions, multiple lookup tables are required"): 4x256^3 (paper-preset
generator) and 4x512^3 (64 offset copies of a paper-shaped 128^3 sample),
HBM-resident, fp16 ln(1+c), checked against the oracle on sampled planes.

usage (GPU): python scripts/big_volume.py > profiles/r01_big_volume.json
"""
from __future__ import annotations

import json
import sys
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))


def volume(n: int) -> np.ndarray:
    from synth import gen_cosmo
    if n <= 256:
        return gen_cosmo(1001, n=n)
    base = gen_cosmo(1001)
    k = n // 128
    off = np.arange(k ** 3, dtype=np.int16).reshape(k, k, k)
    x = np.empty((4, n, n, n), dtype=np.int16)
    for tz in range(k):
        for ty in range(k):
            for tx in range(k):
                x[:, tz * 128:(tz + 1) * 128, ty * 128:(ty + 1) * 128, tx * 128:(tx + 1) * 128] = \
                    base + 7 * off[tz, ty, tx]
    return x


def main():
    import torch

    import oracle
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    peak = json.loads((ROOT / "MEASURED_PEAKS.json").read_text())["hbm_gbs"] \
        if (ROOT / "MEASURED_PEAKS.json").exists() else 6650.0
    rows = []
    for n, batch in ((128, 64), (256, 16), (512, 2)):
        x = volume(n)
        b = spp.spp_encode_cosmo(x)
        nU, T, G, kw = spp.spp_stream_info("cosmo", b)
        src = [torch.from_numpy(b).cuda() for _ in range(batch)]   # distinct HBM copies
        dec = Decoder("cosmo", x.shape)
        out = dec.alloc_out(batch)
        for _ in range(2):
            dec.decode(src, out=out)
        torch.cuda.synchronize()
        dec.check_status()
        ok = all(np.array_equal(out[0][:, z:z + 1].cpu().numpy().view(np.uint16),
                                oracle.cosmo_direct(np.ascontiguousarray(x[:, z:z + 1]), 1, "f16").view(np.uint16))
                 for z in (0, n // 2, n - 1))
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        s.record()
        steps = 5
        for _ in range(steps):
            dec.decode(src, out=out)
        e.record()
        torch.cuda.synchronize()
        dt = s.elapsed_time(e) / 1e3 / steps
        alg = batch * (b.size + out[0].numel() * 2)
        rows.append({"shape": [4, n, n, n], "batch": batch, "encoded_MB": b.size / 1e6, "ratio": 2 * x.size / b.size,
                     "nU": nU, "slabs": T, "G_slab0": G, "kw_slab0": kw, "samples_per_s": batch / dt,
                     "GBps_alg": alg / dt / 1e9, "frac_of_measured_hbm": alg / dt / 1e9 / peak, "parity_planes": ok})
        print(json.dumps(rows[-1]), file=sys.stderr, flush=True)
        del src, out
        torch.cuda.empty_cache()
    print(json.dumps({"what": "CosmoFlow decode at 128^3 / 256^3 / 512^3 decompositions (multi-LUT), fp16, "
                      "HBM-resident distinct copies", "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
