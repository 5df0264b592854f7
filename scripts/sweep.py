"""C5 (BASELINE.json configs[4]): value-distribution sweep — compression ratio
vs device-resident decode throughput, CosmoFlow 4x128^3 -> fp16.

For each generator preset (lambda x rho_c grid of SURVEY.md §8d C5, plus the
all-zero volume) a pool of samples is encoded on the host, replicated into a
batch of distinct HBM buffers, decoded with spp_decode_batch (CUDA events,
warm-up first) and checked against the oracle's plain definition on one
sample.  Output: one JSON object with a row per preset.
"""
import argparse
import json
import sys
import time
from pathlib import Path

import numpy as np

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))


def main():
    from synth import gen_cosmo

    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=128)
    ap.add_argument("--pool", type=int, default=4)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--policies", default="default,localized",
                    help="encoder policies per preset: default (FORMAT.md 1.3), localized (1.4)")
    ap.add_argument("--only", default="", help="comma-separated preset names to run (default: all)")
    a = ap.parse_args()
    grid = [(lam, rho) for lam in (0.01, 0.05, 1.0, 2.0, 16.0, 64.0) for rho in (0.9, 0.7, 0.0)]
    rows = []
    peak = json.loads((Path(__file__).resolve().parent.parent / "MEASURED_PEAKS.json").read_text())["hbm_gbs"] \
        if (Path(__file__).resolve().parent.parent / "MEASURED_PEAKS.json").exists() else 6650.0
    cases = [("zeros", None, None)] + [(f"lam{lam}_rho{rho}", lam, rho) for lam, rho in grid]
    policies = a.policies.split(",")
    if a.only:
        cases = [c for c in cases if c[0] in a.only.split(",")]
    for name, lam, rho in cases:
        if lam is None:
            xs = [np.zeros((4, 128, 128, 128), dtype=np.int16)]
        else:
            xs = [gen_cosmo(3001 + i, "paper", lam=lam, rho_c=rho) for i in range(a.pool)]
        for policy in policies:
            rows.append(measure(a, name, policy, lam, rho, xs, peak))
            print(json.dumps(rows[-1]), file=sys.stderr, flush=True)
    print(json.dumps({"config": "C5 sweep, CosmoFlow 4x128^3 -> fp16, batch %d, pool %d" % (a.batch, a.pool),
                      "rows": rows}, indent=1))


def measure(a, name, policy, lam, rho, xs, peak):
    import torch

    import oracle
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    t0 = time.time()
    bufs = [spp.spp_encode_cosmo(x, localize=(policy == "localized")) for x in xs]
    info = [spp.spp_stream_info("cosmo", b) for b in bufs]
    P = len(bufs)
    slots = [((b.size + 255) // 256) * 256 for b in bufs]
    offs = np.zeros(a.batch + 1, dtype=np.int64)
    for i in range(a.batch):
        offs[i + 1] = offs[i] + slots[i % P]
    src = torch.empty(int(offs[-1]), dtype=torch.uint8, device="cuda")
    for i in range(a.batch):
        src[int(offs[i]): int(offs[i]) + bufs[i % P].size].copy_(torch.from_numpy(bufs[i % P]))
    ptrs = torch.from_numpy(offs[:a.batch] + src.data_ptr()).cuda()
    dec = Decoder("cosmo", (4, 128, 128, 128))
    out = dec.alloc_out(a.batch)
    for _ in range(3):
        dec.decode(ptrs, out=out, n=a.batch)
    torch.cuda.synchronize()
    dec.check_status()
    ok = bool(np.array_equal(out[0].cpu().numpy().view(np.uint16),
                             oracle.cosmo_direct(xs[0], 1, "f16").view(np.uint16)))
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    s.record()
    for _ in range(a.steps):
        dec.decode(ptrs, out=out, n=a.batch)
    e.record()
    torch.cuda.synchronize()
    dt = s.elapsed_time(e) / 1e3 / a.steps
    in_b = sum(bufs[i % P].size for i in range(a.batch))
    out_b = out.numel() * 2
    row = {"preset": name, "policy": policy, "lambda": lam, "rho_c": rho,
           "ratio": float(np.mean([x.nbytes / b.size for x, b in zip(xs, bufs)])),
           "nU": int(np.mean([i[0] for i in info])), "slabs": int(max(i[1] for i in info)),
           "G_slab0": int(np.mean([i[2] for i in info])), "kw_slab0": int(info[0][3]),
           "samples_per_s": a.batch / dt, "GBps_alg": (in_b + out_b) / dt / 1e9,
           "frac_of_measured_hbm": (in_b + out_b) / dt / 1e9 / peak, "parity_sample0": ok,
           "setup_s": time.time() - t0}
    del src, out, ptrs
    torch.cuda.empty_cache()
    return row


if __name__ == "__main__":
    main()
