#!/usr/bin/env python
"""BASELINE.json configs[0] / configs[2]: one sample,
encoded on the host and decoded on one GPU, next to the CPU oracle.

Reports, per format: host encode ms (product encoder and the oracle's), the
oracle's decode ms on one thread, and the GPU decode latency of the single
sample (prologue + main kernel) replayed from a CUDA graph, for each output
type.  A repeated single sample stays L2-warm, so this is latency, not
bandwidth (the roofline numbers come from the C2 / C4 batches in bench.py).
Every GPU output is checked bit for bit against the oracle.

usage (GPU): python scripts/single_sample.py > profiles/r01_single_sample.json
"""
from __future__ import annotations

import json
import sys
import time
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))


def timed(fn, reps=3):
    best = float("inf")
    out = None
    for _ in range(reps):
        t0 = time.perf_counter()
        out = fn()
        best = min(best, time.perf_counter() - t0)
    return out, best * 1e3


def gpu_latency_us(dec, src, out, reps=200):
    import torch
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    ptrs = torch.tensor([t.data_ptr() for t in src], dtype=torch.int64, device="cuda")
    with torch.cuda.stream(s):
        for _ in range(3):
            dec.decode(ptrs, out=out, n=len(src))
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        dec.decode(ptrs, out=out, n=len(src))
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    with torch.cuda.stream(s):
        g.replay()
        e0.record(s)
        for _ in range(reps):
            g.replay()
        e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / reps


def main():
    import torch

    import oracle
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    from synth import deepcam_stats, gen_cosmo, gen_deepcam
    rows = {}
    # ---- C1: one CosmoFlow sample 4x128^3 (paper preset, seed 1001)
    x = gen_cosmo(1001)
    b, enc_ms = timed(lambda: spp.spp_encode_cosmo(x))
    _, enc_orc_ms = timed(lambda: oracle.cosmo_encode(x), reps=1)
    be, enc_esc_ms = timed(lambda: spp.spp_encode_cosmo(x, escape=True))
    nU, T, G, kw = spp.spp_stream_info("cosmo", b)
    r = {"shape": list(x.shape), "encoded_bytes": int(b.size), "ratio": x.nbytes / b.size, "nU": nU, "slabs": T,
         "G": G, "kw": kw, "encode_ms": enc_ms, "encode_oracle_ms": enc_orc_ms,
         "encode_escaped_ms": enc_esc_ms, "ratio_escaped": x.nbytes / be.size, "gpu_us": {}, "parity": {}}
    for out, tr in (("f16", 1), ("f32", 1), ("i16", 0)):
        want, oms = timed(lambda: oracle.cosmo_decode(b, x.shape, tr, out), reps=2)
        r[f"oracle_decode_ms_{out}"] = oms
        for esc, buf in ((False, b), (True, be)):
            dec = Decoder("cosmo", x.shape, out=out, transform=tr, escape_keys=esc)
            src = [torch.from_numpy(buf).cuda()]
            o = dec.alloc_out(1)
            key = out + ("_escaped" if esc else "")
            r["gpu_us"][key] = gpu_latency_us(dec, src, o)
            dec.check_status()
            got = o[0].cpu().numpy()
            r["parity"][key] = bool(np.array_equal(got.view(np.uint16 if got.itemsize == 2 else np.uint32),
                                                   want.view(np.uint16 if want.itemsize == 2 else np.uint32)))
    rows["C1_cosmo"] = r
    print(json.dumps({"C1_cosmo": r}), file=sys.stderr, flush=True)
    # ---- C3: one DeepCAM sample 16x768x1152 (seed 2001), per-channel normalisation
    y = gen_deepcam(2001)
    mean, rstd = deepcam_stats(y)
    d, enc_ms = timed(lambda: spp.spp_encode_deepcam(y))
    _, enc_orc_ms = timed(lambda: oracle.deepcam_encode(y), reps=1)
    raw, seg, nseg, dbytes = spp.spp_stream_info("deepcam", d)
    r = {"shape": list(y.shape), "encoded_bytes": int(d.size), "ratio": y.nbytes / d.size, "raw_lines": raw,
         "seg_lines": seg, "segments": nseg, "encode_ms": enc_ms, "encode_oracle_ms": enc_orc_ms, "gpu_us": {},
         "parity": {}}
    for out in ("f16", "f32"):
        want, oms = timed(lambda: oracle.deepcam_decode(d, y.shape, mean, rstd, out), reps=1)
        r[f"oracle_decode_ms_{out}"] = oms
        dec = Decoder("deepcam", y.shape, out=out)
        dec.set_normalisation(mean, rstd)
        src = [torch.from_numpy(d).cuda()]
        o = dec.alloc_out(1)
        r["gpu_us"][out] = gpu_latency_us(dec, src, o, reps=50)
        dec.check_status()
        got = o[0].cpu().numpy()
        nan = np.isnan(want)
        iv = np.uint16 if got.itemsize == 2 else np.uint32
        r["parity"][out] = bool(np.array_equal(np.isnan(got), nan) and
                                np.array_equal(got[~nan].view(iv), want[~nan].view(iv)))
    rows["C3_deepcam"] = r
    print(json.dumps({"what": "single-sample encode / decode (BASELINE configs[0], configs[2]); GPU latency from "
                      "CUDA-graph replays of one sample (L2-warm: latency, not bandwidth)", **rows}, indent=1))


if __name__ == "__main__":
    main()
