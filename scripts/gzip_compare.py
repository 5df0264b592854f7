#!/usr/bin/env python
"""Our encoded size vs general-purpose gzip on the synthetic sets (SURVEY.md
§8f f4, the comparison half; "roughly 4x, compared with a 5x
compression using the general-purpose gzip", "the gzipped files are
roughly 75% the size of our encoded samples").

For each sample: raw bytes (int16 CDHW counts / fp32 CHW fields), the product
encoder's stream, and zlib (gzip's DEFLATE, level 6 = gzip's default) of the
raw bytes in the CosmoFlow TFRecord layout (channels-last int16) and in
CDHW; plus single-thread host gunzip time per sample (the paper's gzip arm
decompresses on the CPU only).  CPU-only; prints one JSON document.
"""
from __future__ import annotations

import json
import sys
import time
import zlib
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))


def gz(raw: bytes):
    c = zlib.compress(raw, 6)
    t0 = time.perf_counter()
    zlib.decompress(c)
    return len(c), time.perf_counter() - t0


def main():
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import gen_cosmo, gen_deepcam
    rows = []
    for i in range(3):
        x = gen_cosmo(1001 + i)
        enc = spp.spp_encode_cosmo(x).size
        g_cl, t_cl = gz(np.ascontiguousarray(np.moveaxis(x, 0, -1)).tobytes())   # TFRecord: channels-last
        g_cf, _ = gz(x.tobytes())
        rows.append({"app": "cosmoflow", "seed": 1001 + i, "raw": x.nbytes, "ours": int(enc),
                     "gzip_channels_last": g_cl, "gzip_cdhw": g_cf, "ratio_ours": x.nbytes / enc,
                     "ratio_gzip": x.nbytes / g_cl, "gzip_over_ours": g_cl / enc, "gunzip_s_1thread": t_cl})
    for i in range(2):
        x = gen_deepcam(2001 + i)
        enc = spp.spp_encode_deepcam(x).size
        g, t = gz(x.tobytes())
        rows.append({"app": "deepcam", "seed": 2001 + i, "raw": x.nbytes, "ours": int(enc), "gzip": g,
                     "ratio_ours": x.nbytes / enc, "ratio_gzip": x.nbytes / g, "gzip_over_ours": g / enc,
                     "gunzip_s_1thread": t, "note": "ours is lossy (P:86); gzip is lossless"})
    print(json.dumps({"what": "encoded size vs zlib level 6 (gzip default) on the synthetic samples",
                      "paper": {"cosmoflow_ours": "~4x (P:98)", "cosmoflow_gzip": "5x (P:60, P:98)",
                                "gzip_over_ours": "~0.75 (P:219)"}, "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
