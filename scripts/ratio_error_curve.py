#!/usr/bin/env python
"""DeepCAM compression ratio vs reconstruction error over the encoder's policy
knobs ("roughly 3% of values
with more than 10% error").  Encodes paper-shaped samples with
spp_encode_deepcam_ex at several emin lookahead windows / REPEAT thresholds,
decodes them with the product GPU path (fp32 output, no normalisation, so the
output is x-hat itself) and reports bytes/value, ratio, the paper's statistic
(fraction of values with relative error > 10%, reading S19) overall and on the
sparse precipitation-like channel, and the median relative error.

usage (GPU): python scripts/ratio_error_curve.py [--samples 2] > profiles/r01_deepcam_ratio_error.json
"""
from __future__ import annotations

import argparse
import json
import sys
from pathlib import Path

import numpy as np
import torch

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))


def rel_err(x: np.ndarray, xh: np.ndarray) -> np.ndarray:
    r = np.abs(xh.astype(np.float64) - x) / np.maximum(np.abs(x.astype(np.float64)), 1e-300)
    r[(x == 0) & (xh == 0)] = 0.0          # reading S19: x = 0 counts only if x-hat != 0
    return r


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--samples", type=int, default=2)
    ap.add_argument("--H", type=int, default=768)
    args = ap.parse_args()
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    from synth import DEEPCAM_CHANNELS, gen_deepcam

    xs = [gen_deepcam(2001 + i, H=args.H) for i in range(args.samples)]
    C, H, W = xs[0].shape
    precip = [c for c in range(C) if DEEPCAM_CHANNELS[c % len(DEEPCAM_CHANNELS)][0] == "precipitation"]
    dec = Decoder("deepcam", (C, H, W), out="f32")
    rows = []
    settings = [(la, 0, 0) for la in (4, 8, 16, 36, 64, 128, 256, 1152)] + [(64, 4, 0), (64, 64, 0)]
    # FORMAT.md 2.5 error budget: a line with >= k values above 10% error stays RAW
    settings += [(0, 0, k) for k in (256, 64, 16, 4, 1)]
    settings += [(0, 0, -k) for k in (64, 16, 4, 1)]   # negative: the same budgets with RAW16 lines (2.6)
    settings += [(0, 0, 10000 + k) for k in (64, 16, 4, 1)]   # +10000: budgets with RAW segments (2.7)
    settings += [(0, 0, -(10000 + k)) for k in (16, 1)]       # both
    for la, rm, budget in settings:
        nbytes, bad, tot, bad_p, tot_p, med = 0, 0, 0, 0, 0, []
        nseg = 0
        nraw = 0
        for x in xs:
            b = spp.spp_encode_deepcam(x, la, rm, err_budget=abs(budget) % 10000, raw16=budget < 0,
                                       raw_segments=abs(budget) > 10000)
            nbytes += b.size
            info = spp.spp_stream_info("deepcam", b)
            nraw += info[0]
            nseg += info[2]
            src = torch.from_numpy(b).cuda()
            xh = dec.decode([src])[0].cpu().numpy()
            torch.cuda.synchronize()
            dec.check_status()
            r = rel_err(x, xh)
            bad += int((r > 0.1).sum())
            tot += r.size
            bad_p += int((r[precip] > 0.1).sum())
            tot_p += r[precip].size
            med.append(float(np.median(r)))
        vals = args.samples * C * H * W
        rows.append({"lookahead": la or 64, "repeat_min": rm or 16, "err_budget": abs(budget) % 10000,
                     "raw16": budget < 0, "raw_segments": abs(budget) > 10000,
                     "bytes_per_value": nbytes / vals,
                     "ratio_vs_fp32": 4.0 * vals / nbytes, "frac_rel_err_gt_10pct": bad / tot,
                     "frac_rel_err_gt_10pct_precip_channel": bad_p / max(1, tot_p),
                     "frac_rel_err_gt_10pct_other_channels": (bad - bad_p) / max(1, tot - tot_p),
                     "median_rel_err": float(np.median(med)), "segments_per_line": nseg / (args.samples * C * H),
                     "raw_lines": nraw})
        print(json.dumps(rows[-1]), file=sys.stderr, flush=True)
    print(json.dumps({"what": "DeepCAM ratio vs error over encoder knobs (FORMAT.md 2.4 defaults: lookahead 64, "
                      "repeat_min 16; FORMAT.md 2.5 err_budget k at rel_err 0.1, 0 = off); decoded by libspp on the GPU (fp32 x-hat)",
                      "samples": args.samples, "shape": [C, H, W], "paper": "about 3% of values > 10% error (P:86)",
                      "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
