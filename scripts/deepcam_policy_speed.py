#!/usr/bin/env python
"""HBM-resident KD decode rate of DeepCAM streams written with different
encoder policies (FORMAT.md 2.4 default; 2.5 error budget; 2.6 RAW16; 2.7 RAW
segments): lines that leave the one-pass path (RAW, RAW16, mode 3) take KD's
general line path.  Batch of distinct HBM copies, fp16 normalised output.

usage (GPU): python scripts/deepcam_policy_speed.py > profiles/r01_deepcam_policy_speed.json
"""
import json
import sys
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))


def main():
    import torch

    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    from synth import deepcam_stats, gen_deepcam
    peak = json.loads((ROOT / "MEASURED_PEAKS.json").read_text())["hbm_gbs"] \
        if (ROOT / "MEASURED_PEAKS.json").exists() else 6650.0
    xs = [gen_deepcam(2001 + i) for i in range(2)]
    mean, rstd = deepcam_stats(xs[0])
    B = 256
    rows = []
    for name, kw in (("default", {}), ("budget1", dict(err_budget=1)), ("budget1_raw16", dict(err_budget=1, raw16=True)),
                     ("budget1_raw16_onepass", dict(err_budget=1, raw16=True, _onepass=True)),
                     ("budget1_rawseg", dict(err_budget=1, raw_segments=True)),
                     ("budget16_rawseg", dict(err_budget=16, raw_segments=True)),
                     ("budget1_rawseg_general", dict(err_budget=1, raw_segments=True, _general=True))):
        kw = dict(kw)
        general = kw.pop("_general", False)  # mode-3 lines on the general line path (opts.raw_segments = 0)
        onepass = kw.pop("_onepass", False)  # RAW16 lines on the opts.raw_segments instance
        bufs = [spp.spp_encode_deepcam(x, **kw) for x in xs]
        dec = Decoder("deepcam", xs[0].shape, raw_segments=(bool(kw.get("raw_segments")) and not general) or onepass)
        dec.set_normalisation(mean, rstd)
        out = dec.alloc_out(B)
        src = [torch.from_numpy(bufs[i % 2]).cuda() for i in range(B)]
        for _ in range(2):
            dec.decode(src, out=out)
        torch.cuda.synchronize()
        dec.check_status()
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        s.record()
        for _ in range(5):
            dec.decode(src, out=out)
        e.record()
        torch.cuda.synchronize()
        dt = s.elapsed_time(e) / 1e3 / 5
        alg = sum(bufs[i % 2].size for i in range(B)) + out.numel() * 2
        rows.append({"policy": name, "bytes_per_value": float(np.mean([b.size for b in bufs])) / xs[0].size,
                     "samples_per_s": B / dt, "frac_of_measured_hbm": alg / dt / 1e9 / peak,
                     "lines_off_onepass": int(sum(spp.spp_stream_info("deepcam", bufs[0])[:1]))})
        print(json.dumps(rows[-1]), file=sys.stderr, flush=True)
        del src, out
        torch.cuda.empty_cache()
    print(json.dumps({"what": "KD decode rate per DeepCAM encoder policy (batch 256, fp16)", "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
