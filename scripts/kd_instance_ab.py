"""A/B of the two W = 1152 KD instances on the default DeepCAM stream (mode-1
lines only): the mode-1 instance vs the opts.raw_segments instance (which also
takes FORMAT.md 2.6/2.7 lines in one pass).  Alternating runs, batch 1024,
CUDA events.  usage (GPU): python scripts/kd_instance_ab.py"""
import json
import sys
from pathlib import Path

import numpy as np

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))


def main():
    import torch
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    from synth import deepcam_stats, gen_deepcam
    xs = [gen_deepcam(2001 + i) for i in range(4)]
    bufs = [spp.spp_encode_deepcam(x) for x in xs]
    mean, rstd = deepcam_stats(xs[0])
    B = 1024
    slot = max(b.size for b in bufs) + 256
    src = torch.empty(B * slot, dtype=torch.uint8, device="cuda")
    for i in range(B):
        src[i * slot: i * slot + bufs[i % 4].size].copy_(torch.from_numpy(bufs[i % 4]))
    ptrs = torch.arange(B, dtype=torch.int64, device="cuda") * slot + src.data_ptr()
    res = {False: [], True: []}
    decs = {rs: Decoder("deepcam", xs[0].shape, raw_segments=rs) for rs in (False, True)}
    out = decs[False].alloc_out(B)
    for d in decs.values():
        d.set_normalisation(mean, rstd)
        for _ in range(3):
            d.decode(ptrs, out=out, n=B)
    torch.cuda.synchronize()
    for rep in range(6):
        for rs in (False, True):
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record()
            for _ in range(10):
                decs[rs].decode(ptrs, out=out, n=B)
            e.record()
            torch.cuda.synchronize()
            res[rs].append(B * 10 / (s.elapsed_time(e) / 1e3))
    for d in decs.values():
        d.check_status()
    print(json.dumps({"mode1_instance": float(np.median(res[False])), "raw_segments_instance": float(np.median(res[True])),
                      "ratio": float(np.median(res[True]) / np.median(res[False])), "runs": {str(k): v for k, v in res.items()}}))


if __name__ == "__main__":
    main()
