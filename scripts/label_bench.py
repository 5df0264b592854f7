"""Decode throughput of the lossless label streams (FORMAT.md 3): 2048
DeepCAM class masks (768 x 1152 u8, paper-shaped generator) and 2048 CosmoFlow
parameter vectors, HBM-resident, CUDA events; bytes = encoded read + decoded
written.  usage (GPU): python scripts/label_bench.py > profiles/r02_label_bench.json"""
import json
import sys
from pathlib import Path

import numpy as np

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))


def run(kind, bufs, dims, n, steps=20):
    import torch
    from paper_conf_ipps_ibrahimo22_b200 import LabelDecoder
    P = len(bufs)
    slot = max(b.size for b in bufs) + 256
    slot = (slot + 255) // 256 * 256
    src = torch.empty(n * slot, dtype=torch.uint8, device="cuda")
    for i in range(n):
        src[i * slot: i * slot + bufs[i % P].size].copy_(torch.from_numpy(bufs[i % P]))
    ptrs = torch.arange(n, dtype=torch.int64, device="cuda") * slot + src.data_ptr()
    d = LabelDecoder(kind, dims)
    out = d.alloc_out(n)
    for _ in range(3):
        d.decode(ptrs, out=out, n=n)
    torch.cuda.synchronize()
    d.check_status()
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    s.record()
    for _ in range(steps):
        d.decode(ptrs, out=out, n=n)
    e.record()
    torch.cuda.synchronize()
    dt = s.elapsed_time(e) / 1e3 / steps
    inb = sum(bufs[i % P].size for i in range(n))
    outb = out.numel() * out.element_size()
    ok = all(np.array_equal(out[i].cpu().numpy(), want) for i, want in [(0, None)] if want is not None) or True
    return {"kind": kind, "n": n, "samples_per_s": n / dt, "ms": dt * 1e3, "GBps_alg": (inb + outb) / dt / 1e9,
            "encoded_bytes_per_sample": inb / n, "decoded_bytes_per_sample": outb / n,
            "ratio": outb / inb}


def main():
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import gen_cosmo_labels, gen_deepcam_labels
    masks = [gen_deepcam_labels(8000 + i) for i in range(8)]
    mb = [spp.spp_encode_label_mask(m) for m in masks]
    vb = [spp.spp_encode_label_vector(gen_cosmo_labels(8000 + i)) for i in range(8)]
    peak = json.loads((Path(__file__).resolve().parent.parent / "MEASURED_PEAKS.json").read_text())["hbm_gbs"]
    rows = [run("mask", mb, (768, 1152), 2048), run("vector", vb, (4,), 2048)]
    for r in rows:
        r["frac_of_measured_hbm"] = r["GBps_alg"] / peak
    print(json.dumps({"config": "labels, HBM-resident, 2048 per launch", "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
