"""Run a few decodes of one workload (for ncu captures; never a bench number)."""
import argparse
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp  # noqa: E402
from synth import deepcam_stats, gen_cosmo, gen_deepcam  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("workload", choices=["cosmo", "deepcam"])
ap.add_argument("--n", type=int, default=64)
ap.add_argument("--iters", type=int, default=3)
ap.add_argument("--out", default="f16")
a = ap.parse_args()
if a.workload == "cosmo":
    xs = [gen_cosmo(1001 + i) for i in range(4)]
    bufs = [spp.spp_encode_cosmo(x) for x in xs]
    dims = xs[0].shape
    stats = None
else:
    xs = [gen_deepcam(2001 + i) for i in range(2)]
    bufs = [spp.spp_encode_deepcam(x) for x in xs]
    dims = xs[0].shape
    stats = deepcam_stats(xs[0])
srcs = [torch.from_numpy(bufs[i % len(bufs)]).cuda() for i in range(a.n)]
dec = Decoder(a.workload, dims, out=a.out)
if stats is not None:
    dec.set_normalisation(*stats)
out = dec.alloc_out(a.n)
for _ in range(a.iters):
    dec.decode(srcs, out=out)
torch.cuda.synchronize()
dec.check_status()
print("ok", a.workload, a.n)
