"""Full-size decodes for compute-sanitizer (memcheck / racecheck / synccheck):
   compute-sanitizer --tool racecheck python scripts/sanitize_fullsize.py deepcam
Cases: `deepcam` (one 16x768x1152 paper-shaped sample, fp16 normalised and fp32,
on both W = 1152 KD instances), `deepcam_long` (lines longer than KD's ring and
W > 8192: the global line path), `cosmo` (4x256^3, six tables; escaped keys).
Each case prints the status words (0 = ok)."""
import sys
from pathlib import Path

import numpy as np

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp  # noqa: E402
from synth import deepcam_stats, gen_cosmo, gen_deepcam  # noqa: E402


def run(fmt_name, bufs, dims, shift=None, scale=None, **kw):
    dec = Decoder(fmt_name, dims, **kw)
    if shift is not None:
        dec.set_normalisation(shift, scale)
    srcs = [torch.from_numpy(b).cuda() for b in bufs]
    sizes = torch.tensor([b.size for b in bufs], dtype=torch.int64, device="cuda")
    dec.decode(srcs, src_bytes=sizes)
    torch.cuda.synchronize()
    return int(dec.status.item())


case = sys.argv[1] if len(sys.argv) > 1 else "deepcam"
if case in ("deepcam_default", "deepcam_bigline"):
    # racecheck isolation: the default stream (no line longer than one ring slot)
    # vs a stream with RAW lines (each takes the whole ring)
    y = gen_deepcam(2001, H=192)
    mean, rstd = deepcam_stats(y)
    b = spp.spp_encode_deepcam(y) if case == "deepcam_default" else spp.spp_encode_deepcam(y, err_budget=4)
    print(case, spp.spp_stream_info("deepcam", b), run("deepcam", [b, b], y.shape, mean, rstd, out="f16"))
elif case == "deepcam":
    y = gen_deepcam(2001)
    mean, rstd = deepcam_stats(y)
    d = spp.spp_encode_deepcam(y)
    r = spp.spp_encode_deepcam(y, err_budget=4, raw16=True, raw_segments=True)
    for rs in (False, True):
        print("deepcam f16", rs, run("deepcam", [d, d], y.shape, mean, rstd, out="f16", raw_segments=rs))
        print("deepcam f32", rs, run("deepcam", [d], y.shape, out="f32", raw_segments=rs))
        print("deepcam budget/raw16/rawseg f16", rs, run("deepcam", [r], y.shape, mean, rstd, raw_segments=rs))
elif case == "deepcam_long":
    from tests import fmt
    from tests.test_gpu_limits import _many_short_raw_segments_line, _one_per_position_line
    rng = np.random.default_rng(77)
    lines = [_one_per_position_line(rng, 1152, 1), _one_per_position_line(rng, 1152, 3),
             _many_short_raw_segments_line(rng, 1152), fmt.build_raw_line(rng.standard_normal(1152).astype(np.float32))]
    b = fmt.build_deepcam_stream(1, 4, 1152, lines, A=1)
    for rs in (False, True):
        print("deepcam long lines", rs, run("deepcam", [b, b], (1, 4, 1152), raw_segments=rs))
    W = 12000
    x = (np.sin(np.linspace(0, 30, W)) * 50 + rng.standard_normal((2, 2, W))).astype(np.float32)
    w = spp.spp_encode_deepcam(x)
    print("deepcam W=12000", run("deepcam", [w], x.shape, out="f16"))
elif case == "cosmo":
    x = gen_cosmo(1001, n=256)
    b = spp.spp_encode_cosmo(x)
    print("cosmo 256^3", run("cosmo", [b], x.shape))
    e = spp.spp_encode_cosmo(gen_cosmo(1001), escape=True)
    print("cosmo escaped", run("cosmo", [e, e], (4, 128, 128, 128), escape_keys=True))
