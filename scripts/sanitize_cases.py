"""Small decodes (valid and corrupted streams) for compute-sanitizer runs:
   compute-sanitizer --tool memcheck|racecheck|synccheck python scripts/sanitize_cases.py
Corrupt streams must be reported through the status word with no
out-of-bounds access (SURVEY.md §5 failure detection)."""
import sys
from pathlib import Path

import numpy as np

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))
import torch  # noqa: E402

from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp  # noqa: E402
from synth import gen_cosmo, gen_deepcam  # noqa: E402
from tests import fmt  # noqa: E402


def run(fmt_name, bufs, dims, **kw):
    dec = Decoder(fmt_name, dims, **kw)
    srcs = [torch.from_numpy(b).cuda() for b in bufs]
    sizes = torch.tensor([b.size for b in bufs], dtype=torch.int64, device="cuda")
    dec.decode(srcs, src_bytes=sizes)
    torch.cuda.synchronize()
    return int(dec.status.item())


x = gen_cosmo(1001, n=32)
b = spp.spp_encode_cosmo(x)
h = fmt.cosmo_header(b)
bad = b.copy(); bad[h["slabs"][0]["keys_off"]:h["slabs"][0]["keys_off"] + 64] = 0xFF
trunc = b[: b.size // 2].copy()
lut = b.copy(); lut[h["slabs"][0]["lut_off"]:h["slabs"][0]["lut_off"] + 16] = 0xFF
print("cosmo ok", run("cosmo", [b, b], x.shape))
print("cosmo bad keys", run("cosmo", [b, bad], x.shape))
print("cosmo bad lut", run("cosmo", [lut, b], x.shape, out="f32"))
print("cosmo truncated", run("cosmo", [b, trunc], x.shape))
# many slabs (FORMAT.md 1.4 localized tables; kw 0 / 1 / 8 in one stream): the
# producer warp streams key tiles across slab and sample boundaries
v = gen_cosmo(3006, "sparse", n=64)
v[:, :16] = 3
v[:, 48:] = np.random.default_rng(1).integers(0, 3000, size=(4, 16, 64, 64))
loc = spp.spp_encode_cosmo(v, localize=True)
print("cosmo localized", run("cosmo", [loc, spp.spp_encode_cosmo(gen_cosmo(3001, "sparse", n=64), localize=True), loc],
                             v.shape))
y = gen_deepcam(2001, H=16)
d = spp.spp_encode_deepcam(y)
hd = fmt.deepcam_header(d)
dbad = d.copy(); dbad[hd["payload_off"] + 2: hd["payload_off"] + 4] = 0xFF      # nseg huge
dtr = d[: d.size // 3].copy()
ddir = d.copy(); ddir[hd["dir_off"] + 8: hd["dir_off"] + 12] = 0xFF             # bad directory entry
print("deepcam ok", run("deepcam", [d, d], y.shape))
print("deepcam bad nseg", run("deepcam", [d, dbad], y.shape))
print("deepcam truncated", run("deepcam", [dtr, d], y.shape))
print("deepcam bad dir", run("deepcam", [d, ddir], y.shape, out="f32"))
# mode-3 lines (FORMAT.md 2.7): RAW segments on the one-pass path; a RAW
# segment declared in a mode-1 line and a RAW segment longer than the line's
# bytes must be reported, not read past
r = spp.spp_encode_deepcam(y, err_budget=1, raw_segments=True)
hr = fmt.deepcam_header(r)
l3 = next(l for l in range(hr["L"]) if fmt.deepcam_line(r, hr, l)["mode"] == 3)
o3 = hr["payload_off"] + int(hr["dir"][l3])
rm1 = r.copy(); rm1[o3] = 1
rlen = r.copy()
seg = next(s for s, g in enumerate(fmt.deepcam_line(r, hr, l3)["segs"]) if g["kind"] == 2)
rlen[o3 + 4 + 4 * seg: o3 + 6 + 4 * seg] = np.frombuffer(np.uint16(1152).tobytes(), np.uint8)
for rs in (False, True):  # general line path / one-pass instance (opts.raw_segments)
    print("deepcam raw segments ok", rs, run("deepcam", [r, r], y.shape, raw_segments=rs))
    print("deepcam raw segment in mode 1", rs, run("deepcam", [r, rm1], y.shape, raw_segments=rs))
    print("deepcam raw segment too long", rs, run("deepcam", [rlen, r], y.shape, out="f32", raw_segments=rs))
# lossless labels (FORMAT.md 3): valid, wrong kind, bad run sum, truncated (src_bytes)
from paper_conf_ipps_ibrahimo22_b200 import LabelDecoder  # noqa: E402
from synth import gen_deepcam_labels  # noqa: E402
m = gen_deepcam_labels(9, H=32, W=256)
lb = spp.spp_encode_label_mask(m)
hl = fmt.label_header(lb)
lk = lb.copy(); lk[6] = 2
ls = lb.copy(); ls[hl["payload_off"] + int(hl["dir"][3]) + 4] ^= 0x40
lt = lb[: lb.size // 2].copy()


def run_labels(bufs):
    d = LabelDecoder("mask", m.shape)
    srcs = [torch.from_numpy(b).cuda() for b in bufs]
    sizes = torch.tensor([b.size for b in bufs], dtype=torch.int64, device="cuda")
    d.decode(srcs, src_bytes=sizes)
    torch.cuda.synchronize()
    return int(d.status.item())


print("labels ok", run_labels([lb, lb]))
print("labels bad kind", run_labels([lb, lk]))
print("labels bad run sum", run_labels([ls, lb]))
print("labels truncated", run_labels([lb, lt]))
