"""KD under sustained load (experiment, not product): the C4 launch (2048
DeepCAM samples -> fp16, HBM-resident) repeated back to back, and again with
idle gaps, CUDA events around every launch, nvidia-smi (SM / memory clocks,
power, throttle reasons) sampled every 50 ms.  Shows whether the bench's KD
time is set by the power budget (sw_power_cap) rather than by the kernel.
usage (GPU): python scripts/kd_power_trace.py > profiles/<round>_kd_power_trace.json"""
import json
import subprocess
import sys
import threading
import time
from pathlib import Path

import numpy as np

sys.path.insert(0, str(Path(__file__).resolve().parent.parent))


class Trace:
    Q = "timestamp,clocks.sm,clocks.mem,power.draw,clocks_event_reasons.sw_power_cap,temperature.gpu"

    def __enter__(self):
        self.lines = []
        self.proc = subprocess.Popen(["nvidia-smi", "--id=0", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                      "-lms", "50"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        self.t = threading.Thread(target=lambda: [self.lines.append(ln.strip()) for ln in self.proc.stdout],
                                  daemon=True)
        self.t.start()
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        time.sleep(0.2)
        self.proc.terminate()
        self.proc.wait(timeout=3)

    def rows(self):
        out = []
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 6:
                continue
            try:
                out.append({"sm_mhz": float(f[1]), "mem_mhz": float(f[2]), "power_w": float(f[3]),
                            "power_cap": f[4].lower() == "active", "temp_c": float(f[5])})
            except ValueError:
                continue
        return out


def main():
    import torch
    from bench import make_pool
    from paper_conf_ipps_ibrahimo22_b200 import Decoder

    B, dims = 2048, (16, 768, 1152)
    bufs, stats, _ = make_pool("deepcam", 16, 2001, threads=16)
    sizes = [int(b.size) for b in bufs]
    slot = [((s + 255) // 256) * 256 for s in sizes]
    offs = np.zeros(B + 1, dtype=np.int64)
    for i in range(B):
        offs[i + 1] = offs[i] + slot[i % len(bufs)]
    src = torch.empty(int(offs[-1]), dtype=torch.uint8, device="cuda")
    for i in range(B):
        src[int(offs[i]): int(offs[i]) + sizes[i % len(bufs)]].copy_(torch.from_numpy(bufs[i % len(bufs)]))
    ptrs = torch.from_numpy(offs[:B] + src.data_ptr()).cuda()
    dec = Decoder("deepcam", dims, out="f16")
    dec.set_normalisation(stats[0], stats[1])
    out = dec.alloc_out(B)
    alg = int(offs[-1]) + out.numel() * 2
    peak = json.loads((Path(__file__).resolve().parent.parent / "MEASURED_PEAKS.json").read_text())["hbm_gbs"]
    for _ in range(3):
        dec.decode(ptrs, out=out, n=B)
    torch.cuda.synchronize()
    dec.check_status()
    res = {"what": "KD C4 launch (2048 x 16x768x1152 -> fp16) repeated; per-launch CUDA-event ms; nvidia-smi at 50 ms",
           "alg_bytes_per_launch": alg, "peak_gbs": peak}
    for name, n, gap in (("back_to_back", 60, 0.0), ("idle_gaps_250ms", 12, 0.25)):
        time.sleep(3.0)  # cool down between the two regimes
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
        with Trace() as tr:
            for a, b in ev:
                a.record()
                dec.decode(ptrs, out=out, n=B)
                b.record()
                if gap:
                    torch.cuda.synchronize()
                    time.sleep(gap)
            torch.cuda.synchronize()
        ms = [a.elapsed_time(b) for a, b in ev]
        smi = tr.rows()
        res[name] = {"launch_ms": [round(x, 3) for x in ms],
                     "frac_first": alg / (ms[0] * 1e-3) / 1e9 / peak,
                     "frac_median": alg / (float(np.median(ms)) * 1e-3) / 1e9 / peak,
                     "frac_last10": alg / (float(np.mean(ms[-10:])) * 1e-3) / 1e9 / peak,
                     "smi_samples": len(smi),
                     "sm_mhz_median": float(np.median([r["sm_mhz"] for r in smi])) if smi else None,
                     "mem_mhz_median": float(np.median([r["mem_mhz"] for r in smi])) if smi else None,
                     "power_w_median": float(np.median([r["power_w"] for r in smi])) if smi else None,
                     "power_w_max": max(r["power_w"] for r in smi) if smi else None,
                     "power_cap_fraction": (sum(r["power_cap"] for r in smi) / len(smi)) if smi else None,
                     "temp_c_max": max(r["temp_c"] for r in smi) if smi else None,
                     "smi": smi}
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
