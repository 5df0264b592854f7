"""Probe the GPU box: device properties, host cores, pinned/pageable H2D bandwidth.

Used once per round to fill BASELINE.md / DESIGN.md's streamed-mode roofline.
"""
import json, os, subprocess, time
import torch

def bw(nbytes, pinned, reps=5):
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=pinned)
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d.copy_(h, non_blocking=pinned); torch.cuda.synchronize()
    best = 0.0
    for _ in range(reps):
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        s.record(); d.copy_(h, non_blocking=pinned); e.record(); e.synchronize()
        best = max(best, nbytes / (s.elapsed_time(e) * 1e-3) / 1e9)
    d2h = 0.0
    for _ in range(reps):
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        s.record(); h.copy_(d, non_blocking=pinned); e.record(); e.synchronize()
        d2h = max(d2h, nbytes / (s.elapsed_time(e) * 1e-3) / 1e9)
    return best, d2h

p = torch.cuda.get_device_properties(0)
out = {"name": p.name, "sms": p.multi_processor_count, "total_mem_gb": p.total_memory / 1e9,
       "l2_bytes": getattr(p, "L2_cache_size", None),
       "smem_per_block_optin": getattr(p, "shared_memory_per_block_optin", None),
       "smem_per_sm": getattr(p, "shared_memory_per_multiprocessor", None),
       "regs_per_sm": getattr(p, "regs_per_multiprocessor", None),
       "cpu_count": os.cpu_count(), "sched_affinity": len(os.sched_getaffinity(0))}
try:
    out["lscpu"] = subprocess.run(["lscpu"], capture_output=True, text=True).stdout.splitlines()[:20]
except Exception as ex:
    out["lscpu"] = str(ex)
for mb in (4, 16, 64, 256, 1024):
    n = mb << 20
    out[f"h2d_pinned_{mb}MB"], out[f"d2h_pinned_{mb}MB"] = bw(n, True)
    if mb <= 256:
        out[f"h2d_pageable_{mb}MB"], _ = bw(n, False, reps=3)
try:
    out["topo"] = subprocess.run(["nvidia-smi", "topo", "-m"], capture_output=True, text=True).stdout
except Exception as ex:
    out["topo"] = str(ex)
print(json.dumps(out, indent=1))
