#!/usr/bin/env python
"""bench.py — throughput of the fused decode + preprocess hot path on B200.

Default workload (BASELINE.json configs[1], "C2"): a CosmoFlow batch of 512
samples (4x128^3 int16 counts, paper-shaped generator) encoded on the host,
decoded + ln(1+c)-normalised to fp16 CDHW tensors in HBM by libspp.  A step is
one spp_decode_batch over the whole batch (2 kernel launches).  The default
run appends the DeepCAM C4 workload (BASELINE configs[3]: 2048 samples
16x768x1152 -> fp16, per-channel normalisation) as "secondary", at every N;
``--workload deepcam`` makes C4 the headline.

  value      MODE A — compressed set RESIDENT IN HBM: samples/s, whole job (sum
             over ranks / max-over-ranks device time), CUDA events on the decode
             stream
  e2e        MODE B — compressed set in PINNED HOST memory, through the public
             streamed API spp_decode_host: PCIe H2D on a copy stream overlapped
             with decode (Fig. 1 b.4 + b.5), plus a D2H read of the status
             word each step; per rank: H2D GB/s and overlap max(t_h2d, t_dec)/t_e2e
  roofline   dominant kernel (KC / KD): algorithmic bytes (compressed read +
             decoded written) per launch / its CUDA-event duration, vs the
             measured HBM copy peak (MEASURED_PEAKS.json); frac_nominal vs the
             north star's ~8 TB/s
  cpu_baseline  the plain C oracle (oracle/) decoding a bounded sample on the
             host's cores, one sample per thread (rank 0, N = 1 only)

Multi-GPU: one process per GPU (torchrun), NCCL.  Each rank is bound to the CPU
cores of its GPU's NUMA node before it allocates pinned memory.  ``--scaling
weak`` (default; "samples per GPU"): every rank decodes its own
batch of 512 / 2048.  ``--scaling strong``: the fixed 512 / 2048 set split by
shard_indices.  No collective on the data path: NCCL only for the barriers
around the timed regions and MAX all-reduces of the elapsed times.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time
from concurrent.futures import ThreadPoolExecutor
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent
sys.path.insert(0, str(ROOT))

METRIC = json.loads((ROOT / "BASELINE.json").read_text())["metric"]
NOMINAL_HBM_GBS = 8000.0  # BASELINE.json north_star: "roughly 8 TB/s" (reading S26)


def _peaks():
    p = ROOT / "MEASURED_PEAKS.json"
    if p.exists():
        d = json.loads(p.read_text())
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy_ read+write)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


WORKLOADS = {
    "cosmo": dict(cfg="C2", batch=512, pool=16, seed=1001, dims=(4, 128, 128, 128),
                  desc="BASELINE configs[1]: CosmoFlow batch of 512 samples, 4x128^3 int16 counts "
                       "(paper preset: lognormal density + coupled Poisson), decoded + ln(1+c) to fp16 CDHW. "
                       "value = mode A (compressed set resident in HBM); e2e = mode B (host-resident pinned "
                       "set streamed H2D through spp_decode_host)"),
    "deepcam": dict(cfg="C4", batch=2048, pool=8, seed=2001, dims=(16, 768, 1152),
                    desc="BASELINE configs[3]: DeepCAM epoch shard of 2048 samples, 16x768x1152 fp32 "
                         "(paper-shaped channel mix), decoded + per-channel (x-mean)/std to fp16 CHW. "
                         "value = mode A (compressed set resident in HBM); e2e = mode B (host-resident pinned "
                         "set streamed H2D through spp_decode_host)"),
}


# ----------------------------------------------------------------------------- placement
def _cpulist(s: str) -> set[int]:
    out = set()
    for part in s.strip().split(","):
        if not part:
            continue
        if "-" in part:
            a, b = part.split("-")
            out.update(range(int(a), int(b) + 1))
        else:
            out.add(int(part))
    return out


def bind_to_gpu_numa(dev_index: int) -> dict:
    """Bind this process to the CPU cores local to GPU `dev_index` (its NUMA
    node, from sysfs by PCI address, else NVML) before any pinned allocation,
    so the rank's pinned host pool and its copy threads live next to its PCIe
    root (host<->device bandwidth bounds the streamed path)."""
    import torch
    info = {"bound": False}
    try:
        p = torch.cuda.get_device_properties(dev_index)
        pci = f"{p.pci_domain_id:04x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
        info["pci"] = pci
        base = Path("/sys/bus/pci/devices") / pci
        cpus = set()
        if (base / "local_cpulist").exists():
            cpus = _cpulist((base / "local_cpulist").read_text())
        if (base / "numa_node").exists():
            info["numa_node"] = int((base / "numa_node").read_text().strip())
        if not cpus:
            try:
                import pynvml
                pynvml.nvmlInit()
                h = pynvml.nvmlDeviceGetHandleByPciBusId(pci.encode())
                words = pynvml.nvmlDeviceGetCpuAffinity(h, (os.cpu_count() + 63) // 64)
                for wi, w in enumerate(words):
                    cpus.update(wi * 64 + b for b in range(64) if (w >> b) & 1)
            except Exception as ex:  # noqa: BLE001
                info["nvml"] = str(ex)[:80]
        allowed = os.sched_getaffinity(0)
        use = cpus & allowed
        if use and use != allowed:
            os.sched_setaffinity(0, use)
            info["bound"] = True
        info["cpus"] = len(os.sched_getaffinity(0))
    except Exception as ex:  # noqa: BLE001
        info["error"] = str(ex)[:120]
    return info


# ----------------------------------------------------------------------------- setup
def make_pool(workload: str, pool: int, seed: int, threads: int, escape: bool = False):
    """Generate + encode `pool` distinct samples (host, product encoder)."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import deepcam_stats, gen_cosmo, gen_deepcam

    def one(i):
        if workload == "cosmo":
            x = gen_cosmo(seed + i)
            return spp.spp_encode_cosmo(x, escape=escape), None, None
        x = gen_deepcam(seed + i)
        return spp.spp_encode_deepcam(x), (deepcam_stats(x) if i == 0 else None), (x if i == 0 else None)

    with ThreadPoolExecutor(max_workers=threads) as ex:
        res = list(ex.map(one, range(pool)))
    return [r[0] for r in res], res[0][1], res[0][2]


def stream_stats(workload: str, bufs) -> dict:
    """Per-sample format statistics of the pool (SURVEY §5 metrics): CosmoFlow
    |U|, slabs, G and kw of slab 0; DeepCAM line-mode histogram and segments."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    info = np.array([spp.spp_stream_info(workload, b) for b in bufs], dtype=np.float64)
    if workload == "cosmo":
        return {"nU_mean": float(info[:, 0].mean()), "slabs_mean": float(info[:, 1].mean()),
                "G_slab0_mean": float(info[:, 2].mean()), "kw_slab0": sorted({int(v) for v in info[:, 3]}),
                "bytes_per_sample_mean": float(np.mean([b.size for b in bufs]))}
    lines = info[:, 0] + info[:, 1]
    return {"raw_lines_per_sample": float(info[:, 0].mean()), "seg_lines_per_sample": float(info[:, 1].mean()),
            "segments_per_seg_line": float(info[:, 2].sum() / max(1.0, info[:, 1].sum())),
            "delta_bytes_per_value": float(info[:, 3].sum() / (lines.sum() * 1152)),
            "bytes_per_sample_mean": float(np.mean([b.size for b in bufs]))}


class Clocks:
    """nvidia-smi sampler running during the timed region."""

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        time.sleep(0.3)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        time.sleep(0.15)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for k, v in zip(names, f[4:8]):
                if v.lower() == "active":
                    reasons.add(k)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": mx, "reasons": ["unsampled"], "samples": 0}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def cpu_baseline(workload: str, bufs, dims, stats, seconds: float = 12.0):
    """The plain C oracle (as it stands) on this host's cores, one sample per thread."""
    import oracle
    cores = len(os.sched_getaffinity(0)) or os.cpu_count() or 1

    def work(i):
        b = bufs[i % len(bufs)]
        if workload == "cosmo":
            oracle.cosmo_decode(b, dims, 1, "f16")
        else:
            oracle.deepcam_decode(b, dims, stats[0], stats[1], "f16")
        return 1

    oracle.lib()
    # (i) one core, one sample at a time, briefly
    one, t1 = 0, time.perf_counter()
    while one < 2 or time.perf_counter() - t1 < min(2.0, seconds / 4):
        work(one)
        one += 1
    one_rate = one / (time.perf_counter() - t1)
    # (ii) every host core, one sample per thread (PAPER.md P:106's CPU assignment)
    done = 0
    t0 = time.perf_counter()
    with ThreadPoolExecutor(max_workers=cores) as ex:
        while time.perf_counter() - t0 < seconds:
            done += sum(ex.map(work, range(done, done + cores)))
    dt = time.perf_counter() - t0
    return {"value": done / dt, "unit": "samples/s", "cores": cores, "kind": "oracle",
            "value_1core": one_rate,
            "sample": f"{done} {workload} samples (oracle/spp_oracle.c sequential decoder, fp16 out), "
                      f"one per thread on {cores} threads, {dt:.1f} s wall; value_1core: {one} samples on one "
                      "thread"}


def _gather(obj, dist):
    if dist is None:
        return [obj]
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, obj)
    return out


def _sum_over_ranks(v: int, dist, dev) -> int:
    if dist is None:
        return int(v)
    import torch
    t = torch.tensor([int(v)], dtype=torch.int64, device=None if dist.get_backend() == "gloo" else dev)
    dist.all_reduce(t)
    return int(t.item())


# ----------------------------------------------------------------------------- GPU arm
def run_gpu(args, rank: int, world: int, local_rank: int, dist):
    import ctypes

    import torch
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, HostPipeline, spp
    from paper_conf_ipps_ibrahimo22_b200.shard import max_over_ranks, rank_seed_base, shard_indices

    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    W = WORKLOADS[args.workload]
    dims = W["dims"]
    strong = args.scaling == "strong"
    B_total = args.batch or W["batch"]
    # weak: every rank its own batch of B_total samples (distinct seeds);
    # strong: the one B_total set split across ranks (the same seeds everywhere)
    B = len(shard_indices(B_total, rank, world)) if strong else B_total
    if B < 1:
        raise ValueError(f"--scaling strong with a batch of {B_total} leaves rank {rank} of {world} without samples")
    t_setup = time.perf_counter()
    esc = args.escape_keys and args.workload == "cosmo"
    seed = W["seed"] if strong else rank_seed_base(W["seed"], rank)
    bufs, stats, x0 = make_pool(args.workload, args.pool or W["pool"], seed, escape=esc,
                                threads=max(1, len(os.sched_getaffinity(0))))
    sizes = [int(b.size) for b in bufs]
    P = len(bufs)
    # sample j of this rank = pool entry (global index % P); B distinct device
    # buffers (one allocation, 256-B aligned slots): inputs + outputs per step far
    # exceed the 126 MB L2, no flush needed
    gidx = shard_indices(B_total, rank, world) if strong else list(range(B))
    pj = [g % P for g in gidx]
    slot = [((s + 255) // 256) * 256 for s in sizes]
    offs = np.zeros(B + 1, dtype=np.int64)
    for i in range(B):
        offs[i + 1] = offs[i] + slot[pj[i]]
    src_all = torch.empty(int(offs[-1]), dtype=torch.uint8, device=dev)
    pool_dev = [torch.from_numpy(b).to(dev) for b in bufs]
    for i in range(B):
        src_all[int(offs[i]): int(offs[i]) + sizes[pj[i]]].copy_(pool_dev[pj[i]])
    del pool_dev
    ptrs = torch.from_numpy(offs[:B] + src_all.data_ptr()).to(dev)
    dec = Decoder(args.workload, dims, out="f16", escape_keys=esc)
    if args.workload == "deepcam":
        dec.set_normalisation(stats[0], stats[1])
    out = dec.alloc_out(B)
    in_bytes = int(sum(sizes[p] for p in pj))
    out_bytes = out.numel() * out.element_size()
    stream = torch.cuda.current_stream()
    # timing events recorded by the library around its two kernels
    nev = args.steps
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(nev)]
    for trio in evs:           # torch creates CUDA events lazily: force creation
        for e in trio:
            e.record(stream)
    torch.cuda.synchronize()
    ev_arrays = [(ctypes.c_void_p * 3)(*[e.cuda_event for e in trio]) for trio in evs]
    assert all(e.cuda_event for trio in evs for e in trio)
    setup_s = time.perf_counter() - t_setup

    def step(i=None):
        dec.opts.timing_events = ctypes.cast(ev_arrays[i], ctypes.c_void_p).value if i is not None else None
        dec.decode(ptrs, out=out, n=B)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    dec.check_status()
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(local_rank) as clk:
        start.record(stream)
        for i in range(args.steps):
            step(i)
        end.record(stream)
        torch.cuda.synchronize()
    if dist:
        dist.barrier()
    elapsed = start.elapsed_time(end) / 1e3
    dec.check_status()
    k_main = float(np.mean([evs[i][1].elapsed_time(evs[i][2]) for i in range(nev)])) / 1e3
    k_pro = float(np.mean([evs[i][0].elapsed_time(evs[i][1]) for i in range(nev)])) / 1e3
    tmax = max_over_ranks(elapsed, dist, dev)          # device-timed, max over ranks
    units = _sum_over_ranks(B, dist, dev)               # samples all ranks decode per step
    value = units * args.steps / tmax

    # DeepCAM codec error statistics on pool sample 0 (reading S19; "3% of
    # values with > 10% error"): fp32 x̂ without normalisation vs the original
    err = None
    if x0 is not None:
        d32 = Decoder("deepcam", dims, out="f32")
        xh = d32.decode([torch.from_numpy(bufs[0]).to(dev)])[0].cpu().numpy()
        d32.check_status()
        x = x0.astype(np.float64)
        ae = np.abs(xh.astype(np.float64) - x)
        with np.errstate(divide="ignore", invalid="ignore"):
            big = np.where(x == 0, xh != 0, ae > 0.1 * np.abs(x))
        err = {"frac_rel_err_gt_10pct": float(big.mean()), "max_abs_err": float(ae.max()),
               "mean_abs_err": float(ae.mean()), "sample": "pool sample 0, decoded fp32 x̂ vs the fp32 original"}

    # ---- MODE B, end to end: pinned host -> H2D (copy stream) overlapped with decode
    e2e_steps = max(1, min(args.steps, args.e2e_steps))
    # the compressed pool packed back to back in one pinned buffer (samples are
    # 16-B multiples): consecutive samples of a chunk leave in one PCIe copy
    hoffs = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int64)
    host_all = torch.empty(int(hoffs[-1]), dtype=torch.uint8).pin_memory()
    for i, b in enumerate(bufs):
        host_all[int(hoffs[i]): int(hoffs[i + 1])].copy_(torch.from_numpy(b))
    host = [host_all[int(hoffs[i]): int(hoffs[i + 1])] for i in range(P)]
    host_srcs = [host[p] for p in pj]
    slot_bytes = max(sizes) * args.chunk + 4096
    pipe = HostPipeline(dec, slot_bytes=slot_bytes, nslots=3, max_chunk=args.chunk)
    st_host = torch.zeros(1, dtype=torch.int32).pin_memory()
    for _ in range(2):
        pipe.decode(host_srcs, out)
        st_host.copy_(dec.status, non_blocking=True)
        torch.cuda.synchronize()
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    s2, e2 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s2.record(stream)
    for _ in range(e2e_steps):
        pipe.decode(host_srcs, out)
        st_host.copy_(dec.status, non_blocking=True)   # D2H read of the step's result (status word)
    e2.record(stream)
    torch.cuda.synchronize()
    assert int(st_host.item()) == 0, "decode status"
    e2e_launches = pipe.launches()
    pipe.close()
    t_e2e = s2.elapsed_time(e2) / 1e3 / e2e_steps          # this rank, per step
    t2 = max_over_ranks(t_e2e * e2e_steps, dist, dev)
    e2e_value = units * e2e_steps / t2
    # the same bytes as plain H2D copies (the chunks the pipeline moves: runs of
    # back-to-back pool samples), alone on a copy stream: this rank's link rate
    cs = torch.cuda.Stream(device=dev)
    stage = torch.empty(int(hoffs[-1]), dtype=torch.uint8, device=dev)
    runs = []
    i = 0
    while i < B:
        k = 1
        while i + k < B and k < args.chunk and pj[i + k] == pj[i + k - 1] + 1:
            k += 1
        runs.append((int(hoffs[pj[i]]), int(hoffs[pj[i + k - 1] + 1])))
        i += k
    if dist:
        dist.barrier()      # every rank copies at once: the contended link rate
    torch.cuda.synchronize()
    h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(cs):
        h0.record(cs)
        for a, b_ in runs:
            stage[a:b_].copy_(host_all[a:b_], non_blocking=True)
        h1.record(cs)
    torch.cuda.synchronize()
    t_h2d = h0.elapsed_time(h1) / 1e3
    t_dec = elapsed / args.steps
    del stage
    rank_info = {"rank": rank, "batch": B, "decode_ms": t_dec * 1e3, "kernel_ms": k_main * 1e3,
                 "e2e_ms": t_e2e * 1e3, "h2d_ms": t_h2d * 1e3, "h2d_gbs": in_bytes / t_h2d / 1e9,
                 "e2e_h2d_gbs": in_bytes / t_e2e / 1e9, "overlap": max(t_h2d, t_dec) / t_e2e,
                 "clocks": clk.summary()}
    ranks = _gather(rank_info, dist)

    peak, peak_src = _peaks()
    alg = in_bytes + out_bytes
    achieved = alg / k_main / 1e9
    traffic = None
    tf = ROOT / "profiles" / f"ncu_traffic_{args.workload}{'_escape' if esc else ''}.json"
    if tf.exists():
        try:
            traffic = json.loads(tf.read_text()).get("traffic_bytes_per_launch")
        except Exception:
            traffic = None
    kname = ("kc_expand (KC, escaped-key instance)" if esc else "kc_expand (KC)") if args.workload == "cosmo" \
        else "kd_decode_ws (KD)"
    res = {
        "value": value, "ms_per_step": tmax / args.steps * 1e3, "elapsed_s": tmax,
        "gbs_alg": alg * units / B * args.steps / tmax / 1e9,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "kernel": kname,
                     "frac_nominal_8tbs": achieved / NOMINAL_HBM_GBS,
                     "alg_bytes_per_launch": alg, "kernel_ms": k_main * 1e3, "prologue_ms": k_pro * 1e3,
                     "kernel_share_of_step": k_main / (elapsed / args.steps), "peak_source": peak_src,
                     "rank": rank},
        "e2e": {"value": e2e_value, "unit": "samples/s", "h2d_bytes_per_step": in_bytes,
                "d2h_bytes_per_step": 4, "steps": e2e_steps, "chunk": args.chunk, "gpu_launches": e2e_launches,
                "h2d_gbs_rank0": rank_info["h2d_gbs"], "overlap_rank0": rank_info["overlap"],
                "api": "spp_decode_host (pinned host sources, chunked H2D on a copy stream, decode on the caller's "
                       "stream)"},
        "per_rank": ranks,
        "gpu_launches": spp.spp_decode_launches(args.workload) * args.steps,
        "clocks": clk.summary(),
        "batch": B, "units_per_step": units, "in_bytes": in_bytes, "out_bytes": out_bytes, "pool": P,
        "setup_s": setup_s, "stream_stats": stream_stats(args.workload, bufs), "codec_error": err,
        "compression_ratio": float(np.prod(dims)) * (2 if args.workload == "cosmo" else 4) * P / sum(sizes),
    }
    del out, src_all
    torch.cuda.empty_cache()
    return res, bufs, stats


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=None)
    ap.add_argument("--warmup", type=int, default=None)
    ap.add_argument("--impl", choices=["spp", "reference"], default="spp")
    ap.add_argument("--workload", choices=["cosmo", "deepcam"], default="cosmo")
    ap.add_argument("--scaling", choices=["weak", "strong"], default="weak",
                    help="weak: every rank decodes its own batch (PAPER.md P:221 samples per GPU); strong: the "
                         "fixed batch split across ranks")
    ap.add_argument("--secondary", choices=["auto", "none"], default="auto",
                    help="append the DeepCAM C4 numbers to the CosmoFlow line (every N)")
    ap.add_argument("--batch", type=int, default=None)
    ap.add_argument("--secondary-batch", type=int, default=None, help="DeepCAM batch of the secondary (default 2048)")
    ap.add_argument("--pool", type=int, default=None)
    ap.add_argument("--chunk", type=int, default=16, help="samples per H2D chunk in the e2e pipeline")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--escape-keys", action="store_true",
                    help="CosmoFlow streams with FORMAT.md 1.5 escaped 1-byte keys (beyond the paper's 1/2-byte "
                         "keys) and the decode kernel that stages them")
    args = ap.parse_args()
    if args.steps is None:
        args.steps = 200 if args.workload == "cosmo" else 30
    if args.warmup is None:
        args.warmup = 10 if args.workload == "cosmo" else 3
    args.warmup = max(3, args.warmup)

    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local_rank = int(os.environ.get("LOCAL_RANK", 0))
    W = WORKLOADS[args.workload]

    if args.impl == "reference":
        if rank != 0:
            return
        run_reference(args, W)
        return

    import torch
    dist = None
    backend = os.environ.get("SPP_DIST_BACKEND", "nccl")
    if world > 1 and backend != "nccl":
        # SPP_DIST_BACKEND=gloo (tests only) lets several ranks share one GPU
        local_rank %= max(1, torch.cuda.device_count())
    placement = bind_to_gpu_numa(local_rank)  # before any pinned allocation or worker thread
    if world > 1:
        import torch.distributed as td
        torch.cuda.set_device(local_rank)
        if backend == "nccl":
            os.environ.setdefault("NCCL_DEBUG", "INFO")   # the driver checks nranks in the NCCL log
            td.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            td.init_process_group(backend)
        dist = td
    placements = _gather(placement, dist)
    res, bufs, stats = run_gpu(args, rank, world, local_rank, dist)
    sec = None
    if args.secondary == "auto" and args.workload == "cosmo":
        a2 = argparse.Namespace(**vars(args))
        a2.workload, a2.steps, a2.warmup, a2.e2e_steps = "deepcam", min(20, args.steps), 3, 2
        a2.batch = args.secondary_batch
        r2, b2, s2 = run_gpu(a2, rank, world, local_rank, dist)
        sec = {"workload": WORKLOADS["deepcam"]["desc"], "cfg": "C4", "value": r2["value"], "unit": "samples/s",
               "ms_per_step": r2["ms_per_step"], "gbs_alg": r2["gbs_alg"], "roofline": r2["roofline"],
               "e2e": r2["e2e"], "per_rank": r2["per_rank"], "clocks": r2["clocks"],
               "compression_ratio": r2["compression_ratio"], "stream_stats": r2["stream_stats"],
               "codec_error": r2["codec_error"], "batch_per_rank": r2["batch"], "units_per_step": r2["units_per_step"],
               "steps": a2.steps, "gpu_launches": r2["gpu_launches"],
               "cpu_baseline": (cpu_baseline("deepcam", b2, WORKLOADS["deepcam"]["dims"], s2,
                                             seconds=min(8.0, args.cpu_seconds)) if world == 1 and rank == 0
                                else None)}
    variant = None
    if sec is not None and not args.escape_keys and world == 1 and args.batch is None:
        # the same C2 workload with FORMAT.md 1.5 escaped keys (beyond the paper's format):
        # fewer bytes per sample, so a faster streamed (PCIe-bound) path
        a3 = argparse.Namespace(**vars(args))
        a3.escape_keys, a3.steps, a3.e2e_steps = True, 50, 3
        r3, _, _ = run_gpu(a3, rank, world, local_rank, dist)
        variant = {"key_format": "FORMAT.md 1.5 escaped 1-byte keys", "value": r3["value"], "unit": "samples/s",
                   "ms_per_step": r3["ms_per_step"], "roofline": r3["roofline"], "e2e": r3["e2e"],
                   "compression_ratio": r3["compression_ratio"], "clocks": r3["clocks"], "steps": a3.steps}
    if rank != 0:
        if dist:
            dist.destroy_process_group()
        return
    cpu = cpu_baseline(args.workload, bufs, W["dims"], stats, seconds=args.cpu_seconds) if world == 1 else None
    line = {
        "metric": METRIC, "value": res["value"], "unit": "samples/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": res["ms_per_step"], "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "u16" if args.workload == "cosmo" else "f32",
        "data": "synthetic",
        "config": {"workload": W["desc"], "cfg": W["cfg"], "value_mode": "A: compressed set resident in HBM",
                   "e2e_mode": "B: compressed set in pinned host memory, streamed H2D (spp_decode_host)",
                   "batch_per_rank": res["batch"], "samples_per_step_all_ranks": res["units_per_step"],
                   "out_dtype": "f16",
                   "pool_distinct_samples": res["pool"], "compression_ratio": res["compression_ratio"],
                   "key_format": ("FORMAT.md 1.5 escaped 1-byte keys" if args.escape_keys and args.workload == "cosmo"
                                  else ("FORMAT.md 1.3 (the paper's 1/2-byte keys)" if args.workload == "cosmo"
                                        else "FORMAT.md 2 (A = 36 aligned segments)")),
                   "stream_stats": res["stream_stats"], "codec_error": res["codec_error"],
                   "GB_per_s_alg_total": res["gbs_alg"], "in_bytes_per_step_rank0": res["in_bytes"],
                   "out_bytes_per_step_rank0": res["out_bytes"],
                   "l2": "no flush: inputs+outputs per step far exceed the 126 MB L2 (distinct HBM buffers)",
                   "parallelism": f"sample shards ({args.scaling} scaling), 1 process per GPU ({world}), no data-path "
                                  "collective",
                   "placement": placements},
        "roofline": res["roofline"], "cpu_baseline": cpu, "e2e": res["e2e"], "gpu_launches": res["gpu_launches"],
        "clocks": res["clocks"], "per_rank": res["per_rank"],
    }
    if sec:
        line["secondary"] = sec
    if variant:
        line["variant_escape_keys"] = variant
    if dist:  # NCCL's teardown log lines (NCCL_DEBUG=INFO, stdout) come before the JSON line
        dist.destroy_process_group()
    print(json.dumps(line), flush=True)


def run_reference(args, W):
    """--impl reference: the oracle as it stands on the host cores, one bounded
    sample of the workload per step (cores samples, one per thread)."""
    import oracle
    from synth import deepcam_stats, gen_cosmo, gen_deepcam
    cores = os.cpu_count() or 1
    npool = 4
    if args.workload == "cosmo":
        xs = [gen_cosmo(W["seed"] + i) for i in range(npool)]
        bufs = [oracle.cosmo_encode(x) for x in xs]
        stats = None
    else:
        xs = [gen_deepcam(W["seed"] + i) for i in range(npool)]
        bufs = [oracle.deepcam_encode(x) for x in xs]
        stats = deepcam_stats(xs[0])
    per_step = cores

    def work(i):
        b = bufs[i % npool]
        if args.workload == "cosmo":
            oracle.cosmo_decode(b, W["dims"], 1, "f16")
        else:
            oracle.deepcam_decode(b, W["dims"], stats[0], stats[1], "f16")

    # keep the whole run to a few minutes: shrink the sample if a step is long
    with ThreadPoolExecutor(max_workers=cores) as ex:
        t0 = time.perf_counter()
        list(ex.map(work, range(per_step)))
        one = time.perf_counter() - t0
        budget = 150.0
        steps, warm = args.steps, args.warmup
        while per_step > 1 and one * (steps + warm) > budget:
            per_step //= 2
            one /= 2
        for _ in range(warm):
            list(ex.map(work, range(per_step)))
        t0 = time.perf_counter()
        for _ in range(steps):
            list(ex.map(work, range(per_step)))
        dt = time.perf_counter() - t0
    value = per_step * steps / dt
    desc = (f"{per_step} {args.workload} samples per step (oracle/spp_oracle.c sequential decoder, fp16 out, "
            f"one sample per thread, {min(per_step, cores)} threads)")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": args.gpus,
            "steps": steps, "warmup": warm, "ms_per_step": dt / steps * 1e3, "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "u16" if args.workload == "cosmo" else "f32",
            "data": "synthetic", "config": {"workload": W["desc"], "cfg": W["cfg"], "reference": "CPU oracle"},
            "cpu_baseline": {"value": value, "unit": "samples/s", "cores": min(per_step, cores), "kind": "oracle",
                             "sample": desc},
            "e2e": {"value": value, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
