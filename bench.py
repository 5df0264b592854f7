#!/usr/bin/env python
"""bench.py — throughput of the fused decode + preprocess hot path on B200.

Default workload (BASELINE.json configs[1], "C2"): a CosmoFlow batch of 512
samples (4x128^3 int16 counts, paper-shaped generator) encoded on the host,
decoded + ln(1+c)-normalised to fp16 CDHW tensors in HBM by libspp.  A step is
one spp_decode_batch over the whole batch (2 kernel launches).  ``--workload
deepcam`` runs C4 (2048 DeepCAM samples 16x768x1152 -> fp16, per-channel
normalisation); the default run appends a C4 measurement as "secondary".

  value      samples/s, whole job (sum over ranks / max-over-ranks device time),
             inputs resident in HBM, CUDA events on the decode stream
  e2e        same metric through spp_decode_host: pinned host memory -> PCIe H2D
             on a copy stream overlapped with decode (b.4 + b.5), plus a D2H read
             of the status word each step
  roofline   dominant kernel (KC / KD): algorithmic bytes (compressed read +
             decoded written) per launch / its CUDA-event duration, vs the
             measured HBM copy peak (MEASURED_PEAKS.json)
  cpu_baseline  the plain C oracle (oracle/) decoding a bounded sample on the
             host's cores, one sample per thread

Multi-GPU: one process per GPU (torchrun), each rank decodes its own batch
(weak scaling, no collective on the data path; NCCL barrier + MAX all-reduce of
the elapsed time only).
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


def _peaks():
    p = ROOT / "MEASURED_PEAKS.json"
    if p.exists():
        d = json.loads(p.read_text())
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy_ read+write)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


WORKLOADS = {
    "cosmo": dict(cfg="C2", batch=512, pool=16, seed=1001, dims=(4, 128, 128, 128),
                  desc="BASELINE configs[1]: CosmoFlow batch of 512 samples, 4x128^3 int16 counts "
                       "(paper preset: lognormal density + coupled Poisson), host-resident compressed set, "
                       "decoded + ln(1+c) to fp16 CDHW"),
    "deepcam": dict(cfg="C4", batch=2048, pool=8, seed=2001, dims=(16, 768, 1152),
                    desc="BASELINE configs[3]: DeepCAM epoch shard of 2048 samples, 16x768x1152 fp32 "
                         "(paper-shaped channel mix), decoded + per-channel (x-mean)/std to fp16 CHW"),
}


# ----------------------------------------------------------------------------- setup
def make_pool(workload: str, pool: int, seed: int, threads: int, escape: bool = False):
    """Generate + encode `pool` distinct samples (host, product encoder)."""
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import deepcam_stats, gen_cosmo, gen_deepcam

    def one(i):
        if workload == "cosmo":
            x = gen_cosmo(seed + i)
            return spp.spp_encode_cosmo(x, escape=escape), None
        x = gen_deepcam(seed + i)
        return spp.spp_encode_deepcam(x), (deepcam_stats(x) if i == 0 else None)

    with ThreadPoolExecutor(max_workers=threads) as ex:
        res = list(ex.map(one, range(pool)))
    bufs = [r[0] for r in res]
    stats = res[0][1]
    return bufs, stats


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
    cores = os.cpu_count() or 1
    shape = dims if workload == "cosmo" else dims

    def work(i):
        b = bufs[i % len(bufs)]
        if workload == "cosmo":
            oracle.cosmo_decode(b, shape, 1, "f16")
        else:
            oracle.deepcam_decode(b, shape, stats[0], stats[1], "f16")
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


# ----------------------------------------------------------------------------- GPU arm
def run_gpu(args, rank: int, world: int, local_rank: int, dist):
    import torch
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, HostPipeline, spp

    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    l2_granted = spp.spp_set_l2_persisting(int(args.l2_persist_mb * 2**20)) if args.l2_persist_mb > 0 else 0
    W = WORKLOADS[args.workload]
    B = args.batch or W["batch"]
    dims = W["dims"]
    t_setup = time.perf_counter()
    from paper_conf_ipps_ibrahimo22_b200.shard import aggregate_throughput, max_over_ranks, rank_seed_base
    esc = args.escape_keys and args.workload == "cosmo"
    bufs, stats = make_pool(args.workload, args.pool or W["pool"], rank_seed_base(W["seed"], rank), escape=esc,
                            threads=max(1, (os.cpu_count() or 1) // max(1, world)))
    sizes = [int(b.size) for b in bufs]
    P = len(bufs)
    # B distinct device buffers (one big allocation, 256-B aligned slots): the
    # whole set (inputs + outputs) is far larger than L2, no flush needed
    slot = [((s + 255) // 256) * 256 for s in sizes]
    offs = np.zeros(B + 1, dtype=np.int64)
    for i in range(B):
        offs[i + 1] = offs[i] + slot[i % P]
    src_all = torch.empty(int(offs[-1]), dtype=torch.uint8, device=dev)
    pool_dev = [torch.from_numpy(b).to(dev) for b in bufs]
    for i in range(B):
        src_all[int(offs[i]): int(offs[i]) + sizes[i % P]].copy_(pool_dev[i % P])
    del pool_dev
    ptrs = torch.from_numpy(offs[:B] + src_all.data_ptr()).to(dev)
    dec = Decoder(args.workload, dims, out="f16", escape_keys=esc)
    if args.workload == "deepcam":
        dec.set_normalisation(stats[0], stats[1])
    out = dec.alloc_out(B)
    in_bytes = int(sum(sizes[i % P] for i in range(B)))
    out_bytes = out.numel() * out.element_size()
    stream = torch.cuda.current_stream()
    # timing events recorded by the library around its two kernels
    nev = args.steps
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(nev)]
    import ctypes
    for trio in evs:           # torch creates CUDA events lazily: force creation
        for e in trio:
            e.record(stream)
    torch.cuda.synchronize()
    ev_arrays = [(ctypes.c_void_p * 3)(*[e.cuda_event for e in trio]) for trio in evs]
    assert all(e.cuda_event for trio in evs for e in trio)
    setup_s = time.perf_counter() - t_setup

    def step(i=None):
        if i is not None:
            dec.opts.timing_events = ctypes.cast(ev_arrays[i], ctypes.c_void_p).value
        else:
            dec.opts.timing_events = None
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
    value = aggregate_throughput(B, world, args.steps, tmax)

    # ---- end to end: pinned host -> H2D (copy stream) overlapped with decode
    e2e_steps = max(1, min(args.steps, args.e2e_steps))
    # the compressed pool packed back to back in one pinned buffer (samples are
    # 16-B multiples): consecutive samples of a chunk leave in one PCIe copy
    hoffs = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int64)
    host_all = torch.empty(int(hoffs[-1]), dtype=torch.uint8).pin_memory()
    for i, b in enumerate(bufs):
        host_all[int(hoffs[i]): int(hoffs[i + 1])].copy_(torch.from_numpy(b))
    host = [host_all[int(hoffs[i]): int(hoffs[i + 1])] for i in range(P)]
    host_srcs = [host[i % P] for i in range(B)]
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
    t2 = max_over_ranks(s2.elapsed_time(e2) / 1e3, dist, dev)
    e2e_value = aggregate_throughput(B, world, e2e_steps, t2)

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
        else "kd_decode (KD)"
    res = {
        "value": value, "ms_per_step": tmax / args.steps * 1e3, "elapsed_s": tmax,
        "gbs_alg": world * alg * args.steps / tmax / 1e9,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "kernel": kname,
                     "alg_bytes_per_launch": alg, "kernel_ms": k_main * 1e3, "prologue_ms": k_pro * 1e3,
                     "kernel_share_of_step": k_main / (tmax / args.steps), "peak_source": peak_src},
        "e2e": {"value": e2e_value, "unit": "samples/s", "h2d_bytes_per_step": in_bytes,
                "d2h_bytes_per_step": 4, "steps": e2e_steps, "chunk": args.chunk, "gpu_launches": e2e_launches},
        "gpu_launches": spp.spp_decode_launches(args.workload) * args.steps,
        "clocks": clk.summary(),
        "batch": B, "in_bytes": in_bytes, "out_bytes": out_bytes, "pool": P, "setup_s": setup_s,
        "l2_persist_bytes": l2_granted,
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
    ap.add_argument("--secondary", choices=["auto", "none"], default="auto",
                    help="append the other workload's numbers (rank 0 line) when running the default")
    ap.add_argument("--batch", type=int, default=None)
    ap.add_argument("--pool", type=int, default=None)
    ap.add_argument("--chunk", type=int, default=16, help="samples per H2D chunk in the e2e pipeline")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--escape-keys", action="store_true",
                    help="CosmoFlow streams with FORMAT.md 1.5 escaped 1-byte keys (beyond the paper's 1/2-byte "
                         "keys) and the decode kernel that stages them")
    ap.add_argument("--l2-persist-mb", type=float, default=float(os.environ.get("SPP_L2_PERSIST_MB", "0")),
                    help="L2 persisting set-aside for the CosmoFlow LUT rows (spp_set_l2_persisting)")
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

    dist = None
    if world > 1:
        import torch
        import torch.distributed as td
        # one process per GPU over NCCL.  SPP_DIST_BACKEND=gloo (tests only) lets
        # several ranks share one GPU: the device is local_rank modulo the count
        backend = os.environ.get("SPP_DIST_BACKEND", "nccl")
        if backend != "nccl":
            local_rank %= max(1, torch.cuda.device_count())
        torch.cuda.set_device(local_rank)
        if backend == "nccl":
            td.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            td.init_process_group(backend)
        dist = td
    res, bufs, stats = run_gpu(args, rank, world, local_rank, dist)
    sec = None
    if args.secondary == "auto" and world == 1 and args.workload == "cosmo" and args.batch is None:
        a2 = argparse.Namespace(**vars(args))
        a2.workload, a2.steps, a2.warmup, a2.e2e_steps = "deepcam", 20, 3, 2
        r2, b2, s2 = run_gpu(a2, rank, world, local_rank, dist)
        sec = {"workload": WORKLOADS["deepcam"]["desc"], "value": r2["value"], "unit": "samples/s",
               "ms_per_step": r2["ms_per_step"], "gbs_alg": r2["gbs_alg"], "roofline": r2["roofline"],
               "e2e": r2["e2e"], "clocks": r2["clocks"], "compression_ratio": r2["compression_ratio"],
               "batch": r2["batch"], "steps": a2.steps,
               "cpu_baseline": cpu_baseline("deepcam", b2, WORKLOADS["deepcam"]["dims"], s2,
                                            seconds=min(8.0, args.cpu_seconds))}
    variant = None
    if sec is not None and not args.escape_keys:
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
        "warmup": args.warmup, "ms_per_step": res["ms_per_step"], "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u16" if args.workload == "cosmo" else "f32", "data": "synthetic",
        "config": {"workload": W["desc"], "cfg": W["cfg"], "batch_per_gpu": res["batch"], "out_dtype": "f16",
                   "pool_distinct_samples": res["pool"], "compression_ratio": res["compression_ratio"],
                   "key_format": ("FORMAT.md 1.5 escaped 1-byte keys" if args.escape_keys and args.workload == "cosmo"
                                  else "FORMAT.md 1.3 (the paper's 1/2-byte keys)"),
                   "GB_per_s_alg_total": res["gbs_alg"], "in_bytes_per_step": res["in_bytes"],
                   "out_bytes_per_step": res["out_bytes"],
                   "l2": "no flush: inputs+outputs per step far exceed the 126 MB L2 (distinct HBM buffers)",
                   "parallelism": f"sample shards, 1 process per GPU ({world})"},
        "roofline": res["roofline"], "cpu_baseline": cpu, "e2e": res["e2e"], "gpu_launches": res["gpu_launches"],
        "clocks": res["clocks"],
    }
    if sec:
        line["secondary"] = sec
    if variant:
        line["variant_escape_keys"] = variant
    print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


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
            "scaling": "weak", "vs_baseline": None, "dtype": "u16" if args.workload == "cosmo" else "f32",
            "data": "synthetic", "config": {"workload": W["desc"], "cfg": W["cfg"], "reference": "CPU oracle"},
            "cpu_baseline": {"value": value, "unit": "samples/s", "cores": min(per_step, cores), "kind": "oracle",
                             "sample": desc},
            "e2e": {"value": value, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
