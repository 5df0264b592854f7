#!/usr/bin/env python
"""The paper's CPU decoder variant as a comparison point (
PAPER.md P:106 "on the CPU we assign different samples to different threads",
P:211 "the GPU plugin is up to 1.5x faster than the CPU").

scripts/cpu_plugin.c (gcc -O3 -march=native, one sample per call) decodes the
same encoded sets the GPU bench uses, one sample per thread on every host
core, fp16 output; this script times it and, with --gpu, the GPU path on the
same samples (device-resident and streamed from pinned memory).  It is not
part of the product and is checked against the oracle by
tests/test_cpu_plugin.py.

usage: python scripts/cpu_plugin.py [--gpu] > profiles/r01_cpu_plugin.json
"""
from __future__ import annotations

import argparse
import ctypes as C
import json
import os
import subprocess
import sys
import time
from concurrent.futures import ThreadPoolExecutor
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))
SRC = ROOT / "scripts" / "cpu_plugin.c"
OUTDIR = ROOT / "scripts" / "_cpu_plugin_build"


def load(native: bool = True) -> C.CDLL:
    """Compile for this host (the .so is not shipped: -march=native)."""
    OUTDIR.mkdir(exist_ok=True)
    lib = OUTDIR / ("libcpu_plugin_native.so" if native else "libcpu_plugin.so")
    if not lib.exists() or lib.stat().st_mtime < SRC.stat().st_mtime:
        flags = ["-O3", "-ffp-contract=off", "-fno-fast-math", "-std=gnu11", "-shared", "-fPIC"]
        if native:
            flags.append("-march=native")
        subprocess.run(["gcc", *flags, "-o", str(lib), str(SRC), "-lm"], check=True)
    L = C.CDLL(str(lib))
    L.cpu_cosmo_decode_f16.argtypes = [C.c_void_p, C.c_size_t, C.c_void_p]
    L.cpu_cosmo_decode_f16.restype = C.c_int
    L.cpu_deepcam_decode_f16.argtypes = [C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p, C.c_void_p]
    L.cpu_deepcam_decode_f16.restype = C.c_int
    return L


def cosmo_decode(L, buf: np.ndarray, shape) -> np.ndarray:
    out = np.empty(shape, dtype=np.float16)
    assert L.cpu_cosmo_decode_f16(buf.ctypes.data, buf.size, out.ctypes.data) == 0
    return out


def deepcam_decode(L, buf: np.ndarray, shape, shift=None, scale=None) -> np.ndarray:
    out = np.empty(shape, dtype=np.float16)
    sh = None if shift is None else np.ascontiguousarray(shift, dtype=np.float32)
    sc = None if scale is None else np.ascontiguousarray(scale, dtype=np.float32)
    assert L.cpu_deepcam_decode_f16(buf.ctypes.data, buf.size, None if sh is None else sh.ctypes.data,
                                    None if sc is None else sc.ctypes.data, out.ctypes.data) == 0
    return out


def time_cpu(fn, bufs, seconds: float, threads: int):
    """One sample per thread, each thread decoding into its own output."""
    done = [0] * threads
    stop = time.perf_counter() + seconds

    def worker(t):
        i = t
        while time.perf_counter() < stop:
            fn(bufs[i % len(bufs)], t)
            done[t] += 1
            i += threads
    t0 = time.perf_counter()
    with ThreadPoolExecutor(max_workers=threads) as ex:
        list(ex.map(worker, range(threads)))
    return sum(done) / (time.perf_counter() - t0), sum(done)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seconds", type=float, default=8.0)
    ap.add_argument("--gpu", action="store_true")
    a = ap.parse_args()
    from paper_conf_ipps_ibrahimo22_b200 import spp
    from synth import deepcam_stats, gen_cosmo, gen_deepcam
    L = load()
    cores = os.cpu_count() or 1
    rows = {}
    cos = [spp.spp_encode_cosmo(gen_cosmo(1001 + i)) for i in range(4)]
    ys = [gen_deepcam(2001 + i) for i in range(2)]
    mean, rstd = deepcam_stats(ys[0])
    dcs = [spp.spp_encode_deepcam(y) for y in ys]
    for name, bufs, shape, fn in (
            ("cosmo", cos, (4, 128, 128, 128), None), ("deepcam", dcs, (16, 768, 1152), None)):
        outs = [np.empty(shape, dtype=np.float16) for _ in range(cores)]
        if name == "cosmo":
            def dec(b, t, _o=outs):
                L.cpu_cosmo_decode_f16(b.ctypes.data, b.size, _o[t].ctypes.data)
        else:
            sh, sc = mean.astype(np.float32), rstd.astype(np.float32)

            def dec(b, t, _o=outs):
                L.cpu_deepcam_decode_f16(b.ctypes.data, b.size, sh.ctypes.data, sc.ctypes.data, _o[t].ctypes.data)
        one, n1 = time_cpu(dec, bufs, min(a.seconds, 4.0), 1)
        allc, na = time_cpu(dec, bufs, a.seconds, cores)
        rows[name] = {"cpu_1thread_samples_per_s": one, "cpu_all_cores_samples_per_s": allc, "cores": cores,
                      "samples_timed": na, "bytes_per_sample_in": float(np.mean([b.size for b in bufs]))}
        print(json.dumps({name: rows[name]}), file=sys.stderr, flush=True)
    if a.gpu:
        import torch
        from paper_conf_ipps_ibrahimo22_b200 import Decoder, HostPipeline
        for name, bufs, shape in (("cosmo", cos, (4, 128, 128, 128)), ("deepcam", dcs, (16, 768, 1152))):
            B = 256 if name == "cosmo" else 64
            dec = Decoder(name, shape)
            if name == "deepcam":
                dec.set_normalisation(mean, rstd)
            out = dec.alloc_out(B)
            dsrc = [torch.from_numpy(bufs[i % len(bufs)]).cuda() for i in range(B)]
            for _ in range(2):
                dec.decode(dsrc, out=out)
            torch.cuda.synchronize()
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record()
            for _ in range(5):
                dec.decode(dsrc, out=out)
            e.record()
            torch.cuda.synchronize()
            res = B * 5 / (s.elapsed_time(e) / 1e3)
            sizes = [b.size for b in bufs]
            offs = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int64)
            host_all = torch.empty(int(offs[-1]), dtype=torch.uint8).pin_memory()
            for i, b in enumerate(bufs):
                host_all[int(offs[i]): int(offs[i + 1])].copy_(torch.from_numpy(b))
            hs = [host_all[int(offs[i]): int(offs[i + 1])] for i in range(len(bufs))]
            srcs = [hs[i % len(bufs)] for i in range(B)]
            pipe = HostPipeline(dec, slot_bytes=max(sizes) * 16 + 4096, nslots=3, max_chunk=16)
            pipe.decode(srcs, out)
            torch.cuda.synchronize()
            s.record()
            for _ in range(3):
                pipe.decode(srcs, out)
            e.record()
            torch.cuda.synchronize()
            e2e = B * 3 / (s.elapsed_time(e) / 1e3)
            dec.check_status()
            # the CPU plugin's output equals the GPU's for the first sample
            got = out[0].cpu().numpy()
            cpu = cosmo_decode(L, bufs[0], shape) if name == "cosmo" else deepcam_decode(L, bufs[0], shape, mean, rstd)
            pipe.close()
            # the CPU plugin must then ship DECODED fp16 samples over PCIe: pinned H2D rate
            dec_bytes = int(np.prod(shape)) * 2
            hbuf = torch.empty(dec_bytes * 4, dtype=torch.uint8).pin_memory()
            dbuf = torch.empty(dec_bytes * 4, dtype=torch.uint8, device="cuda")
            dbuf.copy_(hbuf, non_blocking=True)
            torch.cuda.synchronize()
            s.record()
            for _ in range(10):
                dbuf.copy_(hbuf, non_blocking=True)
            e.record()
            torch.cuda.synchronize()
            h2d = dec_bytes * 4 * 10 / (s.elapsed_time(e) / 1e3)
            cpu_e2e = min(rows[name]["cpu_all_cores_samples_per_s"], h2d / dec_bytes)
            rows[name].update({"gpu_resident_samples_per_s": res, "gpu_streamed_samples_per_s": e2e,
                               "pinned_h2d_GBps": h2d / 1e9,
                               "cpu_plugin_e2e_bound_samples_per_s": cpu_e2e,
                               "gpu_streamed_over_cpu_plugin_e2e_bound": e2e / cpu_e2e,
                               "gpu_streamed_over_cpu_all_cores": e2e / rows[name]["cpu_all_cores_samples_per_s"],
                               "gpu_resident_over_cpu_all_cores": res / rows[name]["cpu_all_cores_samples_per_s"],
                               "same_bits_as_gpu": bool(np.array_equal(got.view(np.uint16), cpu.view(np.uint16)))})
            print(json.dumps({name: rows[name]}), file=sys.stderr, flush=True)
    print(json.dumps({"what": "paper's CPU decoder variant (one sample per thread, P:106) vs the GPU path; fp16 out; "
                      "paper-shaped synthetic samples; cpu_plugin_e2e_bound = min(CPU decode rate, pinned H2D rate "
                      "of the decoded fp16 sample), since the CPU plugin ships decoded samples to the GPU", "paper": "GPU plugin up to 1.5x faster than the CPU plugin "
                      "for unstaged DeepCAM data (P:211)", "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
