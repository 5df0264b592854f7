#!/usr/bin/env python
"""End-to-end overlap of the decode loader with a training step (SURVEY.md
§8f f1; Fig. 1 b.5 -> training; the paper's DALI role).

Times, with CUDA events on the consumer stream (after warm-up):
  train     : AMP training steps on one fixed, already-decoded batch
  loader    : DecodeLoader alone (next() + a trivial consumer read)
  both      : DecodeLoader feeding the same training step
and reports the exposed loader cost (both - train) per step.  The models are
small stand-ins with the paper's input shapes (CosmoFlow: 3-D conv stack on
4x128^3; DeepCAM: 2-D conv stack on 16x768x1152), random init, synthetic data.

usage: python scripts/train_overlap.py [--workload cosmo|deepcam] [--source device|host]
"""
from __future__ import annotations

import argparse
import json
import sys
import time
from pathlib import Path

import numpy as np
import torch
import torch.nn as nn

ROOT = Path(__file__).resolve().parent.parent
sys.path.insert(0, str(ROOT))


def cosmo_net():
    layers, c = [], 4
    for co in (16, 32, 64, 64, 128):
        layers += [nn.Conv3d(c, co, 3, padding=1), nn.LeakyReLU(0.3), nn.MaxPool3d(2)]
        c = co
    return nn.Sequential(*layers, nn.Flatten(), nn.Linear(128 * 4 * 4 * 4, 128), nn.LeakyReLU(0.3),
                         nn.Linear(128, 4))


def deepcam_net():
    layers, c = [], 16
    for co in (32, 64, 128, 128):
        layers += [nn.Conv2d(c, co, 3, stride=2, padding=1), nn.BatchNorm2d(co), nn.ReLU()]
        c = co
    return nn.Sequential(*layers, nn.Conv2d(c, 3, 1), nn.Upsample(scale_factor=16, mode="bilinear"))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", choices=["cosmo", "deepcam"], default="cosmo")
    ap.add_argument("--source", choices=["device", "host"], default="device")
    ap.add_argument("--batch", type=int, default=None)
    ap.add_argument("--pool", type=int, default=8)
    ap.add_argument("--samples", type=int, default=64, help="shard size (pool replicated)")
    ap.add_argument("--steps", type=int, default=20)
    args = ap.parse_args()
    from paper_conf_ipps_ibrahimo22_b200 import Decoder, spp
    from paper_conf_ipps_ibrahimo22_b200.loader import DecodeLoader, EncodedShard, EpochSampler
    from synth import deepcam_stats, gen_cosmo, gen_deepcam

    dev = torch.device("cuda:0")
    B = args.batch or (8 if args.workload == "cosmo" else 2)
    if args.workload == "cosmo":
        pool = [spp.spp_encode_cosmo(gen_cosmo(1001 + i)) for i in range(args.pool)]
        dims, stats = (4, 128, 128, 128), None
        net, target_fn = cosmo_net(), (lambda y: torch.zeros(y.shape[0], 4, device=dev))
    else:
        xs = [gen_deepcam(2001 + i) for i in range(args.pool)]
        pool = [spp.spp_encode_deepcam(x) for x in xs]
        dims, stats = (16, 768, 1152), deepcam_stats(xs[0])
        del xs
        net = deepcam_net()
        target_fn = lambda y: torch.zeros(y.shape[0], 768, 1152, dtype=torch.long, device=dev)
    bufs = [pool[i % len(pool)] for i in range(args.samples)]
    net = net.to(dev).to(memory_format=torch.channels_last_3d if args.workload == "cosmo" else torch.channels_last)
    opt = torch.optim.SGD(net.parameters(), lr=1e-3, momentum=0.9)
    scaler = torch.amp.GradScaler("cuda")
    loss_fn = nn.MSELoss() if args.workload == "cosmo" else nn.CrossEntropyLoss()

    def train_step(x):
        with torch.autocast("cuda", dtype=torch.float16):
            y = net(x)
            loss = loss_fn(y.float(), target_fn(x))
        opt.zero_grad(set_to_none=True)
        scaler.scale(loss).backward()
        scaler.step(opt)
        scaler.update()
        return loss

    dec = Decoder(args.workload, dims, out="f16")
    if stats is not None:
        dec.set_normalisation(stats[0], stats[1])
    shard = EncodedShard(bufs, device_resident=(args.source == "device"), device=dev)
    ld = DecodeLoader(dec, shard, B, EpochSampler(len(bufs), seed=0), source=args.source, depth=2)
    nb = len(ld)
    steps = min(args.steps, nb)

    def timed(fn, n):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        s.record()
        fn(n)
        e.record()
        torch.cuda.synchronize()
        return s.elapsed_time(e) / n

    fixed = next(iter(ld))[0].clone()
    for _ in range(3):
        train_step(fixed)

    def run_train(n):
        for _ in range(n):
            train_step(fixed)

    def run_loader(n):
        for k, (b, _) in enumerate(ld):
            b[:1].view(-1)[:1].float()          # a trivial consumer read
            if k + 1 == n:
                break

    def run_both(n):
        for k, (b, _) in enumerate(ld):
            train_step(b)
            if k + 1 == n:
                break

    run_loader(steps)
    run_both(steps)
    t_train = timed(run_train, steps)
    t_loader = timed(run_loader, steps)
    t_both = timed(run_both, steps)
    res = {"workload": args.workload, "source": args.source, "batch": B, "steps": steps,
           "ms_train_step": t_train, "ms_loader_batch": t_loader, "ms_loader_plus_train": t_both,
           "ms_exposed_loader": t_both - t_train, "exposed_frac_of_step": (t_both - t_train) / t_both,
           "loader_samples_per_s_alone": B / t_loader * 1e3, "cuda_graph": args.source == "device",
           "loader_launches": ld.launches, "note": "stand-in conv nets with the paper's input shapes, AMP fp16, "
           "random init, synthetic data; CUDA events on the consumer stream"}
    ld.close()
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
