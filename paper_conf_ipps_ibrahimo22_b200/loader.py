"""Training-data loader over the compressed sample formats.

This is the role the paper gives its DALI plugins (§VI, P:104-110;
Fig. 1 b.2-b.5): the compressed set stays in (pinned) host memory or in
HBM, and every training step receives a decoded, preprocessed fp16 batch that
was produced on the GPU while the previous step was computing.

  EncodedShard   one rank's compressed samples packed into one pinned host
                 buffer (and optionally one HBM buffer), 256-B aligned slots
  EpochSampler   seeded per-epoch permutation split across ranks like
                 torch's DistributedSampler (i-th rank takes every world-th
                 index of the permutation; equal counts per rank)
  DecodeLoader   iterator of decoded batches: a ring of `depth` output slots
                 decoded on a side stream ahead of the consumer.  Source
                 "device": the shard is HBM-resident and each batch is one
                 CUDA-graph replay of spp_decode_batch (KC0+KC or KD0+KD) after
                 a tiny H2D copy of the batch's pointer table.  Source "host":
                 each batch streams its compressed bytes H2D through
                 spp_decode_host (copy stream overlapped with decode, b.4+b.5).

Python here only schedules: every byte of every batch is produced by libspp's
kernels (there is no CPU decode path).  A yielded batch tensor is valid until
the next ``next()`` call (its slot is then recycled), the DALI convention;
``clone()`` it to keep it.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from . import Decoder, HostPipeline, SppError

_ALIGN = 256


class EncodedShard:
    """Compressed samples of one rank, packed for pinned-host / HBM residency."""

    def __init__(self, buffers, pin: bool | None = None, device=None, device_resident: bool = False):
        import torch
        self.torch = torch
        if not buffers:
            raise ValueError("empty shard")
        self.sizes = np.array([int(b.size) for b in buffers], dtype=np.int64)
        if np.any(self.sizes % 16) or np.any(self.sizes < 32):
            raise ValueError("encoded streams are whole 16-B multiples of at least 32 bytes")
        slots = (self.sizes + _ALIGN - 1) // _ALIGN * _ALIGN
        self.offsets = np.zeros(len(buffers), dtype=np.int64)
        self.offsets[1:] = np.cumsum(slots)[:-1]
        total = int(slots.sum())
        pin = torch.cuda.is_available() if pin is None else pin
        self.host = torch.empty(total, dtype=torch.uint8, pin_memory=pin)
        h = self.host.numpy()
        for i, b in enumerate(buffers):
            o = int(self.offsets[i])
            h[o:o + int(self.sizes[i])] = np.asarray(b, dtype=np.uint8)
        # DeepCAM streams whose header flags (FORMAT.md 2.1 bit 0) announce RAW16 /
        # RAW-segment lines: the loader then selects the KD instance that decodes
        # them in one pass (opts.raw_segments)
        self.extended_line_modes = any(bytes(np.asarray(b[:4], np.uint8)) == b"SPPD" and int(b[6]) & 1
                                       for b in buffers)
        self.device_buf = None
        if device_resident:
            self.device_buf = self.host.to(device or "cuda", non_blocking=False)

    def __len__(self) -> int:
        return len(self.sizes)

    @property
    def nbytes(self) -> int:
        return int(self.sizes.sum())

    def max_sample_bytes(self) -> int:
        return int(self.sizes.max())

    def host_view(self, i: int):
        o = int(self.offsets[i])
        return self.host[o:o + int(self.sizes[i])]

    def device_ptrs(self, idx) -> np.ndarray:
        """Device addresses of samples `idx` in the HBM-resident copy."""
        if self.device_buf is None:
            raise RuntimeError("shard is not device-resident")
        return self.offsets[np.asarray(idx, dtype=np.int64)] + self.device_buf.data_ptr()


@dataclass
class EpochSampler:
    """Seeded per-epoch permutation of n samples, split across `world` ranks.

    Every rank sees the same permutation (seed + epoch) and takes positions
    rank, rank + world, ...; the permutation is truncated to a multiple of
    world so every rank gets n // world indices (drop_last semantics of
    DistributedSampler).  Batches are consecutive runs of a rank's indices;
    a trailing partial batch is dropped when drop_last.
    """

    n: int
    rank: int = 0
    world: int = 1
    seed: int = 0
    shuffle: bool = True

    def __post_init__(self):
        if self.world < 1 or not 0 <= self.rank < self.world or self.n < self.world:
            raise ValueError("bad sampler geometry")

    def indices(self, epoch: int) -> np.ndarray:
        perm = (np.random.default_rng([self.seed, epoch]).permutation(self.n) if self.shuffle
                else np.arange(self.n))
        per = self.n // self.world
        return perm[: per * self.world][self.rank::self.world]

    def batches(self, epoch: int, batch_size: int, drop_last: bool = True) -> list[np.ndarray]:
        idx = self.indices(epoch)
        nb = len(idx) // batch_size if drop_last else -(-len(idx) // batch_size)
        return [idx[k * batch_size:(k + 1) * batch_size] for k in range(nb)]


class DecodeLoader:
    """Iterator of decoded, preprocessed batches (fp16 by default) in HBM.

    decoder   : a ``Decoder`` (format, dims, output type, DeepCAM normalisation)
    shard     : the rank's ``EncodedShard``
    sampler   : ``EpochSampler`` over len(shard)
    source    : "device" (shard HBM-resident; needs shard.device_buf) or "host"
    depth     : output slots in the ring (>= 2: one in use, one being decoded)
    cuda_graph: capture each slot's decode once and replay it (device source)
    check     : read the device status word every `check` batches (0: at epoch end only)
    labels    : optional (LabelDecoder, EncodedShard) of the samples' lossless label
                streams (FORMAT.md 3), the shard HBM-resident (labels are small:
                ~20 KB per DeepCAM mask, 48 B per CosmoFlow vector); each batch's labels
                are decoded on the same stream right after its samples and the
                iterator yields (batch, labels, indices) instead of (batch, indices)

    Each complete pass advances the epoch by one (``set_epoch`` overrides it),
    so consecutive passes see different permutations.
    """

    def __init__(self, decoder: Decoder, shard: EncodedShard, batch_size: int, sampler: EpochSampler,
                 source: str = "device", depth: int = 2, cuda_graph: bool = True, drop_last: bool = True,
                 chunk: int = 16, check: int = 0, labels=None):
        import torch
        self.torch = torch
        if depth < 2:
            raise ValueError("depth >= 2")
        if source not in ("device", "host"):
            raise ValueError("source is 'device' or 'host'")
        if source == "device" and shard.device_buf is None:
            raise ValueError("device source needs a device-resident shard")
        if sampler.n != len(shard):
            raise ValueError("sampler size != shard size")
        self.dec, self.shard, self.B, self.sampler = decoder, shard, int(batch_size), sampler
        if decoder.fmt == "deepcam" and shard.extended_line_modes and not decoder.opts.raw_segments:
            decoder.opts.raw_segments = 1
            decoder.version += 1
        self.source, self.depth, self.drop_last, self.check = source, depth, drop_last, check
        self.use_graph = cuda_graph and source == "device"
        dev = decoder.device
        self.stream = torch.cuda.Stream(device=dev)
        self.out = [decoder.alloc_out(self.B) for _ in range(depth)]
        self.ready = [torch.cuda.Event() for _ in range(depth)]
        self.free = [torch.cuda.Event() for _ in range(depth)]
        self.free_pending = [False] * depth
        self.epoch = 0
        self.launches = 0       # libspp kernel launches enqueued by this loader
        self.batches_done = 0
        self.pipe = None
        self.lab = None
        if labels is not None:
            ldec, lshard = labels
            if lshard.device_buf is None or len(lshard) != len(shard):
                raise ValueError("labels: an HBM-resident shard with one label stream per sample")
            self.lab = ldec
            self.lab_shard = lshard
            self.lab_out = [ldec.alloc_out(self.B) for _ in range(depth)]
            self.lab_ptr_host = [torch.zeros(self.B, dtype=torch.int64, pin_memory=True) for _ in range(depth)]
            self.lab_ptr_dev = [torch.zeros(self.B, dtype=torch.int64, device=dev) for _ in range(depth)]
            self.lab_copied = [torch.cuda.Event() for _ in range(depth)]
            self.lab_copied_pending = [False] * depth
        if source == "device":
            self.ptr_host = [torch.zeros(self.B, dtype=torch.int64, pin_memory=True) for _ in range(depth)]
            self.ptr_dev = [torch.zeros(self.B, dtype=torch.int64, device=dev) for _ in range(depth)]
            self.copied = [torch.cuda.Event() for _ in range(depth)]
            self.copied_pending = [False] * depth
            decoder.workspace(self.B)           # allocate before any capture
            self.graphs = [None] * depth
            self.graph_version = decoder.version  # graphs hold the decoder's buffer addresses
        else:
            self.pipe = HostPipeline(decoder, slot_bytes=shard.max_sample_bytes() * chunk + 4096, nslots=3,
                                     max_chunk=chunk)

    # ------------------------------------------------------------------ enqueue
    def _decode_device(self, s: int, idx: np.ndarray, n: int):
        t = self.torch
        if self.copied_pending[s]:
            self.copied[s].synchronize()        # the slot's previous pointer upload has been consumed
        ph = self.ptr_host[s].numpy()
        ph[:n] = self.shard.device_ptrs(idx)
        self.ptr_dev[s].copy_(self.ptr_host[s], non_blocking=True)
        self.copied[s].record(self.stream)
        self.copied_pending[s] = True
        if self.use_graph and n == self.B:
            if self.graph_version != self.dec.version:
                # the decoder replaced its workspace or normalisation tensors since
                # capture: replaying would read freed memory / stale constants
                self.stream.synchronize()
                self.graphs = [None] * self.depth
                self.graph_version = self.dec.version
            if self.graphs[s] is None:
                self.dec.decode(self.ptr_dev[s], out=self.out[s], n=n)   # warm-up outside capture
                g = t.cuda.CUDAGraph()
                self.stream.synchronize()
                with t.cuda.graph(g, stream=self.stream):
                    self.dec.decode(self.ptr_dev[s], out=self.out[s], n=n)
                self.graphs[s] = g
            self.graphs[s].replay()
        else:
            self.dec.decode(self.ptr_dev[s], out=self.out[s], n=n)

    def _enqueue(self, k: int):
        s = k % self.depth
        idx = self._batches[k]
        t = self.torch
        with t.cuda.stream(self.stream):
            if self.free_pending[s]:
                self.stream.wait_event(self.free[s])   # the consumer is done with the slot's last batch
                self.free_pending[s] = False
            if self.source == "device":
                self._decode_device(s, idx, len(idx))
                self.launches += self.dec_launches()
            else:
                srcs = [self.shard.host_view(int(i)) for i in idx]
                self.pipe.decode(srcs, self.out[s], stream=self.stream)
                self.launches += self.pipe.launches()
            if self.lab is not None:
                self._decode_labels(s, idx, len(idx))
            self.ready[s].record(self.stream)

    def _decode_labels(self, s: int, idx: np.ndarray, n: int):
        if self.lab_copied_pending[s]:
            self.lab_copied[s].synchronize()    # the slot's previous pointer upload has been consumed
        self.lab_ptr_host[s].numpy()[:n] = self.lab_shard.device_ptrs(idx)
        self.lab_ptr_dev[s].copy_(self.lab_ptr_host[s], non_blocking=True)
        self.lab_copied[s].record(self.stream)
        self.lab_copied_pending[s] = True
        self.lab.decode(self.lab_ptr_dev[s], out=self.lab_out[s], n=n, stream=self.stream)
        self.launches += 1

    def dec_launches(self) -> int:
        from . import spp
        return spp.spp_decode_launches(self.dec.fmt)

    # ------------------------------------------------------------------ iteration
    def set_epoch(self, epoch: int):
        self.epoch = int(epoch)

    def __len__(self) -> int:
        return len(self.sampler.batches(self.epoch, self.B, self.drop_last))

    def __iter__(self):
        t = self.torch
        self._batches = self.sampler.batches(self.epoch, self.B, self.drop_last)
        nb = len(self._batches)
        # a previous pass may have stopped early with batches still in use:
        # every slot is free only after the consumer's work so far
        cur = t.cuda.current_stream(self.dec.device)
        for s in range(self.depth):
            self.free[s].record(cur)
            self.free_pending[s] = True
        for k in range(min(self.depth, nb)):
            self._enqueue(k)
        consumer = t.cuda.current_stream(self.dec.device)
        for k in range(nb):
            s = k % self.depth
            consumer.wait_event(self.ready[s])
            n = len(self._batches[k])
            batch = self.out[s] if n == self.B else self.out[s][:n]
            if self.lab is not None:
                yield batch, (self.lab_out[s] if n == self.B else self.lab_out[s][:n]), self._batches[k]
            else:
                yield batch, self._batches[k]
            # the consumer has enqueued its work on batch k: the slot is free after that work
            consumer = t.cuda.current_stream(self.dec.device)
            self.free[s].record(consumer)
            self.free_pending[s] = True
            self.batches_done += 1
            if self.check and self.batches_done % self.check == 0:
                self.dec.check_status()
            if k + self.depth < nb:
                self._enqueue(k + self.depth)
        self.stream.synchronize()
        self.dec.check_status()
        if self.lab is not None:
            self.lab.check_status()
        self.epoch += 1

    def close(self):
        if self.pipe is not None:
            self.pipe.close()
            self.pipe = None


__all__ = ["EncodedShard", "EpochSampler", "DecodeLoader", "SppError"]
