"""paper_conf_ipps_ibrahimo22_b200 — B200-native decode + preprocess of the
CosmoFlow / DeepCAM compressed sample formats of Ibrahim & Oliker (IPDPS'22).

The product is ``libspp.so`` (C ABI, include/spp.h; sm_100a CUDA kernels in
``csrc/``).  This package is its thin Python face: ``spp`` mirrors the C
names, ``Decoder`` / ``HostPipeline`` wrap device memory, workspaces and
streams with PyTorch (plumbing only: every byte of the hot path is produced by
libspp's kernels).
"""
from __future__ import annotations

from . import spp
from .spp import (FMT, OUT, SppError, spp_decode_batch, spp_decode_host, spp_decode_opts_init,
                  spp_encode_cosmo, spp_encode_deepcam, spp_stream_info, spp_version)

__all__ = ["spp", "Decoder", "HostPipeline", "LabelDecoder", "SppError", "spp_encode_cosmo", "spp_encode_deepcam",
           "spp_decode_batch", "spp_decode_host", "spp_decode_opts_init", "spp_stream_info", "spp_version",
           "sample_shape"]


def sample_shape(fmt: str, dims):
    """Decoded tensor shape of one sample: [C, D, H, W] (cosmo) or [C, H, W] (deepcam)."""
    return tuple(dims) if fmt == "cosmo" else (dims[0], dims[-2], dims[-1])


_TORCH_DT = {"f16": "float16", "f32": "float32", "i16": "int16"}


class Decoder:
    """Device-resident batch decode through ``spp_decode_batch``.

    ``dims``: (4, D, H, W) for cosmo, (C, H, W) for deepcam.  Sources are CUDA
    uint8 tensors (one per sample, 16-B aligned) or one device int64 tensor of
    pointers.  The workspace and status word are torch allocations reused
    across calls.
    """

    def __init__(self, fmt: str, dims, out: str = "f16", transform: int | None = None, device=None,
                 escape_keys: bool = False, raw_segments: bool = False):
        import torch
        self.torch = torch
        spp.load()
        self.fmt = fmt
        self.dims = tuple(int(d) for d in dims)
        Cc, D, H, W = (self.dims if fmt == "cosmo" else (self.dims[0], 1, self.dims[1], self.dims[2]))
        self.out = out
        self.opts = spp_decode_opts_init(fmt, Cc, D, H, W, out=out, transform=transform)
        self.opts.escape_keys = int(bool(escape_keys))  # FORMAT.md 1.5 streams: the staging kernel
        self.opts.raw_segments = int(bool(raw_segments))  # FORMAT.md 2.7 streams: the mode-3 KD instance
        self.device = torch.device(device or "cuda")
        self.status = torch.zeros(1, dtype=torch.int32, device=self.device)
        self._ws = None
        self._ws_n = 0
        self.shift = None
        self.scale = None
        # bumped whenever a device buffer a captured decode refers to is replaced
        # (workspace, shift/scale): CUDA graphs captured earlier must be dropped
        self.version = 0

    def set_normalisation(self, shift, scale):
        """DeepCAM per-channel (shift, scale) as device fp32 tensors [C] (or None)."""
        t = self.torch
        self.shift = None if shift is None else t.as_tensor(shift, dtype=t.float32, device=self.device).contiguous()
        self.scale = None if scale is None else t.as_tensor(scale, dtype=t.float32, device=self.device).contiguous()
        self.version += 1

    def workspace(self, n: int):
        need = spp.spp_decode_workspace_size(self.fmt, n, self.opts)
        if self._ws is None or self._ws.numel() < need:
            self._ws = self.torch.empty(max(need, 256), dtype=self.torch.uint8, device=self.device)
            self.version += 1
        return self._ws, need

    def alloc_out(self, n: int):
        t = self.torch
        return t.empty((n, *sample_shape(self.fmt, self.dims)), dtype=getattr(t, _TORCH_DT[self.out]),
                       device=self.device)

    def pointer_table(self, srcs):
        t = self.torch
        return t.tensor([s.data_ptr() for s in srcs], dtype=t.int64, device=self.device)

    def decode(self, srcs, out=None, n: int | None = None, src_bytes=None, stream=None):
        """Enqueue the decode of n samples on `stream` (default: current stream)."""
        t = self.torch
        ptrs = srcs if isinstance(srcs, t.Tensor) and srcs.dtype == t.int64 else self.pointer_table(srcs)
        n = int(ptrs.numel()) if n is None else n
        if out is None:
            out = self.alloc_out(n)
        ws, need = self.workspace(n)
        o = self.opts
        o.workspace = ws.data_ptr()
        o.workspace_size = ws.numel()
        o.status = self.status.data_ptr()
        o.shift = None if self.shift is None else self.shift.data_ptr()
        o.scale = None if self.scale is None else self.scale.data_ptr()
        o.src_bytes = None if src_bytes is None else src_bytes.data_ptr()
        st = (stream or t.cuda.current_stream()).cuda_stream
        spp_decode_batch(self.fmt, ptrs.data_ptr(), n, out.data_ptr(), o, st)
        return out

    def check_status(self):
        """Synchronise on the status word; raise SppError for a corrupt sample."""
        v = int(self.status.item()) & 0xFFFFFFFF
        if v:
            self.status.zero_()
            raise SppError(v & 0xFF, f"sample {v >> 8}")


class LabelDecoder:
    """Device-resident batch decode of label streams through ``spp_decode_labels``
    (FORMAT.md 3; PAPER.md P:175 lossless labels).  kind "mask": dims (H, W),
    output u8 [n, H, W]; kind "vector": dims (W,), output fp32 [n, W]."""

    def __init__(self, kind: str, dims, device=None):
        import torch
        self.torch = torch
        spp.load()
        if kind not in spp.LABEL_KIND:
            raise ValueError("kind is 'mask' or 'vector'")
        self.kind = kind
        self.dims = tuple(int(d) for d in dims)
        self.H, self.W = (self.dims if kind == "mask" else (1, self.dims[-1]))
        self.device = torch.device(device or "cuda")
        self.status = torch.zeros(1, dtype=torch.int32, device=self.device)

    def alloc_out(self, n: int):
        t = self.torch
        if self.kind == "mask":
            return t.empty((n, self.H, self.W), dtype=t.uint8, device=self.device)
        return t.empty((n, self.W), dtype=t.float32, device=self.device)

    def decode(self, srcs, out=None, n: int | None = None, src_bytes=None, stream=None):
        t = self.torch
        ptrs = srcs if isinstance(srcs, t.Tensor) and srcs.dtype == t.int64 else \
            t.tensor([s.data_ptr() for s in srcs], dtype=t.int64, device=self.device)
        n = int(ptrs.numel()) if n is None else n
        if out is None:
            out = self.alloc_out(n)
        st = (stream or t.cuda.current_stream()).cuda_stream
        spp.spp_decode_labels(self.kind, ptrs.data_ptr(), n, out.data_ptr(), self.H, self.W, self.status.data_ptr(),
                              0 if src_bytes is None else src_bytes.data_ptr(), st)
        return out

    def check_status(self):
        v = int(self.status.item()) & 0xFFFFFFFF
        if v:
            self.status.zero_()
            raise SppError(v & 0xFF, f"label sample {v >> 8}")


class HostPipeline:
    """Streamed decode from pinned host memory via ``spp_decode_host`` (b.4+b.5)."""

    def __init__(self, decoder: Decoder, slot_bytes: int, nslots: int = 3, max_chunk: int = 16):
        self.dec = decoder
        self.handle = spp.spp_pipeline_create(decoder.fmt, decoder.opts, slot_bytes, nslots, max_chunk)

    def decode(self, host_srcs, out, stream=None):
        t = self.dec.torch
        o = self.dec.opts
        o.status = self.dec.status.data_ptr()
        o.shift = None if self.dec.shift is None else self.dec.shift.data_ptr()
        o.scale = None if self.dec.scale is None else self.dec.scale.data_ptr()
        st = (stream or t.cuda.current_stream()).cuda_stream
        spp_decode_host(self.handle, [s.data_ptr() for s in host_srcs], [s.numel() for s in host_srcs],
                        out.data_ptr(), o, st)
        return out

    def launches(self) -> int:
        return spp.spp_pipeline_last_launches(self.handle)

    def close(self):
        if self.handle:
            spp.spp_pipeline_destroy(self.handle)
            self.handle = 0

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
