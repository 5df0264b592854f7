// pipeline.cu — streamed decode from host memory (b.4 + b.5 of PAPER.md
// Fig. 1): compressed samples are copied host -> HBM in chunks on a
// dedicated copy stream into a ring of staging slots, and each chunk is
// decoded on the caller's stream as soon as its copy lands, overlapping the
// PCIe transfer of chunk i+1 with the decode of chunk i.
// measured the pageable-vs-pinned gap that motivates pinned sources.
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <new>
#include <vector>

#include "spp.h"
#include "spp_format.h"
#include "spp_internal.h"

struct spp_pipeline {
    int device = 0;
    spp_format fmt = SPP_FMT_COSMO;
    spp_decode_opts opts{};
    size_t slot_bytes = 0;
    int nslots = 0, max_chunk = 0;
    uint8_t *d_stage = nullptr;
    const void **h_ptrs = nullptr;  // pinned [nslots][max_chunk]
    const void **d_ptrs = nullptr;  // device
    uint64_t *h_sizes = nullptr;    // pinned [nslots][max_chunk]
    uint64_t *d_sizes = nullptr;    // device
    void *d_ws = nullptr;
    size_t ws_bytes = 0;
    cudaStream_t copy = nullptr;
    std::vector<cudaEvent_t> copied, freed;
    std::vector<int> freed_pending;
    cudaEvent_t done = nullptr;  // recorded after a call's last decode; the next call's stream waits on it
    bool done_pending = false;
    int last_launches = 0;
};

static void destroy_impl(spp_pipeline *p) {
    if (!p) return;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(p->device);
    if (p->copy) cudaStreamSynchronize(p->copy);
    for (size_t i = 0; i < p->freed.size(); i++) {
        if (p->freed[i]) { cudaEventSynchronize(p->freed[i]); cudaEventDestroy(p->freed[i]); }
        if (p->copied[i]) cudaEventDestroy(p->copied[i]);
    }
    if (p->done) { cudaEventSynchronize(p->done); cudaEventDestroy(p->done); }
    if (p->copy) cudaStreamDestroy(p->copy);
    cudaFree(p->d_stage);
    cudaFree(p->d_ptrs);
    cudaFree(p->d_sizes);
    cudaFree(p->d_ws);
    cudaFreeHost(p->h_ptrs);
    cudaFreeHost(p->h_sizes);
    cudaSetDevice(prev);
    delete p;
}

extern "C" {

spp_status spp_pipeline_create(spp_pipeline **out, spp_format fmt, const spp_decode_opts *opts, size_t slot_bytes,
                               int nslots, int max_chunk) {
    if (!out || !opts || slot_bytes < 64 || nslots < 2 || nslots > 8 || max_chunk < 1) return SPP_ERR_INVALID_ARG;
    if (fmt != SPP_FMT_COSMO && fmt != SPP_FMT_DEEPCAM) return SPP_ERR_INVALID_ARG;
    *out = nullptr;
    spp_pipeline *p = new (std::nothrow) spp_pipeline();
    if (!p) return SPP_ERR_CUDA;
    if (cudaGetDevice(&p->device) != cudaSuccess) { delete p; return SPP_ERR_CUDA; }
    p->fmt = fmt;
    p->opts = *opts;
    p->slot_bytes = spp::round_up16(slot_bytes);
    p->nslots = nslots;
    p->max_chunk = max_chunk;
    p->ws_bytes = spp_decode_workspace_size(fmt, max_chunk, opts);
    const size_t nd = (size_t)nslots * max_chunk;
    bool ok = cudaMalloc(&p->d_stage, p->slot_bytes * nslots) == cudaSuccess &&
              cudaMalloc(&p->d_ptrs, nd * sizeof(void *)) == cudaSuccess &&
              cudaMalloc(&p->d_sizes, nd * sizeof(uint64_t)) == cudaSuccess &&
              cudaMalloc(&p->d_ws, p->ws_bytes ? p->ws_bytes : 256) == cudaSuccess &&
              cudaHostAlloc(&p->h_ptrs, nd * sizeof(void *), cudaHostAllocDefault) == cudaSuccess &&
              cudaHostAlloc(&p->h_sizes, nd * sizeof(uint64_t), cudaHostAllocDefault) == cudaSuccess &&
              cudaStreamCreateWithFlags(&p->copy, cudaStreamNonBlocking) == cudaSuccess;
    p->copied.assign(nslots, nullptr);
    p->freed.assign(nslots, nullptr);
    p->freed_pending.assign(nslots, 0);
    for (int i = 0; ok && i < nslots; i++)
        ok = cudaEventCreateWithFlags(&p->copied[i], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&p->freed[i], cudaEventDisableTiming) == cudaSuccess;
    ok = ok && cudaEventCreateWithFlags(&p->done, cudaEventDisableTiming) == cudaSuccess;
    if (!ok) {
        cudaGetLastError();
        destroy_impl(p);
        return SPP_ERR_CUDA;
    }
    *out = p;
    return SPP_OK;
}

void spp_pipeline_destroy(spp_pipeline *p) { destroy_impl(p); }

int spp_pipeline_last_launches(const spp_pipeline *p) { return p ? p->last_launches : 0; }

spp_status spp_decode_host(spp_pipeline *p, const void *const *h_src, const size_t *src_bytes, int n, void *d_dst,
                           const spp_decode_opts *opts, spp_stream_t stream) {
    if (!p || !opts || n < 0) return SPP_ERR_INVALID_ARG;
    p->last_launches = 0;
    if (n == 0) return SPP_OK;
    if (!h_src || !src_bytes || !d_dst) return SPP_ERR_INVALID_ARG;
    for (int i = 0; i < n; i++) {
        if (!h_src[i] || src_bytes[i] < 64 || (src_bytes[i] & 15)) return SPP_ERR_INVALID_ARG;
        if (src_bytes[i] > p->slot_bytes) return SPP_ERR_BUFFER_TOO_SMALL;
    }
    const size_t out_bytes = spp_decoded_sample_bytes(p->fmt, opts);
    if (!out_bytes) return SPP_ERR_INVALID_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    spp_decode_opts o = *opts;
    o.workspace = p->d_ws;
    o.workspace_size = p->ws_bytes;
    // the previous call may still be decoding on another stream: the shared
    // workspace (per-chunk meta / f(U)) must not be rewritten before it is done
    if (p->done_pending && cudaStreamWaitEvent(st, p->done, 0) != cudaSuccess) return SPP_ERR_CUDA;
    int i = 0, chunk = 0;
    while (i < n) {
        const int slot = chunk % p->nslots;
        if (p->freed_pending[slot]) {
            // the slot's previous chunk must be decoded before its staging and
            // descriptor memory are reused (blocks only when the ring is full)
            if (cudaEventSynchronize(p->freed[slot]) != cudaSuccess) return SPP_ERR_CUDA;
            p->freed_pending[slot] = 0;
        }
        const void **hp = p->h_ptrs + (size_t)slot * p->max_chunk;
        uint64_t *hs = p->h_sizes + (size_t)slot * p->max_chunk;
        uint8_t *stage = p->d_stage + (size_t)slot * p->slot_bytes;
        size_t off = 0;
        int k = 0;
        // samples that sit back to back in host memory travel as one copy
        // (large PCIe transfers run closer to the link rate than per-sample ones)
        const uint8_t *run_src = nullptr;
        size_t run_off = 0, run_len = 0;
        while (i + k < n && k < p->max_chunk && off + src_bytes[i + k] <= p->slot_bytes) {
            const uint8_t *h = static_cast<const uint8_t *>(h_src[i + k]);
            hp[k] = stage + off;
            hs[k] = src_bytes[i + k];
            if (run_len && h == run_src + run_len) {
                run_len += src_bytes[i + k];
            } else {
                if (run_len && cudaMemcpyAsync(stage + run_off, run_src, run_len, cudaMemcpyHostToDevice, p->copy) !=
                                   cudaSuccess)
                    return SPP_ERR_CUDA;
                run_src = h;
                run_off = off;
                run_len = src_bytes[i + k];
            }
            off += src_bytes[i + k];
            k++;
        }
        if (run_len && cudaMemcpyAsync(stage + run_off, run_src, run_len, cudaMemcpyHostToDevice, p->copy) != cudaSuccess)
            return SPP_ERR_CUDA;
        const void **dp = p->d_ptrs + (size_t)slot * p->max_chunk;
        uint64_t *ds = p->d_sizes + (size_t)slot * p->max_chunk;
        if (cudaMemcpyAsync(dp, hp, k * sizeof(void *), cudaMemcpyHostToDevice, p->copy) != cudaSuccess ||
            cudaMemcpyAsync(ds, hs, k * sizeof(uint64_t), cudaMemcpyHostToDevice, p->copy) != cudaSuccess ||
            cudaEventRecord(p->copied[slot], p->copy) != cudaSuccess ||
            cudaStreamWaitEvent(st, p->copied[slot], 0) != cudaSuccess)
            return SPP_ERR_CUDA;
        o.src_bytes = ds;
        // the host holds the headers: a DeepCAM chunk with extended line modes
        // (header flags bit 0, FORMAT.md 2.1) takes the KD instance that decodes
        // them in one pass, whatever opts->raw_segments says
        o.raw_segments = opts->raw_segments;
        if (p->fmt == SPP_FMT_DEEPCAM && !o.raw_segments)
            for (int j = 0; j < k; j++) {
                uint16_t flags;
                memcpy(&flags, static_cast<const uint8_t *>(h_src[i + j]) + 6, 2);
                if (flags & 1u) o.raw_segments = 1;
            }
        spp_status r = spp_decode_batch(p->fmt, dp, k, static_cast<uint8_t *>(d_dst) + (size_t)i * out_bytes, &o,
                                        stream);
        if (r != SPP_OK) return r;
        p->last_launches += spp_decode_launches(p->fmt);
        if (cudaEventRecord(p->freed[slot], st) != cudaSuccess) return SPP_ERR_CUDA;
        p->freed_pending[slot] = 1;
        i += k;
        chunk++;
    }
    if (cudaEventRecord(p->done, st) != cudaSuccess) return SPP_ERR_CUDA;
    p->done_pending = true;
    return SPP_OK;
}

}  // extern "C"
