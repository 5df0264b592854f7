/*
 * spp.h — C ABI of libspp: scientific-sample preprocessing for B200 (sm_100a).
 *
 * The library implements the data-parallel hot path of Ibrahim & Oliker,
 * "Preprocessing Pipeline Optimization for Scientific Deep Learning Workloads"
 * (IPDPS'22; /root/reference/PAPER.md, cited as P:<line>):
 *   b.1  encode each sample once on the host            (Fig. 1 b.1)
 *   b.4  move the compressed bytes host -> HBM           (b.4)
 *   b.5  decode on the GPU, fused with the application's preprocessing, into
 *        an FP16 training tensor
 * for CosmoFlow (LUT format + ln(1+c) on the unique values)
 * and DeepCAM (differential line format + per-channel normalisation,
 * P:72-92).  Byte layouts and arithmetic: FORMAT.md.
 *
 * Conventions (all entry points):
 *  - extern "C", little-endian, sizes in bytes.  No torch types.
 *  - Ownership: every buffer is caller-owned.  The library never allocates or
 *    frees caller memory; scratch comes from opts->workspace.  Only
 *    spp_pipeline_create allocates (its own staging ring and events), freed by
 *    spp_pipeline_destroy.
 *  - Host-checkable argument errors return immediately and enqueue nothing.
 *    Stream corruption is detected on the device and reported through
 *    opts->status (the first error wins); the affected sample's output is
 *    unspecified, no out-of-bounds access happens.
 *  - Device calls are asynchronous on `stream` (a cudaStream_t; NULL = legacy
 *    default stream), on the current CUDA device, never synchronise the host
 *    and never allocate.
 *  - There is no CPU fallback: a device call without a usable sm_100 GPU
 *    returns SPP_ERR_CUDA.
 */
#ifndef SPP_H
#define SPP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *spp_stream_t; /* identical to cudaStream_t */

typedef enum {
    SPP_OK = 0,
    SPP_ERR_INVALID_ARG = 1,      /* null pointer, bad dims, bad enum, misalignment */
    SPP_ERR_BUFFER_TOO_SMALL = 2, /* dst / workspace / staging too small; *encoded_size = required */
    SPP_ERR_CORRUPT = 3,          /* malformed stream (device status, or host-side parse) */
    SPP_ERR_UNSUPPORTED = 4,      /* legal by FORMAT.md but outside the GPU path's limits */
    SPP_ERR_CUDA = 5              /* CUDA runtime error (no device, launch failure, ...) */
} spp_status;

typedef enum { SPP_FMT_COSMO = 1, SPP_FMT_DEEPCAM = 2 } spp_format;

typedef enum {
    SPP_OUT_F16 = 1, /* IEEE binary16, RNE from the fp32 value ("FP16 samples") */
    SPP_OUT_F32 = 2, /* IEEE binary32 */
    SPP_OUT_I16 = 3  /* CosmoFlow with transform = 0 only: the decoded int16 counts */
} spp_out;

/* ------------------------------------------------------------------------ */
/* Host encoders (b.1).  Reentrant and thread-safe, no global state, no
 * CUDA.  On SPP_ERR_BUFFER_TOO_SMALL, *encoded_size holds the required size. */

/* Upper bound of spp_encode_cosmo's output for a C x D x H x W volume. */
size_t spp_cosmo_max_encoded_size(int C, int D, int H, int W);

/* CosmoFlow LUT encoder (FORMAT.md 1.3; P:98-100 unique values and 4-groups,
 * P:106 1/2-byte keys with 8-byte lookup values).
 *   counts : host int16 [C][D][H][W] (CDHW), every value >= 0 (P:96 particle
 *            counts; negative -> SPP_ERR_INVALID_ARG)
 *   C      : must be 4 (four redshifts)
 *   dst    : host buffer of dst_capacity bytes, 16-B aligned not required
 * Output is deterministic: same input -> same bytes. */
spp_status spp_encode_cosmo(const int16_t *counts, int C, int D, int H, int W,
                            void *dst, size_t dst_capacity, size_t *encoded_size);

/* CosmoFlow encoder policy (FORMAT.md 1.3 / 1.4).
 *   localize : 0 (default) = one table for the whole volume, halved along z
 *              only while a table would exceed 65,536 groups (FORMAT.md 1.3);
 *              1 = "localized lookup tables" (multiple tables
 *              P:100): the dyadic z-partition with the fewest encoded bytes,
 *              so slabs whose groups fit 256 take 1-byte keys.  Never
 *              larger than localize = 0.  Any other value -> SPP_ERR_INVALID_ARG.
 * Both policies write FORMAT.md v1 streams; the decoders are unchanged. */
typedef struct {
    int localize;
    int escape_keys;  /* 1 = FORMAT.md 1.5: a slab that would take 2-byte keys stores
                         1-byte keys with the 255 most frequent groups inline and an
                         escape list of the rest, when that is smaller (beyond the
                         paper's 1/2-byte keys); 0 (default) = off */
} spp_cosmo_params;

/* spp_encode_cosmo with an explicit policy (params may be NULL = defaults;
 * escape_keys other than 0/1 -> SPP_ERR_INVALID_ARG);
 * spp_cosmo_max_encoded_size bounds both policies. */
spp_status spp_encode_cosmo_ex(const int16_t *counts, int C, int D, int H, int W,
                               const spp_cosmo_params *params, void *dst, size_t dst_capacity,
                               size_t *encoded_size);

/* Upper bound of spp_encode_deepcam's output for C x H x W. */
size_t spp_deepcam_max_encoded_size(int C, int H, int W);

/* DeepCAM differential line encoder (FORMAT.md 2.4; Fig. 4).
 *   x : host fp32 [C][H][W] (CHW); lines are rows of W values along x.
 *       Non-finite values are legal and force a RAW (uncompressed) line.
 * Lossy within the bound of DESIGN.md reading S19; deterministic. */
spp_status spp_encode_deepcam(const float *x, int C, int H, int W,
                              void *dst, size_t dst_capacity, size_t *encoded_size);

/* Encoder policy knobs (FORMAT.md 2.4).  PAPER.md P:84 fixes
 * the code (1 sign, 3 exponent, 4 mantissa bits, per-segment minimum
 * exponent) but not how segments are chosen; these trade bytes for error:
 *   lookahead  : positions whose differences set a new DIFF segment's emin
 *                (default 64; shorter windows adapt emin faster: smaller
 *                errors next to abrupt changes, more segments).  2..65535.
 *   repeat_min : shortest run of bit-identical values that opens a REPEAT
 *                segment (default 16).  2..65535.
 *   rel_err    : relative-error threshold of the error budget (default 0.1,
 *                the paper's "larger than 10% error"); > 0 and finite.
 *   err_budget : FORMAT.md 2.5 error budget (default 0 = off).  k > 0: a line
 *                whose SEG encoding has k or more values with
 *                |x̂ - x| > rel_err |x| (S19) is written RAW, i.e.
 *                kept uncompressed ("areas with abrupt changes are kept
 *                uncompressed").  Trades bytes for fewer large errors.
 *   raw16      : 1 = a line the error budget keeps uncompressed is stored as
 *                binary16 (FORMAT.md 2.6, half the bytes) when every value is
 *                finite and its fp16 rounding is within rel_err of it; else
 *                fp32 RAW.  0 (default) = fp32 RAW only.  Other values ->
 *                SPP_ERR_INVALID_ARG.
 * A zero field selects its default.  Every setting obeys the per-value
 * error bound of DESIGN.md reading S19 (RAW16 lines: within rel_err) and
 * decodes on the same decoders. */
typedef struct {
    int lookahead;
    int repeat_min;
    float rel_err;
    int err_budget;
    int raw16;
    int raw_segments;  /* 1 = a line over the error budget may keep only its offending
                          A-blocks raw, as RAW segments of a mode-3 line (FORMAT.md 2.7),
                          when that is smaller and within the budget; 0 (default) = off */
    const float *repeat_tol;  /* host fp32[C] or NULL (= all 0): per-channel REPEAT tolerance
                                 (FORMAT.md 2.8; "all neighbouring values are similar",
                                 DESIGN.md S15).  tau_c > 0: a run of values within tau_c of
                                 its first value, |x_j - x_i| <= tau_c, may become a REPEAT
                                 of x_i (decoded error <= tau_c); 0: bit-identical runs only.
                                 Each finite and >= 0, else SPP_ERR_INVALID_ARG. */
    const float *max_abs_err; /* host fp32[C] or NULL (= all 0): per-channel absolute error
                                 bound (FORMAT.md 2.8).  eps_c > 0: every decoded value of
                                 channel c satisfies |x̂ - x| <= eps_c; a SEG line that would
                                 exceed it is kept uncompressed (RAW, or RAW16 / RAW segments
                                 when allowed and within the bound).  0: no bound. */
} spp_deepcam_params;

/* spp_encode_deepcam with explicit policy knobs (params may be NULL = defaults);
 * out-of-range knobs -> SPP_ERR_INVALID_ARG. */
spp_status spp_encode_deepcam_ex(const float *x, int C, int H, int W, const spp_deepcam_params *params,
                                 void *dst, size_t dst_capacity, size_t *encoded_size);

/* Host-side parse of one encoded sample's header (no CUDA).  For CosmoFlow
 * info[0..3] = nU, nslab, G of slab 0, kw of slab 0; for DeepCAM info[0..3] =
 * number of RAW lines, SEG lines, total segments, total delta bytes.
 * Returns SPP_ERR_CORRUPT on a malformed stream. */
spp_status spp_stream_info(spp_format fmt, const void *src, size_t src_bytes, int64_t info[4]);

/* ------------------------------------------------------------------------ */
/* Device decode (b.5). */

typedef struct {
    int out;                 /* spp_out: SPP_OUT_F16 (default) | SPP_OUT_F32 | SPP_OUT_I16 */
    int transform;           /* CosmoFlow: 1 = ln(1+c) (default), 0 = identity */
    const float *shift;      /* DeepCAM: device fp32[C] or NULL (= 0)   y = (x - shift) * scale */
    const float *scale;      /* DeepCAM: device fp32[C] or NULL (= 1)   (reading S18) */
    uint32_t *status;        /* optional device word; 0 = ok, else (spp_status | sample << 8) of
                                the first corrupt sample.  The caller zeroes it. */
    const uint64_t *src_bytes; /* optional device u64[n]: size of each source buffer; when given,
                                  every read is bounds-checked against it as well */
    void *workspace;         /* device scratch >= spp_decode_workspace_size(), 256-B aligned */
    size_t workspace_size;
    int C, D, H, W;          /* expected dims (CosmoFlow C=4,D,H,W; DeepCAM C,H,W with D ignored);
                                every sample header must match (else CORRUPT in status) */
    void *const *timing_events; /* optional host array of 3 cudaEvent_t, recorded on `stream`
                                   before the prologue kernel, between the prologue and the main
                                   kernel, and after the main kernel (live per-kernel timing) */
    int escape_keys;         /* CosmoFlow: 1 = the batch may hold FORMAT.md 1.5 escaped-key slabs
                                (spp_encode_cosmo_ex escape_keys = 1): use the kernel variant that
                                stages them.  0 (default): the paper-format kernel, which reports
                                such samples as SPP_ERR_UNSUPPORTED in `status` (odd shapes that
                                take the scalar kernel decode them either way). */
    int raw_segments;        /* DeepCAM: 1 = the batch may hold FORMAT.md 2.7 mode-3 lines
                                (spp_encode_deepcam_ex raw_segments = 1): W = 1152 batches use the
                                KD instance that decodes them (and FORMAT.md 2.6 RAW16 lines) in one
                                warp pass.  0 (default): the mode-1 instance, on which those lines
                                take the general line path (same bits, slower).  Other values -> SPP_ERR_INVALID_ARG.
                                spp_decode_host reads each sample's header flags (FORMAT.md 2.1 bit 0, set
                                by the encoders when such lines exist) and selects this instance itself. */
} spp_decode_opts;

/* Fill opts with defaults for fmt and the given dims (out = F16, transform = 1). */
void spp_decode_opts_init(spp_decode_opts *opts, spp_format fmt, int C, int D, int H, int W);

/* Bytes of device workspace spp_decode_batch needs for n samples. */
size_t spp_decode_workspace_size(spp_format fmt, int n, const spp_decode_opts *opts);

/* Bytes of one decoded sample (C*D*H*W or C*H*W elements times the out size). */
size_t spp_decoded_sample_bytes(spp_format fmt, const spp_decode_opts *opts);

/* Decode + preprocess a batch of n encoded samples resident in HBM.
 *   d_src : DEVICE array of n DEVICE pointers, each to a 16-B aligned stream
 *   d_dst : device output, n samples back to back, [n][C][D][H][W] (CosmoFlow,
 *           CDHW: the transpose is fused) or [n][C][H][W] (DeepCAM),
 *           16-B aligned
 * Launches the sm_100a kernels (CosmoFlow: transform of the unique values then
 * the fused LUT expansion; DeepCAM: header/directory parse then the warp-per-line
 * differential decode) on `stream`.  Returns after enqueueing.
 * L2 residency of the output: CosmoFlow stores it as streaming (evict-first)
 * data; DeepCAM rows are stored with an L2 evict_first hint when the launch
 * writes more than 64 MB (batches) and with normal priority below that, so a
 * small batch's output can still be in L2 for its consumer.  Compressed inputs
 * are read once (CosmoFlow key tiles carry an evict_first hint). */
spp_status spp_decode_batch(spp_format fmt, const void *const *d_src, int n, void *d_dst,
                            const spp_decode_opts *opts, spp_stream_t stream);

/* Number of kernel launches one spp_decode_batch call enqueues (for accounting). */
int spp_decode_launches(spp_format fmt);

/* ------------------------------------------------------------------------ */
/* Streamed decode from host memory (b.4 + b.5): the compressed bytes are
 * copied host -> device in chunks on a copy stream, overlapped with the
 * decode of the previous chunk on `stream` (double/triple buffered staging
 * ring owned by the pipeline).  Host sources should be pinned
 * (cudaHostAlloc / cudaHostRegister) for the copies to be asynchronous. */
typedef struct spp_pipeline spp_pipeline;

/*   slot_bytes : capacity of one staging slot (>= the largest chunk of samples)
 *   nslots     : ring depth (2..8)
 *   max_chunk  : maximum samples per chunk (decode launch)
 * Allocates device staging (nslots * slot_bytes), a pinned descriptor area,
 * a device workspace, events and a copy stream on the current device. */
spp_status spp_pipeline_create(spp_pipeline **out, spp_format fmt, const spp_decode_opts *opts,
                               size_t slot_bytes, int nslots, int max_chunk);
void spp_pipeline_destroy(spp_pipeline *p);

/* Decode n host-resident samples into d_dst (layout as spp_decode_batch).
 * Calls on one pipeline are ordered: each call's first decode waits (on the
 * device) for the previous call's last decode, whatever streams they used, since
 * they share the pipeline's workspace and staging ring.
 *   h_src     : HOST array of n HOST pointers (pinned for async copies)
 *   src_bytes : HOST array of n sizes (multiples of 16)
 *   opts      : as spp_decode_batch; opts->workspace/src_bytes are ignored
 *               (the pipeline owns its workspace)
 * All work is enqueued on `stream` (decode) and the pipeline's copy stream; the
 * call returns when everything is enqueued (it may block only while the
 * staging ring is full).  Samples of one chunk that lie back to back in host
 * memory (h_src[k+1] == h_src[k] + src_bytes[k]) are copied with one
 * transfer. */
spp_status spp_decode_host(spp_pipeline *p, const void *const *h_src, const size_t *src_bytes,
                           int n, void *d_dst, const spp_decode_opts *opts, spp_stream_t stream);

/* Number of decode launches and copies the last spp_decode_host call enqueued. */
int spp_pipeline_last_launches(const spp_pipeline *p);

/* ------------------------------------------------------------------------ */
/* Labels: lossless label coding (FORMAT.md 3; "For both
 * applications, we use lossless compression of the labels").  DeepCAM labels
 * are per-pixel class masks (P:56 semantic segmentation), coded per row as
 * maximal runs of one class or verbatim; CosmoFlow labels are the four
 * cosmological parameters, kept as binary32.  One label stream per
 * sample, independent of the sample stream. */
typedef enum { SPP_LABEL_MASK = 1, SPP_LABEL_VECTOR = 2 } spp_label_kind;

/* Upper bound of an encoded label stream: kind MASK, H x W; kind VECTOR, W values (H = 1). */
size_t spp_label_max_encoded_size(int kind, int H, int W);

/* mask: host u8 [H][W] row-major class values (any 0..255).  Lossless;
 * deterministic.  H, W in 1..65535.  dst/dst_capacity/encoded_size as the
 * sample encoders (SPP_ERR_BUFFER_TOO_SMALL reports the required size). */
spp_status spp_encode_label_mask(const uint8_t *mask, int H, int W, void *dst, size_t dst_capacity,
                                 size_t *encoded_size);

/* v: host fp32 [n], n in 1..65535, stored verbatim (bit-exact, NaN payloads included). */
spp_status spp_encode_label_vector(const float *v, int n, void *dst, size_t dst_capacity, size_t *encoded_size);

/* Decode n label streams resident in HBM (one kernel launch on `stream`):
 *   kind      : SPP_LABEL_MASK -> d_dst u8 [n][H][W]; SPP_LABEL_VECTOR -> d_dst fp32 [n][W] (H must be 1)
 *   d_src     : DEVICE array of n DEVICE pointers, each 16-B aligned
 *   src_bytes : optional device u64[n] bounding each stream's reads (NULL = trust the header)
 *   status    : optional device word, as spp_decode_opts.status (a stream whose header does not match
 *               kind/H/W, or a malformed row, sets SPP_ERR_CORRUPT | sample << 8)
 * Host-checkable errors (n < 0, null pointers, bad kind/dims) return SPP_ERR_INVALID_ARG.
 * Masks are stored with an L2 evict_first hint when the launch writes more than 64 MB. */
spp_status spp_decode_labels(int kind, const void *const *d_src, const uint64_t *src_bytes, int n, void *d_dst,
                             int H, int W, uint32_t *status, spp_stream_t stream);

const char *spp_status_string(spp_status s);

/* Library build identification: "spp <version> sm_100a". */
const char *spp_version(void);

#ifdef __cplusplus
}
#endif

#endif /* SPP_H */
