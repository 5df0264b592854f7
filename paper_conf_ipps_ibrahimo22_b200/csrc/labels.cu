// labels.cu — GPU decode of the lossless label streams (FORMAT.md 3; PAPER.md
// P:175 "For both applications, we use lossless compression of the labels").
//
//   KL  kl_decode_mask  persistent warps, one mask row at a time (rows are
//                       independent, like DeepCAM data lines).  Rows of
//                       <= 32 runs (W % 16 == 0, W <= 2048) are filled in
//                       registers and leave by TMA bulk store
//                       (kl_run_row_staged); other RUN rows: the row's
//                       run starts (warp scan of the run lengths) are set in a
//                       per-warp bitmap of 1,024 positions; lane l owns 32
//                       consecutive positions, so the run of position p is
//                       (starts before the lane) + popc(bits <= p) - 1, and the
//                       lane writes its 32 class bytes with two 16-B stores.
//                       RAW rows are copied with 16-B loads/stores.
//   KL  kl_decode_vec   one thread per value (CosmoFlow's 4 parameters per
//                       sample): binary32 copied verbatim.
// Output: masks u8 [n][H][W]; vectors fp32 [n][W].  Corrupt streams set the
// status word (first error wins) and never read outside [src, src + total).
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <type_traits>

#include "common.cuh"
#include "spp_format.h"
#include "spp_internal.h"

namespace spp {
namespace {

constexpr uint32_t kLabelMagic = 0x4C505053u;  // "SPPL"
constexpr int kLabelHeader = 32;
constexpr int kKlWarps = 8;  // warps per CTA
constexpr uint32_t kKlChunk = 4096;  // positions per bitmap pass (128 words per warp)
constexpr uint32_t kKlFastW = 2048;  // staged rows: W % 16 == 0, W <= 2048 (<= 16 words, 64 positions per lane)
constexpr uint32_t kKlStageW = 2304;  // staging bytes per buffer: one row, or a row pair of W <= 1152
constexpr uint32_t kKlFastRuns = 32;  // staged RUN rows: one run per lane
constexpr uint32_t kKlPairRuns = 16;  // row pairs: one run per lane of a half-warp
#ifndef SPP_KL_GROUP_MINB  // CTAs per SM the row-group instances' registers target
#define SPP_KL_GROUP_MINB 4
#endif
#ifndef SPP_KL_QUADS  // 1: try 4-row groups (<= 8 runs per row) before pairs (measured 2.4% slower: r02b9)
#define SPP_KL_QUADS 0
#endif
// L2 policy of the staged rows' TMA bulk stores: evict_first when the launch writes
// more than kRowEfBytes (+4% on 2048 masks, profiles/r02b2_*, r02b3_*), normal below
// (a loader batch's labels stay L2-resident for their consumer)
#ifndef SPP_KL_ROW_EF
#define SPP_KL_ROW_EF 1
#endif
constexpr uint64_t kRowEfBytes = 64ull << 20;
__device__ __forceinline__ void kl_store(void *dst, const void *src, uint32_t bytes, uint64_t pol) {
    bulk_s2g_hint(dst, src, bytes, pol);
}

// inclusive warp scan, the shuffle's in-range predicate guarding the add
__device__ __forceinline__ uint32_t scan_u32(uint32_t v) {
#pragma unroll
    for (int d = 1; d < kWarp; d <<= 1)
        asm("{\n.reg .u32 t;\n.reg .pred p;\nshfl.sync.up.b32 t|p, %0, %1, 0, 0xffffffff;\n@p add.u32 %0, %0, t;\n}\n"
            : "+r"(v)
            : "r"(d));
    return v;
}

__device__ __forceinline__ void bulk_wait_read_1() { asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); }

// Staged RUN row (nrun <= 32, W % 16 == 0, W <= 2048; the paper's masks have
// 1-5 runs per row): lane r holds run r (length, value); one warp scan gives
// the run starts, each start sets one bit in the bitmap of the lane owning its
// position (lane l owns words [wpl l, wpl l + wpl) of the row: <= 64
// positions, two bitmap words); a popc scan of those words gives the run at
// each lane's first position, and the lane's words are filled in registers,
// written to the warp's staging row and leave with one TMA bulk store.
template <int WPL>  // words (4 positions) per lane: W = 1152 -> 9
__device__ __forceinline__ bool kl_run_row_staged(const uint8_t *p, uint32_t bytes, uint32_t nrun, uint32_t W,
                                                  uint32_t magic, uint32_t *bm, uint32_t bm_s,
                                                  uint8_t *stage, uint32_t stage_s, uint8_t *row, int lane,
                                                  uint64_t pol) {
    if (4ull + 3ull * nrun > bytes) return false;
    const bool have = (uint32_t)lane < nrun;
    const uint32_t len = have ? __ldg(reinterpret_cast<const uint16_t *>(p + 4) + lane) : 0u;
    const uint32_t val = have ? __ldg(p + 4 + 2 * nrun + lane) : 0u;
    const uint32_t incl = scan_u32(len), st = incl - len;
    const bool bad = __any_sync(0xffffffffu, have && len == 0) || __shfl_sync(0xffffffffu, incl, 31) != W;
    if (bad) return false;
    constexpr uint32_t rlen = 4u * WPL;  // positions per lane
    sts_u2(bm_s + 8u * (uint32_t)lane, make_uint2(0u, 0u));
    __syncwarp();
    if (have) {
        const uint32_t o = __umulhi(st, magic);  // st / rlen (exact: st < 2^16, rlen <= 64)
        const uint32_t b = st - o * rlen;
        atomicOr(bm + 2 * o + (b >> 5), 1u << (b & 31));
    }
    __syncwarp();
    const uint2 mm = lds_u2(bm_s + 8u * (uint32_t)lane);
    const uint32_t c = __popc(mm.x) + __popc(mm.y);
    const uint32_t before = scan_u32(c) - c;  // run starts before this lane's first position
    uint32_t idx = before + (mm.x & 1u) - 1u;  // run of the first position (run 0 starts at 0)
    uint64_t rest = ((uint64_t)mm.y << 32 | mm.x) & ~1ull;
    uint32_t v = __shfl_sync(0xffffffffu, val, idx & 31) * 0x01010101u;
    uint32_t out[WPL];
#pragma unroll
    for (int k = 0; k < WPL; k++) out[k] = v;
    const uint32_t tmax = __reduce_max_sync(0xffffffffu, c - (mm.x & 1u));
    for (uint32_t t = 0; t < tmax; t++) {  // one pass per run starting inside the lane's words
        const bool has = rest != 0;
        const uint32_t j = has ? (uint32_t)__ffsll((long long)rest) - 1u : 0u;
        idx += has;
        v = __shfl_sync(0xffffffffu, val, idx & 31) * 0x01010101u;
        rest &= rest - 1;
        if (has) {
            const uint32_t kj = j >> 2;
            const uint32_t keep = (j & 3) ? 0xFFFFFFFFu >> (32 - 8 * (j & 3)) : 0u;  // bytes of word kj before j
#pragma unroll
            for (int k = 0; k < WPL; k++) {
                const uint32_t m = (uint32_t)k > kj ? 0u : ((uint32_t)k == kj ? keep : 0xFFFFFFFFu);
                out[k] = (out[k] & m) | (v & ~m);
            }
        }
    }
    const uint32_t lo = rlen * (uint32_t)lane;
    const uint32_t nw = lo + rlen <= W ? (uint32_t)WPL : (lo < W ? (W - lo) / 4 : 0u);  // the last lanes: part / none
#pragma unroll
    for (int k = 0; k < WPL; k++)
        if ((uint32_t)k < nw) sts_f32(stage_s + lo + 4u * k, __uint_as_float(out[k]));
    fence_proxy_async_smem();  // this lane's staged words -> visible to the bulk store
    __syncwarp();
    if (lane == 0) kl_store(row, stage, W, pol);
    return true;
}

// inclusive scan within each LPR-lane segment of the warp (LPR = 16: half-warps, 8: quarters)
template <int LPR>
__device__ __forceinline__ uint32_t scan_seg_u32(uint32_t v) {
#pragma unroll
    for (int d = 1; d < LPR; d <<= 1)
        asm("{\n.reg .u32 t;\n.reg .pred p;\nshfl.sync.up.b32 t|p, %0, %1, %2, 0xffffffff;\n@p add.u32 %0, %0, t;\n}\n"
            : "+r"(v)
            : "r"(d), "n"((32 - LPR) << 8));
    return v;
}
// 0xFFFFFFFF << n with PTX shl semantics (n >= 32 gives 0)
__device__ __forceinline__ uint32_t ones_shl(uint32_t n) {
    uint32_t r;
    asm("shl.b32 %0, %1, %2;" : "=r"(r) : "r"(0xFFFFFFFFu), "r"(n));
    return r;
}

// G consecutive RUN rows (G = 2 or 4), at most 32/G runs each (W % 128 == 0,
// G W <= 2 kKlStageW): each LPR = 32/G-lane segment of the warp decodes one
// row exactly as kl_run_row_staged does with a whole warp -- lane hl holds run
// hl, a segment scan gives the starts, each start sets one bit in the bitmap
// of the lane owning its position (W / LPR positions per lane), a popc scan
// gives the run at each lane's first position, the lane fills its WPLG words
// in registers -- and the G rows, adjacent in dst, leave by ONE TMA bulk store.
// Every warp-collective step (scans, ballots, the bitmap round trip, the proxy
// fence and the store) is paid once per G rows.  p, bytes, nrun are the lane's
// segment's row.  Returns the rows decoded: bit LPR r set = row g + r.
template <int G, int WPLG>  // W = 1152: G = 2 -> 18 words per lane, G = 4 -> 36
__device__ __forceinline__ uint32_t kl_run_group_staged(const uint8_t *p, uint32_t bytes, uint32_t nrun, uint32_t W,
                                                        uint32_t magicg, uint32_t *bm, uint32_t bm_s, uint8_t *stage,
                                                        uint32_t stage_s, uint8_t *row0, int lane, uint64_t pol) {
    constexpr uint32_t LPR = 32 / G;                    // lanes per row
    constexpr uint32_t rlen = 4u * WPLG;                // positions per lane
    constexpr int NB = (int)((rlen + 31) / 32);         // bitmap words per lane
    constexpr int BMS = NB <= 4 ? 4 : 8;                // ... allocated in 16-B units
    constexpr uint32_t leaders = G == 2 ? 0x00010001u : 0x01010101u;
    const uint32_t hl = (uint32_t)lane & (LPR - 1), hb = (uint32_t)lane & ~(LPR - 1), h = (uint32_t)lane / LPR;
    const bool fits = 4ull + 3ull * nrun <= bytes;
    const bool have = fits && hl < nrun;
    const uint32_t len = have ? __ldg(reinterpret_cast<const uint16_t *>(p + 4) + hl) : 0u;
    const uint32_t val = have ? __ldg(p + 4 + 2 * nrun + hl) : 0u;
    const uint32_t incl = scan_seg_u32<LPR>(len), st = incl - len;
    const uint32_t tot = __shfl_sync(0xffffffffu, incl, (int)(hb | (LPR - 1)));
    const uint32_t zero_len = __ballot_sync(0xffffffffu, have && len == 0);
    const bool okh = fits && ((zero_len >> hb) & ((1u << LPR) - 1u)) == 0 && tot == W;
    const uint32_t okm = __ballot_sync(0xffffffffu, okh) & leaders;
#pragma unroll
    for (int w = 0; w < BMS; w += 4) sts_u4(bm_s + 4u * (BMS * (uint32_t)lane + w), make_uint4(0u, 0u, 0u, 0u));
    __syncwarp();
    if (have && okh) {
        const uint32_t o = __umulhi(st, magicg);  // st / rlen (exact: st < 2^16, rlen <= 144)
        const uint32_t b = st - o * rlen;
        atomicOr(bm + BMS * (hb | o) + (b >> 5), 1u << (b & 31));
    }
    __syncwarp();
    uint32_t mw[BMS];
#pragma unroll
    for (int w = 0; w < BMS; w += 4) {
        const uint4 q = lds_u4(bm_s + 4u * (BMS * (uint32_t)lane + w));
        mw[w] = q.x, mw[w + 1] = q.y, mw[w + 2] = q.z, mw[w + 3] = q.w;
    }
    uint32_t c = 0;
#pragma unroll
    for (int w = 0; w < NB; w++) c += __popc(mw[w]);
    const uint32_t first = mw[0] & 1u;
    const uint32_t before = scan_seg_u32<LPR>(c) - c;  // run starts before this lane's first position
    uint32_t idx = before + first - 1u;                 // run of the first position (run 0 starts at 0)
    mw[0] &= ~1u;
    uint32_t v = __shfl_sync(0xffffffffu, val, (int)(hb | (idx & (LPR - 1)))) * 0x01010101u;
    uint32_t out[WPLG];
#pragma unroll
    for (int k = 0; k < WPLG; k++) out[k] = v;
    const uint32_t tmax = __reduce_max_sync(0xffffffffu, c - first);
    for (uint32_t t = 0; t < tmax; t++) {  // one pass per run starting inside the lane's words
        bool has = false;
        uint32_t j = 0;
#pragma unroll
        for (int w = 0; w < NB; w++) {  // the lowest remaining start
            if (!has && mw[w]) {
                j = 32u * w + __ffs(mw[w]) - 1u;
                mw[w] &= mw[w] - 1;
                has = true;
            }
        }
        idx += has;
        v = __shfl_sync(0xffffffffu, val, (int)(hb | (idx & (LPR - 1)))) * 0x01010101u;
        if (has) {
            const int j8 = 8 * (int)j;
#pragma unroll
            for (int k = 0; k < WPLG; k++) {  // bytes at or after j take v
                const uint32_t take = ones_shl((uint32_t)max(j8 - 32 * k, 0));
                out[k] = (out[k] & ~take) | (v & take);
            }
        }
    }
    const uint32_t lo = stage_s + h * W + rlen * hl;
    static_assert((WPLG & 1) == 0, "row groups stage 8-byte pairs of words");
#pragma unroll
    for (int k = 0; k < WPLG; k += 2) sts_u2(lo + 4u * k, make_uint2(out[k], out[k + 1]));
    fence_proxy_async_smem();  // this lane's staged words -> visible to the bulk store
    __syncwarp();
    if (lane == 0 && okm) {
        if (okm == leaders) {
            kl_store(row0, stage, G * W, pol);
        } else {
#pragma unroll
            for (int r = 0; r < G; r++)
                if ((okm >> (LPR * r)) & 1u) kl_store(row0 + r * W, stage + r * W, W, pol);
        }
    }
    return okm;
}

// header check shared by both kinds: returns total (0 if invalid)
__device__ __forceinline__ uint64_t label_header_ok(const uint8_t *b, uint64_t limit, uint32_t kind, uint32_t H,
                                                    uint32_t W) {
    if (b == nullptr || (reinterpret_cast<uintptr_t>(b) & 15) != 0 || limit < (uint64_t)kLabelHeader) return 0;
    const uint4 h0 = *reinterpret_cast<const uint4 *>(b);
    const uint4 h1 = *reinterpret_cast<const uint4 *>(b + 16);
    const uint64_t total = (uint64_t)h1.y << 32 | h1.x;
    const bool ok = h0.x == kLabelMagic && (h0.y & 0xFFFFu) == kVersion && (h0.y >> 16) == kind &&
                    (h0.z & 0xFFFFu) == H && (h0.z >> 16) == W && total <= limit && (total & 15) == 0 &&
                    total >= (uint64_t)kLabelHeader;
    return ok ? total : 0;
}

template <int WPL, int WPLQ>  // WPL 0: no staged rows (W % 16 != 0, W > 2048 or an unaligned dst);
                              // WPLQ: words per lane of a 4-row group (W / 32), 0: no row groups
__global__ void __launch_bounds__(kKlWarps * kWarp, WPLQ > 0 ? SPP_KL_GROUP_MINB : 4) kl_decode_mask(const void *const *__restrict__ src,
                                                                   const uint64_t *__restrict__ src_bytes, int n,
                                                                   uint32_t H, uint32_t W, uint8_t *__restrict__ dst,
                                                                   uint32_t *__restrict__ status, uint32_t row_ef) {
    __shared__ uint32_t bitmap[kKlWarps][WPLQ > 0 ? 256 : kKlChunk / 32];  // 4-row groups: 8 words per lane
    __shared__ __align__(128) uint8_t stage_rows[kKlWarps][2][kKlStageW];  // double-buffered staging rows
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t *bm = bitmap[warp];
    const uint32_t bm_s = smem_u32(bm);
    const uint32_t magic = 0xFFFFFFFFu / (4u * (WPL > 0 ? WPL : 1)) + 1u;
    constexpr int WPL2 = WPLQ / 2;  // words per lane of a row pair
    const uint32_t magic2 = 0xFFFFFFFFu / (4u * (WPL2 > 0 ? WPL2 : 1)) + 1u;
    const uint32_t magic4 = 0xFFFFFFFFu / (4u * (WPLQ > 0 ? WPLQ : 1)) + 1u;
    uint32_t nstaged = 0;  // rows this warp has stored by TMA (buffer nstaged & 1 next)
    uint64_t pol;
    if (row_ef) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    else asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
    const uint64_t T = (uint64_t)n * H;
    const uint64_t NW = (uint64_t)gridDim.x * kKlWarps, gw = (uint64_t)blockIdx.x * kKlWarps + warp;
    const uint64_t g0 = gw * T / NW, g1 = (gw + 1) * T / NW;
    const uint64_t P = kLabelHeader + ((4ull * (H + 1) + 15) & ~15ull);
    const bool vec16 = (W & 15) == 0;  // rows start 16-B aligned in dst
    // Row window: lane k holds row (wbase + k)'s payload address, byte count and
    // first word (mode, nrun), loaded and validated by all lanes at once every
    // 32 rows, so a row's dependent loads (header -> directory -> row header)
    // are paid once per 32 rows instead of per row.
    uint64_t wbase = 0, w_p = 0;
    uint32_t w_bytes = 0, w_hdr = 0, w_ok = 0;
    auto load_window = [&](uint64_t wb) {
        wbase = wb;
        const uint64_t gk = wb + lane;
        w_ok = 0;
        if (gk < g1) {
            const uint64_t sk = gk / H;
            const uint32_t yk = (uint32_t)(gk - sk * H);
            const uint8_t *b = static_cast<const uint8_t *>(src[sk]);
            uint64_t total = label_header_ok(b, src_bytes ? src_bytes[sk] : ~0ull, SPP_LABEL_MASK, H, W);
            if (total && P > total) total = 0;
            if (total) {
                const uint32_t *dir = reinterpret_cast<const uint32_t *>(b + kLabelHeader);
                const uint32_t da = __ldg(dir + yk), db = __ldg(dir + yk + 1);
                if (db >= da && ((da | db) & 15u) == 0 && (uint64_t)db <= total - P && db - da >= 16) {
                    w_p = reinterpret_cast<uint64_t>(b + P + da);
                    w_bytes = db - da;
                    w_hdr = __ldg(reinterpret_cast<const uint32_t *>(w_p));
                    w_ok = 1;
                }
            }
            if (!w_ok) report(status, SPP_ERR_CORRUPT, (int64_t)sk);
        }
    };
    for (uint64_t g = g0; g < g1; g++) {
        if constexpr (WPLQ > 0) {
            // G consecutive RUN rows of <= 32/G runs each (4, else 2): one 32/G-lane segment
            // per row, one bulk store per group.  The group's staging buffer is the warp's
            // whole staging area, so every staged store first waits for the previous one
            // to have read shared memory (bulk_wait_read_all below).
            auto group_ok = [&](int G, uint32_t maxruns, int kk) {
                const int src = kk + min(lane, G - 1);  // lanes >= G repeat row G - 1
                const uint32_t hr = __shfl_sync(0xffffffffu, w_hdr, src);
                const bool good = __shfl_sync(0xffffffffu, w_ok, src) && (hr & 0xFFu) == 1u && (hr >> 16) >= 1 &&
                                  (hr >> 16) <= maxruns;
                return __all_sync(0xffffffffu, good) != 0;
            };
            auto run_group = [&](auto gtag, int kk) {
                constexpr int G = decltype(gtag)::value;
                constexpr uint32_t LPR = 32 / G;
                const int kh = kk + lane / (int)LPR;
                const uint8_t *p = reinterpret_cast<const uint8_t *>(__shfl_sync(0xffffffffu, w_p, kh));
                const uint32_t bytes = __shfl_sync(0xffffffffu, w_bytes, kh);
                const uint32_t nrun = __shfl_sync(0xffffffffu, w_hdr, kh) >> 16;
                uint8_t *stage = &stage_rows[warp][0][0];
                if (lane == 0) bulk_wait_read_all();  // the previous store has read the staging area
                __syncwarp();
                constexpr int WG = G == 4 ? (WPLQ > 0 ? WPLQ : 2) : (WPL2 > 0 ? WPL2 : 2);
                const uint32_t okm = kl_run_group_staged<G, WG>(p, bytes, nrun, W, G == 4 ? magic4 : magic2, bm,
                                                                bm_s, stage, smem_u32(stage), dst + g * (uint64_t)W,
                                                                lane, pol);
                if (lane == 0)
                    for (int r = 0; r < G; r++)
                        if (!((okm >> (LPR * r)) & 1u)) report(status, SPP_ERR_CORRUPT, (int64_t)((g + r) / H));
            };
            if (SPP_KL_QUADS && g + 3 < g1) {
                if (g == g0 || g + 3 >= wbase + kWarp) load_window(g);
                const int kk = (int)(g - wbase);
                if (group_ok(4, 8, kk)) {
                    run_group(std::integral_constant<int, 4>{}, kk);
                    g += 3;
                    continue;
                }
            }
            if (g + 1 < g1) {
                if (g == g0 || g + 1 >= wbase + kWarp) load_window(g);
                const int kk = (int)(g - wbase);
                if (group_ok(2, kKlPairRuns, kk)) {
                    run_group(std::integral_constant<int, 2>{}, kk);
                    g += 1;
                    continue;
                }
            }
        }
        if (g == g0 || g >= wbase + kWarp) load_window(g);
        const int kk = (int)(g - wbase);
        bool ok = __shfl_sync(0xffffffffu, w_ok, kk) != 0;
        if (!ok) continue;  // reported by the window load
        const uint8_t *p = reinterpret_cast<const uint8_t *>(__shfl_sync(0xffffffffu, w_p, kk));
        const uint64_t bytes = __shfl_sync(0xffffffffu, w_bytes, kk);
        const uint32_t hdr = __shfl_sync(0xffffffffu, w_hdr, kk);
        uint8_t *row = dst + g * (uint64_t)W;
        const uint32_t mode = hdr & 0xFFu;
        if (ok && mode == 0) {  // verbatim row
            ok = 16ull + W <= bytes;
            if (ok) {
                if (vec16) {
                    const uint4 *s4 = reinterpret_cast<const uint4 *>(p + 16);
                    for (uint32_t k = lane; k < W / 16; k += kWarp) reinterpret_cast<uint4 *>(row)[k] = __ldg(s4 + k);
                } else {
                    for (uint32_t k = lane; k < W; k += kWarp) row[k] = __ldg(p + 16 + k);
                }
            }
        } else if (WPL > 0 && ok && mode == 1 && (hdr >> 16) >= 1 && (hdr >> 16) <= kKlFastRuns) {
            uint8_t *stage = stage_rows[warp][WPLQ > 0 ? 0 : nstaged & 1];
            if (lane == 0) {  // the store that last used this buffer has read it
                if constexpr (WPLQ > 0) bulk_wait_read_all();  // (a group store may cover both buffers)
                else bulk_wait_read_1();
            }
            __syncwarp();
            ok = kl_run_row_staged<(WPL > 0 ? WPL : 1)>(p, (uint32_t)bytes, hdr >> 16, W, magic, bm, bm_s, stage, smem_u32(stage),
                                        row, lane, pol);
            nstaged += ok;
        } else if (ok && mode == 1) {  // maximal runs
            const uint32_t nrun = hdr >> 16;
            ok = nrun >= 1 && nrun <= W && 4ull + 3ull * nrun <= bytes;
            const uint16_t *lens = reinterpret_cast<const uint16_t *>(p + 4);
            const uint8_t *vals = p + 4 + 2 * nrun;
            // positions in chunks of kKlChunk: one pass over the runs sets the
            // chunk's run starts in the warp's bitmap (and validates the lengths);
            // lane l then owns the 32-position windows l, l + 32, ... of the chunk
            for (uint32_t c0 = 0; ok && c0 < W; c0 += kKlChunk) {
                for (uint32_t k = lane; k < kKlChunk / 32; k += kWarp) bm[k] = 0;
                __syncwarp();
                uint32_t before = 0, run_end = 0;
                bool bad = false;
                for (uint32_t r0 = 0; r0 < nrun && (c0 == 0 || run_end <= c0 + kKlChunk); r0 += kWarp) {
                    const uint32_t r = r0 + lane;
                    const uint32_t len = r < nrun ? __ldg(lens + r) : 0u;
                    bad |= r < nrun && len == 0;
                    const uint32_t incl = scan_u32(len);
                    const uint32_t st = run_end + incl - len;
                    if (r < nrun && st >= c0 && st < c0 + kKlChunk) atomicOr(&bm[(st - c0) >> 5], 1u << (st & 31));
                    before += __popc(__ballot_sync(0xffffffffu, r < nrun && st < c0));
                    run_end += __shfl_sync(0xffffffffu, incl, 31);
                }
                if (c0 == 0) ok = !__any_sync(0xffffffffu, bad) && run_end == W;  // the first pass saw every run
                __syncwarp();
                if (!ok) break;
                uint32_t carry = before;
                for (uint32_t w0 = 0; w0 < kKlChunk / 32 && c0 + 32 * w0 < W; w0 += kWarp) {
                    const uint32_t word = bm[w0 + lane];
                    const uint32_t c = __popc(word);
                    const uint32_t incl = scan_u32(c);
                    const uint32_t base = carry + incl - c;  // run starts before this lane's window
                    carry += __shfl_sync(0xffffffffu, incl, 31);
                    const uint32_t p0 = c0 + 32 * (w0 + lane);
                    if (p0 < W) {
                        // the run of p0, then one fill per run starting inside the window
                        // (a mask row has a handful of runs: usually none starts here)
                        uint32_t idx = base + (word & 1u) - 1;
                        uint32_t v = __ldg(vals + min(idx, nrun - 1)) * 0x01010101u;
                        uint32_t out[8];
#pragma unroll
                        for (int k = 0; k < 8; k++) out[k] = v;
                        for (uint32_t w = word & ~1u; w; w &= w - 1) {
                            const uint32_t j = __ffs(w) - 1;  // a run starts at p0 + j: bytes j.. take its value
                            idx++;
                            v = __ldg(vals + min(idx, nrun - 1)) * 0x01010101u;
#pragma unroll
                            for (int k = 0; k < 8; k++) {
                                const int sh = (int)j - 4 * k;  // bytes 4k..4k+3 at or after j
                                const uint32_t m = sh <= 0 ? 0xFFFFFFFFu : (sh >= 4 ? 0u : 0xFFFFFFFFu << (8 * sh));
                                out[k] = (out[k] & ~m) | (v & m);
                            }
                        }
                        if (vec16 && p0 + 32 <= W) {
                            reinterpret_cast<uint4 *>(row + p0)[0] = make_uint4(out[0], out[1], out[2], out[3]);
                            reinterpret_cast<uint4 *>(row + p0)[1] = make_uint4(out[4], out[5], out[6], out[7]);
                        } else {
#pragma unroll
                            for (int k = 0; k < 8; k++)
#pragma unroll
                                for (int bb = 0; bb < 4; bb++)
                                    if (p0 + 4 * k + bb < W) row[p0 + 4 * k + bb] = (uint8_t)(out[k] >> (8 * bb));
                        }
                    }
                }
                __syncwarp();
            }
        } else {
            ok = false;
        }
        if (!ok && lane == 0) report(status, SPP_ERR_CORRUPT, (int64_t)(g / H));
    }
    if (lane == 0) bulk_wait_all();  // shared memory must outlive the last row stores
}

__global__ void kl_decode_vec(const void *const *__restrict__ src, const uint64_t *__restrict__ src_bytes, int n,
                              uint32_t W, float *__restrict__ dst, uint32_t *__restrict__ status) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (uint64_t)n * W) return;
    const uint64_t s = i / W;
    const uint32_t k = (uint32_t)(i - s * W);
    const uint8_t *b = static_cast<const uint8_t *>(src[s]);
    const uint64_t total = label_header_ok(b, src_bytes ? src_bytes[s] : ~0ull, SPP_LABEL_VECTOR, 1, W);
    if (!total || total < kLabelHeader + 4ull * W) {
        if (k == 0) report(status, SPP_ERR_CORRUPT, (int64_t)s);
        return;
    }
    dst[i] = __ldg(reinterpret_cast<const float *>(b + kLabelHeader) + k);
}

}  // namespace

spp_status labels_decode(int kind, const void *const *d_src, const uint64_t *src_bytes, int n, void *d_dst,
                         int H, int W, uint32_t *status, cudaStream_t stream) {
    DeviceProps dp;
    spp_status st = current_device_props(&dp);
    if (st != SPP_OK) return st;
    if (kind == SPP_LABEL_VECTOR) {
        const uint64_t total = (uint64_t)n * W;
        kl_decode_vec<<<(unsigned)((total + 255) / 256), 256, 0, stream>>>(d_src, src_bytes, n, (uint32_t)W,
                                                                           static_cast<float *>(d_dst), status);
    } else {
        const uint64_t rows = (uint64_t)n * H;
        // staged rows leave by TMA bulk store: 16-B aligned rows of a multiple of 16 bytes
        const bool staged = (W % 16) == 0 && W <= (int)kKlFastW && (reinterpret_cast<uintptr_t>(d_dst) & 15) == 0;
        const int wpl = staged ? (W / 4 + kWarp - 1) / kWarp : 0;
        // row groups (4 or 2 rows per warp, one bulk store per group): W % 128 == 0, 4W <= 2 kKlStageW
        const bool groups = staged && W % 128 == 0 && 4 * W <= 2 * (int)kKlStageW;
        void (*kern)(const void *const *, const uint64_t *, int, uint32_t, uint32_t, uint8_t *, uint32_t *,
                     uint32_t) = nullptr;
        switch (groups ? 100 + wpl : wpl) {
#define SPP_KL_CASE(k) \
    case k: kern = kl_decode_mask<k, 0>; break;
#define SPP_KL_GROUP(k) \
    case 100 + k: kern = kl_decode_mask<k, 4 * k>; break;
            SPP_KL_CASE(0) SPP_KL_CASE(1) SPP_KL_CASE(2) SPP_KL_CASE(3) SPP_KL_CASE(4) SPP_KL_CASE(5) SPP_KL_CASE(6)
            SPP_KL_CASE(7) SPP_KL_CASE(8) SPP_KL_CASE(9) SPP_KL_CASE(10) SPP_KL_CASE(11) SPP_KL_CASE(12)
            SPP_KL_CASE(13) SPP_KL_CASE(14) SPP_KL_CASE(15) SPP_KL_CASE(16)
            SPP_KL_GROUP(1) SPP_KL_GROUP(2) SPP_KL_GROUP(3) SPP_KL_GROUP(4) SPP_KL_GROUP(5) SPP_KL_GROUP(6)
            SPP_KL_GROUP(7) SPP_KL_GROUP(8) SPP_KL_GROUP(9)
#undef SPP_KL_CASE
#undef SPP_KL_GROUP
            default: return SPP_ERR_INVALID_ARG;
        }
        // 8 CTAs per SM: about two waves of the pair instance (4 resident per SM); measured
        // 3% faster than one resident wave (profiles/r02b2_*): later CTAs fill SMs whose
        // first CTAs finished early
        const uint64_t ctas = std::min<uint64_t>((uint64_t)dp.sms * 8, (rows + kKlWarps - 1) / kKlWarps);
        const unsigned grid = (unsigned)std::max<uint64_t>(1, ctas);
        const uint32_t row_ef = SPP_KL_ROW_EF && rows * (uint64_t)W > kRowEfBytes;
        kern<<<grid, kKlWarps * kWarp, 0, stream>>>(d_src, src_bytes, n, (uint32_t)H, (uint32_t)W,
                                                    static_cast<uint8_t *>(d_dst), status, row_ef);
    }
    return cudaGetLastError() == cudaSuccess ? SPP_OK : SPP_ERR_CUDA;
}

}  // namespace spp
