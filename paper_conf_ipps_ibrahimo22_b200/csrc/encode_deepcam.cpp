// encode_deepcam.cpp — host DeepCAM differential line encoder (step b.1,
// PAPER.md P:32), FORMAT.md 2.4.
//
// PAPER.md §V.A (Fig. 4): each line along x is split into
// segments; a segment has a pivot/head value and 8-bit differences (1 sign, 3
// exponent bits relative to the segment's minimum exponent, 4 mantissa bits).
// Lines with abrupt transitions or too many segments stay uncompressed (RAW);
// runs of identical values use a special encoding (REPEAT); the encoder picks
// whichever is smaller ("best space-saving").  Closed-loop: each difference is
// taken against the value the decoder will reconstruct, so errors do not
// accumulate along the line.
#include <math.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <cmath>
#include <utility>
#include <cstdlib>
#include <thread>
#include <vector>

#include "spp.h"
#include "spp_format.h"

namespace {

using namespace spp::deepcam;
using spp::round_up16;

// magnitude of the 7-bit exponent|mantissa field (FORMAT.md 2.2), ascending in b
struct CodeTable {
    int mag[128];
    CodeTable() {
        for (int b = 0; b < 128; b++) {
            int E = b >> 4, M = b & 15;
            mag[b] = E == 0 ? M : (16 + M) << (E - 1);
        }
    }
    // byte whose value is nearest to t; ties toward the smaller magnitude
    inline int quantise(double t, int *value) const {
        double a = fabs(t);
        int lo = 0, hi = 127;  // largest b with mag[b] <= a
        while (lo < hi) {
            int mid = (lo + hi + 1) >> 1;
            if (mag[mid] <= a) lo = mid; else hi = mid - 1;
        }
        int b = lo;
        if (b < 127 && (mag[b + 1] - a) < (a - mag[b])) b++;
        if (mag[b] == 0) { *value = 0; return 0; }
        *value = t < 0 ? -mag[b] : mag[b];
        return t < 0 ? (b | 0x80) : b;
    }
};
const CodeTable kCodes;

inline uint32_t fbits(float f) { uint32_t u; memcpy(&u, &f, 4); return u; }

// exact ceil(log2(q)), q > 0
inline int ceil_log2(double q) {
    int e;
    double f = frexp(q, &e);
    return f == 0.5 ? e - 1 : e;
}

struct Seg { uint16_t len; uint8_t kind, emin_b; float head; };

// segment alignment (FORMAT.md 2.4): the GPU decodes 36 (W = 1152, one line per
// warp pass) or 8 positions per lane; aligned segment starts keep every lane
// inside one segment
inline int alignment_for(int W) { return W == 1152 ? 36 : (W % 8 == 0 ? 8 : 1); }

struct LineEncoder {
    int W, A;
    int lookahead, repeat_min;  // FORMAT.md 2.4 policy knobs (defaults 64, 16)
    double tau = 0.0;           // FORMAT.md 2.8 REPEAT tolerance of the line's channel (0: bit-identical runs)
    const float *xl = nullptr;  // the line being encoded (tolerant runs scan it)
    std::vector<int> run;
    std::vector<Seg> segs;
    std::vector<uint8_t> deltas;
    LineEncoder(int w, int a, int la, int rm)
        : W(w), A(a), lookahead(la), repeat_min(rm), run(w), segs(), deltas() {
        segs.reserve(w);
        deltas.reserve(w);
    }

    // REPEAT candidate at i, cut at the range end E (E = W for a whole line):
    // bit-identical values (tau = 0, FORMAT.md 2.4) or values within tau of x[i]
    // ("all neighbouring values are similar"; FORMAT.md 2.8)
    int rep(int i, int E) const {
        int r;
        if (tau == 0.0) {
            r = run[i] < E - i ? run[i] : E - i;
        } else {
            const double h = xl[i];
            r = 1;
            while (i + r < E && fabs((double)xl[i + r] - h) <= tau) r++;
        }
        return i + r == E ? r : (r / A) * A;
    }

    // SEG payload size, or -1 when no aligned segmentation exists (RAW)
    int64_t encode(const float *x) {
        segs.clear();
        deltas.clear();
        xl = x;
        run[W - 1] = 1;
        for (int i = W - 2; i >= 0; i--) run[i] = fbits(x[i]) == fbits(x[i + 1]) ? run[i + 1] + 1 : 1;
        if (!encode_range(x, 0, W)) return -1;
        return (int64_t)round_up16(4 + 8 * (uint64_t)segs.size() + deltas.size());
    }

    // the FORMAT.md 2.4 greedy policy over positions [i, E), appended to segs /
    // deltas (2.7 re-encodes the ranges between RAW segments); false when no
    // aligned segmentation exists
    bool encode_range(const float *x, int i, const int E) {
        while (i < E) {
            const int rl = rep(i, E);
            if (rl >= repeat_min) {
                segs.push_back(Seg{(uint16_t)rl, kRepeat, 0, x[i]});
                i += rl;
                continue;
            }
            const float h = x[i];
            double m = 0.0;
            const int jend = (i + lookahead < E) ? i + lookahead : E;
            for (int j = i + 1; j < jend; j++) {
                double d = fabs((double)x[j] - (double)x[j - 1]);
                if (d > m) m = d;
            }
            int emin = -149;
            if (m > 0.0) {
                emin = ceil_log2(m / (double)kMaxCode);
                emin = emin < -149 ? -149 : (emin > 96 ? 96 : emin);
            }
            const size_t nd0 = deltas.size();
            int end;
            for (;;) {  // (re)encode the segment starting at i
                deltas.resize(nd0);
                const float unit = ldexpf(1.0f, emin);
                int64_t S = 0;
                float prev = h;
                int j = i + 1;
                bool overflow = false;
                for (; j < E; j++) {
                    if (j % A == 0 && rep(j, E) >= repeat_min) break;
                    double t = ldexp((double)x[j] - (double)prev, -emin);
                    if (fabs(t) > kMaxCode + 0.5) { overflow = true; break; }
                    int k;
                    int b = kCodes.quantise(t, &k);
                    if (llabs(S + k) > kMaxAbsS) { overflow = true; break; }
                    S += k;
                    prev = h + (float)S * unit;                // decoder's x̂_j (fp32, one rounding)
                    deltas.push_back((uint8_t)b);
                }
                if (!overflow) { end = j; break; }
                end = (j / A) * A;
                if (end > i) { deltas.resize(nd0 + (size_t)(end - i - 1)); break; }
                if (emin >= 96) return false;
                emin++;
            }
            segs.push_back(Seg{(uint16_t)(end - i), kDiff, (uint8_t)(emin + kEminBias), h});
            i = end;
        }
        return true;
    }
};

// x̂ of the line just encoded, by the decoder's arithmetic (FORMAT.md 2.3; RAW
// segments of 2.7 decode to their stored values)
void rebuild(const LineEncoder &e, const float *x, std::vector<float> &xh) {
    xh.resize(e.W);
    int pos = 0;
    size_t d = 0;
    for (const Seg &g : e.segs) {
        if (g.kind == kRawSeg) {
            std::copy(x + pos, x + pos + g.len, xh.begin() + pos);
            d += 4 * (size_t)g.len;
        } else if (g.kind == kRepeat) {
            std::fill(xh.begin() + pos, xh.begin() + pos + g.len, g.head);
        } else {
            const float unit = ldexpf(1.0f, (int)g.emin_b - kEminBias);
            int64_t S = 0;
            xh[pos] = g.head;
            for (int j = 1; j < g.len; j++) {
                const uint8_t b = e.deltas[d++];
                const int mag = kCodes.mag[b & 127];
                S += (b & 0x80) ? -mag : mag;
                xh[pos + j] = g.head + (float)S * unit;
            }
        }
        pos += g.len;
    }
}

// Error bounds of a decoded value (binary64 on the binary32 operands):
// relative (FORMAT.md 2.5, "> 10% error", S19: |x̂ - x| > rel |x|)
// and the per-channel absolute bound eps of FORMAT.md 2.8 (|x̂ - x| > eps, eps > 0)
struct Bounds {
    double rel, eps;
    bool use_rel;  // the error budget is on
    bool rel_over(float xh, float x) const { return fabs((double)xh - (double)x) > rel * fabs((double)x); }
    bool abs_over(float xh, float x) const { return eps > 0.0 && fabs((double)xh - (double)x) > eps; }
    // (values over rel, values over eps) of a rebuilt line
    std::pair<int, int> count(const std::vector<float> &xh, const float *x, int W) const {
        int r = 0, a = 0;
        for (int k = 0; k < W; k++) {
            r += rel_over(xh[k], x[k]);
            a += abs_over(xh[k], x[k]);
        }
        return {r, a};
    }
};

// FORMAT.md 2.7: the A-blocks of `e0`'s encoding holding a value over the bounds
// become RAW segments (a run of them, one segment); the ranges between are
// re-encoded by the 2.4 policy, into `e`.  False if no aligned segmentation exists.
bool encode_rawseg(const LineEncoder &e0, const std::vector<float> &xh0, LineEncoder &e, const float *x,
                   const Bounds &bd) {
    const int W = e0.W, A = e0.A;
    e.segs.clear();
    e.deltas.clear();
    e.run = e0.run;
    e.tau = e0.tau;
    e.xl = x;
    const int nb = (W + A - 1) / A;
    auto block_bad = [&](int b) {
        for (int k = b * A; k < W && k < (b + 1) * A; k++)
            if ((bd.use_rel && bd.rel_over(xh0[k], x[k])) || bd.abs_over(xh0[k], x[k])) return true;
        return false;
    };
    int b = 0;
    while (b < nb) {
        const bool bad = block_bad(b);
        int b2 = b + 1;
        while (b2 < nb && block_bad(b2) == bad) b2++;
        const int s0 = b * A, e1 = b2 * A < W ? b2 * A : W;
        if (bad) {
            e.segs.push_back(Seg{(uint16_t)(e1 - s0), kRawSeg, 0, x[s0]});
            const size_t at = e.deltas.size();
            e.deltas.resize(at + 4 * (size_t)(e1 - s0));
            memcpy(e.deltas.data() + at, x + s0, 4 * (size_t)(e1 - s0));
        } else if (!e.encode_range(x, s0, e1)) {
            return false;
        }
        b = b2;
    }
    return true;
}

// binary32 -> binary16, round to nearest even (FORMAT.md 2.6 RAW16 lines)
inline uint16_t f32_to_f16(float f) {
    _Float16 h = (_Float16)f;
    uint16_t u;
    memcpy(&u, &h, 2);
    return u;
}
inline float f16_to_f32(uint16_t u) {
    _Float16 h;
    memcpy(&h, &u, 2);
    return (float)h;
}
// FORMAT.md 2.6 / 2.8: every value finite and its binary16 rounding within the bounds
bool raw16_ok(const float *x, int W, const Bounds &bd) {
    for (int k = 0; k < W; k++) {
        if (!isfinite(x[k])) return false;
        const float h = f16_to_f32(f32_to_f16(x[k]));
        if (!isfinite(h) || bd.rel_over(h, x[k]) || bd.abs_over(h, x[k])) return false;
    }
    return true;
}

inline bool all_finite(const float *x, int W) {
    for (int k = 0; k < W; k++)
        if (!isfinite(x[k])) return false;
    return true;
}

}  // namespace

extern "C" size_t spp_deepcam_max_encoded_size(int C, int H, int W) {
    if (C < 1 || H < 1 || W < 1) return 0;
    uint64_t L = (uint64_t)C * H;
    return (size_t)(spp::kHeaderBytes + round_up16(4 * (L + 1)) + L * round_up16(16 + 4 * (uint64_t)W));
}

extern "C" spp_status spp_encode_deepcam(const float *x, int C, int H, int W, void *dst,
                                         size_t dst_capacity, size_t *encoded_size) {
    return spp_encode_deepcam_ex(x, C, H, W, nullptr, dst, dst_capacity, encoded_size);
}

extern "C" spp_status spp_encode_deepcam_ex(const float *x, int C, int H, int W, const spp_deepcam_params *params,
                                            void *dst, size_t dst_capacity, size_t *encoded_size) {
    if (!x || !encoded_size || C < 1 || H < 1 || W < 1 || C > 65535 || H > 65535 || W > 65535)
        return SPP_ERR_INVALID_ARG;
    const int la = params && params->lookahead ? params->lookahead : kLookahead;
    const int rm = params && params->repeat_min ? params->repeat_min : kRepeatMin;
    const float rel = params && params->rel_err != 0.0f ? params->rel_err : 0.1f;
    const int budget = params ? params->err_budget : 0;
    const int raw16 = params ? params->raw16 : 0;
    const int rawseg = params ? params->raw_segments : 0;
    const float *tol = params ? params->repeat_tol : nullptr;      // FORMAT.md 2.8, fp32[C] or NULL
    const float *abs_err = params ? params->max_abs_err : nullptr;  // FORMAT.md 2.8, fp32[C] or NULL
    if (raw16 != 0 && raw16 != 1) return SPP_ERR_INVALID_ARG;
    if (rawseg != 0 && rawseg != 1) return SPP_ERR_INVALID_ARG;
    const uint64_t raw16_size = round_up16(16 + 2 * (uint64_t)W);
    if (la < 2 || la > 65535 || rm < 2 || rm > 65535) return SPP_ERR_INVALID_ARG;
    if (budget < 0 || !(rel > 0.0f) || !(rel < 1e30f)) return SPP_ERR_INVALID_ARG;
    for (int c = 0; c < C; c++)
        if ((tol && !(tol[c] >= 0.0f && std::isfinite(tol[c]))) || (abs_err && !(abs_err[c] >= 0.0f && std::isfinite(abs_err[c]))))
            return SPP_ERR_INVALID_ARG;
    const uint64_t L = (uint64_t)C * H;
    const uint64_t dir_off = spp::kHeaderBytes;
    const uint64_t payload_off = round_up16(dir_off + 4 * (L + 1));
    const uint64_t raw_size = round_up16(16 + 4 * (uint64_t)W);
    const int A = alignment_for(W);
    // Lines encode independently, so both passes run over contiguous
    // line ranges on host threads (SPP_ENCODE_THREADS, default: the hardware
    // concurrency); the output is identical for any thread count.
    unsigned nthr = std::thread::hardware_concurrency();
    if (const char *e = getenv("SPP_ENCODE_THREADS")) nthr = (unsigned)atoi(e);
    nthr = std::max(1u, std::min<unsigned>(nthr ? nthr : 1u, (unsigned)((L + 63) / 64)));
    auto parallel_lines = [&](auto &&body) {  // body(l0, l1) on [l0, l1)
        if (nthr == 1) {
            body((uint64_t)0, L);
            return;
        }
        std::vector<std::thread> th;
        for (unsigned i = 0; i < nthr; i++)
            th.emplace_back([&, i]() { body(L * i / nthr, L * (i + 1) / nthr); });
        for (auto &t : th) t.join();
    };
    // Per-line choice (FORMAT.md 2.4-2.8): the line mode (0 RAW, 1 SEG in `enc`,
    // 2 RAW16, 3 SEG with RAW segments in `enc3`) and its payload bytes.  A SEG
    // line over the error budget (2.5) or with a value over its channel's absolute
    // bound (2.8) is kept uncompressed: RAW16 (2.6) when its binary16 rounding is
    // within the bounds, or RAW segments (2.7) when smaller and within the bounds.
    struct Work {
        LineEncoder enc, enc3;
        std::vector<float> xh;
    };
    auto choose = [&](Work &w, uint64_t l, const float *xl, uint64_t &sz) -> uint8_t {
        sz = raw_size;
        if (!all_finite(xl, W)) return kModeRaw;
        const int ch = (int)(l / (uint64_t)H);
        const Bounds bd{(double)rel, abs_err ? (double)abs_err[ch] : 0.0, budget > 0};
        w.enc.tau = tol ? (double)tol[ch] : 0.0;
        const int64_t seg = w.enc.encode(xl);
        if (seg >= 0 && (bd.use_rel || bd.eps > 0.0)) {
            rebuild(w.enc, xl, w.xh);
            const auto [nrel, nabs] = bd.count(w.xh, xl, W);
            if ((bd.use_rel && nrel >= budget) || nabs > 0) {
                uint8_t mode = kModeRaw;
                if (raw16 && raw16_ok(xl, W, bd)) { mode = kModeRaw16; sz = raw16_size; }
                if (rawseg && encode_rawseg(w.enc, w.xh, w.enc3, xl, bd)) {
                    const uint64_t s3 = round_up16(4 + 8 * (uint64_t)w.enc3.segs.size() + w.enc3.deltas.size());
                    if (s3 < sz) {
                        std::vector<float> xh3;
                        rebuild(w.enc3, xl, xh3);
                        const auto [r3, a3] = bd.count(xh3, xl, W);
                        if ((!bd.use_rel || r3 < budget) && a3 == 0) { mode = kModeSegRaw; sz = s3; }
                    }
                }
                return mode;
            }
        }
        if (seg >= 0 && (uint64_t)seg < raw_size) { sz = (uint64_t)seg; return kModeSeg; }
        return kModeRaw;
    };
    // pass 1: per-line mode and size
    std::vector<uint8_t> mode(L);
    std::vector<uint32_t> dir(L + 1);
    std::vector<uint64_t> line_size(L);
    parallel_lines([&](uint64_t l0, uint64_t l1) {
        Work w{LineEncoder(W, A, la, rm), LineEncoder(W, A, la, rm), {}};
        for (uint64_t l = l0; l < l1; l++) mode[l] = choose(w, l, x + l * (uint64_t)W, line_size[l]);
    });
    uint64_t cur = 0;
    for (uint64_t l = 0; l < L; l++) {
        if (cur > 0xFFFFFFFFull) return SPP_ERR_UNSUPPORTED;
        dir[l] = (uint32_t)cur;
        cur += line_size[l];
    }
    if (cur > 0xFFFFFFFFull) return SPP_ERR_UNSUPPORTED;
    dir[L] = (uint32_t)cur;
    const uint64_t total = payload_off + cur;
    *encoded_size = (size_t)total;
    if (!dst || dst_capacity < total) return SPP_ERR_BUFFER_TOO_SMALL;
    uint8_t *out = (uint8_t *)dst;
    memset(out, 0, (size_t)total);
    uint32_t u32;
    uint16_t u16;
    u32 = spp::kDeepcamMagic; memcpy(out, &u32, 4);
    u16 = spp::kVersion; memcpy(out + 4, &u16, 2);
    // flags bit 0 (FORMAT.md 2.1): the stream holds RAW16 / mode-3 lines (2.6 / 2.7)
    u16 = std::any_of(mode.begin(), mode.end(), [](uint8_t m) { return m == kModeRaw16 || m == kModeSegRaw; }) ? 1 : 0;
    memcpy(out + 6, &u16, 2);
    u16 = (uint16_t)C; memcpy(out + kC, &u16, 2);
    u16 = (uint16_t)H; memcpy(out + kH, &u16, 2);
    u16 = (uint16_t)W; memcpy(out + kW, &u16, 2);
    u16 = (uint16_t)A; memcpy(out + kAlign, &u16, 2);
    u32 = (uint32_t)L; memcpy(out + kL, &u32, 4);
    memcpy(out + kDirOff, &dir_off, 8);
    memcpy(out + kPayloadOff, &payload_off, 8);
    memcpy(out + kTotal, &total, 8);
    memcpy(out + dir_off, dir.data(), 4 * (L + 1));
    // pass 2: payloads (the choice is deterministic: recomputed per line)
    parallel_lines([&](uint64_t l0, uint64_t l1) {
        Work w{LineEncoder(W, A, la, rm), LineEncoder(W, A, la, rm), {}};
        for (uint64_t l = l0; l < l1; l++) {
            const float *xl = x + l * (uint64_t)W;
            uint8_t *p = out + payload_off + dir[l];
            p[0] = mode[l];
            if (mode[l] == kModeRaw) {
                memcpy(p + 16, xl, 4 * (size_t)W);
                continue;
            }
            if (mode[l] == kModeRaw16) {
                for (int k = 0; k < W; k++) {
                    const uint16_t h = f32_to_f16(xl[k]);
                    memcpy(p + 16 + 2 * (size_t)k, &h, 2);
                }
                continue;
            }
            uint64_t sz;
            choose(w, l, xl, sz);
            const LineEncoder &e = mode[l] == kModeSegRaw ? w.enc3 : w.enc;
            const uint16_t nseg = (uint16_t)e.segs.size();
            memcpy(p + 2, &nseg, 2);
            for (int s = 0; s < nseg; s++) {
                const Seg &g = e.segs[s];
                memcpy(p + 4 + 4 * s, &g.len, 2);
                p[4 + 4 * s + 2] = g.kind;
                p[4 + 4 * s + 3] = g.emin_b;
                memcpy(p + 4 + 4 * (size_t)nseg + 4 * s, &g.head, 4);
            }
            memcpy(p + 4 + 8 * (size_t)nseg, e.deltas.data(), e.deltas.size());
        }
    });
    return SPP_OK;
}
