// encode_labels.cpp — host label encoders (step b.1) for the
// lossless label coding of P:175 ("For both applications, we use lossless
// compression of the labels"), FORMAT.md 3.
//
// DeepCAM: per-pixel class masks (P:56 semantic segmentation).  Each row is
// its list of maximal runs of one class (a row of 1152 pixels with a few
// cyclones and rivers has a handful of runs), or verbatim bytes when the run
// list is not smaller.  Rows are independent, like DeepCAM data lines.
// CosmoFlow: the four cosmological parameters, kept as binary32.
#include <stdint.h>
#include <string.h>

#include <vector>

#include "spp.h"
#include "spp_format.h"

namespace {

using spp::round_up16;

constexpr uint32_t kLabelMagic = 0x4C505053u;  // "SPPL"

// bytes of the row's run list (mode 1) and the run count
inline uint64_t run_row_bytes(const uint8_t *r, int W, uint32_t *nrun) {
    uint32_t n = 1;
    for (int x = 1; x < W; x++) n += r[x] != r[x - 1];
    *nrun = n;
    return round_up16(4 + 3 * (uint64_t)n);
}

void put16(uint8_t *p, uint16_t v) { memcpy(p, &v, 2); }
void put32(uint8_t *p, uint32_t v) { memcpy(p, &v, 4); }
void put64(uint8_t *p, uint64_t v) { memcpy(p, &v, 8); }

void write_header(uint8_t *o, uint16_t kind, int H, int W, uint64_t total) {
    put32(o, kLabelMagic);
    put16(o + 4, spp::kVersion);
    put16(o + 6, kind);
    put16(o + 8, (uint16_t)H);
    put16(o + 10, (uint16_t)W);
    put64(o + 16, total);
}

}  // namespace

extern "C" size_t spp_label_max_encoded_size(int kind, int H, int W) {
    if (H < 1 || W < 1) return 0;
    if (kind == SPP_LABEL_VECTOR) return (size_t)round_up16(32 + 4 * (uint64_t)W);
    if (kind != SPP_LABEL_MASK) return 0;
    return (size_t)(32 + round_up16(4 * ((uint64_t)H + 1)) + (uint64_t)H * round_up16(16 + (uint64_t)W));
}

extern "C" spp_status spp_encode_label_mask(const uint8_t *mask, int H, int W, void *dst, size_t dst_capacity,
                                            size_t *encoded_size) {
    if (!mask || !encoded_size || H < 1 || W < 1 || H > 65535 || W > 65535) return SPP_ERR_INVALID_ARG;
    const uint64_t raw_row = round_up16(16 + (uint64_t)W);
    const uint64_t P = 32 + round_up16(4 * ((uint64_t)H + 1));
    std::vector<uint32_t> nrun(H);
    std::vector<uint32_t> dir(H + 1);
    uint64_t cur = 0;
    for (int y = 0; y < H; y++) {
        if (cur > 0xFFFFFFFFull) return SPP_ERR_UNSUPPORTED;
        dir[y] = (uint32_t)cur;
        const uint64_t rb = run_row_bytes(mask + (uint64_t)y * W, W, &nrun[y]);
        if (rb >= raw_row) nrun[y] = 0;  // verbatim row (RAW on a tie)
        cur += nrun[y] ? rb : raw_row;
    }
    if (cur > 0xFFFFFFFFull) return SPP_ERR_UNSUPPORTED;
    dir[H] = (uint32_t)cur;
    const uint64_t total = P + cur;
    *encoded_size = (size_t)total;
    if (!dst || dst_capacity < total) return SPP_ERR_BUFFER_TOO_SMALL;
    uint8_t *o = static_cast<uint8_t *>(dst);
    memset(o, 0, (size_t)total);
    write_header(o, SPP_LABEL_MASK, H, W, total);
    memcpy(o + 32, dir.data(), 4 * ((size_t)H + 1));
    for (int y = 0; y < H; y++) {
        const uint8_t *r = mask + (uint64_t)y * W;
        uint8_t *p = o + P + dir[y];
        if (!nrun[y]) {
            p[0] = 0;
            memcpy(p + 16, r, (size_t)W);
            continue;
        }
        p[0] = 1;
        put16(p + 2, (uint16_t)nrun[y]);
        uint8_t *lens = p + 4, *vals = p + 4 + 2 * (size_t)nrun[y];
        uint32_t k = 0;
        int x0 = 0;
        for (int x = 1; x <= W; x++) {
            if (x < W && r[x] == r[x0]) continue;
            put16(lens + 2 * (size_t)k, (uint16_t)(x - x0));
            vals[k++] = r[x0];
            x0 = x;
        }
    }
    return SPP_OK;
}

extern "C" spp_status spp_encode_label_vector(const float *v, int n, void *dst, size_t dst_capacity,
                                              size_t *encoded_size) {
    if (!v || !encoded_size || n < 1 || n > 65535) return SPP_ERR_INVALID_ARG;
    const uint64_t total = round_up16(32 + 4 * (uint64_t)n);
    *encoded_size = (size_t)total;
    if (!dst || dst_capacity < total) return SPP_ERR_BUFFER_TOO_SMALL;
    uint8_t *o = static_cast<uint8_t *>(dst);
    memset(o, 0, (size_t)total);
    write_header(o, SPP_LABEL_VECTOR, 1, n, total);
    memcpy(o + 32, v, 4 * (size_t)n);  // binary32 verbatim (the host is little-endian)
    return SPP_OK;
}
