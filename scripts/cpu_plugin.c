/* cpu_plugin.c — an optimised CPU decoder for the two formats: the paper's
 * CPU plugin variant ("two variants ... one for the CPU and
 * another for the GPU ... on the CPU we assign different samples to different
 * threads"), kept as a COMPARISON POINT.  It is not part of
 * the product (libspp has no CPU decode path) and shares no code with it or
 * with oracle/; tests/test_cpu_plugin.py checks it bit for bit against the
 * oracle, scripts/cpu_plugin.py times it against the GPU.
 *
 * One call decodes one sample (FORMAT.md 1.2 / 2.3) into fp16 training
 * layout; callers run one sample per thread.  Build: gcc -O3 -march=native
 * -ffp-contract=off -fno-fast-math -shared -fPIC (no FTZ/DAZ). */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define RD(T, p) (*(const T *)(const void *)(p))

static inline uint16_t h16(float f) {
    _Float16 h = (_Float16)f; /* IEEE RNE from binary32 (F16C with -march=native) */
    uint16_t u;
    memcpy(&u, &h, 2);
    return u;
}

/* CosmoFlow: out[c][v] = RNE16(RN32(log1p(U[LUT[key[v]].c]))), CDHW.  Returns 0
 * or -1 on a malformed stream (light checks: this is a timing comparison). */
int cpu_cosmo_decode_f16(const uint8_t *s, size_t size, uint16_t *out) {
    if (size < 64 || RD(uint32_t, s) != 0x43505053u) return -1;
    const int D = RD(uint16_t, s + 10), H = RD(uint16_t, s + 12), W = RD(uint16_t, s + 14);
    const uint32_t nU = RD(uint32_t, s + 16), T = RD(uint32_t, s + 20);
    const uint64_t U_off = RD(uint64_t, s + 24), slab_off = RD(uint64_t, s + 32);
    const uint64_t plane = (uint64_t)H * W, N = (uint64_t)D * plane;
    if (nU == 0 || nU > 32768 || U_off + 2ull * nU > size || slab_off + 32ull * T > size) return -1;
    uint16_t hU[32768];
    for (uint32_t i = 0; i < nU; i++) hU[i] = h16((float)log1p((double)RD(int16_t, s + U_off + 2ull * i)));
    uint64_t *tup = NULL; /* per slab: 4 fp16 outputs of each group */
    size_t tup_cap = 0;
    for (uint32_t t = 0; t < T; t++) {
        const uint8_t *sl = s + slab_off + 32ull * t;
        const uint32_t z0 = RD(uint32_t, sl), z1 = RD(uint32_t, sl + 4), G = RD(uint32_t, sl + 8);
        const int kw = sl[12];
        const uint64_t lut_off = RD(uint64_t, sl + 16), keys_off = RD(uint64_t, sl + 24);
        const uint64_t v0 = (uint64_t)z0 * plane, Nt = (uint64_t)(z1 - z0) * plane;
        uint16_t *o0 = out + v0, *o1 = out + N + v0, *o2 = out + 2 * N + v0, *o3 = out + 3 * N + v0;
        if (kw == 8) {
            const uint16_t *r = (const uint16_t *)(const void *)(s + keys_off);
            for (uint64_t v = 0; v < Nt; v++) o0[v] = hU[r[v]];
            for (uint64_t v = 0; v < Nt; v++) o1[v] = hU[r[Nt + v]];
            for (uint64_t v = 0; v < Nt; v++) o2[v] = hU[r[2 * Nt + v]];
            for (uint64_t v = 0; v < Nt; v++) o3[v] = hU[r[3 * Nt + v]];
            continue;
        }
        if (G > tup_cap) {
            free(tup);
            tup_cap = G;
            tup = (uint64_t *)malloc(8 * (size_t)G);
        }
        const uint16_t *lut = (const uint16_t *)(const void *)(s + lut_off);
        for (uint32_t g = 0; g < G; g++)
            tup[g] = (uint64_t)hU[lut[4 * g]] | (uint64_t)hU[lut[4 * g + 1]] << 16 |
                     (uint64_t)hU[lut[4 * g + 2]] << 32 | (uint64_t)hU[lut[4 * g + 3]] << 48;
        if (kw == 0) {
            const uint64_t e = tup[0];
            for (uint64_t v = 0; v < Nt; v++) {
                o0[v] = (uint16_t)e; o1[v] = (uint16_t)(e >> 16); o2[v] = (uint16_t)(e >> 32); o3[v] = (uint16_t)(e >> 48);
            }
        } else if (kw == 1) {
            const uint8_t *k = s + keys_off;
            for (uint64_t v = 0; v < Nt; v++) {
                const uint64_t e = tup[k[v]];
                o0[v] = (uint16_t)e; o1[v] = (uint16_t)(e >> 16); o2[v] = (uint16_t)(e >> 32); o3[v] = (uint16_t)(e >> 48);
            }
        } else {
            const uint16_t *k = (const uint16_t *)(const void *)(s + keys_off);
            for (uint64_t v = 0; v < Nt; v++) {
                const uint64_t e = tup[k[v]];
                o0[v] = (uint16_t)e; o1[v] = (uint16_t)(e >> 16); o2[v] = (uint16_t)(e >> 32); o3[v] = (uint16_t)(e >> 48);
            }
        }
    }
    free(tup);
    return 0;
}

/* DeepCAM: out[c][y][x] = RNE16(RN32(RN32(x̂ - shift[c]) * scale[c])), CHW,
 * x̂ per FORMAT.md 2.3 (exact integer prefix, one fp32 rounding). */
int cpu_deepcam_decode_f16(const uint8_t *s, size_t size, const float *shift, const float *scale, uint16_t *out) {
    if (size < 64 || RD(uint32_t, s) != 0x44505053u) return -1;
    const int C = RD(uint16_t, s + 8), H = RD(uint16_t, s + 10), W = RD(uint16_t, s + 12);
    const uint64_t dir_off = RD(uint64_t, s + 24), payload_off = RD(uint64_t, s + 32);
    const uint32_t *dir = (const uint32_t *)(const void *)(s + dir_off);
    int code[256];
    for (int b = 0; b < 256; b++) {
        const int E = (b >> 4) & 7, M = b & 15, m = E == 0 ? M : (16 + M) << (E - 1);
        code[b] = (b & 0x80) ? -m : m;
    }
    float *xh = (float *)malloc(4 * (size_t)W);
    if (!xh) return -1;
    for (int c = 0; c < C; c++) {
        const float sh = shift ? shift[c] : 0.0f, sc = scale ? scale[c] : 1.0f;
        for (int y = 0; y < H; y++) {
            const uint64_t l = (uint64_t)c * H + y;
            const uint8_t *p = s + payload_off + dir[l];
            if (p[0] == 0) {
                memcpy(xh, p + 16, 4 * (size_t)W);
            } else if (p[0] == 2) {  /* RAW16 (FORMAT.md 2.6) */
                for (int x = 0; x < W; x++) {
                    _Float16 h;
                    memcpy(&h, p + 16 + 2 * (size_t)x, 2);
                    xh[x] = (float)h;
                }
            } else {
                const int nseg = RD(uint16_t, p + 2);
                const uint8_t *desc = p + 4, *heads = p + 4 + 4 * nseg, *d = p + 4 + 8 * nseg;
                int pos = 0;
                for (int k = 0; k < nseg; k++) {
                    const int len = RD(uint16_t, desc + 4 * k), kind = desc[4 * k + 2];
                    const float h = RD(float, heads + 4 * k);
                    if (kind == 0) {
                        for (int j = 0; j < len; j++) xh[pos + j] = h;
                    } else {
                        const float unit = ldexpf(1.0f, (int)desc[4 * k + 3] - 150);
                        int32_t S = 0;
                        xh[pos] = h;
                        for (int j = 1; j < len; j++) {
                            S += code[*d++];
                            xh[pos + j] = h + (float)S * unit;
                        }
                    }
                    pos += len;
                }
            }
            uint16_t *o = out + l * (uint64_t)W;
            for (int x = 0; x < W; x++) o[x] = h16((xh[x] - sh) * sc);
        }
    }
    free(xh);
    return 0;
}
