/*
 * spp_oracle.c — plain, slow, obviously-correct CPU oracle for the hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  The
 * product path (paper_conf_ipps_ibrahimo22_b200/) never calls it and shares
 * no code, header, table or constant generator with it.
 *
 * It follows FORMAT.md (our byte-level reading of PAPER.md) and PAPER.md:
 *   - CosmoFlow: plain definition out = RN(ln(1 + count)) (P:30, P:80, P:100,
 *     lossless per P:175) AND a sequential parser/decoder of the LUT format
 *     (P:98-100), AND the LUT encoder policy (FORMAT.md 1.3).
 *   - DeepCAM: the differential line decoder step by step (Fig. 4
 *     P:90) and the encoder policy (FORMAT.md 2.4).
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math -std=c11 -shared -fPIC
 * (no FMA contraction, no FTZ/DAZ: fp32 subnormals are real here).
 *
 * Parity pins for every function live in tests/test_oracle_pins.py; see
 * DESIGN.md "Oracle and pins".  Return codes: 0 ok, 1 invalid argument,
 * 2 buffer too small, 3 corrupt stream.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_OK 0
#define ORC_EINVAL 1
#define ORC_ESMALL 2
#define ORC_ECORRUPT 3

#define OUT_F16 1
#define OUT_F32 2
#define OUT_I16 3

/* ------------------------------------------------------------------ */
/* little-endian field access (byte by byte: no alignment assumptions) */
static uint16_t rd16(const uint8_t *p) { return (uint16_t)(p[0] | (p[1] << 8)); }
static uint32_t rd32(const uint8_t *p) {
    return (uint32_t)p[0] | ((uint32_t)p[1] << 8) | ((uint32_t)p[2] << 16) | ((uint32_t)p[3] << 24);
}
static uint64_t rd64(const uint8_t *p) { return (uint64_t)rd32(p) | ((uint64_t)rd32(p + 4) << 32); }
static void wr16(uint8_t *p, uint16_t v) { p[0] = (uint8_t)v; p[1] = (uint8_t)(v >> 8); }
static void wr32(uint8_t *p, uint32_t v) { for (int i = 0; i < 4; i++) p[i] = (uint8_t)(v >> (8 * i)); }
static void wr64(uint8_t *p, uint64_t v) { wr32(p, (uint32_t)v); wr32(p + 4, (uint32_t)(v >> 32)); }
static float f32_of_bits(uint32_t u) { float f; memcpy(&f, &u, 4); return f; }
static uint32_t bits_of_f32(float f) { uint32_t u; memcpy(&u, &f, 4); return u; }
static uint64_t up16(uint64_t x) { return (x + 15) & ~(uint64_t)15; }

/* ------------------------------------------------------------------ */
/* IEEE binary32 -> binary16, round to nearest, ties to even.
 * Pinned against numpy's float16 conversion (library routine). */
/* binary16 -> binary32 (exact: every half is a float), FORMAT.md 2.6 */
float orc_f16_to_f32(uint16_t h) {
    int sgn = h >> 15, E = (h >> 10) & 31, M = h & 1023;
    float v;
    if (E == 0) v = ldexpf((float)M, -24);                       /* zero / subnormal */
    else if (E == 31) v = M ? NAN : INFINITY;
    else v = ldexpf((float)(1024 + M), E - 25);
    return sgn ? -v : v;
}

uint16_t orc_f32_to_f16(float f) {
    uint32_t x = bits_of_f32(f);
    uint32_t sign = (x >> 16) & 0x8000u;
    uint32_t exp = (x >> 23) & 0xFFu;
    uint32_t man = x & 0x7FFFFFu;
    if (exp == 0xFF) {                       /* Inf / NaN */
        if (man == 0) return (uint16_t)(sign | 0x7C00u);
        return (uint16_t)(sign | 0x7E00u | (man >> 13));
    }
    int e = (int)exp - 127;                  /* unbiased exponent */
    if (e > 15) return (uint16_t)(sign | 0x7C00u);   /* overflow (rounding handled below for e==15) */
    if (e >= -14) {                          /* normal half */
        uint32_t m = man;                    /* 23 bits -> keep 10 */
        uint32_t keep = m >> 13, rest = m & 0x1FFFu;
        uint32_t h = ((uint32_t)(e + 15) << 10) | keep;
        if (rest > 0x1000u || (rest == 0x1000u && (keep & 1u))) h += 1;   /* may carry into exponent / Inf */
        return (uint16_t)(sign | h);
    }
    /* subnormal half (or zero): value = full_m * 2^(e-23), target unit 2^-24 */
    if (e < -25) return (uint16_t)sign;      /* < 2^-25: rounds to 0 (2^-25 exactly is a tie -> even 0) */
    uint32_t full = (exp == 0) ? man : (man | 0x800000u);
    /* value / 2^-24 = full * 2^(e - 23 + 24) = full * 2^(e + 1) */
    int shift = -(e + 1);                    /* right shift amount, 14..24 */
    uint32_t keep = full >> shift;
    uint32_t rest = full & ((1u << shift) - 1u);
    uint32_t half = 1u << (shift - 1);
    if (rest > half || (rest == half && (keep & 1u))) keep += 1;
    return (uint16_t)(sign | keep);
}

/* ------------------------------------------------------------------ */
/* CosmoFlow transform ("log(count+1)"; reading S1/S2): fp64 log1p then
 * one rounding to fp32.  Pinned exhaustively against mpmath. */
float orc_cosmo_f32(int count) { return (float)log1p((double)count); }

static int emit_cosmo(int16_t count, int transform, int out_kind, void *out, size_t i) {
    if (out_kind == OUT_I16) {
        if (transform) return ORC_EINVAL;
        ((int16_t *)out)[i] = count;
        return ORC_OK;
    }
    float v = transform ? orc_cosmo_f32(count) : (float)count;
    if (out_kind == OUT_F32) ((float *)out)[i] = v;
    else if (out_kind == OUT_F16) ((uint16_t *)out)[i] = orc_f32_to_f16(v);
    else return ORC_EINVAL;
    return ORC_OK;
}

/* Plain definition (lossless codec): out[i] = f(counts[i]). */
int orc_cosmo_direct(const int16_t *counts, int64_t n, int transform, int out_kind, void *out) {
    if (!counts || !out || n < 0) return ORC_EINVAL;
    for (int64_t i = 0; i < n; i++) {
        if (counts[i] < 0) return ORC_EINVAL;
        int rc = emit_cosmo(counts[i], transform, out_kind, out, (size_t)i);
        if (rc) return rc;
    }
    return ORC_OK;
}

/* ---------------- CosmoFlow encoder (FORMAT.md 1.3) ---------------- */
static int cmp_i16(const void *a, const void *b) {
    int x = *(const int16_t *)a, y = *(const int16_t *)b;
    return (x > y) - (x < y);
}
static int cmp_u64(const void *a, const void *b) {
    uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
    return (x > y) - (x < y);
}
typedef struct { uint64_t tup; int64_t freq; } group_t;
static int cmp_group(const void *a, const void *b) {
    const group_t *x = a, *y = b;
    if (x->freq != y->freq) return (x->freq < y->freq) - (x->freq > y->freq);  /* freq descending */
    return (x->tup > y->tup) - (x->tup < y->tup);                              /* tuple ascending */
}
static int64_t find_u64(const uint64_t *arr, int64_t n, uint64_t key) {
    int64_t lo = 0, hi = n - 1;
    while (lo <= hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (arr[mid] == key) return mid;
        if (arr[mid] < key) lo = mid + 1; else hi = mid - 1;
    }
    return -1;
}

typedef struct { int z0, z1; } zrange_t;

static int cmp_i64_desc(const void *a, const void *b) {
    int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
    return (x < y) - (x > y);
}
/* FORMAT.md 1.5: voxels of a slab whose key would be >= 255 (escaped) = all
 * voxels minus those of the 255 most frequent groups; `sorted` holds the
 * slab's tuples in ascending order */
static int64_t escaped_count(const uint64_t *sorted, int64_t Nt, int64_t G) {
    int64_t *f = malloc(8 * (size_t)G), g = -1, top = 0;
    for (int64_t i = 0; i < Nt; i++) {
        if (i == 0 || sorted[i] != sorted[i - 1]) f[++g] = 0;
        f[g]++;
    }
    qsort(f, (size_t)G, 8, cmp_i64_desc);
    for (int64_t k = 0; k < G && k < 255; k++) top += f[k];
    free(f);
    return Nt - top;
}
/* FORMAT.md 1.5 key bytes of an escaped-key slab: eidx, low bytes, escapes */
static uint64_t escaped_bytes(int64_t Nt, int64_t n_esc) {
    uint64_t nb = ((uint64_t)Nt + 255) / 256;
    return up16(4 * (nb + 1)) + up16((uint64_t)Nt) + up16(2 * (uint64_t)n_esc);
}

/* count distinct 4-tuples over planes [z0,z1) */
static int64_t count_groups(const uint64_t *tup, int64_t plane, int z0, int z1, uint64_t *scratch) {
    int64_t n = (int64_t)(z1 - z0) * plane;
    memcpy(scratch, tup + (int64_t)z0 * plane, (size_t)n * 8);
    qsort(scratch, (size_t)n, 8, cmp_u64);
    int64_t g = 0;
    for (int64_t i = 0; i < n; i++) if (i == 0 || scratch[i] != scratch[i - 1]) g++;
    return g;
}

static void split_slabs(const uint64_t *tup, int64_t plane, int z0, int z1, uint64_t *scratch,
                        zrange_t *out, int *nout) {
    int64_t g = count_groups(tup, plane, z0, z1, scratch);
    if (g > 65536 && z1 - z0 > 1) {
        int mid = z0 + (z1 - z0) / 2;
        split_slabs(tup, plane, z0, mid, scratch, out, nout);
        split_slabs(tup, plane, mid, z1, scratch, out, nout);
        return;
    }
    out[*nout].z0 = z0;
    out[*nout].z1 = z1;
    (*nout)++;
}

/* FORMAT.md 1.4 ("localized lookup tables", "multiple lookup
 * tables", P:106 1-byte keys): bytes of [z0,z1) written as one slab — its
 * 32-B table entry plus LUT and keys, or the RAW planes (rules of 1.3). */
static uint64_t slab_bytes(int64_t G, int64_t Nt) {
    int kw = G == 1 ? 0 : (G <= 256 ? 1 : 2);
    if (G > 65536 || 8 * G + kw * Nt >= 8 * Nt) return 32 + up16(8 * (uint64_t)Nt);
    return 32 + up16(8 * (uint64_t)G) + (kw ? up16((uint64_t)kw * (uint64_t)Nt) : 0);
}

/* FORMAT.md 1.4: among the partitions reachable by halving [z0,z1) at
 * z0 + (z1-z0)/2, the one with the fewest bytes; the whole slab is kept unless
 * the halves are strictly smaller.  Appends the slabs in z order. */
static uint64_t split_localized(const uint64_t *tup, int64_t plane, int z0, int z1, uint64_t *scratch,
                                zrange_t *out, int *nout) {
    int64_t g = count_groups(tup, plane, z0, z1, scratch);
    uint64_t whole = slab_bytes(g, (int64_t)(z1 - z0) * plane);
    if (z1 - z0 > 1) {
        int mid = z0 + (z1 - z0) / 2;
        int n0 = *nout;
        uint64_t halves = split_localized(tup, plane, z0, mid, scratch, out, nout);
        halves += split_localized(tup, plane, mid, z1, scratch, out, nout);
        if (halves < whole) return halves;
        *nout = n0;                     /* drop the halves, keep the whole slab */
    }
    out[*nout].z0 = z0;
    out[*nout].z1 = z1;
    (*nout)++;
    return whole;
}

size_t orc_cosmo_max_encoded_size(int D, int H, int W) {
    uint64_t N = (uint64_t)D * H * W;
    /* header + U + slab table + worst case per slab: RAW planes (8 B/voxel) */
    return (size_t)(64 + up16(2 * 32768) + up16(32 * (uint64_t)D) + 8 * N + 16 * (uint64_t)D + 64);
}

int orc_cosmo_encode_ex(const int16_t *counts, int D, int H, int W, int policy, uint8_t *dst, size_t cap,
                        size_t *size);
int orc_cosmo_encode(const int16_t *counts, int D, int H, int W, uint8_t *dst, size_t cap, size_t *size) {
    return orc_cosmo_encode_ex(counts, D, H, W, 0, dst, cap, size);
}

/* FORMAT.md 1.3; policy bit 0: 1.4 localized tables, bit 1: 1.5 escaped keys */
int orc_cosmo_encode_ex(const int16_t *counts, int D, int H, int W, int policy, uint8_t *dst, size_t cap,
                        size_t *size) {
    if (policy < 0 || policy > 3) return ORC_EINVAL;
    const int localize = policy & 1, escape = (policy >> 1) & 1;
    if (!counts || !size || D < 1 || H < 1 || W < 1 || D > 65535 || H > 65535 || W > 65535) return ORC_EINVAL;
    const int C = 4;
    int64_t plane = (int64_t)H * W, N = (int64_t)D * plane;
    for (int64_t i = 0; i < C * N; i++) if (counts[i] < 0) return ORC_EINVAL;
    /* 1. unique values */
    int16_t *U = malloc((size_t)(C * N) * 2);
    memcpy(U, counts, (size_t)(C * N) * 2);
    qsort(U, (size_t)(C * N), 2, cmp_i16);
    int64_t nU = 0;
    for (int64_t i = 0; i < C * N; i++) if (i == 0 || U[i] != U[nU - 1]) U[nU++] = U[i];
    /* index of each count in U (direct table over 0..32767) */
    int32_t *idx_of = malloc(32768 * 4);
    for (int64_t i = 0; i < nU; i++) idx_of[U[i]] = (int32_t)i;
    /* 4-tuples of U-indices per voxel, lexicographic order = numeric order of packed u64 */
    uint64_t *tup = malloc((size_t)N * 8);
    for (int64_t v = 0; v < N; v++) {
        uint64_t t = 0;
        for (int c = 0; c < C; c++) t = (t << 16) | (uint64_t)idx_of[counts[c * N + v]];
        tup[v] = t;
    }
    uint64_t *scratch = malloc((size_t)N * 8);
    zrange_t *sl = malloc(sizeof(zrange_t) * (size_t)D);
    int nslab = 0;
    if (localize) split_localized(tup, plane, 0, D, scratch, sl, &nslab);
    else split_slabs(tup, plane, 0, D, scratch, sl, &nslab);

    /* 2. lay out: header, U, slab table, then per slab LUT + keys */
    uint64_t off = 64;
    uint64_t U_off = off; off = up16(off + 2 * (uint64_t)nU);
    uint64_t slab_off = off; off = up16(off + 32 * (uint64_t)nslab);
    int rc = ORC_OK;
    /* first pass computes sizes; second pass writes (re-derives groups) */
    uint8_t *out = NULL;
    for (int pass = 0; pass < 2 && rc == ORC_OK; pass++) {
        uint64_t cur = off;
        for (int t = 0; t < nslab; t++) {
            int64_t Nt = (int64_t)(sl[t].z1 - sl[t].z0) * plane;
            const uint64_t *tt = tup + (int64_t)sl[t].z0 * plane;
            memcpy(scratch, tt, (size_t)Nt * 8);
            qsort(scratch, (size_t)Nt, 8, cmp_u64);
            int64_t G = 0;
            for (int64_t i = 0; i < Nt; i++) if (i == 0 || scratch[i] != scratch[i - 1]) G++;
            int kw = G == 1 ? 0 : (G <= 256 ? 1 : 2);
            if (G > 65536 || 8 * G + kw * Nt >= 8 * Nt) { kw = 8; }
            int64_t n_esc = 0;
            if (escape && kw == 2) {                     /* FORMAT.md 1.5: escaped 1-byte keys if smaller */
                n_esc = escaped_count(scratch, Nt, G);
                if (escaped_bytes(Nt, n_esc) < up16(2 * (uint64_t)Nt)) kw = 3;
            }
            uint64_t lut_off = 0, keys_off = 0;
            if (kw != 8) { lut_off = cur; cur = up16(cur + 8 * (uint64_t)G); }
            if (kw == 3) { keys_off = cur; cur += escaped_bytes(Nt, n_esc); }
            else if (kw != 0) { keys_off = cur; cur = up16(cur + (uint64_t)(kw == 8 ? 8 : kw) * (uint64_t)Nt); }
            if (pass == 1) {
                uint8_t *s = out + slab_off + 32 * (uint64_t)t;
                wr32(s, (uint32_t)sl[t].z0); wr32(s + 4, (uint32_t)sl[t].z1);
                wr32(s + 8, kw == 8 ? 0u : (uint32_t)G); s[12] = (uint8_t)kw;
                wr64(s + 16, lut_off); wr64(s + 24, keys_off);
                if (kw == 8) {
                    for (int c = 0; c < C; c++)
                        for (int64_t v = 0; v < Nt; v++) {
                            int16_t cnt = counts[c * N + (int64_t)sl[t].z0 * plane + v];
                            wr16(out + keys_off + 2 * ((uint64_t)c * Nt + v), (uint16_t)idx_of[cnt]);
                        }
                } else {
                    /* distinct tuples with frequencies, ordered by (freq desc, tuple asc) */
                    group_t *grp = malloc(sizeof(group_t) * (size_t)G);
                    int64_t g = -1;
                    for (int64_t i = 0; i < Nt; i++) {
                        if (i == 0 || scratch[i] != scratch[i - 1]) { g++; grp[g].tup = scratch[i]; grp[g].freq = 0; }
                        grp[g].freq++;
                    }
                    qsort(grp, (size_t)G, sizeof(group_t), cmp_group);
                    /* key of a tuple: its rank in grp; lookup via sorted distinct tuples */
                    uint64_t *uniq = malloc(8 * (size_t)G);
                    int64_t *key_of = malloc(8 * (size_t)G);
                    int64_t u = 0;
                    for (int64_t i = 0; i < Nt; i++) if (i == 0 || scratch[i] != scratch[i - 1]) uniq[u++] = scratch[i];
                    for (int64_t k = 0; k < G; k++) key_of[find_u64(uniq, G, grp[k].tup)] = k;
                    for (int64_t k = 0; k < G; k++)
                        for (int c = 0; c < C; c++)
                            wr16(out + lut_off + 8 * (uint64_t)k + 2 * (uint64_t)c,
                                 (uint16_t)((grp[k].tup >> (16 * (3 - c))) & 0xFFFFu));
                    uint64_t nb = ((uint64_t)Nt + 255) / 256;
                    uint64_t low_off = keys_off + up16(4 * (nb + 1)), esc_off = low_off + up16((uint64_t)Nt);
                    int64_t seen = 0;
                    for (int64_t v = 0; v < Nt && kw != 0; v++) {
                        int64_t k = key_of[find_u64(uniq, G, tt[v])];
                        if (kw == 1) out[keys_off + (uint64_t)v] = (uint8_t)k;
                        else if (kw == 2) wr16(out + keys_off + 2 * (uint64_t)v, (uint16_t)k);
                        else {                           /* kw = 3: escape keys >= 255 */
                            if (v % 256 == 0) wr32(out + keys_off + 4 * ((uint64_t)v / 256), (uint32_t)seen);
                            out[low_off + (uint64_t)v] = (uint8_t)(k < 255 ? k : 255);
                            if (k >= 255) wr16(out + esc_off + 2 * (uint64_t)seen++, (uint16_t)k);
                        }
                    }
                    if (kw == 3) wr32(out + keys_off + 4 * nb, (uint32_t)seen);
                    free(grp); free(uniq); free(key_of);
                }
            }
        }
        if (pass == 0) {
            *size = (size_t)cur;
            if (!dst || cap < cur) { rc = ORC_ESMALL; break; }
            out = dst;
            memset(out, 0, (size_t)cur);
            wr32(out, 0x43505053u); wr16(out + 4, 1); wr16(out + 6, 0);
            wr16(out + 8, (uint16_t)C); wr16(out + 10, (uint16_t)D); wr16(out + 12, (uint16_t)H); wr16(out + 14, (uint16_t)W);
            wr32(out + 16, (uint32_t)nU); wr32(out + 20, (uint32_t)nslab);
            wr64(out + 24, U_off); wr64(out + 32, slab_off); wr64(out + 40, cur);
            for (int64_t i = 0; i < nU; i++) wr16(out + U_off + 2 * (uint64_t)i, (uint16_t)U[i]);
        }
    }
    free(U); free(idx_of); free(tup); free(scratch); free(sl);
    return rc;
}

/* ---------------- CosmoFlow sequential decoder (FORMAT.md 1.2) ------------- */
int orc_cosmo_decode(const uint8_t *src, size_t size, int transform, int out_kind, void *out,
                     int expC, int expD, int expH, int expW) {
    if (!src || !out) return ORC_EINVAL;
    if (out_kind == OUT_I16 && transform) return ORC_EINVAL;
    if (size < 64 || rd32(src) != 0x43505053u || rd16(src + 4) != 1) return ORC_ECORRUPT;
    int C = rd16(src + 8), D = rd16(src + 10), H = rd16(src + 12), W = rd16(src + 14);
    if (C != 4 || D < 1 || H < 1 || W < 1) return ORC_ECORRUPT;
    if (C != expC || D != expD || H != expH || W != expW) return ORC_ECORRUPT;
    uint32_t nU = rd32(src + 16), T = rd32(src + 20);
    uint64_t U_off = rd64(src + 24), slab_off = rd64(src + 32), total = rd64(src + 40);
    if (total > size || nU < 1 || nU > 32768 || T < 1 || T > (uint32_t)D) return ORC_ECORRUPT;
    if (U_off + 2 * (uint64_t)nU > total || slab_off + 32 * (uint64_t)T > total) return ORC_ECORRUPT;
    int64_t plane = (int64_t)H * W, N = (int64_t)D * plane;
    uint32_t zexp = 0;
    for (uint32_t t = 0; t < T; t++) {
        const uint8_t *s = src + slab_off + 32 * (uint64_t)t;
        uint32_t z0 = rd32(s), z1 = rd32(s + 4), G = rd32(s + 8);
        int kw = s[12];
        uint64_t lut_off = rd64(s + 16), keys_off = rd64(s + 24);
        if (z0 != zexp || z1 <= z0 || z1 > (uint32_t)D) return ORC_ECORRUPT;
        zexp = z1;
        int64_t Nt = (int64_t)(z1 - z0) * plane;
        if (kw == 0 && G != 1) return ORC_ECORRUPT;
        if (kw == 1 && (G < 1 || G > 256)) return ORC_ECORRUPT;
        if (kw == 2 && (G < 1 || G > 65536)) return ORC_ECORRUPT;
        if (kw == 3 && (G < 1 || G > 65536)) return ORC_ECORRUPT;
        if (kw == 8 && G != 0) return ORC_ECORRUPT;
        if (kw != 0 && kw != 1 && kw != 2 && kw != 3 && kw != 8) return ORC_ECORRUPT;
        if (kw != 8 && lut_off + 8 * (uint64_t)G > total) return ORC_ECORRUPT;
        /* kw = 3 (FORMAT.md 1.5): eidx u32[nb+1], low u8[Nt], esc u16[eidx[nb]] */
        uint64_t nb = ((uint64_t)Nt + 255) / 256, low_off = 0, esc_off = 0, n_esc = 0, seen = 0;
        if (kw == 3) {
            low_off = keys_off + up16(4 * (nb + 1));
            esc_off = low_off + up16((uint64_t)Nt);
            if (esc_off > total || rd32(src + keys_off) != 0) return ORC_ECORRUPT;
            n_esc = rd32(src + keys_off + 4 * nb);
            if (esc_off + 2 * n_esc > total) return ORC_ECORRUPT;
        } else if (kw != 0 && keys_off + (uint64_t)(kw == 8 ? 8 : kw) * (uint64_t)Nt > total) {
            return ORC_ECORRUPT;
        }
        for (int64_t v = 0; v < Nt; v++) {
            uint32_t g = 0;
            if (kw == 3) {                               /* escaped 1-byte keys, voxel order */
                if (v % 256 == 0 && rd32(src + keys_off + 4 * ((uint64_t)v / 256)) != seen) return ORC_ECORRUPT;
                g = src[low_off + (uint64_t)v];
                if (g == 255) {
                    if (seen >= n_esc) return ORC_ECORRUPT;
                    g = rd16(src + esc_off + 2 * seen++);
                }
            }
            for (int c = 0; c < C; c++) {
                uint32_t e;
                if (kw == 8) {
                    e = rd16(src + keys_off + 2 * ((uint64_t)c * Nt + v));
                } else {
                    if (kw != 3)
                        g = kw == 0 ? 0 : (kw == 1 ? src[keys_off + v] : rd16(src + keys_off + 2 * (uint64_t)v));
                    if (g >= G) return ORC_ECORRUPT;
                    e = rd16(src + lut_off + 8 * (uint64_t)g + 2 * (uint64_t)c);
                }
                if (e >= nU) return ORC_ECORRUPT;
                int16_t count = (int16_t)rd16(src + U_off + 2 * (uint64_t)e);
                int rc = emit_cosmo(count, transform, out_kind, out,
                                    (size_t)((int64_t)c * N + (int64_t)z0 * plane + v));
                if (rc) return rc;
            }
        }
        if (kw == 3 && seen != n_esc) return ORC_ECORRUPT;
    }
    if (zexp != (uint32_t)D) return ORC_ECORRUPT;
    return ORC_OK;
}

/* ---------------- DeepCAM 8-bit delta code (FORMAT.md 2.2) ---------- */
int orc_deepcam_code(int b) {
    int sgn = (b >> 7) & 1, E = (b >> 4) & 7, M = b & 15;
    int mag = (E == 0) ? M : ((16 + M) << (E - 1));
    return sgn ? -mag : mag;
}

/* ---------------- DeepCAM line decoder (FORMAT.md 2.3) --------------------- */
/* Decodes line l of the stream into xhat[W] (before normalisation). */
int orc_deepcam_decode_line(const uint8_t *src, size_t size, int l, float *xhat) {
    if (!src || !xhat || size < 64 || rd32(src) != 0x44505053u || rd16(src + 4) != 1) return ORC_ECORRUPT;
    int C = rd16(src + 8), H = rd16(src + 10), W = rd16(src + 12), A = rd16(src + 14);
    uint32_t L = rd32(src + 16);
    uint64_t dir_off = rd64(src + 24), payload_off = rd64(src + 32), total = rd64(src + 40);
    if (C < 1 || H < 1 || W < 1 || L != (uint32_t)C * (uint32_t)H || total > size) return ORC_ECORRUPT;
    if (A < 1 || W % A != 0) return ORC_ECORRUPT;            /* segment alignment (FORMAT.md 2.1) */
    if (l < 0 || (uint32_t)l >= L) return ORC_EINVAL;
    if (dir_off + 4 * ((uint64_t)L + 1) > total) return ORC_ECORRUPT;
    uint32_t a = rd32(src + dir_off + 4 * (uint64_t)l), b = rd32(src + dir_off + 4 * (uint64_t)l + 4);
    if (b < a || (a & 15) || (b & 15) || payload_off + b > total) return ORC_ECORRUPT;
    const uint8_t *p = src + payload_off + a;
    uint64_t len_line = b - a;
    if (len_line < 16) return ORC_ECORRUPT;
    int mode = p[0];
    if (mode == 0) {                                     /* RAW */
        if (16 + 4 * (uint64_t)W > len_line) return ORC_ECORRUPT;
        for (int x = 0; x < W; x++) xhat[x] = f32_of_bits(rd32(p + 16 + 4 * (uint64_t)x));
        return ORC_OK;
    }
    if (mode == 2) {                                     /* RAW16 (FORMAT.md 2.6) */
        if (16 + 2 * (uint64_t)W > len_line) return ORC_ECORRUPT;
        for (int x = 0; x < W; x++) xhat[x] = orc_f16_to_f32(rd16(p + 16 + 2 * (uint64_t)x));
        return ORC_OK;
    }
    if (mode != 1 && mode != 3) return ORC_ECORRUPT;        /* 3: SEG with RAW segments (FORMAT.md 2.7) */
    int nseg = rd16(p + 2);
    if (nseg < 1 || nseg > W || 4 + 8 * (uint64_t)nseg > len_line) return ORC_ECORRUPT;
    uint64_t dpos = 4 + 8 * (uint64_t)nseg;             /* next delta byte */
    int pos = 0;
    for (int s = 0; s < nseg; s++) {
        const uint8_t *d = p + 4 + 4 * (uint64_t)s;
        int len = rd16(d), kind = d[2], emin_b = d[3];
        float h = f32_of_bits(rd32(p + 4 + 4 * (uint64_t)nseg + 4 * (uint64_t)s));
        if (len < 1 || pos + len > W || pos % A != 0) return ORC_ECORRUPT;
        if (kind == 0) {                                 /* REPEAT: broadcast the head */
            for (int j = 0; j < len; j++) xhat[pos + j] = h;
        } else if (kind == 1) {                          /* DIFF */
            if (emin_b < 1 || emin_b > 246) return ORC_ECORRUPT;
            if (dpos + (uint64_t)(len - 1) > len_line) return ORC_ECORRUPT;
            int emin = emin_b - 150;
            float unit = ldexpf(1.0f, emin);             /* 2^emin, exact (subnormal at -149) */
            int64_t S = 0;
            xhat[pos] = h;
            for (int j = 1; j < len; j++) {
                S += orc_deepcam_code(p[dpos + (uint64_t)(j - 1)]);
                xhat[pos + j] = h + (float)S * unit;     /* fp32: exact product, one rounding */
            }
            dpos += (uint64_t)(len - 1);
        } else if (kind == 2 && mode == 3) {             /* RAW segment: len binary32 values */
            if (dpos + 4 * (uint64_t)len > len_line) return ORC_ECORRUPT;
            for (int j = 0; j < len; j++) xhat[pos + j] = f32_of_bits(rd32(p + dpos + 4 * (uint64_t)j));
            dpos += 4 * (uint64_t)len;
        } else {
            return ORC_ECORRUPT;
        }
        pos += len;
    }
    if (pos != W) return ORC_ECORRUPT;
    if (up16(dpos) > len_line) return ORC_ECORRUPT;
    return ORC_OK;
}

/* Whole-sample decode with per-channel normalisation (FORMAT.md 2.3, S18). */
int orc_deepcam_decode(const uint8_t *src, size_t size, const float *shift, const float *scale,
                       int out_kind, void *out, int expC, int expH, int expW) {
    if (!src || !out || (out_kind != OUT_F16 && out_kind != OUT_F32)) return ORC_EINVAL;
    if (size < 64 || rd32(src) != 0x44505053u) return ORC_ECORRUPT;
    int C = rd16(src + 8), H = rd16(src + 10), W = rd16(src + 12);
    if (C != expC || H != expH || W != expW) return ORC_ECORRUPT;
    float *xhat = malloc(sizeof(float) * (size_t)W);
    int rc = ORC_OK;
    for (int c = 0; c < C && rc == ORC_OK; c++) {
        float sh = shift ? shift[c] : 0.0f, sc = scale ? scale[c] : 1.0f;
        for (int y = 0; y < H && rc == ORC_OK; y++) {
            int l = c * H + y;
            rc = orc_deepcam_decode_line(src, size, l, xhat);
            if (rc) break;
            for (int x = 0; x < W; x++) {
                float t = xhat[x] - sh;                   /* first rounding */
                float v = t * sc;                         /* second rounding */
                size_t i = ((size_t)c * H + y) * W + x;
                if (out_kind == OUT_F32) ((float *)out)[i] = v;
                else ((uint16_t *)out)[i] = orc_f32_to_f16(v);
            }
        }
    }
    free(xhat);
    return rc;
}

/* ---------------- DeepCAM encoder (FORMAT.md 2.4) -------------------------- */
static int mags[128];                                    /* code magnitudes, ascending in b */
static void init_mags(void) { for (int b = 0; b < 128; b++) mags[b] = orc_deepcam_code(b); }

/* nearest code byte to t (|t| <= 1984.5), ties toward the smaller magnitude */
static int quantise(double t) {
    double a = fabs(t);
    int best = 0;                                        /* mags[] ascending: scan up to a */
    while (best < 127 && mags[best + 1] <= a) best++;    /* mags[best] <= a < mags[best+1] */
    if (best < 127 && (mags[best + 1] - a) < (a - mags[best])) best++;  /* strictly nearer; tie -> smaller */
    if (mags[best] == 0) return 0;
    return t < 0 ? (best | 0x80) : best;
}

/* ceil(log2(q)) for q > 0, exact via frexp */
static int ceil_log2(double q) {
    int e;
    double f = frexp(q, &e);                            /* q = f * 2^e, 0.5 <= f < 1 */
    return (f == 0.5) ? e - 1 : e;
}

/* Encode one line (FORMAT.md 2.4) with segment alignment A; returns the SEG
 * byte size, or -1 if no aligned segmentation exists (the line is then RAW). */
typedef struct { int len, kind, emin_b; float head; } seg_t;

/* The run that may become a REPEAT segment at i, cut at the range end E
 * (E = W for a whole line).  tau = 0: the run of bit-identical values
 * (FORMAT.md 2.4, run[] precomputed).  tau > 0 (FORMAT.md 2.8, "all
 * neighbouring values are similar", reading S15): the longest run of values
 * within tau of x[i], |x[j] - x[i]| <= tau in binary64. */
static int run_at(const float *x, const int *run, int i, int E, double tau) {
    if (tau == 0.0) return run[i] < E - i ? run[i] : E - i;
    int k = 1;
    while (i + k < E && fabs((double)x[i + k] - (double)x[i]) <= tau) k++;
    return k;
}
static int rep_len(const float *x, const int *run, int i, int E, int A, double tau) {
    int r = run_at(x, run, i, E, tau);
    return (i + r == E) ? r : (r / A) * A;
}

/* The greedy policy of FORMAT.md 2.4 over positions [i0, E) of a line (E = W
 * for the whole line; 2.7 encodes the ranges between RAW segments), appending
 * to segs / deltas.  Returns -1 when no aligned segmentation exists. */
static int encode_range(const float *x, int i0, int E, int A, int lookahead, int repeat_min, seg_t *segs,
                        int *nseg_io, uint8_t *deltas, int64_t *nd_io, const int *run, double tau) {
    int nseg = *nseg_io;
    int64_t nd = *nd_io;
    int i = i0;
    while (i < E) {
        int rl = rep_len(x, run, i, E, A, tau);
        if (rl >= repeat_min) {
            segs[nseg].len = rl; segs[nseg].kind = 0; segs[nseg].emin_b = 0; segs[nseg].head = x[i];
            nseg++;
            i += rl;
            continue;
        }
        float h = x[i];
        double m = 0.0;
        for (int j = i + 1; j < E && j < i + lookahead; j++) {
            double d = fabs((double)x[j] - (double)x[j - 1]);
            if (d > m) m = d;
        }
        int emin = -149;
        if (m > 0.0) {
            emin = ceil_log2(m / 1984.0);
            if (emin < -149) emin = -149;
            if (emin > 96) emin = 96;
        }
        int64_t nd0 = nd;
        int end;
        for (;;) {                                       /* (re)encode the segment from i */
            float unit = ldexpf(1.0f, emin);
            int64_t S = 0;
            float prev = h;
            int j = i + 1, overflow = 0;
            nd = nd0;
            while (j < E) {
                if (j % A == 0 && rep_len(x, run, j, E, A, tau) >= repeat_min) break;
                double t = ldexp((double)x[j] - (double)prev, -emin);
                if (fabs(t) > 1984.5) { overflow = 1; break; }
                int b = quantise(t);
                int k = orc_deepcam_code(b);
                if (llabs(S + k) > 1983LL * 1984LL) { overflow = 1; break; }
                S += k;
                prev = h + (float)S * unit;
                if (deltas) deltas[nd] = (uint8_t)b;
                nd++;
                j++;
            }
            if (!overflow) { end = j; break; }
            end = (j / A) * A;
            if (end > i) { nd = nd0 + (end - i - 1); break; }   /* drop deltas of positions >= end */
            if (emin >= 96) return -1;                          /* no aligned segmentation: RAW */
            emin++;                                             /* overflow inside the first A values */
        }
        segs[nseg].len = end - i; segs[nseg].kind = 1; segs[nseg].emin_b = emin + 150; segs[nseg].head = h;
        nseg++;
        i = end;
    }
    *nseg_io = nseg;
    *nd_io = nd;
    return 0;
}

static int64_t encode_line(const float *x, int W, int A, int lookahead, int repeat_min, seg_t *segs,
                           int *nseg_out, uint8_t *deltas, int64_t *ndelta_out, int *run, double tau) {
    /* run lengths of bit-identical values */
    run[W - 1] = 1;
    for (int i = W - 2; i >= 0; i--)
        run[i] = (bits_of_f32(x[i]) == bits_of_f32(x[i + 1])) ? run[i + 1] + 1 : 1;
    int nseg = 0;
    int64_t nd = 0;
    if (encode_range(x, 0, W, A, lookahead, repeat_min, segs, &nseg, deltas, &nd, run, tau) < 0) return -1;
    *nseg_out = nseg;
    *ndelta_out = nd;
    return (int64_t)up16(4 + 8 * (uint64_t)nseg + (uint64_t)nd);
}

int orc_deepcam_align(int W) { return W == 1152 ? 36 : (W % 8 == 0 ? 8 : 1); }

size_t orc_deepcam_max_encoded_size(int C, int H, int W) {
    uint64_t L = (uint64_t)C * H;
    return (size_t)(64 + up16(4 * (L + 1)) + L * up16(16 + 4 * (uint64_t)W));
}

int orc_deepcam_encode_a(const float *x, int C, int H, int W, int A, uint8_t *dst, size_t cap, size_t *size);
int orc_deepcam_encode_p(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, uint8_t *dst,
                         size_t cap, size_t *size);

int orc_deepcam_encode(const float *x, int C, int H, int W, uint8_t *dst, size_t cap, size_t *size) {
    return orc_deepcam_encode_a(x, C, H, W, orc_deepcam_align(W), dst, cap, size);
}

/* same policy with an explicit alignment A (W % A == 0) */
int orc_deepcam_encode_a(const float *x, int C, int H, int W, int A, uint8_t *dst, size_t cap, size_t *size) {
    return orc_deepcam_encode_p(x, C, H, W, A, 64, 16, dst, cap, size);
}

/* ... and explicit policy knobs: the emin lookahead window and the shortest
 * REPEAT run (FORMAT.md 2.4 uses 64 and 16) */
int orc_deepcam_encode_q(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, float rel_err,
                         int err_budget, uint8_t *dst, size_t cap, size_t *size);
int orc_deepcam_encode_p(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, uint8_t *dst,
                         size_t cap, size_t *size) {
    return orc_deepcam_encode_q(x, C, H, W, A, lookahead, repeat_min, 0.1f, 0, dst, cap, size);
}
int orc_deepcam_encode_r(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, float rel_err,
                         int err_budget, int raw16, uint8_t *dst, size_t cap, size_t *size);
int orc_deepcam_encode_s(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, float rel_err,
                         int err_budget, int raw16, int rawseg, uint8_t *dst, size_t cap, size_t *size);
int orc_deepcam_encode_r(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, float rel_err,
                         int err_budget, int raw16, uint8_t *dst, size_t cap, size_t *size) {
    return orc_deepcam_encode_s(x, C, H, W, A, lookahead, repeat_min, rel_err, err_budget, raw16, 0, dst, cap, size);
}
int orc_deepcam_encode_q(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, float rel_err,
                         int err_budget, uint8_t *dst, size_t cap, size_t *size) {
    return orc_deepcam_encode_r(x, C, H, W, A, lookahead, repeat_min, rel_err, err_budget, 0, dst, cap, size);
}

/* x̂ of an encoded SEG line, position by position, exactly as the decoder of
 * FORMAT.md 2.3 rebuilds it (RAW segments of 2.7: their stored values). */
static void line_xhat(const float *x, const seg_t *segs, int nseg, const uint8_t *deltas, float *xh) {
    int pos = 0;
    int64_t d = 0;
    for (int s = 0; s < nseg; s++) {
        float h = segs[s].head;
        if (segs[s].kind == 2) {                           /* RAW segment: exact (FORMAT.md 2.7) */
            for (int j = 0; j < segs[s].len; j++) xh[pos + j] = x[pos + j];
            d += 4 * (int64_t)segs[s].len;
        } else if (segs[s].kind == 0) {                    /* REPEAT: the head */
            for (int j = 0; j < segs[s].len; j++) xh[pos + j] = h;
        } else {                                           /* DIFF: h, then RN(h + S * 2^emin) */
            float unit = ldexpf(1.0f, segs[s].emin_b - 150);
            int64_t S = 0;
            xh[pos] = h;
            for (int j = 1; j < segs[s].len; j++) {
                S += orc_deepcam_code(deltas[d++]);
                xh[pos + j] = h + (float)S * unit;
            }
        }
        pos += segs[s].len;
    }
}

/* The two error bounds a value is checked against (binary64 on binary32
 * operands).  Relative (FORMAT.md 2.5; "areas with abrupt changes are kept
 * uncompressed", "roughly 3% of the values with larger than 10% error";
 * DESIGN.md S19): |x̂ - x| > rel |x|, so x = 0 counts iff x̂ != 0.  Absolute
 * (FORMAT.md 2.8, per channel): |x̂ - x| > eps, eps > 0. */
static int over_rel(float xh, float x, double rel) { return fabs((double)xh - (double)x) > rel * fabs((double)x); }
static int over_abs(float xh, float x, double eps) { return eps > 0.0 && fabs((double)xh - (double)x) > eps; }

/* FORMAT.md 2.6: every value finite and its RNE binary16 rounding within rel
 * of it (and within eps when eps > 0, FORMAT.md 2.8) */
static int raw16_ok(const float *x, int W, double rel, double eps) {
    for (int k = 0; k < W; k++) {
        if (!isfinite(x[k])) return 0;
        float h = orc_f16_to_f32(orc_f32_to_f16(x[k]));
        if (!isfinite(h) || over_rel(h, x[k], rel) || over_abs(h, x[k], eps)) return 0;
    }
    return 1;
}

/* FORMAT.md 2.7 encoder step: the blocks [bA, bA + A) holding a flagged value
 * of the 2.4 encoding (flag[] filled by the caller) become RAW segments (a run
 * of them, one segment); the ranges between are re-encoded by the 2.4 policy.
 * Returns the line's SEG size, or -1. */
static int64_t encode_line_rawseg(const float *x, int W, int A, int lookahead, int repeat_min, const uint8_t *flag,
                                  const int *run, double tau, seg_t *segs, int *nseg_out, uint8_t *deltas,
                                  int64_t *nd_out) {
    int nb = (W + A - 1) / A, nseg = 0;
    int64_t nd = 0;
    int b = 0;
    while (b < nb) {
        int bad_b = 0;
        for (int k = b * A; k < W && k < (b + 1) * A; k++) bad_b |= flag[k];
        int b2 = b + 1;
        for (; b2 < nb; b2++) {
            int bb = 0;
            for (int k = b2 * A; k < W && k < (b2 + 1) * A; k++) bb |= flag[k];
            if (bb != bad_b) break;
        }
        int s0 = b * A, e0 = b2 * A < W ? b2 * A : W;
        if (bad_b) {
            segs[nseg].len = e0 - s0; segs[nseg].kind = 2; segs[nseg].emin_b = 0; segs[nseg].head = x[s0];
            nseg++;
            for (int k = s0; k < e0; k++) { wr32(deltas + nd, bits_of_f32(x[k])); nd += 4; }
        } else if (encode_range(x, s0, e0, A, lookahead, repeat_min, segs, &nseg, deltas, &nd, run, tau) < 0) {
            return -1;
        }
        b = b2;
    }
    *nseg_out = nseg;
    *nd_out = nd;
    return (int64_t)up16(4 + 8 * (uint64_t)nseg + (uint64_t)nd);
}

typedef struct {
    int A, lookahead, repeat_min, err_budget, raw16, rawseg;
    double rel;
    seg_t *segs, *segs2;
    uint8_t *deltas, *deltas2, *flag;
    int *run;
    float *xh;
    int nseg, nseg2;
    int64_t nd, nd2;
} enc_ctx;

/* The line's encoding (FORMAT.md 2.4-2.8): 0 RAW, 1 SEG (segs/deltas), 2 RAW16,
 * 3 SEG with RAW segments (segs2/deltas2); *size = its payload bytes.
 * tau / eps: the line's channel's REPEAT tolerance and absolute bound (2.8). */
static int decide_line(const float *x, int W, enc_ctx *c, double tau, double eps, uint64_t *size) {
    uint64_t raw_size = up16(16 + 4 * (uint64_t)W), raw16_size = up16(16 + 2 * (uint64_t)W);
    for (int k = 0; k < W; k++)
        if (!isfinite(x[k])) { *size = raw_size; return 0; }     /* non-finite: RAW (2.4 step 1) */
    int64_t seg_size = encode_line(x, W, c->A, c->lookahead, c->repeat_min, c->segs, &c->nseg, c->deltas, &c->nd,
                                   c->run, tau);
    if (seg_size >= 0 && (c->err_budget > 0 || eps > 0.0)) {
        line_xhat(x, c->segs, c->nseg, c->deltas, c->xh);
        int nrel = 0, nabs = 0;
        for (int k = 0; k < W; k++) { nrel += over_rel(c->xh[k], x[k], c->rel); nabs += over_abs(c->xh[k], x[k], eps); }
        if ((c->err_budget > 0 && nrel >= c->err_budget) || nabs > 0) {
            /* kept uncompressed (2.5 / 2.8): RAW, RAW16 (2.6) or RAW segments (2.7) */
            int mode = 0;
            uint64_t sz = raw_size;
            if (c->raw16 && raw16_ok(x, W, c->rel, eps)) { mode = 2; sz = raw16_size; }
            if (c->rawseg) {
                for (int k = 0; k < W; k++)
                    c->flag[k] = (c->err_budget > 0 && over_rel(c->xh[k], x[k], c->rel)) || over_abs(c->xh[k], x[k], eps);
                int64_t rs = encode_line_rawseg(x, W, c->A, c->lookahead, c->repeat_min, c->flag, c->run, tau, c->segs2,
                                                &c->nseg2, c->deltas2, &c->nd2);
                if (rs >= 0 && (uint64_t)rs < sz) {
                    line_xhat(x, c->segs2, c->nseg2, c->deltas2, c->xh);
                    int r2 = 0, a2 = 0;
                    for (int k = 0; k < W; k++) { r2 += over_rel(c->xh[k], x[k], c->rel); a2 += over_abs(c->xh[k], x[k], eps); }
                    if ((c->err_budget == 0 || r2 < c->err_budget) && a2 == 0) { mode = 3; sz = (uint64_t)rs; }
                }
            }
            *size = sz;
            return mode;
        }
    }
    if (seg_size >= 0 && (uint64_t)seg_size < raw_size) { *size = (uint64_t)seg_size; return 1; }
    *size = raw_size;                                    /* RAW on a tie (2.4 step 3) */
    return 0;
}

int orc_deepcam_encode_t(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, float rel_err,
                         int err_budget, int raw16, int rawseg, const float *repeat_tol, const float *max_abs_err,
                         uint8_t *dst, size_t cap, size_t *size);
int orc_deepcam_encode_s(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, float rel_err,
                         int err_budget, int raw16, int rawseg, uint8_t *dst, size_t cap, size_t *size) {
    return orc_deepcam_encode_t(x, C, H, W, A, lookahead, repeat_min, rel_err, err_budget, raw16, rawseg, NULL, NULL,
                                dst, cap, size);
}

/* The DeepCAM encoder (FORMAT.md 2.4-2.8) with every knob.  repeat_tol /
 * max_abs_err: NULL or fp32[C], each finite and >= 0 (0 = off). */
int orc_deepcam_encode_t(const float *x, int C, int H, int W, int A, int lookahead, int repeat_min, float rel_err,
                         int err_budget, int raw16, int rawseg, const float *repeat_tol, const float *max_abs_err,
                         uint8_t *dst, size_t cap, size_t *size) {
    if (!x || !size || C < 1 || H < 1 || W < 1 || C > 65535 || H > 65535 || W > 65535) return ORC_EINVAL;
    if (raw16 != 0 && raw16 != 1) return ORC_EINVAL;
    if (rawseg != 0 && rawseg != 1) return ORC_EINVAL;
    if (lookahead < 2 || lookahead > 65535 || repeat_min < 2 || repeat_min > 65535) return ORC_EINVAL;
    if (err_budget < 0 || !(rel_err > 0.0f) || !(rel_err < 1e30f)) return ORC_EINVAL;
    if ((uint64_t)C * H > 0xFFFFFFFFull || A < 1 || W % A != 0) return ORC_EINVAL;
    for (int c = 0; c < C; c++) {
        if (repeat_tol && !(repeat_tol[c] >= 0.0f && repeat_tol[c] < INFINITY)) return ORC_EINVAL;
        if (max_abs_err && !(max_abs_err[c] >= 0.0f && max_abs_err[c] < INFINITY)) return ORC_EINVAL;
    }
    init_mags();
    uint64_t L = (uint64_t)C * H;
    uint64_t dir_off = 64, payload_off = up16(dir_off + 4 * (L + 1));
    enc_ctx c = {A, lookahead, repeat_min, err_budget, raw16, rawseg, (double)rel_err, NULL, NULL, NULL, NULL, NULL,
                 NULL, NULL, 0, 0, 0, 0};
    c.segs = malloc(sizeof(seg_t) * (size_t)W);
    c.segs2 = malloc(sizeof(seg_t) * (size_t)W);
    c.deltas = malloc((size_t)W);
    c.deltas2 = malloc(5 * (size_t)W);
    c.flag = malloc((size_t)W);
    c.run = malloc(sizeof(int) * (size_t)W);
    c.xh = malloc(sizeof(float) * (size_t)W);
    /* pass 1: sizes */
    uint64_t pay = 0;
    for (uint64_t l = 0; l < L; l++) {
        int ch = (int)(l / (uint64_t)H);
        uint64_t sz;
        decide_line(x + l * (uint64_t)W, W, &c, repeat_tol ? repeat_tol[ch] : 0.0, max_abs_err ? max_abs_err[ch] : 0.0,
                    &sz);
        pay += sz;
    }
    uint64_t total = payload_off + pay;
    *size = (size_t)total;
    int rc = ORC_OK;
    if (total > 0xFFFFFFFFull + payload_off) rc = ORC_EINVAL;
    else if (!dst || cap < total) rc = ORC_ESMALL;
    if (rc == ORC_OK) {
        memset(dst, 0, (size_t)total);
        wr32(dst, 0x44505053u); wr16(dst + 4, 1); wr16(dst + 6, 0);   /* flags: bit 0 set below (FORMAT.md 2.1) */
        wr16(dst + 8, (uint16_t)C); wr16(dst + 10, (uint16_t)H); wr16(dst + 12, (uint16_t)W);
        wr16(dst + 14, (uint16_t)A);
        wr32(dst + 16, (uint32_t)L);
        wr64(dst + 24, dir_off); wr64(dst + 32, payload_off); wr64(dst + 40, total);
        uint64_t cur = 0;
        for (uint64_t l = 0; l < L; l++) {
            wr32(dst + dir_off + 4 * l, (uint32_t)cur);
            const float *xl = x + l * (uint64_t)W;
            uint8_t *p = dst + payload_off + cur;
            int ch = (int)(l / (uint64_t)H);
            uint64_t sz;
            int mode = decide_line(xl, W, &c, repeat_tol ? repeat_tol[ch] : 0.0, max_abs_err ? max_abs_err[ch] : 0.0,
                                   &sz);
            p[0] = (uint8_t)mode;
            if (mode == 0) {
                for (int k = 0; k < W; k++) wr32(p + 16 + 4 * (uint64_t)k, bits_of_f32(xl[k]));
            } else if (mode == 2) {
                for (int k = 0; k < W; k++) wr16(p + 16 + 2 * (uint64_t)k, orc_f32_to_f16(xl[k]));
            } else {
                const seg_t *sg = mode == 1 ? c.segs : c.segs2;
                int ns = mode == 1 ? c.nseg : c.nseg2;
                wr16(p + 2, (uint16_t)ns);
                for (int s = 0; s < ns; s++) {
                    wr16(p + 4 + 4 * s, (uint16_t)sg[s].len);
                    p[4 + 4 * s + 2] = (uint8_t)sg[s].kind;
                    p[4 + 4 * s + 3] = (uint8_t)sg[s].emin_b;
                    wr32(p + 4 + 4 * (uint64_t)ns + 4 * s, bits_of_f32(sg[s].head));
                }
                memcpy(p + 4 + 8 * (uint64_t)ns, mode == 1 ? c.deltas : c.deltas2, (size_t)(mode == 1 ? c.nd : c.nd2));
            }
            if (mode == 2 || mode == 3) wr16(dst + 6, 1);     /* an extended line mode is present */
            cur += sz;
        }
        wr32(dst + dir_off + 4 * L, (uint32_t)cur);
    }
    free(c.segs); free(c.segs2); free(c.deltas); free(c.deltas2); free(c.flag); free(c.run); free(c.xh);
    return rc;
}

/* ---------------- labels (FORMAT.md 3; "lossless compression of the labels") */
/* Plain definitions: a mask row is coded as its maximal runs of equal values
 * (or verbatim when that is not smaller); decoding is the identity. */
size_t orc_label_max_encoded_size(int kind, int H, int W) {
    if (W < 1 || H < 1) return 0;
    if (kind == 2) return (size_t)up16(32 + 4 * (uint64_t)W);
    return (size_t)(32 + up16(4 * ((uint64_t)H + 1)) + (uint64_t)H * up16(16 + (uint64_t)W));
}

int orc_label_encode_mask(const uint8_t *m, int H, int W, uint8_t *dst, size_t cap, size_t *size) {
    if (!m || !size || H < 1 || W < 1 || H > 65535 || W > 65535) return ORC_EINVAL;
    uint64_t P = 32 + up16(4 * ((uint64_t)H + 1));
    /* pass 1: row sizes */
    uint64_t pay = 0;
    for (int y = 0; y < H; y++) {
        const uint8_t *r = m + (uint64_t)y * W;
        uint64_t nrun = 1;
        for (int x = 1; x < W; x++) if (r[x] != r[x - 1]) nrun++;
        uint64_t run_size = up16(4 + 3 * nrun), raw_size = up16(16 + (uint64_t)W);
        pay += run_size < raw_size ? run_size : raw_size;
    }
    uint64_t total = P + pay;
    *size = (size_t)total;
    if (total - P > 0xFFFFFFFFull) return ORC_EINVAL;
    if (!dst || cap < total) return ORC_ESMALL;
    memset(dst, 0, (size_t)total);
    wr32(dst, 0x4C505053u); wr16(dst + 4, 1); wr16(dst + 6, 1);
    wr16(dst + 8, (uint16_t)H); wr16(dst + 10, (uint16_t)W); wr64(dst + 16, total);
    uint64_t cur = 0;
    for (int y = 0; y < H; y++) {
        wr32(dst + 32 + 4 * (uint64_t)y, (uint32_t)cur);
        const uint8_t *r = m + (uint64_t)y * W;
        uint8_t *p = dst + P + cur;
        uint64_t nrun = 1;
        for (int x = 1; x < W; x++) if (r[x] != r[x - 1]) nrun++;
        uint64_t run_size = up16(4 + 3 * nrun), raw_size = up16(16 + (uint64_t)W);
        if (run_size < raw_size) {
            p[0] = 1; wr16(p + 2, (uint16_t)nrun);
            int k = 0, start = 0;
            for (int x = 1; x <= W; x++) {
                if (x == W || r[x] != r[x - 1]) {          /* run [start, x) ends */
                    wr16(p + 4 + 2 * (uint64_t)k, (uint16_t)(x - start));
                    p[4 + 2 * nrun + (uint64_t)k] = r[start];
                    k++;
                    start = x;
                }
            }
            cur += run_size;
        } else {
            p[0] = 0;
            memcpy(p + 16, r, (size_t)W);
            cur += raw_size;
        }
    }
    wr32(dst + 32 + 4 * (uint64_t)H, (uint32_t)cur);
    return ORC_OK;
}

int orc_label_encode_vector(const float *v, int n, uint8_t *dst, size_t cap, size_t *size) {
    if (!v || !size || n < 1 || n > 65535) return ORC_EINVAL;
    uint64_t total = up16(32 + 4 * (uint64_t)n);
    *size = (size_t)total;
    if (!dst || cap < total) return ORC_ESMALL;
    memset(dst, 0, (size_t)total);
    wr32(dst, 0x4C505053u); wr16(dst + 4, 1); wr16(dst + 6, 2);
    wr16(dst + 8, 1); wr16(dst + 10, (uint16_t)n); wr64(dst + 16, total);
    for (int i = 0; i < n; i++) wr32(dst + 32 + 4 * (uint64_t)i, bits_of_f32(v[i]));
    return ORC_OK;
}

/* Sequential decoder of one label stream: kind 1 -> u8 [H][W], kind 2 -> f32 [W]. */
int orc_label_decode(const uint8_t *src, size_t size, int kind, int H, int W, void *out) {
    if (!src || !out || size < 32 || rd32(src) != 0x4C505053u || rd16(src + 4) != 1) return ORC_ECORRUPT;
    if (rd16(src + 6) != kind || rd16(src + 8) != H || rd16(src + 10) != W || H < 1 || W < 1) return ORC_ECORRUPT;
    uint64_t total = rd64(src + 16);
    if (total > size || (total & 15)) return ORC_ECORRUPT;
    if (kind == 2) {
        if (H != 1 || total < 32 + 4 * (uint64_t)W) return ORC_ECORRUPT;
        for (int i = 0; i < W; i++) ((float *)out)[i] = f32_of_bits(rd32(src + 32 + 4 * (uint64_t)i));
        return ORC_OK;
    }
    if (kind != 1) return ORC_ECORRUPT;
    uint64_t P = 32 + up16(4 * ((uint64_t)H + 1));
    if (P > total) return ORC_ECORRUPT;
    uint8_t *m = (uint8_t *)out;
    for (int y = 0; y < H; y++) {
        uint32_t a = rd32(src + 32 + 4 * (uint64_t)y), b = rd32(src + 32 + 4 * (uint64_t)y + 4);
        if (b < a || (a & 15) || (b & 15) || b > total - P || b - a < 16) return ORC_ECORRUPT;
        const uint8_t *p = src + P + a;
        uint64_t len = b - a;
        uint8_t *r = m + (uint64_t)y * W;
        if (p[0] == 0) {
            if (16 + (uint64_t)W > len) return ORC_ECORRUPT;
            memcpy(r, p + 16, (size_t)W);
        } else if (p[0] == 1) {
            uint64_t nrun = rd16(p + 2);
            if (nrun < 1 || nrun > (uint64_t)W || 4 + 3 * nrun > len) return ORC_ECORRUPT;
            uint64_t x = 0;
            for (uint64_t k = 0; k < nrun; k++) {
                uint64_t l = rd16(p + 4 + 2 * k);
                if (l < 1 || x + l > (uint64_t)W) return ORC_ECORRUPT;
                for (uint64_t j = 0; j < l; j++) r[x + j] = p[4 + 2 * nrun + k];
                x += l;
            }
            if (x != (uint64_t)W) return ORC_ECORRUPT;
        } else {
            return ORC_ECORRUPT;
        }
    }
    return ORC_OK;
}

/* ---------------- array helpers for the Python tests ---------------------- */
void orc_f32_to_f16_array(const float *in, int64_t n, uint16_t *out) {
    for (int64_t i = 0; i < n; i++) out[i] = orc_f32_to_f16(in[i]);
}
