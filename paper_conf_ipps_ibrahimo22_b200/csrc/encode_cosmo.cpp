// encode_cosmo.cpp — host CosmoFlow LUT encoder (step b.1 of PAPER.md Fig. 1,
// P:32), FORMAT.md 1.3.
//
// PAPER.md §V.B: the number of unique values per 128^3 sample is a
// few hundred and the four redshifts are coupled, so the distinct 4-groups
// (tens of thousands) index a per-sample lookup table; §VI: keys of
// 1 or 2 bytes, 8-byte lookup values.  Groups are hashed in one pass (open
// addressing), ordered by descending frequency (hot groups first — the GPU
// stages that prefix in shared memory), and keys written in a second pass.
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <functional>
#include <vector>

#include "spp.h"
#include "spp_format.h"

namespace {

using spp::round_up16;

inline void put16(uint8_t *p, uint16_t v) { memcpy(p, &v, 2); }
inline void put32(uint8_t *p, uint32_t v) { memcpy(p, &v, 4); }
inline void put64(uint8_t *p, uint64_t v) { memcpy(p, &v, 8); }

// Open-addressing hash set of 64-bit tuples -> dense slot ids.
struct GroupTable {
    std::vector<uint64_t> keys;
    std::vector<uint32_t> slot;  // slot id + 1 (0 = empty)
    std::vector<uint64_t> tuple_of;
    std::vector<int64_t> freq;
    uint64_t mask = 0;

    void reset(size_t expect) {
        size_t cap = 1024;
        while (cap < 2 * expect) cap <<= 1;
        keys.assign(cap, 0);
        slot.assign(cap, 0);
        mask = cap - 1;
        tuple_of.clear();
        freq.clear();
    }
    static uint64_t hash(uint64_t x) {
        x ^= x >> 33;
        x *= 0xff51afd7ed558ccdULL;
        x ^= x >> 33;
        x *= 0xc4ceb9fe1a85ec53ULL;
        x ^= x >> 33;
        return x;
    }
    void grow() {
        std::vector<uint64_t> ok;
        std::vector<uint32_t> os;
        ok.swap(keys);
        os.swap(slot);
        size_t cap = ok.size() * 2;
        keys.assign(cap, 0);
        slot.assign(cap, 0);
        mask = cap - 1;
        for (size_t i = 0; i < ok.size(); i++) {
            if (!os[i]) continue;
            uint64_t h = hash(ok[i]) & mask;
            while (slot[h]) h = (h + 1) & mask;
            keys[h] = ok[i];
            slot[h] = os[i];
        }
    }
    uint32_t insert(uint64_t t) {
        uint64_t h = hash(t) & mask;
        while (slot[h]) {
            if (keys[h] == t) {
                uint32_t s = slot[h] - 1;
                freq[s]++;
                return s;
            }
            h = (h + 1) & mask;
        }
        uint32_t s = (uint32_t)tuple_of.size();
        keys[h] = t;
        slot[h] = s + 1;
        tuple_of.push_back(t);
        freq.push_back(1);
        if (tuple_of.size() * 2 > keys.size()) grow();
        return s;
    }
};

// FORMAT.md 1.5: eidx u32[nb+1] + low u8[Nt] + escaped u16[n_esc], 16-B sections
uint64_t escaped_key_bytes(int64_t Nt, int64_t n_esc) {
    const uint64_t nb = ((uint64_t)Nt + 255) / 256;
    return round_up16(4 * (nb + 1)) + round_up16((uint64_t)Nt) + round_up16(2 * (uint64_t)n_esc);
}

struct Slab {
    int z0, z1;
    int64_t G, n_esc;
    int kw;
    uint64_t lut_off, keys_off;
    std::vector<uint64_t> lut;       // ordered 4-tuples (hot first)
    std::vector<uint32_t> key_of_slot;
};

struct Ctx {
    const uint64_t *tup;
    int64_t plane;
    GroupTable tab;
    std::vector<uint32_t> vslot;     // per voxel slot (for the slab being built)
};

int64_t count_groups(Ctx &c, int z0, int z1) {
    int64_t n = (int64_t)(z1 - z0) * c.plane;
    c.tab.reset(std::min<int64_t>(n, 1 << 17));
    const uint64_t *t = c.tup + (int64_t)z0 * c.plane;
    for (int64_t v = 0; v < n; v++) c.tab.insert(t[v]);
    return (int64_t)c.tab.tuple_of.size();
}

void split(Ctx &c, int z0, int z1, std::vector<std::pair<int, int>> &out) {
    int64_t G = count_groups(c, z0, z1);
    if (G > spp::cosmo::kMaxG2 && z1 - z0 > 1) {
        int mid = z0 + (z1 - z0) / 2;
        split(c, z0, mid, out);
        split(c, mid, z1, out);
        return;
    }
    out.push_back({z0, z1});
}

// Exact encoded bytes of [z0, z1) as ONE slab (FORMAT.md 1.3 steps 3 and 5):
// its 32-B slab-table entry + LUT + keys, or the RAW planes of the escape.
uint64_t slab_cost(int64_t G, int64_t Nt) {
    const int kw = G == 1 ? 0 : (G <= spp::cosmo::kMaxG1 ? 1 : 2);
    if (G > spp::cosmo::kMaxG2 || 8 * G + kw * Nt >= 8 * Nt)
        return spp::cosmo::kSlabBytes + round_up16(8ull * (uint64_t)Nt);
    return spp::cosmo::kSlabBytes + round_up16(8ull * (uint64_t)G) +
           (kw ? round_up16((uint64_t)kw * (uint64_t)Nt) : 0);
}

// FORMAT.md 1.4 localized tables ("localized lookup tables", P:100
// "multiple lookup tables", P:106 1-byte keys): the z-partition of [z0, z1)
// into dyadic slabs (same halving as 1.3) with the fewest encoded bytes; a
// slab is kept whole unless splitting is strictly smaller.  Leaves appended
// in z order; returns the bytes of the chosen partition.
uint64_t split_localized(Ctx &c, int z0, int z1, std::vector<std::pair<int, int>> &out) {
    const int64_t G = count_groups(c, z0, z1);
    const uint64_t whole = slab_cost(G, (int64_t)(z1 - z0) * c.plane);
    if (z1 - z0 == 1) {
        out.push_back({z0, z1});
        return whole;
    }
    const int mid = z0 + (z1 - z0) / 2;
    std::vector<std::pair<int, int>> parts;
    const uint64_t halves = split_localized(c, z0, mid, parts) + split_localized(c, mid, z1, parts);
    if (halves < whole) {
        out.insert(out.end(), parts.begin(), parts.end());
        return halves;
    }
    out.push_back({z0, z1});
    return whole;
}

}  // namespace

extern "C" size_t spp_cosmo_max_encoded_size(int C, int D, int H, int W) {
    if (C != 4 || D < 1 || H < 1 || W < 1) return 0;
    uint64_t N = (uint64_t)D * H * W;
    return (size_t)(spp::kHeaderBytes + round_up16(2ull * spp::cosmo::kMaxU) +
                    round_up16(32ull * (uint64_t)D) + 8 * N + 16ull * (uint64_t)D + 64);
}

extern "C" spp_status spp_encode_cosmo(const int16_t *counts, int C, int D, int H, int W, void *dst,
                                       size_t dst_capacity, size_t *encoded_size) {
    return spp_encode_cosmo_ex(counts, C, D, H, W, nullptr, dst, dst_capacity, encoded_size);
}

extern "C" spp_status spp_encode_cosmo_ex(const int16_t *counts, int C, int D, int H, int W,
                                          const spp_cosmo_params *params, void *dst, size_t dst_capacity,
                                          size_t *encoded_size) {
    const int localize = params ? params->localize : 0;
    const int escape = params ? params->escape_keys : 0;
    if ((localize != 0 && localize != 1) || (escape != 0 && escape != 1)) return SPP_ERR_INVALID_ARG;
    if (!counts || !encoded_size || C != 4 || D < 1 || H < 1 || W < 1 || D > 65535 || H > 65535 ||
        W > 65535)
        return SPP_ERR_INVALID_ARG;
    const int64_t plane = (int64_t)H * W, N = (int64_t)D * plane;
    // 1. unique values U (ascending) and value -> index
    std::vector<uint8_t> present(32768, 0);
    for (int64_t i = 0; i < 4 * N; i++) {
        int16_t v = counts[i];
        if (v < 0) return SPP_ERR_INVALID_ARG;
        present[(uint16_t)v] = 1;
    }
    std::vector<uint16_t> idx_of(32768, 0);
    std::vector<int16_t> U;
    for (int v = 0; v < 32768; v++)
        if (present[v]) {
            idx_of[v] = (uint16_t)U.size();
            U.push_back((int16_t)v);
        }
    // 2. packed 4-tuples of U-indices (lexicographic order == numeric order)
    std::vector<uint64_t> tup((size_t)N);
    const int16_t *c0 = counts, *c1 = counts + N, *c2 = counts + 2 * N, *c3 = counts + 3 * N;
    for (int64_t v = 0; v < N; v++)
        tup[v] = ((uint64_t)idx_of[c0[v]] << 48) | ((uint64_t)idx_of[c1[v]] << 32) |
                 ((uint64_t)idx_of[c2[v]] << 16) | (uint64_t)idx_of[c3[v]];
    Ctx ctx{tup.data(), plane, {}, {}};
    std::vector<std::pair<int, int>> ranges;
    if (localize)
        split_localized(ctx, 0, D, ranges);
    else
        split(ctx, 0, D, ranges);

    // 3. per slab: groups ordered by (freq desc, tuple asc), key width, layout
    const int T = (int)ranges.size();
    std::vector<Slab> slabs(T);
    uint64_t off = spp::kHeaderBytes;
    const uint64_t U_off = off;
    off = round_up16(off + 2 * U.size());
    const uint64_t slab_off = off;
    off = round_up16(off + (uint64_t)spp::cosmo::kSlabBytes * T);
    for (int t = 0; t < T; t++) {
        Slab &s = slabs[t];
        s.z0 = ranges[t].first;
        s.z1 = ranges[t].second;
        const int64_t Nt = (int64_t)(s.z1 - s.z0) * plane;
        count_groups(ctx, s.z0, s.z1);
        GroupTable &tab = ctx.tab;
        s.G = (int64_t)tab.tuple_of.size();
        s.kw = s.G == 1 ? 0 : (s.G <= spp::cosmo::kMaxG1 ? 1 : 2);
        if (s.G > spp::cosmo::kMaxG2 || 8 * s.G + s.kw * Nt >= 8 * Nt) s.kw = spp::cosmo::kRawSlab;
        s.n_esc = 0;
        if (escape && s.kw == 2) {
            // FORMAT.md 1.5: escaped 1-byte keys when smaller (keys >= 255 go to a u16 list)
            std::vector<int64_t> f(tab.freq.begin(), tab.freq.end());
            const size_t top = std::min<size_t>(255, f.size());
            std::partial_sort(f.begin(), f.begin() + top, f.end(), std::greater<int64_t>());
            int64_t hot = 0;
            for (size_t k = 0; k < top; k++) hot += f[k];
            s.n_esc = Nt - hot;
            if (escaped_key_bytes(Nt, s.n_esc) < round_up16(2ull * (uint64_t)Nt)) s.kw = spp::cosmo::kEscaped;
        }
        if (s.kw != spp::cosmo::kRawSlab) {
            std::vector<uint32_t> order((size_t)s.G);
            for (uint32_t i = 0; i < (uint32_t)s.G; i++) order[i] = i;
            std::sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) {
                if (tab.freq[a] != tab.freq[b]) return tab.freq[a] > tab.freq[b];
                return tab.tuple_of[a] < tab.tuple_of[b];
            });
            s.lut.resize((size_t)s.G);
            s.key_of_slot.resize((size_t)s.G);
            for (uint32_t k = 0; k < (uint32_t)s.G; k++) {
                s.lut[k] = tab.tuple_of[order[k]];
                s.key_of_slot[order[k]] = k;
            }
            s.lut_off = off;
            off = round_up16(off + 8 * (uint64_t)s.G);
        } else {
            s.G = 0;
            s.lut_off = 0;
        }
        if (s.kw == spp::cosmo::kEscaped) {
            s.keys_off = off;
            off += escaped_key_bytes(Nt, s.n_esc);
        } else if (s.kw != 0) {
            s.keys_off = off;
            off = round_up16(off + (uint64_t)(s.kw == spp::cosmo::kRawSlab ? 8 : s.kw) * (uint64_t)Nt);
        } else {
            s.keys_off = 0;
        }
    }
    const uint64_t total = off;
    *encoded_size = (size_t)total;
    if (!dst || dst_capacity < total) return SPP_ERR_BUFFER_TOO_SMALL;

    // 4. write
    uint8_t *out = (uint8_t *)dst;
    memset(out, 0, (size_t)total);
    put32(out, spp::kCosmoMagic);
    put16(out + 4, spp::kVersion);
    put16(out + spp::cosmo::kC, 4);
    put16(out + spp::cosmo::kD, (uint16_t)D);
    put16(out + spp::cosmo::kH, (uint16_t)H);
    put16(out + spp::cosmo::kW, (uint16_t)W);
    put32(out + spp::cosmo::kNU, (uint32_t)U.size());
    put32(out + spp::cosmo::kNSlab, (uint32_t)T);
    put64(out + spp::cosmo::kUOff, U_off);
    put64(out + spp::cosmo::kSlabOff, slab_off);
    put64(out + spp::cosmo::kTotal, total);
    memcpy(out + U_off, U.data(), 2 * U.size());
    for (int t = 0; t < T; t++) {
        Slab &s = slabs[t];
        uint8_t *st = out + slab_off + (uint64_t)spp::cosmo::kSlabBytes * t;
        put32(st, (uint32_t)s.z0);
        put32(st + 4, (uint32_t)s.z1);
        put32(st + 8, (uint32_t)s.G);
        st[12] = (uint8_t)s.kw;
        put64(st + 16, s.lut_off);
        put64(st + 24, s.keys_off);
        const int64_t Nt = (int64_t)(s.z1 - s.z0) * plane;
        const int64_t base = (int64_t)s.z0 * plane;
        if (s.kw == spp::cosmo::kRawSlab) {
            uint16_t *raw = (uint16_t *)(out + s.keys_off);
            for (int c = 0; c < 4; c++) {
                const int16_t *src = counts + (int64_t)c * N + base;
                for (int64_t v = 0; v < Nt; v++) raw[(int64_t)c * Nt + v] = idx_of[src[v]];
            }
            continue;
        }
        uint16_t *lut = (uint16_t *)(out + s.lut_off);
        for (int64_t k = 0; k < s.G; k++)
            for (int c = 0; c < 4; c++) lut[4 * k + c] = (uint16_t)(s.lut[k] >> (16 * (3 - c)));
        if (s.kw == 0) continue;
        // re-hash this slab to map voxels -> slots (slot ids are insertion order,
        // identical to the pass that built key_of_slot)
        count_groups(ctx, s.z0, s.z1);
        GroupTable &tab = ctx.tab;
        const uint64_t *tt = tup.data() + base;
        if (s.kw == 1) {
            uint8_t *keys = out + s.keys_off;
            for (int64_t v = 0; v < Nt; v++) {
                uint64_t h = GroupTable::hash(tt[v]) & tab.mask;
                while (tab.keys[h] != tt[v]) h = (h + 1) & tab.mask;
                keys[v] = (uint8_t)s.key_of_slot[tab.slot[h] - 1];
            }
        } else if (s.kw == 2) {
            uint16_t *keys = (uint16_t *)(out + s.keys_off);
            for (int64_t v = 0; v < Nt; v++) {
                uint64_t h = GroupTable::hash(tt[v]) & tab.mask;
                while (tab.keys[h] != tt[v]) h = (h + 1) & tab.mask;
                keys[v] = (uint16_t)s.key_of_slot[tab.slot[h] - 1];
            }
        } else {  // FORMAT.md 1.5 escaped keys
            const uint64_t nb = ((uint64_t)Nt + 255) / 256;
            uint32_t *eidx = (uint32_t *)(out + s.keys_off);
            uint8_t *low = out + s.keys_off + round_up16(4 * (nb + 1));
            uint16_t *esc = (uint16_t *)(low + round_up16((uint64_t)Nt));
            uint32_t seen = 0;
            for (int64_t v = 0; v < Nt; v++) {
                if ((v & 255) == 0) eidx[v >> 8] = seen;
                uint64_t h = GroupTable::hash(tt[v]) & tab.mask;
                while (tab.keys[h] != tt[v]) h = (h + 1) & tab.mask;
                const uint32_t k = s.key_of_slot[tab.slot[h] - 1];
                low[v] = (uint8_t)(k < 255 ? k : 255);
                if (k >= 255) esc[seen++] = (uint16_t)k;
            }
            eidx[nb] = seen;
        }
    }
    return SPP_OK;
}
