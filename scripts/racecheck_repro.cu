// racecheck_repro.cu — minimal reproducer for the compute-sanitizer racecheck
// reports on KD's input ring: a producer refills a shared
// slot by 1-D TMA after every consumer lane has read it and arrived on the
// slot's "empty" mbarrier, which the producer waits on (release/acquire).
// The same protocol is run in variants that add, one at a time, what KD does
// beyond KC's (racecheck-clean) key ring:
//   0  one producer thread, blocking try_wait on "empty", no cluster (KC-like)
//   1  as 0, launched as a cluster of 2 CTAs (KD needs it for st.async)
//   2  as 1, plus a 16-B st.async record on the slot's "full" barrier (KD's line record)
//   3  as 2, the producer polls "empty" with test_wait (KD's producer loop)
//   4  KD's protocol: a producer warp, lane k serving consumer warp k (two)
//   5  as 4, plus lines that take the whole ring (KD's RAW / oversize lines)
//   6  as 4 with a blocking try_wait per producer lane instead of test_wait
//   7  as 4 with each lane's test_wait issued while it is the only active lane
//   8  as 4 with one producer WARP per consumer (lane 0 of each producer warp)
// Every variant is correctly ordered by the PTX memory model (mbarrier
// arrive = release, try_wait/test_wait = acquire; the TMA write is issued after
// the acquire).  build: nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/rr scripts/racecheck_repro.cu
// run:   compute-sanitizer --tool racecheck /tmp/rr <variant>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

constexpr int kSlots = 2, kSlotBytes = 1024, kIters = 64;

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void expect_tx(uint64_t *b, uint32_t n) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void arrive(uint64_t *b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(b)) : "memory");
}
__device__ __forceinline__ void wait(uint64_t *b, uint32_t ph) {
    asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(
                     sa(b)),
                 "r"(ph)
                 : "memory");
}
__device__ __forceinline__ bool test(uint64_t *b, uint32_t ph) {
    uint32_t r;
    asm volatile("{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0, 1, 0, p;\n}\n"
                 : "=r"(r)
                 : "r"(sa(b)), "r"(ph)
                 : "memory");
    return r;
}
__device__ __forceinline__ void tma(void *d, const void *s, uint32_t n, uint64_t *b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(sa(d)),
                 "l"(s), "r"(n), "r"(sa(b))
                 : "memory");
}
__device__ __forceinline__ void st_async(void *d, uint4 v, uint64_t *b) {
    asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(sa(d)),
                 "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "r"(sa(b))
                 : "memory");
}

// V0..V3 as listed above (one consumer warp, one producer thread).  V4: KD's
// exact ring protocol, a producer WARP whose lane k serves consumer warp k (two
// consumer warps), test_wait polling with used/parity bits, st.async records,
// cluster launch.  V5: V4 plus "big" lines (every 4th) that take the whole ring:
// the producer waits for every slot, arms only the current slot's full barrier
// with both slots' bytes, the consumer releases every slot.
template <int V>
__global__ void ring(const uint8_t *__restrict__ src, uint32_t *__restrict__ out) {
    constexpr int NC = V >= 4 ? 2 : 1;  // consumer warps
    constexpr bool BLOCKING = V == 6;   // V6: V4 with a blocking try_wait per producer lane
    constexpr bool SERIAL = V == 7;     // V7: V4 with the lanes' empty-barrier tests taken one lane at a time
    __shared__ __align__(128) uint8_t slot[NC][kSlots][kSlotBytes];
    __shared__ __align__(16) uint4 rec[NC][kSlots];
    __shared__ uint64_t full[NC][kSlots], empty[NC][kSlots];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
        for (int c = 0; c < NC; c++)
            for (int i = 0; i < kSlots; i++) {
                mbar_init(&full[c][i], 1);
                mbar_init(&empty[c][i], 32);
            }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto is_big = [](int i) { return V == 5 && (i % 4) == 3; };
    if (V == 8 && warp >= NC) {  // one producer warp per consumer, lane 0
        if (lane != 0) return;
        const int c = warp - NC;
        uint32_t used = 0, par = 0;
        for (int i = 0, s = 0; i < kIters; i++, s = (s + 1) % kSlots) {
            if ((used >> s) & 1u) {
                while (!test(&empty[c][s], (par >> s) & 1u)) {
                }
            }
            expect_tx(&full[c][s], kSlotBytes + 16);
            st_async(&rec[c][s], make_uint4(i, 0, 0, 0), &full[c][s]);
            tma(slot[c][s], src + (size_t)i * kSlotBytes, kSlotBytes, &full[c][s]);
            par ^= (1u << s) & used;
            used |= 1u << s;
        }
        return;
    }
    if (warp == NC) {  // producer
        if (V < 4) {
            if (lane != 0) return;
            for (int i = 0; i < kIters; i++) {
                const int s = i % kSlots;
                if (i >= kSlots) {
                    const uint32_t ph = ((i / kSlots) - 1) & 1;
                    if (V >= 3) {
                        while (!test(&empty[0][s], ph)) {
                        }
                    } else {
                        wait(&empty[0][s], ph);
                    }
                }
                expect_tx(&full[0][s], kSlotBytes + (V >= 2 ? 16 : 0));
                if (V >= 2) st_async(&rec[0][s], make_uint4(i, 0, 0, 0), &full[0][s]);
                tma(slot[0][s], src + (size_t)i * kSlotBytes, kSlotBytes, &full[0][s]);
            }
            return;
        }
        // V4/V5: KD's producer loop, lane k for consumer k
        bool active = lane < NC;
        int i = 0, s = 0;
        uint32_t used = 0, par = 0;
        while (__any_sync(0xffffffffu, active)) {
            if (active) {
                const bool big = is_big(i);
                bool ready = true;
                for (int j = 0; j < kSlots; j++)
                    if ((big || j == s) && ((used >> j) & 1u)) {
                        if (BLOCKING) {
                            wait(&empty[lane][j], (par >> j) & 1u);
                        } else if (SERIAL) {
                            for (int k = 0; k < NC; k++)
                                if (k == lane) ready = ready && test(&empty[lane][j], (par >> j) & 1u);
                        } else {
                            ready = ready && test(&empty[lane][j], (par >> j) & 1u);
                        }
                    }
                if (ready) {
                    const uint32_t bytes = big ? kSlots * kSlotBytes : kSlotBytes;
                    expect_tx(&full[lane][s], bytes + 16);
                    st_async(&rec[lane][s], make_uint4(i, big, 0, 0), &full[lane][s]);
                    tma(big ? slot[lane][0] : slot[lane][s], src + (size_t)i * kSlotBytes, bytes, &full[lane][s]);
                    const uint32_t took = big ? (1u << kSlots) - 1u : 1u << s;
                    par ^= took & used;
                    used |= took;
                    s = (s + 1) % kSlots;
                    active = ++i < kIters;
                }
            }
        }
        return;
    }
    uint32_t acc = 0;  // consumer warp `warp`
    uint32_t fph = 0;
    for (int i = 0; i < kIters; i++) {
        const int s = i % kSlots;
        wait(&full[warp][s], (fph >> s) & 1u);
        fph ^= 1u << s;
        const bool big = V >= 2 ? rec[warp][s].y != 0 : false;
        const uint32_t *w = reinterpret_cast<const uint32_t *>(big ? slot[warp][0] : slot[warp][s]);
        const int nw = (big ? kSlots : 1) * kSlotBytes / 4;
        for (int k = lane; k < nw; k += 32) acc += w[k];
        if (V >= 2) acc += rec[warp][s].x;
        __syncwarp();
        if (big) {
            for (int j = 0; j < kSlots; j++) arrive(&empty[warp][j]);
        } else {
            arrive(&empty[warp][s]);
        }
    }
    out[blockIdx.x * 64 + warp * 32 + lane] = acc;
}

int main(int argc, char **argv) {
    const int v = argc > 1 ? atoi(argv[1]) : 0;
    uint8_t *src;
    uint32_t *out;
    cudaMalloc(&src, (size_t)(kIters + kSlots) * kSlotBytes);
    cudaMemset(src, 1, (size_t)(kIters + kSlots) * kSlotBytes);
    cudaMalloc(&out, 2 * 64 * 4);
    cudaMemset(out, 0, 2 * 64 * 4);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2);
    cfg.blockDim = dim3(v == 8 ? 128 : (v >= 4 ? 96 : 64));
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 2;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = v >= 1 ? 1 : 0;
    cudaError_t e = v == 0   ? cudaLaunchKernelEx(&cfg, ring<0>, (const uint8_t *)src, out)
                    : v == 1 ? cudaLaunchKernelEx(&cfg, ring<1>, (const uint8_t *)src, out)
                    : v == 2 ? cudaLaunchKernelEx(&cfg, ring<2>, (const uint8_t *)src, out)
                    : v == 3 ? cudaLaunchKernelEx(&cfg, ring<3>, (const uint8_t *)src, out)
                    : v == 4 ? cudaLaunchKernelEx(&cfg, ring<4>, (const uint8_t *)src, out)
                    : v == 5 ? cudaLaunchKernelEx(&cfg, ring<5>, (const uint8_t *)src, out)
                    : v == 6 ? cudaLaunchKernelEx(&cfg, ring<6>, (const uint8_t *)src, out)
                    : v == 7 ? cudaLaunchKernelEx(&cfg, ring<7>, (const uint8_t *)src, out)
                             : cudaLaunchKernelEx(&cfg, ring<8>, (const uint8_t *)src, out);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    uint32_t h[128];
    cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
    uint64_t sum = 0;
    for (int i = 0; i < 128; i++) sum += h[i];
    printf("variant %d: %s, checksum %llu\n", v, cudaGetErrorString(e), (unsigned long long)sum);
    return e == cudaSuccess ? 0 : 1;
}
