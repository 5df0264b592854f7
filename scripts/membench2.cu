// membench2.cu — attainable HBM bandwidth by STORE PATH for the decode kernels'
// traffic mixes (experiment, not product).  Round-2 follow-up of membench.cu:
// that bench used one LDG.128 + plain STG.128 per thread and found 5.54 TB/s
// for KC's 1:4 read:write mix; this one asks whether another store path (.cs,
// 256-bit STG, TMA bulk stores from shared memory) or a TMA-fed input moves
// that ceiling.  GB/s = (bytes read + bytes written) / time, CUDA events,
// best of 5 after 2 warm-ups, 2 GiB of output per launch (>> L2).
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o membench2 scripts/membench2.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x)                                                                       \
    do {                                                                            \
        cudaError_t e = (x);                                                        \
        if (e != cudaSuccess) {                                                     \
            printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); \
            return 1;                                                               \
        }                                                                           \
    } while (0)

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

// ---- register-path kernels: in = 2 B per voxel, out = 4 planes x 2 B per voxel (KC shape)
// WR = number of output planes (1: 1:1 copy, 2: 1:2 (KD-like), 4: 1:4 (KC-like));
// ST: 0 plain STG.128, 1 STG.128.cs, 2 STG.256.cs (8 words per lane)
template <int WR, int ST>
__global__ void reg_mix(const uint4 *__restrict__ in, uint4 *__restrict__ out, size_t n_in) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    if (ST == 2) {  // each thread: 32 B in, WR x 32 B out
        for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; 2 * i + 1 < n_in; i += stride) {
            uint4 a = __ldcs(in + 2 * i), b = __ldcs(in + 2 * i + 1);
#pragma unroll
            for (int c = 0; c < WR; c++) {
                uint4 *p = out + (size_t)c * n_in + 2 * i;
                asm volatile("st.global.cs.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(a.x + c),
                             "r"(a.y), "r"(a.z), "r"(a.w), "r"(b.x), "r"(b.y), "r"(b.z), "r"(b.w)
                             : "memory");
            }
        }
        return;
    }
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_in; i += stride) {
        uint4 v = __ldcs(in + i);
#pragma unroll
        for (int c = 0; c < WR; c++) {
            uint4 w = make_uint4(v.x + c, v.y ^ c, v.z, v.w);
            if (ST == 0) out[(size_t)c * n_in + i] = w;
            else __stcs(out + (size_t)c * n_in + i, w);
        }
    }
}

// ---- TMA path: input tiles by cp.async.bulk (mbarrier ring), output either by
// STG.128.cs from registers (OUTTMA = 0) or staged in shared memory and written
// by cp.async.bulk s2g, one bulk copy per plane per tile (OUTTMA = 1).
// Tile = TV voxels = 2*TV input bytes; 256 threads; each thread handles TV/256 voxels.
constexpr int TV = 4096;           // voxels per tile
constexpr int TIN = 2 * TV;        // 8 KB input per tile
constexpr int NST = 4;             // input ring stages
template <int WR, int OUTTMA>
__global__ void __launch_bounds__(256) tma_mix(const uint8_t *__restrict__ in, uint8_t *__restrict__ out,
                                               size_t n_vox) {
    extern __shared__ __align__(128) uint8_t sm[];
    uint8_t *ring = sm;                                  // NST x TIN
    uint8_t *stage = sm + NST * TIN;                     // 2 x WR x TIN (OUTTMA)
    uint64_t *full = reinterpret_cast<uint64_t *>(sm + NST * TIN + (OUTTMA ? 2 * WR * TIN : 0));
    uint64_t *empty = full + NST;
    const int tid = threadIdx.x;
    const size_t ntiles = n_vox / TV;
    if (tid == 0) {
        for (int s = 0; s < NST; s++) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(full + s)));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 256;" ::"r"(sa(empty + s)));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    // tiles of this CTA: blockIdx.x, +gridDim.x, ...
    size_t first = blockIdx.x;
    int issued = 0;
    auto issue = [&](size_t t, int k) {  // k = sequence number
        const int s = k % NST;
        if (k >= NST) {  // wait until consumers released the stage
            const uint32_t ph = ((k / NST) - 1) & 1;
            asm volatile("{\n.reg .pred p;\nW1_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W1_%=;\n}\n" ::"r"(sa(empty + s)), "r"(ph) : "memory");
        }
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(full + s)), "r"(TIN) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         sa(ring + s * TIN)),
                     "l"(in + t * TIN), "r"(TIN), "r"(sa(full + s))
                     : "memory");
    };
    if (tid == 0)
        for (; issued < NST - 1 && first + (size_t)issued * gridDim.x < ntiles; issued++)
            issue(first + (size_t)issued * gridDim.x, issued);
    int k = 0;
    for (size_t t = first; t < ntiles; t += gridDim.x, k++) {
        if (tid == 0 && first + (size_t)issued * gridDim.x < ntiles) {
            issue(first + (size_t)issued * gridDim.x, issued);
            issued++;
        }
        const int s = k % NST;
        const uint32_t ph = (k / NST) & 1;
        asm volatile("{\n.reg .pred p;\nW2_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W2_%=;\n}\n" ::"r"(sa(full + s)), "r"(ph) : "memory");
        // each thread: 2 x 16 B of input (16 voxels) per tile
        uint4 v[TIN / 256 / 16];
#pragma unroll
        for (int j = 0; j < TIN / 256 / 16; j++)
            v[j] = *reinterpret_cast<const uint4 *>(ring + s * TIN + 16 * (tid + 256 * j));
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(empty + s)) : "memory");
        if (OUTTMA) {
            uint8_t *st = stage + (k & 1) * WR * TIN;
            if (tid == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
            __syncthreads();
#pragma unroll
            for (int c = 0; c < WR; c++)
#pragma unroll
                for (int j = 0; j < TIN / 256 / 16; j++)
                    *reinterpret_cast<uint4 *>(st + c * TIN + 16 * (tid + 256 * j)) =
                        make_uint4(v[j].x + c, v[j].y, v[j].z, v[j].w);
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncthreads();
            if (tid == 0) {
                for (int c = 0; c < WR; c++)
                    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(
                                     out + (size_t)c * n_vox * 2 + t * TIN),
                                 "r"(sa(st + c * TIN)), "r"(TIN)
                                 : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
        } else {
#pragma unroll
            for (int c = 0; c < WR; c++)
#pragma unroll
                for (int j = 0; j < TIN / 256 / 16; j++)
                    __stcs(reinterpret_cast<uint4 *>(out + (size_t)c * n_vox * 2 + t * TIN) + tid + 256 * j,
                           make_uint4(v[j].x + c, v[j].y, v[j].z, v[j].w));
        }
    }
    if (OUTTMA && tid == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// ---- write-only by TMA bulk store from a constant smem buffer (store-engine ceiling)
template <int CH>
__global__ void tma_write(uint8_t *__restrict__ out, size_t bytes) {
    extern __shared__ __align__(128) uint8_t sm[];
    if (threadIdx.x != 0) return;
    const size_t n = bytes / CH;
    int inflight = 0;
    for (size_t t = blockIdx.x; t < n; t += gridDim.x) {
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(out + t * CH), "r"(sa(sm)),
                     "r"(CH)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        if (++inflight > 6) asm volatile("cp.async.bulk.wait_group.read 6;" ::: "memory");
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
template <int ST>
__global__ void reg_write(uint4 *__restrict__ out, size_t n) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        uint4 w = make_uint4((uint32_t)i, 1, 2, 3);
        if (ST == 0) out[i] = w;
        else __stcs(out + i, w);
    }
}

template <typename F>
float timeit(F f, double bytes) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    f();
    f();
    float best = 1e30f;
    for (int r = 0; r < 5; r++) {
        cudaEventRecord(a);
        f();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    if (cudaGetLastError() != cudaSuccess) return -1.f;
    return (float)(bytes / (best * 1e-3) / 1e9);
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t out_bytes = (size_t)2 << 30;  // 2 GiB written per launch
    uint8_t *in, *out;
    CK(cudaMalloc(&in, out_bytes));
    CK(cudaMalloc(&out, out_bytes));
    CK(cudaMemset(in, 1, out_bytes));
    CK(cudaMemset(out, 0, out_bytes));
    printf("SMs %d\n", sms);
    // write-only
    {
        size_t n = out_bytes / 16;
        for (int occ : {4, 8}) {
            int g = sms * occ;
            printf("write-only STG.128     grid %4d: %6.0f GB/s\n", g,
                   timeit([&] { reg_write<0><<<g, 256>>>((uint4 *)out, n); }, (double)out_bytes));
            printf("write-only STG.128.cs  grid %4d: %6.0f GB/s\n", g,
                   timeit([&] { reg_write<1><<<g, 256>>>((uint4 *)out, n); }, (double)out_bytes));
        }
        cudaFuncSetAttribute(tma_write<16384>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16384);
        cudaFuncSetAttribute(tma_write<4096>, cudaFuncAttributeMaxDynamicSharedMemorySize, 4096);
        for (int occ : {1, 2, 4, 8}) {
            int g = sms * occ;
            printf("write-only TMA 16KB    grid %4d: %6.0f GB/s\n", g,
                   timeit([&] { tma_write<16384><<<g, 32, 16384>>>(out, out_bytes); }, (double)out_bytes));
            printf("write-only TMA 4KB     grid %4d: %6.0f GB/s\n", g,
                   timeit([&] { tma_write<4096><<<g, 32, 4096>>>(out, out_bytes); }, (double)out_bytes));
        }
    }
    // register-path mixes: WR planes, in = out_bytes / WR
    auto regs = [&](auto wr_tag, auto st_tag, const char *name) {
        constexpr int WR = decltype(wr_tag)::value, ST = decltype(st_tag)::value;
        size_t n_in = out_bytes / WR / 16;
        for (int occ : {4, 8}) {
            int g = sms * occ;
            printf("1:%d reg %-10s grid %4d: %6.0f GB/s\n", WR, name, g,
                   timeit([&] { reg_mix<WR, ST><<<g, 256>>>((const uint4 *)in, (uint4 *)out, n_in); },
                          (double)n_in * 16 * (1 + WR)));
        }
    };
    using I1 = std::integral_constant<int, 1>;
    using I2 = std::integral_constant<int, 2>;
    using I4 = std::integral_constant<int, 4>;
    using S0 = std::integral_constant<int, 0>;
    using S1 = std::integral_constant<int, 1>;
    using S2 = std::integral_constant<int, 2>;
    regs(I1{}, S0{}, "STG");
    regs(I1{}, S1{}, "STG.cs");
    regs(I2{}, S0{}, "STG");
    regs(I2{}, S1{}, "STG.cs");
    regs(I2{}, S2{}, "STG256.cs");
    regs(I4{}, S0{}, "STG");
    regs(I4{}, S1{}, "STG.cs");
    regs(I4{}, S2{}, "STG256.cs");
    // TMA-fed mixes
    auto tmas = [&](auto wr_tag, auto o_tag, const char *name) {
        constexpr int WR = decltype(wr_tag)::value, O = decltype(o_tag)::value;
        size_t n_vox = out_bytes / WR / 2;
        int smem = NST * TIN + (O ? 2 * WR * TIN : 0) + 2 * NST * 8;
        cudaFuncSetAttribute(tma_mix<WR, O>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        for (int occ : {1, 2, 3}) {
            int g = sms * occ;
            float r = timeit([&] { tma_mix<WR, O><<<g, 256, smem>>>(in, out, n_vox); }, (double)n_vox * 2 * (1 + WR));
            printf("1:%d tma-in %-12s grid %4d smem %6d: %6.0f GB/s\n", WR, name, g, smem, r);
        }
    };
    tmas(I1{}, S0{}, "STG.cs");
    tmas(I1{}, S1{}, "TMA-store");
    tmas(I2{}, S0{}, "STG.cs");
    tmas(I2{}, S1{}, "TMA-store");
    tmas(I4{}, S0{}, "STG.cs");
    tmas(I4{}, S1{}, "TMA-store");
    CK(cudaGetLastError());
    return 0;
}
