// membench.cu — attainable HBM bandwidth for the traffic mixes of the decode
// kernels (experiment, not product): read R bytes + write W bytes per unit with
// 16-B vector accesses, persistent grid.  Reports GB/s = (R+W)/t.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o membench scripts/membench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

// each thread: load 16 B of input, write WR x 16 B of output (WR planes like KC)
template <int WR>
__global__ void mix(const uint4 *__restrict__ in, uint4 *__restrict__ out, size_t n_in, size_t plane) {
    size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_in; i += stride) {
        uint4 v = in[i];
#pragma unroll
        for (int c = 0; c < WR; c++) {
            uint4 w = make_uint4(v.x + c, v.y ^ c, v.z, v.w);
            out[c * plane + i] = w;
        }
    }
}

template <int WR>
float run(const uint4 *in, uint4 *out, size_t n_in, int grid, int block) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int i = 0; i < 3; i++) mix<WR><<<grid, block>>>(in, out, n_in, n_in);
    cudaEventRecord(a);
    const int reps = 10;
    for (int i = 0; i < reps; i++) mix<WR><<<grid, block>>>(in, out, n_in, n_in);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    double bytes = (double)n_in * 16 * (1 + WR) * reps;
    return (float)(bytes / (ms * 1e-3) / 1e9);
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t n_in = (size_t)1 << 27;  // 2 GiB in
    uint4 *in, *out;
    cudaMalloc(&in, n_in * 16);
    cudaMalloc(&out, n_in * 16 * 4);
    cudaMemset(in, 1, n_in * 16);
    for (int occ : {2, 4, 8}) {
        int grid = sms * occ, block = 256;
        printf("grid %d: copy 1:1 %.0f GB/s | 1:2 %.0f | 1:4 %.0f GB/s\n", grid, run<1>(in, out, n_in, grid, block),
               run<2>(in, out, n_in, grid, block), run<4>(in, out, n_in, grid, block));
    }
    return 0;
}
