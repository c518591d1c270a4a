// Random-row gather throughput on B200 (the roofline of the graph kernels' per-edge gathers).
// Warp per "row group": 32 indices per coalesced load, L = row_bytes/16 lanes per row, 32/L rows per
// load step, UB steps in flight; sums into registers (no writes except one value per thread).
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

template <int L, int UB>
__global__ void gather(const float4* __restrict__ T, const int* __restrict__ idx, long n_edges, float* out) {
    constexpr int S = 32 / L;
    const int lane = threadIdx.x & 31, slot = lane / L, c = lane % L;
    long warp = (blockIdx.x * (long)blockDim.x + threadIdx.x) >> 5;
    long nwarps = ((long)gridDim.x * blockDim.x) >> 5;
    float4 acc = make_float4(0, 0, 0, 0);
    for (long base = warp * 32 * UB; base < n_edges; base += nwarps * 32 * UB) {
        int my[UB];
#pragma unroll
        for (int b = 0; b < UB; ++b) my[b] = (base + b * 32 + lane < n_edges) ? __ldcs(idx + base + b * 32 + lane) : 0;
#pragma unroll
        for (int b = 0; b < UB; ++b) {
            float4 v[L];
#pragma unroll
            for (int j = 0; j < L; ++j) {
                int u = __shfl_sync(0xffffffff, my[b], j * S + slot);
                v[j] = __ldg(T + (long)u * L + c);
            }
#pragma unroll
            for (int j = 0; j < L; ++j) { acc.x += v[j].x; acc.y += v[j].y; acc.z += v[j].z; acc.w += v[j].w; }
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc.x + acc.y + acc.z + acc.w;
}

template <int L, int UB>
double run(size_t table_bytes, long n_edges, int* d_idx, int blocks) {
    int rows = (int)(table_bytes / (16 * L));
    float4* T; float* out;
    cudaMalloc(&T, (size_t)rows * 16 * L);
    cudaMemset(T, 0, (size_t)rows * 16 * L);
    cudaMalloc(&out, (size_t)blocks * 256 * 4);
    // indices for this table size
    std::vector<int> h(n_edges);
    uint64_t x = 88172645463325252ull;
    for (long i = 0; i < n_edges; ++i) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; h[i] = (int)(x % rows); }
    cudaMemcpy(d_idx, h.data(), n_edges * 4, cudaMemcpyHostToDevice);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    gather<L, UB><<<blocks, 256>>>(T, d_idx, n_edges, out);
    cudaEventRecord(a);
    for (int r = 0; r < 5; ++r) gather<L, UB><<<blocks, 256>>>(T, d_idx, n_edges, out);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); ms /= 5;
    cudaFree(T); cudaFree(out);
    double bytes = (double)n_edges * (16.0 * L + 4);
    return bytes / (ms * 1e-3) / 1e9;
}

int main() {
    long n = 100 * 1000 * 1000;
    int* d_idx; cudaMalloc(&d_idx, n * 4);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    size_t sizes[] = {15u << 20, 60u << 20, 90u << 20, 200u << 20, 1u << 30};
    printf("table_MB  row_B  UB  GB/s(algorithmic: row+4B index per edge)\n");
    for (size_t s : sizes) {
        for (int blocks : {sms * 8, sms * 32}) {
            printf("%6zu  %4d  %d  %8.0f  (blocks %d)\n", s >> 20, 64, 4, run<4, 4>(s, n, d_idx, blocks), blocks);
            printf("%6zu  %4d  %d  %8.0f  (blocks %d)\n", s >> 20, 256, 2, run<16, 2>(s, n, d_idx, blocks), blocks);
            printf("%6zu  %4d  %d  %8.0f  (blocks %d)\n", s >> 20, 176, 2, run<11, 2>(s, n, d_idx, blocks), blocks);
        }
    }
    return 0;
}
