// abl.cu -- NEXT-4: baseline neighbour-access kernels for the PAPER.md §7.2 ablation (Fig. 12)
// on B200.  NOT product code: tools/ablation_sweep.py times these against the product kernel
// (seastar_gcn_fwd with no norms = plain sum of in-neighbour rows) on the Reddit-shaped graph.
//   abl_basic        one thread per destination row, edges then features sequential (the paper's "Basic")
//   abl_edge_atomic  one thread per (edge, feature): binary search of dst in indptr + atomicAdd (DGL/minigun, L397-L399)
//   abl_fa           feature-adaptive: one warp per row, lanes over float4 feature chunks, edges sequential, on
//                    a given row order (perm == NULL: the unsorted user order; else the degree-sorted order)
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_basic(int64_t N, const int32_t* __restrict__ ip, const int32_t* __restrict__ ix,
                        const float* __restrict__ X, int F, int64_t ld, float* __restrict__ Y) {
    const int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (v >= N) return;
    for (int f = 0; f < F; ++f) {
        float acc = 0.f;
        for (int e = ip[v]; e < ip[v + 1]; ++e) acc += X[(int64_t)ix[e] * ld + f];
        Y[v * ld + f] = acc;
    }
}

__global__ void k_edge_atomic(int64_t N, int64_t E, const int32_t* __restrict__ ip, const int32_t* __restrict__ ix,
                              const float* __restrict__ X, int F, int64_t ld, float* __restrict__ Y) {
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t >= E * F) return;
    const int64_t e = t / F;
    const int f = (int)(t % F);
    int64_t lo = 0, hi = N - 1;                      // last row with ip[row] <= e
    while (lo < hi) {
        const int64_t mid = (lo + hi + 1) >> 1;
        if (ip[mid] <= e) lo = mid; else hi = mid - 1;
    }
    atomicAdd(Y + lo * ld + f, X[(int64_t)ix[e] * ld + f]);
}

__global__ void k_fa(int64_t N, const int32_t* __restrict__ perm, const int32_t* __restrict__ off,
                     const int32_t* __restrict__ nbr, const float* __restrict__ X, int F, int64_t ld,
                     float* __restrict__ Y) {
    const int64_t row = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (row >= N) return;
    const int64_t v = perm ? perm[row] : row;
    const int beg = off[row], end = off[row + 1];
    const int C4 = (F + 3) / 4;
    for (int c = lane; c < C4; c += 32) {
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int e = beg; e < end; ++e) {
            const float4 x = __ldg(reinterpret_cast<const float4*>(X + (int64_t)nbr[e] * ld) + c);
            acc.x += x.x; acc.y += x.y; acc.z += x.z; acc.w += x.w;
        }
        reinterpret_cast<float4*>(Y + v * ld)[c] = acc;
    }
}

extern "C" {
int abl_basic(int64_t N, const int32_t* ip, const int32_t* ix, const float* X, int F, int64_t ld, float* Y, void* s) {
    k_basic<<<(unsigned)((N + 255) / 256), 256, 0, (cudaStream_t)s>>>(N, ip, ix, X, F, ld, Y);
    return (int)cudaGetLastError();
}
int abl_edge_atomic(int64_t N, int64_t E, const int32_t* ip, const int32_t* ix, const float* X, int F, int64_t ld,
                    float* Y, void* s) {
    cudaMemsetAsync(Y, 0, sizeof(float) * (size_t)N * ld, (cudaStream_t)s);
    const int64_t n = E * F;
    k_edge_atomic<<<(unsigned)((n + 255) / 256), 256, 0, (cudaStream_t)s>>>(N, E, ip, ix, X, F, ld, Y);
    return (int)cudaGetLastError();
}
int abl_fa(int64_t N, const int32_t* perm, const int32_t* off, const int32_t* nbr, const float* X, int F, int64_t ld,
           float* Y, void* s) {
    k_fa<<<(unsigned)((N * 32 + 255) / 256), 256, 0, (cudaStream_t)s>>>(N, perm, off, nbr, X, F, ld, Y);
    return (int)cudaGetLastError();
}
}
