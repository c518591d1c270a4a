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

// ------------------------------------------------------------------------------------------------------------------
// r2: the remaining §7.2 sweep columns
//   abl_slot   the product kernel's lane mapping (L = F/4 float4 lanes per edge slot, 32/L slots per warp, 4 gathers
//              in flight per lane, one warp per row) under three grid policies: 0 = oversubscribed (a warp per row,
//              the block scheduler balances), 1 = persistent (148 x 8 blocks, warps stride over rows), 2 = persistent
//              with an atomic row counter; hub = rows of degree >= 1024 get a CTA of 8 warps (contiguous slices,
//              warp-order merge) in the same launch
//   abl_tma    TMA tile::gather4: one lane per warp issues cp.async.bulk.tensor.2d ... gather4 for 4 neighbour rows
//              into an 8-stage shared-memory ring (mbarrier complete_tx), all lanes sum from shared memory
// ------------------------------------------------------------------------------------------------------------------
#include <cuda.h>

template <int L>
__device__ __forceinline__ void slot_rows(int beg, int end, const int32_t* __restrict__ nbr, const float* __restrict__ X,
                                          int64_t ld, float4& acc) {
    constexpr int S = 32 / L, UB = 4;
    const int lane = threadIdx.x & 31, slot = lane / L, c = lane % L;
    for (int base = beg; base < end; base += 32) {
        const int n = min(32, end - base);
        const int my = lane < n ? __ldcs(nbr + base + lane) : 0;
#pragma unroll
        for (int j0 = 0; j0 < L; j0 += UB) {
            if (j0 * S >= n) break;
            float4 v[UB];
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) {
                const int k = (j0 + jj) * S + slot;
                const int u = __shfl_sync(0xffffffffu, my, k & 31);
                v[jj] = (k < n && j0 + jj < L) ? __ldg(reinterpret_cast<const float4*>(X + (int64_t)u * ld) + c)
                                               : make_float4(0.f, 0.f, 0.f, 0.f);
            }
#pragma unroll
            for (int jj = 0; jj < UB; ++jj) { acc.x += v[jj].x; acc.y += v[jj].y; acc.z += v[jj].z; acc.w += v[jj].w; }
        }
    }
#pragma unroll
    for (int o = L; o < 32; o <<= 1) {
        acc.x += __shfl_xor_sync(0xffffffffu, acc.x, o); acc.y += __shfl_xor_sync(0xffffffffu, acc.y, o);
        acc.z += __shfl_xor_sync(0xffffffffu, acc.z, o); acc.w += __shfl_xor_sync(0xffffffffu, acc.w, o);
    }
}

template <int L>
__global__ void __launch_bounds__(256) k_slot(int64_t N, const int32_t* __restrict__ perm, const int32_t* __restrict__ off,
                                              const int32_t* __restrict__ nbr, const float* __restrict__ X, int64_t ld,
                                              float* __restrict__ Y, int mode, int64_t nhub, int* counter) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    if (nhub > 0 && (int64_t)blockIdx.x < nhub) {          // hub row: 8 warps, contiguous slices, warp-order merge
        __shared__ float4 red[8][32];
        const int64_t row = blockIdx.x;
        const int b = off[row], e = off[row + 1], len = e - b;
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        slot_rows<L>(b + (int)((int64_t)len * wib / 8), b + (int)((int64_t)len * (wib + 1) / 8), nbr, X, ld, acc);
        red[wib][lane] = acc;
        __syncthreads();
        if (wib == 0 && lane < L) {
            float4 t = red[0][lane];
            for (int w = 1; w < 8; ++w) { t.x += red[w][lane].x; t.y += red[w][lane].y; t.z += red[w][lane].z; t.w += red[w][lane].w; }
            reinterpret_cast<float4*>(Y + (int64_t)perm[row] * ld)[lane] = t;
        }
        return;
    }
    const int64_t wid = (int64_t)(blockIdx.x - nhub) * 8 + wib;
    const int64_t nw = (int64_t)(gridDim.x - nhub) * 8;
    int64_t row = nhub + wid;
    while (row < N) {
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        slot_rows<L>(off[row], off[row + 1], nbr, X, ld, acc);
        if (lane < L) reinterpret_cast<float4*>(Y + (int64_t)perm[row] * ld)[lane] = acc;
        if (mode == 0) break;
        if (mode == 1) row += nw;
        else {
            int r = 0;
            if (lane == 0) r = atomicAdd(counter, 1);
            row = nhub + nw + __shfl_sync(0xffffffffu, r, 0);
        }
    }
}

__device__ __forceinline__ uint32_t s32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

template <int C4>   // float4 chunks per row (F = 4 * C4), C4 | 32
__global__ void __launch_bounds__(256) k_tma_g4(int64_t N, const int32_t* __restrict__ perm, const int32_t* __restrict__ off,
                                                const int32_t* __restrict__ nbr, const __grid_constant__ CUtensorMap tm,
                                                float* __restrict__ Y, int64_t ld) {
    constexpr int D = 8;                                   // stages per warp (4 rows each)
    constexpr int SS = (4 * C4 < 8) ? 8 : 4 * C4;          // stage stride in float4: TMA destinations 128-B aligned
    extern __shared__ __align__(128) float4 ring[];        // [8 warps][D][SS]
    __shared__ __align__(8) uint64_t bar[8][D];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int64_t row = (int64_t)blockIdx.x * 8 + wib;
    float4* st = ring + (size_t)wib * D * SS;
    if (lane == 0)
        for (int i = 0; i < D; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(s32(&bar[wib][i])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncwarp();
    if (row >= N) return;
    const int beg = off[row], end = off[row + 1];
    const int ng = (end - beg + 3) / 4;
    auto issue = [&](int g) {                              // lane 0: gather rows 4g..4g+3 of the row's edges
        int u[4];
        for (int j = 0; j < 4; ++j) u[j] = beg + 4 * g + j < end ? __ldg(nbr + beg + 4 * g + j) : 0;
        uint64_t* b = &bar[wib][g % D];
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s32(b)), "r"(4 * C4 * 16) : "memory");
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
            ::"r"(s32(st + (g % D) * SS)), "l"(reinterpret_cast<uint64_t>(&tm)), "r"(0), "r"(u[0]), "r"(u[1]),
              "r"(u[2]), "r"(u[3]), "r"(s32(b)) : "memory");
    };
    if (lane == 0)
        for (int g = 0; g < D && g < ng; ++g) issue(g);
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int g = 0; g < ng; ++g) {
        const uint32_t a = s32(&bar[wib][g % D]), par = (g / D) & 1;
        asm volatile("{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}"
                     ::"r"(a), "r"(par) : "memory");
        const float4* s = st + (g % D) * SS;
#pragma unroll
        for (int k = 0; k < (4 * C4 + 31) / 32; ++k) {
            const int idx = lane + 32 * k;
            if (idx < 4 * C4 && beg + 4 * g + idx / C4 < end) {
                const float4 v = s[idx];
                acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
            }
        }
        __syncwarp();
        if (lane == 0 && g + D < ng) issue(g + D);
    }
    // lanes l, l + C4, l + 2 C4, ... hold partial sums of chunk l % C4
#pragma unroll
    for (int o = C4; o < 32; o <<= 1) {
        acc.x += __shfl_xor_sync(0xffffffffu, acc.x, o); acc.y += __shfl_xor_sync(0xffffffffu, acc.y, o);
        acc.z += __shfl_xor_sync(0xffffffffu, acc.z, o); acc.w += __shfl_xor_sync(0xffffffffu, acc.w, o);
    }
    if (lane < C4) reinterpret_cast<float4*>(Y + (int64_t)perm[row] * ld)[lane] = acc;
}

extern "C" {
int abl_slot(int64_t N, const int32_t* perm, const int32_t* off, const int32_t* nbr, const float* X, int F, int64_t ld,
             float* Y, int mode, int64_t nhub, int* counter, void* s) {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int64_t rest = N - nhub;
    int64_t blocks = mode == 0 ? (rest + 7) / 8 : (int64_t)sms * 8;
    if (mode == 2) cudaMemsetAsync(counter, 0, sizeof(int), (cudaStream_t)s);
    blocks += nhub;
    const int L = F / 4;
#define SL(LL) k_slot<LL><<<(unsigned)blocks, 256, 0, (cudaStream_t)s>>>(N, perm, off, nbr, X, ld, Y, mode, nhub, counter)
    switch (L) { case 1: SL(1); break; case 2: SL(2); break; case 4: SL(4); break; case 8: SL(8); break;
                 case 16: SL(16); break; default: SL(32); break; }
#undef SL
    return (int)cudaGetLastError();
}

int abl_tma(int64_t N, const int32_t* perm, const int32_t* off, const int32_t* nbr, const float* X, int F, int64_t ld,
            float* Y, void* s) {
    typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                            const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                            CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
    static Enc enc = nullptr;
    if (!enc) {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess) return -1;
        enc = reinterpret_cast<Enc>(p);
    }
    CUtensorMap tm;
    const cuuint64_t dims[2] = {(cuuint64_t)F, (cuuint64_t)N};
    const cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
    const cuuint32_t box[2] = {(cuuint32_t)F, 1};
    const cuuint32_t es[2] = {1, 1};
    CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(X), dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return 1000 + (int)r;
    const int C4 = F / 4;
    const size_t smem = (size_t)8 * 8 * (4 * C4 < 8 ? 8 : 4 * C4) * 16;
    const unsigned blocks = (unsigned)((N + 7) / 8);
#define TG(CC) do { cudaFuncSetAttribute(k_tma_g4<CC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); \
                    k_tma_g4<CC><<<blocks, 256, smem, (cudaStream_t)s>>>(N, perm, off, nbr, tm, Y, ld); } while (0)
    switch (C4) { case 1: TG(1); break; case 2: TG(2); break; case 4: TG(4); break; case 8: TG(8); break;
                  case 16: TG(16); break; case 32: TG(32); break; default: return -2; }
#undef TG
    return (int)cudaGetLastError();
}
}
