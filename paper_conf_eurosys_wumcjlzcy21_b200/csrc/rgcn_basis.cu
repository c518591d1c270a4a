// rgcn_basis.cu -- NEXT-2: R-GCN as the paper ran it (Table 2 L485 and Table 3:
// aifb / mutag / bgs with a featureless input layer; hierarchical per-type aggregation §6.3.5
// L465-L475).  Layer of [53] with basis decomposition, reading #26:
//   W_r = sum_b a[r,b] V_b,  featureless input h_u = one-hot(u)  =>  h_u W_r = sum_b a[r,b] V[u,b,:].
//
// B200 mapping (V is [N, B*F], one contiguous row of B*F floats per vertex):
//   forward  (FWD CSR, warp per destination row): every edge gathers the source's whole V row as
//     B*F/4 float4 chunks spread over the 32 lanes.  Because 32 is a multiple of F/4, lane l always
//     holds feature slice f4 = l % (F/4) (of bases b = l/(F/4) + 32/(F/4)*i), so the per-edge basis
//     combination sum_b a[type,b] V[u,b,f4] is accumulated into ONE float4 per lane; a fixed xor tree
//     over the lanes sharing f4 finishes the row.  a is staged in shared memory; no atomics.
//   dV (REV CSR, warp per source row u): dV[u,b,:] = sum_{e in out(u)} norm_e a[type_e,b] dA[dst_e,:];
//     lanes own the (b, f4) chunks of the output row, every edge is ONE broadcast 16-byte load of
//     dA[dst_e, f4] per lane, no cross-lane reduction, no atomics.
//   da (type-major view, warp per task of one type): da[r,b] = sum_{e: type r} norm_e <V[src_e,b,:], dA[dst_e,:]>;
//     each task keeps B partial sums in registers, writes them once, and the per-type sum over tasks
//     runs over the tasks in a fixed order in fp64 (seg_reduce_cols; deterministic).
// The dense output layer uses W_r = sum_b a[r,b] V_b materialised by seastar_basis_combine and the
// staged R-GCN kernel of rgcn.cu.
#include "common.cuh"

namespace seastar {

struct BasisFwdArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr; const int32_t* typ;
    const int32_t* eid; const float* norm; const float* norm_user;
    int64_t row_begin, row_end, vbase;
    const float* V; int64_t ldv;      // [N, B*F] (gathered by source id)
    const float* a;                    // [R, B]
    int R, B, F4;
    const float* loop; int64_t ldl;   // [n_loc, F] self-loop addend or nullptr
    const float* bias; int act;
    float* Y; int64_t ldy;
};

__device__ __forceinline__ void fma4(float4& acc, float c, const float4& x) {
    acc.x = fmaf(c, x.x, acc.x); acc.y = fmaf(c, x.y, acc.y);
    acc.z = fmaf(c, x.z, acc.z); acc.w = fmaf(c, x.w, acc.w);
}

__device__ __forceinline__ void stage_coeffs(const float* __restrict__ a, int n, float* as) {
    for (int i = threadIdx.x; i < n; i += blockDim.x) as[i] = __ldg(a + i);
}

// One edge of the forward: gather V[u] (NI float4 per lane) and accumulate sum_b a[t,b] w V[u,b,f4].
template <int F4, int NI>
__device__ __forceinline__ void basis_fwd_edge(const BasisFwdArgs& p, const float* as, int lane, int nch,
                                               const int (&bi)[NI], int u, int t, float w, float4& acc) {
    const float* vp = p.V + (int64_t)u * p.ldv + 4 * lane;
    const float* at = as + t * p.B;
    float4 x[NI];
#pragma unroll
    for (int i = 0; i < NI; ++i)
        if (lane + 32 * i < nch) x[i] = ldg4(vp + 128 * i);
#pragma unroll
    for (int i = 0; i < NI; ++i)
        if (lane + 32 * i < nch) fma4(acc, w * at[bi[i]], x[i]);
}

// sum the lanes sharing f4 (fixed xor tree); afterwards lanes < F4 hold the row slice 4*lane..4*lane+3
template <int F4>
__device__ __forceinline__ void reduce_f4(float4& acc) {
#pragma unroll
    for (int o = F4; o < 32; o <<= 1) {
        acc.x += __shfl_xor_sync(0xffffffffu, acc.x, o);
        acc.y += __shfl_xor_sync(0xffffffffu, acc.y, o);
        acc.z += __shfl_xor_sync(0xffffffffu, acc.z, o);
        acc.w += __shfl_xor_sync(0xffffffffu, acc.w, o);
    }
}

__device__ __forceinline__ void basis_fwd_epilogue(const BasisFwdArgs& p, int64_t v, int l4, float4 acc) {
    float z[4] = {acc.x, acc.y, acc.z, acc.w};
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int f = 4 * l4 + q;
        if (p.loop) z[q] += __ldg(p.loop + v * p.ldl + f);
        if (p.bias) z[q] += __ldg(p.bias + f);
        z[q] = act_apply(p.act, z[q]);
    }
    *reinterpret_cast<float4*>(p.Y + v * p.ldy + 4 * l4) = make_float4(z[0], z[1], z[2], z[3]);
}

__device__ __forceinline__ float edge_weight(const float* norm_user, const int32_t* eid, const float* norm, int k) {
    return norm_user ? __ldg(norm_user + __ldg(eid + k)) : __ldg(norm + k);
}

// rows with in-degree < 32: one warp per row, persistent grid (a staged once per CTA).
// NI = chunks per lane (pow2 >= B*F4/32); lane l handles chunk c = l + 32 i (< B*F4), basis c / F4.
template <int F4, int NI>
__global__ void __launch_bounds__(256) k_basis_fwd_w(const BasisFwdArgs p) {
    extern __shared__ float as[];
    stage_coeffs(p.a, p.R * p.B, as);
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int nch = p.B * F4;
    int bi[NI];
#pragma unroll
    for (int i = 0; i < NI; ++i) bi[i] = (lane + 32 * i) / F4;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t row = p.row_begin + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5); row < p.row_end;
         row += nw) {
        const int beg = __ldg(p.off + row), end = __ldg(p.off + row + 1);
        const int64_t v = (int64_t)__ldg(p.perm + row) - p.vbase;
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int base = beg; base < end; base += 32) {
            const int n = min(32, end - base);
            int my_u = 0, my_t = 0;
            float my_w = 0.f;
            if (lane < n) {
                my_u = __ldcs(p.nbr + base + lane);
                my_t = __ldcs(p.typ + base + lane);
                my_w = edge_weight(p.norm_user, p.eid, p.norm, base + lane);
            }
            for (int j = 0; j < n; ++j)
                basis_fwd_edge<F4, NI>(p, as, lane, nch, bi, __shfl_sync(0xffffffffu, my_u, j),
                                       __shfl_sync(0xffffffffu, my_t, j), __shfl_sync(0xffffffffu, my_w, j), acc);
        }
        reduce_f4<F4>(acc);
        if (lane < F4) basis_fwd_epilogue(p, v, lane, acc);
    }
}

// rows with in-degree >= 32: WARPS warps per row (persistent over rows).  The CTA stages the metadata of
// 32*WARPS edges in shared memory and warp w takes edges w, w + WARPS, ...; per-warp results are
// merged in warp order (deterministic).  Long rows no longer serialise on one warp's load latency.
template <int F4, int NI, int WARPS>
__global__ void __launch_bounds__(32 * WARPS) k_basis_fwd_c(const BasisFwdArgs p) {
    constexpr int TB = 32 * WARPS;
    extern __shared__ float smem[];
    float* as = smem;
    int* su = reinterpret_cast<int*>(smem + p.R * p.B);
    int* st = su + TB;
    float* sw = reinterpret_cast<float*>(st + TB);
    float4* red = reinterpret_cast<float4*>(sw + TB + 4);   // [WARPS][F4]; +4 floats keep 16B alignment room
    red = reinterpret_cast<float4*>((reinterpret_cast<uintptr_t>(red) + 15) & ~uintptr_t(15));
    stage_coeffs(p.a, p.R * p.B, as);
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int nch = p.B * F4;
    int bi[NI];
#pragma unroll
    for (int i = 0; i < NI; ++i) bi[i] = (lane + 32 * i) / F4;
    for (int64_t row = p.row_begin + blockIdx.x; row < p.row_end; row += gridDim.x) {
        const int beg = __ldg(p.off + row), end = __ldg(p.off + row + 1);
        const int64_t v = (int64_t)__ldg(p.perm + row) - p.vbase;
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int base = beg; base < end; base += TB) {
            const int n = min(TB, end - base);
            if ((int)threadIdx.x < n) {
                su[threadIdx.x] = __ldcs(p.nbr + base + threadIdx.x);
                st[threadIdx.x] = __ldcs(p.typ + base + threadIdx.x);
                sw[threadIdx.x] = edge_weight(p.norm_user, p.eid, p.norm, base + threadIdx.x);
            }
            __syncthreads();
            for (int j = warp; j < n; j += WARPS) basis_fwd_edge<F4, NI>(p, as, lane, nch, bi, su[j], st[j], sw[j], acc);
            __syncthreads();
        }
        reduce_f4<F4>(acc);
        if (lane < F4) red[warp * F4 + lane] = acc;
        __syncthreads();
        if (warp == 0 && lane < F4) {
            float4 t = red[lane];
#pragma unroll 1
            for (int w = 1; w < WARPS; ++w) {
                const float4 r = red[w * F4 + lane];
                t.x += r.x; t.y += r.y; t.z += r.z; t.w += r.w;
            }
            basis_fwd_epilogue(p, v, lane, t);
        }
        __syncthreads();
    }
}

struct BasisDvArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr; const int32_t* typ;
    const int32_t* eid; const float* norm; const float* norm_user;
    int64_t row_begin, row_end, vbase;
    const float* dA; int64_t ldd;     // [N, F] gathered by destination id
    const float* a;
    int R, B, F4;
    float* dV; int64_t ldv;           // [n_loc, B*F]
};

// EB edges at once: EB broadcast loads of dA[dst, f4] in flight, then the NI x EB FMAs
template <int F4, int NI, int EB>
__device__ __forceinline__ void basis_dv_edges(const BasisDvArgs& p, const float* as, int lane, int nch, int f4,
                                               const int (&bi)[NI], const int (&vv)[EB], const int (&tt)[EB],
                                               const float (&ww)[EB], float4 (&acc)[NI]) {
    float4 d[EB];
#pragma unroll
    for (int k = 0; k < EB; ++k) d[k] = ldg4(p.dA + (int64_t)vv[k] * p.ldd + 4 * f4);
#pragma unroll
    for (int k = 0; k < EB; ++k) {
        const float* at = as + tt[k] * p.B;
#pragma unroll
        for (int i = 0; i < NI; ++i)
            if (lane + 32 * i < nch) fma4(acc[i], ww[k] * at[bi[i]], d[k]);
    }
}

// sources with out-degree < 32: one warp per row, persistent; lanes own the (b, f4) chunks of dV[u]
template <int F4, int NI>
__global__ void __launch_bounds__(256) k_basis_dv_w(const BasisDvArgs p) {
    extern __shared__ float as[];
    stage_coeffs(p.a, p.R * p.B, as);
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int nch = p.B * F4;
    const int f4 = lane % F4;
    int bi[NI];
#pragma unroll
    for (int i = 0; i < NI; ++i) bi[i] = (lane + 32 * i) / F4;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t row = p.row_begin + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5); row < p.row_end;
         row += nw) {
        const int beg = __ldg(p.off + row), end = __ldg(p.off + row + 1);
        const int64_t u = (int64_t)__ldg(p.perm + row) - p.vbase;
        float4 acc[NI];
#pragma unroll
        for (int i = 0; i < NI; ++i) acc[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        const int n = end - beg;                       // < 32
        int my_v = 0, my_t = 0;
        float my_w = 0.f;
        if (lane < n) {
            my_v = __ldcs(p.nbr + beg + lane);
            my_t = __ldcs(p.typ + beg + lane);
            my_w = edge_weight(p.norm_user, p.eid, p.norm, beg + lane);
        }
        int j = 0;
        for (; j + 2 <= n; j += 2) {
            const int vv[2] = {__shfl_sync(0xffffffffu, my_v, j), __shfl_sync(0xffffffffu, my_v, j + 1)};
            const int tt[2] = {__shfl_sync(0xffffffffu, my_t, j), __shfl_sync(0xffffffffu, my_t, j + 1)};
            const float ww[2] = {__shfl_sync(0xffffffffu, my_w, j), __shfl_sync(0xffffffffu, my_w, j + 1)};
            basis_dv_edges<F4, NI, 2>(p, as, lane, nch, f4, bi, vv, tt, ww, acc);
        }
        if (j < n) {
            const int vv[1] = {__shfl_sync(0xffffffffu, my_v, j)};
            const int tt[1] = {__shfl_sync(0xffffffffu, my_t, j)};
            const float ww[1] = {__shfl_sync(0xffffffffu, my_w, j)};
            basis_dv_edges<F4, NI, 1>(p, as, lane, nch, f4, bi, vv, tt, ww, acc);
        }
        float* po = p.dV + u * p.ldv + 4 * lane;
#pragma unroll
        for (int i = 0; i < NI; ++i)
            if (lane + 32 * i < nch) *reinterpret_cast<float4*>(po + 128 * i) = acc[i];
    }
}

// sources with out-degree >= 32: 8 warps per row; warp w takes edges w, w + 8, ... of each 256-edge block
// (4 in flight); the 8 partial dV rows are summed in warp order through shared memory.
template <int F4, int NI>
__global__ void __launch_bounds__(256) k_basis_dv_c(const BasisDvArgs p) {
    constexpr int WARPS = 8, TB = 256, EB = 4;
    extern __shared__ float smem[];
    float* as = smem;
    int* su = reinterpret_cast<int*>(smem + p.R * p.B);
    int* st = su + TB;
    float* sw = reinterpret_cast<float*>(st + TB);
    float4* part = reinterpret_cast<float4*>((reinterpret_cast<uintptr_t>(sw + TB) + 15) & ~uintptr_t(15));
    stage_coeffs(p.a, p.R * p.B, as);
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int nch = p.B * F4;
    const int f4 = lane % F4;
    int bi[NI];
#pragma unroll
    for (int i = 0; i < NI; ++i) bi[i] = (lane + 32 * i) / F4;
    for (int64_t row = p.row_begin + blockIdx.x; row < p.row_end; row += gridDim.x) {
        const int beg = __ldg(p.off + row), end = __ldg(p.off + row + 1);
        const int64_t u = (int64_t)__ldg(p.perm + row) - p.vbase;
        float4 acc[NI];
#pragma unroll
        for (int i = 0; i < NI; ++i) acc[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int base = beg; base < end; base += TB) {
            const int n = min(TB, end - base);
            if ((int)threadIdx.x < n) {
                su[threadIdx.x] = __ldcs(p.nbr + base + threadIdx.x);
                st[threadIdx.x] = __ldcs(p.typ + base + threadIdx.x);
                sw[threadIdx.x] = edge_weight(p.norm_user, p.eid, p.norm, base + threadIdx.x);
            }
            __syncthreads();
            int j = warp;
            for (; j + (EB - 1) * WARPS < n; j += EB * WARPS) {
                int vv[EB], tt[EB];
                float ww[EB];
#pragma unroll
                for (int k = 0; k < EB; ++k) { vv[k] = su[j + k * WARPS]; tt[k] = st[j + k * WARPS]; ww[k] = sw[j + k * WARPS]; }
                basis_dv_edges<F4, NI, EB>(p, as, lane, nch, f4, bi, vv, tt, ww, acc);
            }
            for (; j < n; j += WARPS) {
                const int vv[1] = {su[j]}, tt[1] = {st[j]};
                const float ww[1] = {sw[j]};
                basis_dv_edges<F4, NI, 1>(p, as, lane, nch, f4, bi, vv, tt, ww, acc);
            }
            __syncthreads();
        }
#pragma unroll
        for (int i = 0; i < NI; ++i)
            if (lane + 32 * i < nch) part[warp * nch + lane + 32 * i] = acc[i];
        __syncthreads();
        float* po = p.dV + u * p.ldv;
        for (int c = threadIdx.x; c < nch; c += TB) {
            float4 t = part[c];
#pragma unroll
            for (int w = 1; w < WARPS; ++w) {
                const float4 r = part[w * nch + c];
                t.x += r.x; t.y += r.y; t.z += r.z; t.w += r.w;
            }
            *reinterpret_cast<float4*>(po + 4 * c) = t;
        }
        __syncthreads();
    }
}

struct BasisDaArgs {
    const int32_t* src; const int32_t* eid; const float* norm; const float* norm_user;
    const int32_t* run_off; const int32_t* run_dst; const int32_t* task_run;
    int64_t n_tasks;
    const float* V; int64_t ldv;
    const float* dA; int64_t ldd;
    int B, F4;
    float* part;                       // [n_tasks, B]
};

// one CTA (8 warps) per task of one type: warp w walks the contiguous edge slice
// [es + n*w/8, es + n*(w+1)/8) of the task (its first run found by binary search over run_off),
// gathers V[src] and dots it with dA[run_dst]; the 8 per-warp partial da[type, :] are summed in warp order.
template <int F4, int NI>
__global__ void __launch_bounds__(256) k_basis_da(const BasisDaArgs p) {
    constexpr int WARPS = 8;
    extern __shared__ float red[];                   // [WARPS][B]
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int nch = p.B * F4;
    const int f4 = lane % F4;
    for (int64_t t = blockIdx.x; t < p.n_tasks; t += gridDim.x) {
        const int r0 = __ldg(p.task_run + t), r1 = __ldg(p.task_run + t + 1);
        const int es = __ldg(p.run_off + r0), ee = __ldg(p.run_off + r1);
        const int64_t n = ee - es;
        const int k0 = es + (int)(n * warp / WARPS), k1 = es + (int)(n * (warp + 1) / WARPS);
        float acc[NI];
#pragma unroll
        for (int i = 0; i < NI; ++i) acc[i] = 0.f;
        if (k0 < k1) {
            int lo = r0, hi = r1 - 1;                  // last run with run_off <= k0
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (__ldg(p.run_off + mid) <= k0) lo = mid; else hi = mid - 1;
            }
            int run = lo, rend = __ldg(p.run_off + run + 1);
            float4 d = ldg4(p.dA + (int64_t)__ldg(p.run_dst + run) * p.ldd + 4 * f4);
            for (int k = k0; k < k1; ++k) {
                if (k == rend) {                       // warp-uniform
                    ++run;
                    rend = __ldg(p.run_off + run + 1);
                    d = ldg4(p.dA + (int64_t)__ldg(p.run_dst + run) * p.ldd + 4 * f4);
                }
                const int u = __ldg(p.src + k);
                const float w = edge_weight(p.norm_user, p.eid, p.norm, k);
                const float* vp = p.V + (int64_t)u * p.ldv + 4 * lane;
                float4 x[NI];
#pragma unroll
                for (int i = 0; i < NI; ++i)
                    if (lane + 32 * i < nch) x[i] = ldg4(vp + 128 * i);
#pragma unroll
                for (int i = 0; i < NI; ++i)
                    if (lane + 32 * i < nch) {
                        float dot = x[i].x * d.x;
                        dot = fmaf(x[i].y, d.y, dot);
                        dot = fmaf(x[i].z, d.z, dot);
                        dot = fmaf(x[i].w, d.w, dot);
                        acc[i] = fmaf(w, dot, acc[i]);
                    }
            }
        }
        // sum the F4 lanes of each basis (fixed xor tree); lane f4 == 0 holds basis (lane + 32 i) / F4
#pragma unroll
        for (int o = 1; o < F4; o <<= 1)
#pragma unroll
            for (int i = 0; i < NI; ++i) acc[i] += __shfl_xor_sync(0xffffffffu, acc[i], o);
        if (f4 == 0)
#pragma unroll
            for (int i = 0; i < NI; ++i)
                if (lane + 32 * i < nch) red[warp * p.B + (lane + 32 * i) / F4] = acc[i];
        __syncthreads();
        for (int b = threadIdx.x; b < p.B; b += blockDim.x) {
            float x = red[b];
#pragma unroll
            for (int w = 1; w < WARPS; ++w) x += red[w * p.B + b];
            p.part[t * p.B + b] = x;
        }
        __syncthreads();
    }
}

// W[r][k] = sum_b a[r][b] Vb[b][k]   (fp64 accumulation, fixed order)
__global__ void k_basis_combine(const float* __restrict__ a, const float* __restrict__ Vb, int R, int B, int64_t K,
                                float* __restrict__ W) {
    const int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (idx >= (int64_t)R * K) return;
    const int r = (int)(idx / K);
    const int64_t k = idx % K;
    double x = 0.0;
    for (int b = 0; b < B; ++b) x += (double)__ldg(a + (int64_t)r * B + b) * (double)__ldg(Vb + (int64_t)b * K + k);
    W[idx] = (float)x;
}

// da[r][b] = <dW[r], Vb[b]>: one warp per (r, b), lanes stride k, fixed xor tree
__global__ void k_basis_combine_da(const float* __restrict__ Vb, const float* __restrict__ dW, int R, int B, int64_t K,
                                   float* __restrict__ da) {
    const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (w >= (int64_t)R * B) return;
    const int r = (int)(w / B), b = (int)(w % B);
    double x = 0.0;
    for (int64_t k = lane; k < K; k += 32) x += (double)__ldg(dW + (int64_t)r * K + k) * (double)__ldg(Vb + (int64_t)b * K + k);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    if (lane == 0) da[w] = (float)x;
}

// dVb[b][k] = sum_r a[r][b] dW[r][k]
__global__ void k_basis_combine_dv(const float* __restrict__ a, const float* __restrict__ dW, int R, int B, int64_t K,
                                   float* __restrict__ dVb) {
    const int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (idx >= (int64_t)B * K) return;
    const int b = (int)(idx / K);
    const int64_t k = idx % K;
    double x = 0.0;
    for (int r = 0; r < R; ++r) x += (double)__ldg(a + (int64_t)r * B + b) * (double)__ldg(dW + (int64_t)r * K + k);
    dVb[idx] = (float)x;
}

static inline unsigned blocks_for(int64_t n, int per) { return (unsigned)((n + per - 1) / per); }

// dispatch on (F4, NI); F4 in {1,2,4,8,16,32}, NI = pow2_ceil(ceil(B*F4/32)) <= 16
#define BASIS_NI_CASES(F4V, LAUNCH)     \
    switch (NI) {                       \
        case 1: LAUNCH(F4V, 1); break;  \
        case 2: LAUNCH(F4V, 2); break;  \
        case 4: LAUNCH(F4V, 4); break;  \
        case 8: LAUNCH(F4V, 8); break;  \
        default: LAUNCH(F4V, 16); break; \
    }
#define BASIS_DISPATCH(LAUNCH)                          \
    switch (F4) {                                       \
        case 1: BASIS_NI_CASES(1, LAUNCH); break;       \
        case 2: BASIS_NI_CASES(2, LAUNCH); break;       \
        case 4: BASIS_NI_CASES(4, LAUNCH); break;       \
        case 8: BASIS_NI_CASES(8, LAUNCH); break;       \
        case 16: BASIS_NI_CASES(16, LAUNCH); break;     \
        default: BASIS_NI_CASES(32, LAUNCH); break;     \
    }

static seastar_status check_shape(int64_t B, int64_t F, int32_t R, const char* who) {
    if (!(F >= 4 && F <= 128 && (F & (F - 1)) == 0)) {
        set_error("%s: F must be a power of two in [4, 128] (got %lld)", who, (long long)F);
        return SEASTAR_ERR_INVALID_ARGUMENT;
    }
    if (B < 1 || B * F > 2048) {
        set_error("%s: need 1 <= B and B*F <= 2048 (got B=%lld, F=%lld)", who, (long long)B, (long long)F);
        return SEASTAR_ERR_INVALID_ARGUMENT;
    }
    if ((int64_t)R * B * 4 > 96 * 1024) {
        set_error("%s: the coefficient table a (R*B floats) must fit 96 KB of shared memory", who);
        return SEASTAR_ERR_INVALID_ARGUMENT;
    }
    return SEASTAR_OK;
}

// dynamic shared memory of a CTA kernel: the coefficient table, three TB-entry edge-metadata arrays,
// 16-byte alignment slack and `extra` float4 of reduction space
static inline size_t cta_smem(size_t smem_a, int tb, int extra_f4) {
    return smem_a + (size_t)3 * tb * 4 + 32 + (size_t)extra_f4 * 16;
}

// persistent launch: min(work items, resident CTAs) CTAs; the kernels grid-stride over their items
template <typename Arg>
static seastar_status launch_persistent(void (*kern)(Arg), int64_t items, int threads, size_t smem, cudaStream_t s,
                                        const Arg& a) {
    if (items <= 0) return SEASTAR_OK;
    if (smem > 48 * 1024) SS_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    SS_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, threads, smem));
    if (per_sm < 1) {
        set_error("rgcn_basis: %zu bytes of shared memory per CTA do not fit", smem);
        return SEASTAR_ERR_UNSUPPORTED;
    }
    int64_t blocks = (int64_t)per_sm * num_sms();
    if (blocks > items) blocks = items;
    launch_k(kern, dim3((unsigned)blocks), dim3(threads), smem, s, a);
    return check_launch("rgcn_basis kernel");
}

}  // namespace seastar

using namespace seastar;

extern "C" {

seastar_status seastar_rgcn_basis_fwd(seastar_graph g, const float* V_all, int64_t B, int64_t F, int64_t ldv,
                                      const float* a, const float* norm_user, const float* loop_loc, int64_t ldl,
                                      const float* bias, seastar_act act, float* Y_loc, int64_t ldy,
                                      seastar_stream stream) {
    SS_ARG(g && V_all && a && Y_loc, "rgcn_basis_fwd: NULL argument");
    SS_TRY(check_shape(B, F, g->R, "rgcn_basis_fwd"));
    SS_ARG(g->fwd.type != nullptr, "rgcn_basis_fwd: graph was created without etypes");
    SS_ARG(norm_user || g->fwd.norm, "rgcn_basis_fwd: pass norm_user or create the graph with SEASTAR_GRAPH_RGCN_NORM");
    SS_ARG(ldv >= B * F && ldv % 4 == 0 && aligned16(V_all), "rgcn_basis_fwd: V_all needs ldv >= B*F, ldv %% 4 == 0, 16B alignment");
    SS_ARG(ldy >= F && ldy % 4 == 0 && aligned16(Y_loc), "rgcn_basis_fwd: Y_loc needs ldy >= F, ldy %% 4 == 0, 16B alignment");
    SS_ARG(!loop_loc || ldl >= F, "rgcn_basis_fwd: bad ldl");
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "rgcn_basis_fwd: bad activation");
    SS_TRY(check_device());
    const int64_t rows = g->fwd.n_rows;
    if (rows == 0) return SEASTAR_OK;
    BasisFwdArgs p{};
    p.perm = g->fwd.perm; p.off = g->fwd.off; p.nbr = g->fwd.nbr; p.typ = g->fwd.type; p.eid = g->fwd.eid;
    p.norm = g->fwd.norm; p.norm_user = norm_user;
    p.row_begin = 0; p.row_end = rows; p.vbase = g->row_begin;
    p.V = V_all; p.ldv = ldv; p.a = a; p.R = g->R; p.B = (int)B; p.F4 = (int)(F / 4);
    p.loop = loop_loc; p.ldl = ldl; p.bias = bias; p.act = act; p.Y = Y_loc; p.ldy = ldy;
    const int F4 = p.F4, NI = pow2_ceil((int)((B * F4 + 31) / 32));
    const size_t smem_a = (size_t)g->R * B * sizeof(float);
    cudaStream_t s = to_stream(stream);
    const int64_t hub = g->fwd.bucket_rows[0], mid = g->fwd.bucket_rows[1];
    BasisFwdArgs ph = p, pm = p, pl = p;
    ph.row_begin = 0; ph.row_end = hub;
    pm.row_begin = hub; pm.row_end = mid;
    pl.row_begin = mid; pl.row_end = rows;
#define LAUNCH_FWD(F4V, NIV)                                                                                       \
    do {                                                                                                           \
        if (hub > 0)                                                                                               \
            SS_TRY((launch_persistent(k_basis_fwd_c<F4V, NIV, 16>, hub, 512, cta_smem(smem_a, 512, 16 * F4V), s, ph))); \
        if (mid > hub)                                                                                             \
            SS_TRY((launch_persistent(k_basis_fwd_c<F4V, NIV, 8>, mid - hub, 256, cta_smem(smem_a, 256, 8 * F4V), s, pm))); \
        if (rows > mid) SS_TRY((launch_persistent(k_basis_fwd_w<F4V, NIV>, (rows - mid + 7) / 8, 256, smem_a, s, pl))); \
    } while (0)
    BASIS_DISPATCH(LAUNCH_FWD);
#undef LAUNCH_FWD
    return SEASTAR_OK;
}

size_t seastar_rgcn_basis_bwd_workspace(seastar_graph g, int64_t B) {
    if (!g) return 0;
    return (size_t)(g->tm.n_tasks + 1) * (size_t)B * sizeof(float) + 256;
}

seastar_status seastar_rgcn_basis_bwd(seastar_graph g, const float* V_all, int64_t B, int64_t F, int64_t ldv,
                                      const float* a, const float* norm_user, const float* dA_all, int64_t ldd,
                                      float* dV_loc, float* da, void* workspace, size_t ws_bytes,
                                      seastar_stream stream) {
    SS_ARG(g && a && dA_all, "rgcn_basis_bwd: NULL argument");
    SS_ARG(dV_loc || da, "rgcn_basis_bwd: nothing to compute");
    SS_TRY(check_shape(B, F, g->R, "rgcn_basis_bwd"));
    SS_ARG(g->fwd.type != nullptr, "rgcn_basis_bwd: graph was created without etypes");
    SS_ARG(norm_user || g->fwd.norm, "rgcn_basis_bwd: pass norm_user or create the graph with SEASTAR_GRAPH_RGCN_NORM");
    SS_ARG(ldv >= B * F && ldv % 4 == 0, "rgcn_basis_bwd: need ldv >= B*F, ldv %% 4 == 0");
    SS_ARG(ldd >= F && ldd % 4 == 0 && aligned16(dA_all), "rgcn_basis_bwd: dA_all needs ldd %% 4 == 0, 16B alignment");
    SS_ARG(!dV_loc || aligned16(dV_loc), "rgcn_basis_bwd: dV_loc must be 16B aligned");
    SS_ARG(!da || (V_all && aligned16(V_all)), "rgcn_basis_bwd: da needs V_all (16B aligned)");
    SS_ARG(!da || (workspace && ws_bytes >= seastar_rgcn_basis_bwd_workspace(g, B)), "rgcn_basis_bwd: workspace too small");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    const int F4 = (int)(F / 4), NI = pow2_ceil((int)((B * F4 + 31) / 32));
    const size_t smem = (size_t)g->R * B * sizeof(float);
    if (dV_loc && g->rev.n_rows > 0) {
        BasisDvArgs p{};
        p.perm = g->rev.perm; p.off = g->rev.off; p.nbr = g->rev.nbr; p.typ = g->rev.type; p.eid = g->rev.eid;
        p.norm = g->rev.norm; p.norm_user = norm_user;
        p.row_begin = 0; p.row_end = g->rev.n_rows; p.vbase = g->row_begin;
        p.dA = dA_all; p.ldd = ldd; p.a = a; p.R = g->R; p.B = (int)B; p.F4 = F4; p.dV = dV_loc; p.ldv = ldv;
        if (g->rev.n_rows < g->n_loc())   // owned rows missing from the REV CSR get zero
            SS_CUDA(cudaMemsetAsync(dV_loc, 0, sizeof(float) * (size_t)g->n_loc() * ldv, s));
        const int64_t mid = g->rev.bucket_rows[1], rows = g->rev.n_rows;
        BasisDvArgs pm = p, pl = p;
        pm.row_begin = 0; pm.row_end = mid;
        pl.row_begin = mid; pl.row_end = rows;
        const size_t smem_c = cta_smem(smem, 256, 0) + (size_t)8 * B * F4 * 16;
#define LAUNCH_DV(F4V, NIV)                                                                                      \
    do {                                                                                                         \
        if (mid > 0) SS_TRY((launch_persistent(k_basis_dv_c<F4V, NIV>, mid, 256, smem_c, s, pm)));              \
        if (rows > mid) SS_TRY((launch_persistent(k_basis_dv_w<F4V, NIV>, (rows - mid + 7) / 8, 256, smem, s, pl))); \
    } while (0)
        BASIS_DISPATCH(LAUNCH_DV);
#undef LAUNCH_DV
    } else if (dV_loc) {
        SS_CUDA(cudaMemsetAsync(dV_loc, 0, sizeof(float) * (size_t)g->n_loc() * ldv, s));
    }
    if (da) {
        if (g->tm.n_tasks > 0) {
            BasisDaArgs p{};
            p.src = g->tm.src; p.eid = g->tm.eid; p.norm = g->tm.norm; p.norm_user = norm_user;
            p.run_off = g->tm.run_off; p.run_dst = g->tm.run_dst; p.task_run = g->tm.task_run;
            p.n_tasks = g->tm.n_tasks;
            p.V = V_all; p.ldv = ldv; p.dA = dA_all; p.ldd = ldd; p.B = (int)B; p.F4 = F4;
            p.part = static_cast<float*>(workspace);
            const size_t smem_r = (size_t)8 * B * sizeof(float);
#define LAUNCH_DA(F4V, NIV) SS_TRY((launch_persistent(k_basis_da<F4V, NIV>, g->tm.n_tasks, 256, smem_r, s, p)))
            BASIS_DISPATCH(LAUNCH_DA);
#undef LAUNCH_DA
            seg_reduce_cols(p.part, g->tm.type_task, g->R, (int)B, da, s);
            SS_TRY(check_launch("k_seg_reduce_cols"));
        } else {
            SS_CUDA(cudaMemsetAsync(da, 0, sizeof(float) * (size_t)g->R * B, s));
        }
    }
    return SEASTAR_OK;
}

seastar_status seastar_basis_combine(const float* a, const float* Vb, int32_t R, int32_t B, int64_t K, float* W,
                                     seastar_stream stream) {
    SS_ARG(a && Vb && W, "basis_combine: NULL argument");
    SS_ARG(R >= 1 && B >= 1 && K >= 1, "basis_combine: need R, B, K >= 1");
    SS_TRY(check_device());
    k_basis_combine<<<blocks_for((int64_t)R * K, 256), 256, 0, to_stream(stream)>>>(a, Vb, R, B, K, W);
    return check_launch("k_basis_combine");
}

seastar_status seastar_basis_combine_bwd(const float* a, const float* Vb, const float* dW, int32_t R, int32_t B,
                                         int64_t K, float* da, float* dVb, seastar_stream stream) {
    SS_ARG(a && Vb && dW, "basis_combine_bwd: NULL argument");
    SS_ARG(da || dVb, "basis_combine_bwd: nothing to compute");
    SS_ARG(R >= 1 && B >= 1 && K >= 1, "basis_combine_bwd: need R, B, K >= 1");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    if (da) {
        k_basis_combine_da<<<blocks_for((int64_t)R * B * 32, 256), 256, 0, s>>>(Vb, dW, R, B, K, da);
        SS_TRY(check_launch("k_basis_combine_da"));
    }
    if (dVb) {
        k_basis_combine_dv<<<blocks_for((int64_t)B * K, 256), 256, 0, s>>>(a, dW, R, B, K, dVb);
        SS_TRY(check_launch("k_basis_combine_dv"));
    }
    return SEASTAR_OK;
}

}  // extern "C"
