// gat_common.cuh -- argument blocks and arithmetic shared by the GAT kernel files (gat.cu: generic
// chunked kernels, row kernels and the C ABI; gat_hpl.cu: head-per-lane kernels; gat_h1.cu:
// single-head kernels).  PAPER.md Fig. 2 L95-L123 (GAT), §6.3.4 L461-L463 (backward on the reverse
// CSR).
#pragma once
#include <math.h>

#include "common.cuh"

#ifndef GAT_MB_FWD
#define GAT_MB_FWD 3   // min resident 256-thread blocks per SM (<= 85 regs): measured best on Reddit
#endif
#ifndef GAT_MB_BWD
#define GAT_MB_BWD 3
#endif

namespace seastar {

constexpr float kLog2e = 1.4426950408889634f;
// running-max sentinel of the online softmax: finite, so (z - m) never forms inf - inf; a logit
// below -1e30 (not produced by any finite model) would be treated as an empty row (R25)
constexpr float kNegBig = -1e30f;

__device__ __forceinline__ float lrelu(float x, float slope) { return x > 0.f ? x : slope * x; }

// 2^x on the SFU (rel. err ~2^-22; ex2(-inf) = +0): softmax weights are exp(z - m) = ex2((z - m) log2 e)
__device__ __forceinline__ float ex2(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

struct GatFwdArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr;
    int64_t row_begin, row_end, vbase;
    const float* T; const float* el; const float* er;
    int H, F; int64_t ld; float slope;
    int64_t ldel;            // row stride of el (H, or ld when el is packed into T's padding: el == T + H*F)
    const float* bias; int act;
    float* A; float* Y; float* lse;
    float* B; float* bsum;   // optional: der factors (see k_gat_fwd_hpl)
    // NEXT-3 attention dropout (generic chunked kernels only; deid == nullptr: off): the aggregation weight of
    // edge slot k is a_e * drop_mult(key, eid * H + h), key from (dseed, dsite, *dstep)
    const int32_t* deid; uint64_t dseed; const int32_t* dstep; uint32_t dsite, dthr; float dscale;
    int64_t nlong;   // hub-capable launches: blocks [0, nlong) own one long row each (see k_gat_fwd_hpl)
};

struct GatBwdArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr;
    int64_t row_begin, row_end, vbase;
    const float* T;      // gathered (der) or owned (src-major) rows
    const float* el;     // gathered (der) or owned (src-major)
    const float* D;      // packed records: gathered (src-major) or owned (der)
    int H, F; int64_t ldt, ldd; float slope;
    int64_t ldel;        // row stride of el (see GatFwdArgs)
    float* dT; float* del;   // src-major outputs
    float* der;              // der output
    const int32_t* deid; uint64_t dseed; const int32_t* dstep; uint32_t dsite, dthr; float dscale;   // as GatFwdArgs
    int64_t nlong;
};


// packed backward record D[v] = [dA (H*F, zero-padded to a multiple of 4) | per head (er, lse, c, nl2)]
// with nl2 = -lse * log2(e), so a_e = ex2(LReLU(s_e) log2 e + nl2) is one FFMA + one SFU op.  (Measured in r2: a
// 3-scalar layout [er | c | nl2] without lse saves one of the 12 sectors of the 8x8 record but needs three 32-bit
// loads per head instead of one 128-bit load, and the layer-1 backward went from 2.62 to 2.96 ms -- it is L1-bound.)
__host__ __device__ __forceinline__ int rec_aux_offset(int W) { return (W + 3) & ~3; }

// 32-bit row offset -> 64-bit address in one IMAD.WIDE.U32 (row strides are < 2^31 floats, checked
// at the ABI)
__device__ __forceinline__ const float* row_ptr(const float* base, int r, int64_t ld) {
    return base + (size_t)(uint32_t)r * (uint32_t)ld;
}

// el packed into the first padding columns of T (el == T + H*F, row stride ldt) or a separate [rows, H] table
inline int64_t el_stride(const float* T, const float* el, int H, int F, int64_t ldt) {
    return (el == T + (int64_t)H * F) ? ldt : (int64_t)H;
}

// launchers (return false when the geometry does not apply)
// hub = the index set's long_rows(): those leading rows get a multi-warp CTA each
bool launch_gat_fwd_hpl(const GatFwdArgs& a, int64_t hub, cudaStream_t s);
bool launch_gat_bwd_hpl(const GatBwdArgs& a, int64_t hub, cudaStream_t s);
bool launch_gat_der_hpl(const GatBwdArgs& a, cudaStream_t s);
// mid: rows with degree >= 8 (IndexSet::pow2_rows[0]); rows [split, mid) take 16-lane row groups
bool launch_gat_fwd_h1(const GatFwdArgs& a, int64_t hub, int64_t split, int64_t mid, int64_t n_rows, cudaStream_t s);
bool launch_gat_bwd_h1(const GatBwdArgs& a, int64_t hub, int64_t split, int64_t mid, int64_t n_rows, bool der,
                       cudaStream_t s);

// head-per-lane geometry: H | 32, every head row is whole float4s held by one lane
inline int hpl_f4(int H, int F, int64_t ldt, bool aligned) {
    if (H < 2 || (32 % H) != 0 || (F % 4) != 0 || F > 32 || (ldt % 4) != 0 || !aligned) return 0;
    return F / 4;
}

// single-head geometry: VPL float4 chunks per lane (from {1,2,3,4,6,8}), L = pow2 lanes per edge (<= 4)
inline bool h1_geometry(int H, int F, int64_t ldt, bool aligned, int& vpl, int& L) {
    if (H != 1 || (ldt % 4) != 0 || !aligned || F > 128) return false;
    const int C = (F + 3) / 4;
    int v = (C + 3) / 4;
    v = v <= 4 ? v : (v <= 6 ? 6 : 8);
    vpl = v;
    L = pow2_ceil((C + v - 1) / v);
    return L <= 4;
}

}  // namespace seastar
