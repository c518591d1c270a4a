// gemm_tc.cu -- a4: the dense per-layer transform Y = row_scale * act(X W + bias) on the 5th-generation
// tensor cores (tcgen05, kind::tf32) with an fp32-accurate 3xTF32 split.
//
// Shape: X [M, K] row-major fp32 (M = vertices, up to millions; K = feature width), W [K, N] (N <= 256).
// One CTA computes a 128 x NP tile (NP = N rounded up to 16) over the whole K range:
//   warp 0      : TMA producer -- cp.async.bulk.tensor loads 128 x 32 fp32 X tiles (SWIZZLE_128B) into a
//                 STAGES-deep ring, completion signalled on an mbarrier (expect_tx);
//   warps 2..5  : split -- per stage, X_hi = rna_tf32(X) in place and X_lo = X - X_hi, and the W chunk
//                 (read from L2, written K-major with the same 128B swizzle) as W_hi / W_lo;
//                 then the epilogue (tcgen05.ld of the TMEM accumulator, bias / activation / row scale);
//   warp 1      : TMEM allocation and the MMA issuer -- one elected thread issues, per 8-wide K step,
//                 hi*hi + hi*lo + lo*hi into the fp32 accumulator in TMEM and commits each stage back to
//                 the producer (tcgen05.commit -> mbarrier).
// Because X_hi and W_hi are exactly representable in tf32 the products are independent of how the MMA
// unit rounds its inputs; the dropped lo*lo term is < 2^-22 relative.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <mutex>

#include "common.cuh"

namespace seastar {

struct TcArgs {
    int64_t M, K, N;
    const float* Wsplit;            // [nk][W_hi tile | W_lo tile], each NP x 32 K-major, 128B-swizzled
    float* Y; int64_t ldy;
    const float* bias; const float* row_scale; int act;
    int ksplit = 1;                 // k_gemm_tc2: K splits per tile (partials in part, then k_splitk_reduce)
    float* part = nullptr;          // [ksplit][M][NP]
};
constexpr int kSplitKMax = 8;
// K splits are used only while the row tiles cannot fill two CTAs per SM
static int64_t splitk_max_rows() { return 2 * (int64_t)num_sms() * 128; }

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    const uint32_t a = smem_u32(bar);
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(a), "r"(parity) : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* tm, int x, int y, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
        ::"r"(smem_u32(dst)), "l"(reinterpret_cast<uint64_t>(tm)), "r"(x), "r"(y), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_copy(void* dst, const float* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(reinterpret_cast<uint64_t>(src)), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ float rna_tf32(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return __uint_as_float(r);
}
// K-major operand, 128B swizzle, 8-row groups 1024 B apart (sm100 descriptor version 1)
__device__ __forceinline__ uint64_t smem_desc_k128(const void* p) {
    const uint32_t a = smem_u32(p);
    uint64_t d = (uint64_t)((a >> 4) & 0x3FFF);
    d |= (uint64_t)1 << 16;                 // leading byte offset (unused for swizzled K-major)
    d |= (uint64_t)(1024 >> 4) << 32;       // stride byte offset
    d |= (uint64_t)1 << 46;                 // version
    d |= (uint64_t)2 << 61;                 // SWIZZLE_128B
    return d;
}
__device__ __forceinline__ void mma_tf32(uint32_t tmem, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}" ::"r"(tmem), "l"(da), "l"(db), "r"(idesc),
        "r"(acc));
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

// A operand in TMEM (lane = row, 8 consecutive 32-bit columns per K step), B from shared memory
__device__ __forceinline__ void mma_tf32_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}" ::"r"(tmem_d), "r"(tmem_a), "l"(db), "r"(idesc),
        "r"(acc));
}
// 16 consecutive 32-bit columns of this thread's TMEM lane (warp quarter addressing as tcgen05.ld)
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
        "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]), "r"(v[9]),
        "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
        : "memory");
}

// Add TMEM slot (j & 1) -- the finished accumulation segment j -- into the fp32 register accumulators
// of this thread's row (lane quarter q4), in column order, then hand the slot back to the MMA issuer.
// NA accumulators per slot (k_gemm_tc2 keeps the three 3xTF32 products in separate accumulators, so consecutive
// MMAs never depend on each other): they are summed in a fixed order before the register add.
template <int NP, int NA = 1>
__device__ __forceinline__ void drain_segment(uint32_t tmem, int j, int q4, uint64_t* seg_done, uint64_t* slot_free,
                                              float (&racc)[NP]) {
    const int slot = j & 1;
    mbar_wait(&seg_done[slot], (j >> 1) & 1);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
    for (int c0 = 0; c0 < NP; c0 += 16) {
        float t[16];
#pragma unroll
        for (int ai = 0; ai < NA; ++ai) {
            uint32_t v[16];
            asm volatile(
                "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                  "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
                : "r"(tmem + ((uint32_t)(q4 * 32) << 16) + (uint32_t)((slot * NA + ai) * NP + c0)));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
            for (int q = 0; q < 16; ++q) t[q] = ai == 0 ? __uint_as_float(v[q]) : t[q] + __uint_as_float(v[q]);
        }
#pragma unroll
        for (int q = 0; q < 16; ++q) racc[c0 + q] += t[q];
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    mbar_arrive(&slot_free[slot]);
}

#ifndef TC_SEG
#define TC_SEG 2
#endif
#ifndef TC_TN_SEG
#define TC_TN_SEG 2
#endif
#ifndef TC_TWO_CTAS
#define TC_TWO_CTAS 1
#endif
template <int NP>
struct TcCfg {
    static constexpr int BM = 128, BK = 32;
    // NP <= 64: two co-resident CTAs per SM (2 stages each), so one CTA's prologue / epilogue overlaps
    // the other's TMA stream; wider tiles: one CTA with a deeper ring
    static constexpr int CTAS = (TC_TWO_CTAS && NP <= 64) ? 2 : 1;
    static constexpr int STAGES = CTAS == 2 ? 2 : (NP <= 64 ? 4 : (NP <= 128 ? 3 : 2));
    static constexpr uint32_t A_BYTES = BM * BK * 4;          // 16 KB
    static constexpr uint32_t B_BYTES = NP * BK * 4;          // NP rows of 128 B
    static constexpr uint32_t STAGE_BYTES = 2 * A_BYTES + 2 * B_BYTES;
    // accumulation segments of SEG K chunks ping-pong between two TMEM slots; after each segment the
    // epilogue warps add the slot into fp32 registers (IEEE round-to-nearest), so the tensor core's own
    // accumulation never spans more than SEG * 12 MMAs (this keeps the K = 8,415 / 8,710
    // transforms of the Physics / CoraFull configs within 1e-6)
    static constexpr int SEG = TC_SEG;
    static constexpr uint32_t TMEM_COLS = (2 * NP) <= 32 ? 32 : ((2 * NP) <= 64 ? 64 : ((2 * NP) <= 128 ? 128 : 256));
    static constexpr size_t SMEM = (size_t)STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/;
};

template <int NP>
__global__ void __launch_bounds__(192, TcCfg<NP>::CTAS) k_gemm_tc(const __grid_constant__ CUtensorMap tmX, const TcArgs a) {
    using C = TcCfg<NP>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + (size_t)C::STAGES * C::STAGE_BYTES);
    uint64_t* full = bars;                       // TMA landed
    uint64_t* split = bars + C::STAGES;          // hi/lo written (128 arrivals)
    uint64_t* empty = bars + 2 * C::STAGES;      // MMAs done reading
    uint64_t* seg_done = bars + 3 * C::STAGES;   // [2] segment accumulated in TMEM slot b
    uint64_t* slot_free = seg_done + 2;          // [2] slot b drained into registers (128 arrivals)
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(seg_done + 4);
    auto A_hi = [&](int s) { return smem + (size_t)s * C::STAGE_BYTES; };
    auto A_lo = [&](int s) { return smem + (size_t)s * C::STAGE_BYTES + C::A_BYTES; };
    auto B_hi = [&](int s) { return smem + (size_t)s * C::STAGE_BYTES + 2 * C::A_BYTES; };
    auto B_lo = [&](int s) { return smem + (size_t)s * C::STAGE_BYTES + 2 * C::A_BYTES + C::B_BYTES; };

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t m0 = (int64_t)blockIdx.x * C::BM;
    const int nk = (int)((a.K + C::BK - 1) / C::BK);

    if (threadIdx.x == 0) {
        for (int s = 0; s < C::STAGES; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&split[s], 128);
            mbar_init(&empty[s], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&seg_done[b], 1);
            mbar_init(&slot_free[b], 128);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(C::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        // ---------------- TMA producer ----------------
        if (lane == 0) {
            for (int kc = 0; kc < nk; ++kc) {
                const int s = kc % C::STAGES;
                if (kc >= C::STAGES) mbar_wait(&empty[s], ((kc / C::STAGES) - 1) & 1);
                mbar_expect_tx(&full[s], C::A_BYTES + 2 * C::B_BYTES);
                tma_load_2d(A_hi(s), &tmX, kc * C::BK, (int)m0, &full[s]);
                // the pre-split, pre-swizzled W_hi | W_lo tiles of this K chunk: one contiguous bulk copy
                bulk_copy(B_hi(s), a.Wsplit + (size_t)kc * 2 * C::B_BYTES / sizeof(float), 2 * C::B_BYTES, &full[s]);
            }
        }
    } else if (warp == 1) {
        // ---------------- MMA issuer ----------------
        // instruction descriptor: D f32, A/B tf32, both K-major, N = NP, M = 128
        const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NP >> 3) << 17) | ((128u >> 4) << 24);
        for (int kc = 0; kc < nk; ++kc) {
            const int s = kc % C::STAGES;
            const int j = kc / C::SEG, slot = j & 1;
            const bool first = (kc % C::SEG) == 0;
            if (first && j >= 2) mbar_wait(&slot_free[slot], ((j >> 1) - 1) & 1);   // segment j-2 drained
            mbar_wait(&split[s], (kc / C::STAGES) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            if (lane == 0) {
                const uint64_t ah = smem_desc_k128(A_hi(s)), al = smem_desc_k128(A_lo(s));
                const uint64_t bh = smem_desc_k128(B_hi(s)), bl = smem_desc_k128(B_lo(s));
                const uint32_t d = tmem + (uint32_t)(slot * NP);
#pragma unroll
                for (int ks = 0; ks < C::BK / 8; ++ks) {
                    const uint64_t adv = (uint64_t)((ks * 8 * 4) >> 4);   // 32 B per 8-wide K step
                    mma_tf32(d, al + adv, bh + adv, idesc, (!first || ks > 0) ? 1u : 0u);
                    mma_tf32(d, ah + adv, bl + adv, idesc, 1u);
                    mma_tf32(d, ah + adv, bh + adv, idesc, 1u);
                }
                mma_commit(&empty[s]);
                if ((kc % C::SEG) == C::SEG - 1 || kc == nk - 1) mma_commit(&seg_done[slot]);
            }
            __syncwarp();
        }
    } else {
        // ---------------- split, segment drains (then epilogue) ----------------
        const int t = threadIdx.x - 64;                     // 0..127
        const int q4 = warp & 3;                            // TMEM lane quarter accessible to this warp
        float racc[NP];
#pragma unroll
        for (int j = 0; j < NP; ++j) racc[j] = 0.f;
        for (int kc = 0; kc < nk; ++kc) {
            const int s = kc % C::STAGES;
            const int k0 = kc * C::BK;
            // full[s] also proves the MMAs of this stage's previous use are done (the producer armed it
            // only after empty[s]), so the stage's W buffers may be rewritten now
            mbar_wait(&full[s], (kc / C::STAGES) & 1);
            (void)k0;
            // elementwise over the 16 KB tile, consecutive lanes on consecutive 16 B chunks (conflict-free;
            // the swizzle only permutes chunks, so hi and lo land at the same offsets as their source)
            float4* ph = reinterpret_cast<float4*>(A_hi(s));
            float4* pl = reinterpret_cast<float4*>(A_lo(s));
            float4 xv[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) xv[q] = ph[q * 128 + t];
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const float4 x = xv[q];
                const float4 h = make_float4(rna_tf32(x.x), rna_tf32(x.y), rna_tf32(x.z), rna_tf32(x.w));
                ph[q * 128 + t] = h;
                pl[q * 128 + t] = make_float4(x.x - h.x, x.y - h.y, x.z - h.z, x.w - h.w);
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive(&split[s]);
            // one segment behind the MMAs: drain segment j-1 once segment j is fully split
            if (((kc % C::SEG) == C::SEG - 1 || kc == nk - 1) && kc / C::SEG >= 1)
                drain_segment<NP>(tmem, kc / C::SEG - 1, q4, seg_done, slot_free, racc);
        }
        if (nk > 0) drain_segment<NP>(tmem, (nk - 1) / C::SEG, q4, seg_done, slot_free, racc);
        // ---------------- epilogue: bias, activation, row scale ----------------
        const int r = q4 * 32 + lane;
        const int64_t gm = m0 + r;
        if (gm < a.M) {
            const float rs = a.row_scale ? __ldg(a.row_scale + gm) : 1.f;
            float* y = a.Y + gm * a.ldy;
#pragma unroll
            for (int j = 0; j < NP; ++j) {
                if (j < a.N) {
                    const float z = racc[j] + (a.bias ? __ldg(a.bias + j) : 0.f);
                    y[j] = rs * act_apply(a.act, z);
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 1) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(C::TMEM_COLS));
    }
}

// ------------------------------------------------------------------------------------------------
// k_gemm_tc2: the same product, restructured for HBM streaming.  k_gemm_tc splits X in place,
// so a stage's TMA could only be re-armed after the MMAs had consumed it, and the two stages per CTA kept too little
// of X in flight (0.27 ms for Reddit 602 -> 64, ~1/3 of the HBM bound).  Here:
//   * persistent CTAs (one per SM) loop over 128-row tiles, so the X stream never drains between tiles;
//   * a deep ring of raw X tiles (NR x 16 KB, TMA) is decoupled from the operands: the split warps read their
//     rows, write X_hi / X_lo straight into TMEM (tcgen05.st; the MMAs take A from TMEM), and release the raw stage,
//     so the producer runs up to NR chunks ahead and shared memory carries no hi/lo copies and no A reads by the MMAs
//     (the 3xTF32 operand traffic that bounded k_gemm_tc);
//   * the W_hi | W_lo chunks stream through their own ring (WS stages, bulk copies by a dedicated warp), so their
//     L2 latency never sits between a split and its MMAs;
//   * the epilogue writes 128-bit rows.
// Warp 0: X producer (TMA).  Warp 1: TMEM owner and MMA issuer.  Warps 2-5: split, segment drains, epilogue.
// Warp 6: W producer.
// ------------------------------------------------------------------------------------------------
template <int NP>
struct Tc2Cfg {
    static constexpr int BM = 128, BK = 32;
    static constexpr uint32_t RAW_BYTES = BM * BK * 4;                  // 16 KB
    static constexpr uint32_t A_BYTES = BM * BK * 4;
    static constexpr uint32_t B_BYTES = NP * BK * 4;
    static constexpr uint32_t W_BYTES = 2 * B_BYTES;                    // W_hi | W_lo of one K chunk
    // A stages in TMEM: the split of chunk c waits for the MMAs of chunk c - NH, so NH sets how many
    // commit -> mbarrier round trips are in flight (2 stages: 0.2 ms for Reddit 602 -> 16, latency-bound)
#ifndef TC2_NH
#define TC2_NH 6
#endif
#ifndef TC2_CTAS
#define TC2_CTAS 2   // measured (Reddit 602 -> 16 / 64): 1 CTA 0.20 / 0.30 ms, 2 CTAs 0.128 / 0.203 ms
#endif
    static constexpr int CTAS = (TC2_CTAS == 2 && NP <= 64) ? 2 : 1;       // co-resident CTAs per SM
#ifndef TC2_NA
#define TC2_NA 1     // 3: the three products in separate accumulators (measured: no gain)
#endif
    static constexpr int NA = (TC2_NA == 3 && 6 * NP + 2 * 64 <= 512 / CTAS) ? 3 : 1;   // accumulators per slot
    static constexpr int NH_FIT = (512 / CTAS - 2 * NA * NP) / 64;
    static constexpr int NH = NH_FIT < TC2_NH ? NH_FIT : TC2_NH, WS = 4;   // A stages (TMEM), W stages (smem)
    static constexpr size_t BUDGET = (228 * 1024) / CTAS - 1024 /*reserved*/ - 1024 /*align*/ - 512 /*barriers*/;
    static constexpr int NR_FIT = (int)((BUDGET - WS * W_BYTES) / RAW_BYTES);
    static constexpr int NR = NR_FIT > 12 ? 12 : NR_FIT;
    static constexpr int SEG = TC_SEG;
    // TMEM: two accumulator slots [0, 2 NP), then NH A stages of 64 columns (X_hi: 32, X_lo: 32)
    static constexpr uint32_t A_COL0 = 2 * NA * NP;
    static constexpr uint32_t COLS_USED = 2 * NA * NP + NH * 64;
    static constexpr uint32_t TMEM_COLS = COLS_USED <= 64 ? 64 : (COLS_USED <= 128 ? 128 : (COLS_USED <= 256 ? 256 : 512));
    static constexpr size_t SMEM = (size_t)NR * RAW_BYTES + (size_t)WS * W_BYTES + 1024 + 512;
    static_assert(NH >= 2 && NR >= 2, "k_gemm_tc2 does not fit");
};

template <int NP>
__global__ void __launch_bounds__(224, Tc2Cfg<NP>::CTAS) k_gemm_tc2(const __grid_constant__ CUtensorMap tmX, const TcArgs a) {
    using C = Tc2Cfg<NP>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t* raw_base = smem;
    uint8_t* w_base = raw_base + (size_t)C::NR * C::RAW_BYTES;
    uint64_t* bars = reinterpret_cast<uint64_t*>(w_base + (size_t)C::WS * C::W_BYTES);
    uint64_t* raw_full = bars;                       // [NR] TMA landed
    uint64_t* raw_empty = raw_full + C::NR;          // [NR] split warps done reading (128 arrivals)
    uint64_t* split_full = raw_empty + C::NR;        // [NH] hi/lo written (128 arrivals)
    uint64_t* hl_empty = split_full + C::NH;         // [NH] MMAs done reading
    uint64_t* w_full = hl_empty + C::NH;             // [WS] W chunk landed
    uint64_t* w_empty = w_full + C::WS;              // [WS] MMAs done reading
    uint64_t* seg_done = w_empty + C::WS;            // [2]
    uint64_t* slot_free = seg_done + 2;              // [2] (128 arrivals)
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(slot_free + 2);
    auto RAW = [&](int r) { return raw_base + (size_t)r * C::RAW_BYTES; };
    auto B_hi = [&](int w) { return w_base + (size_t)w * C::W_BYTES; };
    auto B_lo = [&](int w) { return w_base + (size_t)w * C::W_BYTES + C::B_BYTES; };

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int nk = (int)((a.K + C::BK - 1) / C::BK);
    const int tiles = (int)((a.M + C::BM - 1) / C::BM);
    // work item = (128-row tile, K split): split s of a tile covers chunks [s nk / S, (s + 1) nk / S)
    const int S = a.ksplit;
    const int items = tiles * S;
    auto k_lo = [&](int it) { return (it % S) * nk / S; };
    auto k_hi = [&](int it) { return (it % S + 1) * nk / S; };

    if (threadIdx.x == 0) {
        for (int r = 0; r < C::NR; ++r) {
            mbar_init(&raw_full[r], 1);
            mbar_init(&raw_empty[r], 128);
        }
        for (int h = 0; h < C::NH; ++h) {
            mbar_init(&split_full[h], 128);
            mbar_init(&hl_empty[h], 1);
        }
        for (int w = 0; w < C::WS; ++w) {
            mbar_init(&w_full[w], 1);
            mbar_init(&w_empty[w], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&seg_done[b], 1);
            mbar_init(&slot_free[b], 128);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(C::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        // ---------------- X producer: raw tiles, up to NR chunks ahead ----------------
        if (lane == 0) {
            int c = 0;
            for (int it = blockIdx.x; it < items; it += gridDim.x) {
                const int tile = it / S;
                for (int kc = k_lo(it); kc < k_hi(it); ++kc, ++c) {
                    const int r = c % C::NR;
                    if (c >= C::NR) mbar_wait(&raw_empty[r], ((c / C::NR) - 1) & 1);
                    mbar_expect_tx(&raw_full[r], C::RAW_BYTES);
                    tma_load_2d(RAW(r), &tmX, kc * C::BK, tile * C::BM, &raw_full[r]);
                }
            }
        }
    } else if (warp == 6) {
        // ---------------- W producer: pre-split W_hi | W_lo chunks, up to WS chunks ahead ----------------
        if (lane == 0) {
            int c = 0;
            for (int it = blockIdx.x; it < items; it += gridDim.x) {
                for (int kc = k_lo(it); kc < k_hi(it); ++kc, ++c) {
                    const int w = c % C::WS;
                    if (c >= C::WS) mbar_wait(&w_empty[w], ((c / C::WS) - 1) & 1);
                    mbar_expect_tx(&w_full[w], C::W_BYTES);
                    bulk_copy(B_hi(w), a.Wsplit + (size_t)kc * C::W_BYTES / sizeof(float), C::W_BYTES, &w_full[w]);
                }
            }
        }
    } else if (warp == 1) {
        // ---------------- MMA issuer ----------------
        const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NP >> 3) << 17) | ((128u >> 4) << 24);
        int c = 0, J = 0;
        for (int it = blockIdx.x; it < items; it += gridDim.x) {
            const int kc0 = k_lo(it), kc1 = k_hi(it);
            for (int kc = kc0; kc < kc1; ++kc, ++c) {
                const int h = c % C::NH, w = c % C::WS;
                const int j = J + (kc - kc0) / C::SEG, slot = j & 1;
                const bool first = ((kc - kc0) % C::SEG) == 0;
                if (first && j >= 2) mbar_wait(&slot_free[slot], ((j >> 1) - 1) & 1);   // segment j-2 drained
                mbar_wait(&split_full[h], (c / C::NH) & 1);
                mbar_wait(&w_full[w], (c / C::WS) & 1);
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                if (lane == 0) {
                    const uint32_t ah = tmem + C::A_COL0 + (uint32_t)h * 64, al = ah + 32;   // A in TMEM (K-major)
                    const uint64_t bh = smem_desc_k128(B_hi(w)), bl = smem_desc_k128(B_lo(w));
                    const uint32_t d0 = tmem + (uint32_t)(slot * C::NA * NP);
                    const uint32_t d1 = d0 + (C::NA > 1 ? NP : 0), d2 = d0 + (C::NA > 1 ? 2 * NP : 0);
#pragma unroll
                    for (int ks = 0; ks < C::BK / 8; ++ks) {
                        const uint64_t adv = (uint64_t)((ks * 8 * 4) >> 4);
                        const uint32_t init = (!first || ks > 0) ? 1u : 0u;
                        mma_tf32_ts(d0, al + ks * 8, bh + adv, idesc, init);
                        mma_tf32_ts(d1, ah + ks * 8, bl + adv, idesc, C::NA > 1 ? init : 1u);
                        mma_tf32_ts(d2, ah + ks * 8, bh + adv, idesc, C::NA > 1 ? init : 1u);
                    }
                    mma_commit(&hl_empty[h]);
                    mma_commit(&w_empty[w]);
                    if (((kc - kc0) % C::SEG) == C::SEG - 1 || kc == kc1 - 1) mma_commit(&seg_done[slot]);
                }
                __syncwarp();
            }
            J += (kc1 - kc0 + C::SEG - 1) / C::SEG;
        }
    } else {
        // ---------------- split, segment drains, epilogue (warps 2-5) ----------------
        const int t = threadIdx.x - 64;
        const int q4 = warp & 3;
        float racc[NP];
#pragma unroll
        for (int j = 0; j < NP; ++j) racc[j] = 0.f;
        int c = 0, J = 0;
        for (int it = blockIdx.x; it < items; it += gridDim.x) {
            const int tile = it / S;
            const int kc0 = k_lo(it), kc1 = k_hi(it);
            const int nseg = (kc1 - kc0 + C::SEG - 1) / C::SEG;
            for (int kc = kc0; kc < kc1; ++kc, ++c) {
                const int r = c % C::NR, h = c % C::NH;
                mbar_wait(&raw_full[r], (c / C::NR) & 1);
                // this thread's row (TMEM lane) of the 128B-swizzled raw tile: chunk q of row rr sits at
                // rr * 128 + ((q ^ (rr & 7)) * 16) (8 consecutive rows hit 8 different bank groups)
                const int rr = q4 * 32 + lane;
                const uint8_t* prow = RAW(r) + rr * 128;
                float4 xv[8];
#pragma unroll
                for (int q = 0; q < 8; ++q) xv[q] = *reinterpret_cast<const float4*>(prow + ((q ^ (rr & 7)) << 4));
                if (c >= C::NH) mbar_wait(&hl_empty[h], ((c / C::NH) - 1) & 1);   // A stage h is free
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                const uint32_t ta = tmem + ((uint32_t)(q4 * 32) << 16) + C::A_COL0 + (uint32_t)h * 64;
#pragma unroll
                for (int half = 0; half < 2; ++half) {
                    uint32_t hv[16], lv[16];
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const float4 x = xv[4 * half + q];
                        const float xs[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
                        for (int u = 0; u < 4; ++u) {
                            const float hh = rna_tf32(xs[u]);
                            hv[4 * q + u] = __float_as_uint(hh);
                            lv[4 * q + u] = __float_as_uint(xs[u] - hh);
                        }
                    }
                    tmem_st16(ta + half * 16, hv);
                    tmem_st16(ta + 32 + half * 16, lv);
                }
                asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
                asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
                mbar_arrive(&split_full[h]);
                mbar_arrive(&raw_empty[r]);                   // after the raw values were consumed (see k_gemm_tc_tn2)
                if ((((kc - kc0) % C::SEG) == C::SEG - 1 || kc == kc1 - 1) && (kc - kc0) / C::SEG >= 1)
                    drain_segment<NP, C::NA>(tmem, J + (kc - kc0) / C::SEG - 1, q4, seg_done, slot_free, racc);
            }
            if (nseg > 0) drain_segment<NP, C::NA>(tmem, J + nseg - 1, q4, seg_done, slot_free, racc);
            J += nseg;
            const int64_t gm = (int64_t)tile * C::BM + q4 * 32 + lane;
            if (S > 1 && gm < a.M) {
                // K split: the raw partial row (no epilogue) -> part[s][gm][0 .. NP); k_splitk_reduce finishes it
                float4* pp = reinterpret_cast<float4*>(a.part + ((it % S) * a.M + gm) * NP);
#pragma unroll
                for (int j = 0; j < NP; j += 4) pp[j / 4] = make_float4(racc[j], racc[j + 1], racc[j + 2], racc[j + 3]);
            }
            // epilogue: bias, activation, row scale; 128-bit stores when the rows allow it
            if (S == 1 && gm < a.M) {
                const float rs = a.row_scale ? __ldg(a.row_scale + gm) : 1.f;
                float* y = a.Y + gm * a.ldy;
                const bool vec = (a.ldy & 3) == 0 && aligned16(a.Y);
#pragma unroll
                for (int j = 0; j < NP; j += 4) {
                    float z[4];
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        z[q] = rs * act_apply(a.act, racc[j + q] + ((a.bias && j + q < a.N) ? __ldg(a.bias + j + q) : 0.f));
                    if (vec && j + 4 <= a.N) {
                        *reinterpret_cast<float4*>(y + j) = make_float4(z[0], z[1], z[2], z[3]);
                    } else {
#pragma unroll
                        for (int q = 0; q < 4; ++q)
                            if (j + q < a.N) y[j + q] = z[q];
                    }
                }
            }
#pragma unroll
            for (int j = 0; j < NP; ++j) racc[j] = 0.f;
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 1) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(C::TMEM_COLS));
    }
}

// W [K, N] -> per 32-wide K chunk: W_hi = rna_tf32(W) and W_lo = W - W_hi as NP x 32 K-major tiles in the
// 128B-swizzled layout the UMMA descriptor expects (element (n, k) at n*128 + ((k/4 ^ n%8)*16 | (k%4)*4))
__global__ void k_split_w(const float* __restrict__ W, int64_t K, int64_t N, int NP, float* __restrict__ out) {
    const int64_t nk = (K + 31) / 32;
    const int64_t total = nk * NP * 32;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t kc = i / (NP * 32);
        const int r = (int)(i % (NP * 32));
        const int n = r / 32, k = r % 32;
        const int64_t gk = kc * 32 + k;
        const float w = (n < N && gk < K) ? W[gk * N + n] : 0.f;
        const float wh = rna_tf32(w);
        const uint32_t off = (uint32_t)(n * 128 + ((((k >> 2) ^ (n & 7)) << 4) | ((k & 3) << 2))) / 4;
        float* tile = out + kc * 2 * NP * 32;
        tile[off] = wh;
        tile[NP * 32 + off] = w - wh;
    }
}

static size_t wsplit_bytes(int64_t K, int64_t N) {
    const int64_t np = (N + 15) / 16 * 16;
    return ((size_t)((K + 31) / 32) * 2 * np * 32 * sizeof(float) + 255) & ~size_t(255);
}
// + room for the K-split partials of k_gemm_tc2 (K >= 1024, N <= 64: the long-K transforms)
static size_t splitk_part_bytes(int64_t K, int64_t N) {
    if (K < 1024 || N > 64) return 0;
    const int64_t np = (N + 15) / 16 * 16;
    return (size_t)kSplitKMax * (size_t)splitk_max_rows() * (size_t)np * sizeof(float);
}
size_t linear_fwd_tc_workspace(int64_t K, int64_t N) { return wsplit_bytes(K, N) + splitk_part_bytes(K, N) + 256; }

// ------------------------------------------------------------------------------------------------
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
        cudaGetLastError();
    });
    return fn;
}

// K-split finish: Y[m, j] = row_scale[m] * act(sum_s part[s][m][j] + bias[j]), splits summed in order
template <int NP>
__global__ void __launch_bounds__(256) k_splitk_reduce(const float* __restrict__ part, int S, int64_t M, int N,
                                                       const float* __restrict__ bias, const float* __restrict__ row_scale,
                                                       int act, float* __restrict__ Y, int64_t ldy) {
    constexpr int Q = NP / 4;
    const int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (idx >= M * Q) return;
    const int64_t m = idx / Q;
    const int q = (int)(idx % Q);
    float4 z = __ldcs(reinterpret_cast<const float4*>(part + m * NP) + q);
    for (int sp = 1; sp < S; ++sp) {
        const float4 v = __ldcs(reinterpret_cast<const float4*>(part + ((int64_t)sp * M + m) * NP) + q);
        z.x += v.x; z.y += v.y; z.z += v.z; z.w += v.w;
    }
    const float rs = row_scale ? __ldg(row_scale + m) : 1.f;
    const float zz[4] = {z.x, z.y, z.z, z.w};
    float* y = Y + m * ldy + 4 * q;
    float o[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) o[u] = rs * act_apply(act, zz[u] + ((bias && 4 * q + u < N) ? __ldg(bias + 4 * q + u) : 0.f));
    if (4 * q + 4 <= N && (ldy & 3) == 0 && aligned16(Y)) {
        *reinterpret_cast<float4*>(y) = make_float4(o[0], o[1], o[2], o[3]);
    } else {
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (4 * q + u < N) y[u] = o[u];
    }
}

// K splits for k_gemm_tc2 when the row tiles alone cannot fill the grid (CoraFull / Physics / Cora: few rows, long K):
// the split count minimising (waves of work items) x (chunks per item)
static int choose_ksplit(int64_t tiles, int nk, int64_t slots) {
    int best = 1;
    int64_t best_cost = nk;
    for (int S = 2; S <= kSplitKMax; S *= 2) {
        if (nk < 4 * S) break;
        const int64_t cost = ((tiles * S + slots - 1) / slots) * ((nk + S - 1) / S) + 2;   // + the reduce pass
        if (cost < best_cost) { best_cost = cost; best = S; }
    }
    return best;
}
template <int NP>
static seastar_status launch_tc_np(const CUtensorMap& tm, const TcArgs& a, cudaStream_t s) {
    // NP <= 64 (every BASELINE transform): k_gemm_tc2; wider outputs and SEASTAR_TC_V1=1 (A/B): k_gemm_tc
    if constexpr (NP <= 64) {
        const char* v1 = getenv("SEASTAR_TC_V1");
        if (!(v1 && v1[0] == '1')) {
            using C2 = Tc2Cfg<NP>;
            SS_CUDA(cudaFuncSetAttribute(k_gemm_tc2<NP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C2::SMEM));
            const int64_t tiles = (a.M + C2::BM - 1) / C2::BM;
            const int64_t slots = (int64_t)C2::CTAS * num_sms();
            TcArgs b = a;
            b.ksplit = (a.part && a.M <= splitk_max_rows()) ? choose_ksplit(tiles, (int)((a.K + 31) / 32), slots) : 1;
            const int64_t items = tiles * b.ksplit;
            const unsigned grid = (unsigned)(items < slots ? items : slots);
            k_gemm_tc2<NP><<<grid, 224, C2::SMEM, s>>>(tm, b);
            SS_TRY(check_launch("k_gemm_tc2"));
            if (b.ksplit > 1) {
                const int64_t n = a.M * (NP / 4);
                k_splitk_reduce<NP><<<(unsigned)((n + 255) / 256), 256, 0, s>>>(b.part, b.ksplit, a.M, (int)a.N, a.bias,
                                                                             a.row_scale, a.act, a.Y, a.ldy);
                SS_TRY(check_launch("k_splitk_reduce"));
            }
            return SEASTAR_OK;
        }
    }
    using C = TcCfg<NP>;
    // set per call: the attribute is per device, and setting it is a cheap host-side call
    SS_CUDA(cudaFuncSetAttribute(k_gemm_tc<NP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::SMEM));
    const unsigned grid = (unsigned)((a.M + C::BM - 1) / C::BM);
    k_gemm_tc<NP><<<grid, 192, C::SMEM, s>>>(tm, a);
    return check_launch("k_gemm_tc");
}

// returns SEASTAR_ERR_UNSUPPORTED (without launching) when the tensor-core path does not apply
seastar_status linear_fwd_tc(const float* X, int64_t M, int64_t K, int64_t ldx, const float* W, int64_t N,
                             const float* bias, const float* row_scale, int act, float* Y, int64_t ldy,
                             void* ws, size_t ws_bytes, cudaStream_t s) {
    if (getenv("SEASTAR_NO_TCGEN05") || M < 128 || K < 32 || N > 128 || (ldx % 4) != 0 || !aligned16(X) ||
        M >= (1LL << 31) || K >= (1LL << 31) || !ws || !aligned16(ws) || ws_bytes < linear_fwd_tc_workspace(K, N))
        return SEASTAR_ERR_UNSUPPORTED;
    auto enc = encode_fn();
    if (!enc) return SEASTAR_ERR_UNSUPPORTED;
    CUtensorMap tm;
    cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)M};
    cuuint64_t strides[1] = {(cuuint64_t)ldx * sizeof(float)};
    cuuint32_t box[2] = {32, 128};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(X), dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return SEASTAR_ERR_UNSUPPORTED;
    const int np = (int)((N + 15) / 16 * 16);
    float* wsplit = static_cast<float*>(ws);
    {
        const int64_t total = (K + 31) / 32 * np * 32;
        k_split_w<<<(unsigned)((total + 255) / 256), 256, 0, s>>>(W, K, N, np, wsplit);
        SS_TRY(check_launch("k_split_w"));
    }
    TcArgs a{M, K, N, wsplit, Y, ldy, bias, row_scale, act};
    if (splitk_part_bytes(K, N)) a.part = reinterpret_cast<float*>(static_cast<char*>(ws) + wsplit_bytes(K, N));
    switch (np) {
        case 16: return launch_tc_np<16>(tm, a, s);
        case 32: return launch_tc_np<32>(tm, a, s);
        case 48: return launch_tc_np<48>(tm, a, s);
        case 64: return launch_tc_np<64>(tm, a, s);
        case 80: return launch_tc_np<80>(tm, a, s);
        case 96: return launch_tc_np<96>(tm, a, s);
        case 128: return launch_tc_np<128>(tm, a, s);
        default: return SEASTAR_ERR_UNSUPPORTED;
    }
}


// ================================================================================================
// dW = X^T dY on tcgen05 (3xTF32), both operands MN-major straight from TMA -- no transpose pass.
//   D[k, n] (128 x NP32 per CTA) = sum_m X[m, k] dY[m, n] over the CTA's row split.
// A = X^T (M' = k, K' = m): a TMA box of 32 k-columns x 32 m-rows (SWIZZLE_128B_ATOM_32B) lands as
// the canonical MN-major tf32 layout (128 B rows, 32 B chunks swizzled within 4-row groups); the 4
// column blocks of the 128-wide k tile sit LBO = 4 KB apart.  B = dY^T likewise (NP32 / 32 column blocks; columns >= N
// are zero-filled by TMA).  Each 8-row K step advances both descriptors by 1024 B.
// Row splits are multiples of 32 rows, so every 32-row chunk belongs to exactly one split; the
// per-split partials [nsplit][K][N] are summed in split order afterwards (deterministic).
// ================================================================================================
struct TcTnArgs {
    int64_t M, K, N;
    int64_t rows_per_split;
    float* part;                     // [nsplit][K][N]
};

template <int NP32>
struct TcTnCfg {
    static constexpr int BM = 128, BR = 32;                   // k tile, rows per stage
    static constexpr int CTAS = 2, STAGES = 2;
    static constexpr uint32_t A_BYTES = BM * BR * 4;           // 16 KB
    static constexpr uint32_t B_BYTES = NP32 * BR * 4;         // 4 KB per 32 columns
    static constexpr uint32_t STAGE_BYTES = 2 * A_BYTES + 2 * B_BYTES;
    // segments of SEG 32-row chunks ping-pong between two TMEM slots and are drained into fp32
    // registers (drain_segment, as in k_gemm_tc): no TMEM accumulation spans more than SEG * 12 MMAs
    static constexpr int SEG = TC_TN_SEG;
    static constexpr uint32_t TMEM_COLS = 2 * NP32 <= 64 ? 64 : 128;
    static constexpr size_t SMEM = (size_t)STAGES * STAGE_BYTES + 1024 + 256;
};

// MN-major tf32 operand: the only UMMA layout for it is SWIZZLE_128B_BASE32B (layout type 1): 128 B
// rows along MN (32 elements) whose 32 B chunks are XOR-permuted by (row & 3) -- what TMA writes with
// CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B.  LBO = bytes between 32-element MN blocks, SBO = bytes between
// 4-row K groups (512 for densely stacked rows).
__device__ __forceinline__ uint64_t smem_desc_mn32b(const void* p, uint32_t lbo) {
    const uint32_t a = smem_u32(p);
    uint64_t d = (uint64_t)((a >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)(512 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)1 << 61;
    return d;
}

template <int NP32>
__global__ void __launch_bounds__(192, TcTnCfg<NP32>::CTAS)
    k_gemm_tc_tn(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmY, const TcTnArgs a) {
    using C = TcTnCfg<NP32>;
    constexpr int NB = NP32 / 32;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + (size_t)C::STAGES * C::STAGE_BYTES);
    uint64_t* full = bars;
    uint64_t* split = bars + C::STAGES;
    uint64_t* empty = bars + 2 * C::STAGES;
    uint64_t* seg_done = bars + 3 * C::STAGES;   // [2]
    uint64_t* slot_free = seg_done + 2;          // [2] (128 arrivals)
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(seg_done + 4);
    auto A_hi = [&](int s) { return smem + (size_t)s * C::STAGE_BYTES; };
    auto A_lo = [&](int s) { return smem + (size_t)s * C::STAGE_BYTES + C::A_BYTES; };
    auto B_hi = [&](int s) { return smem + (size_t)s * C::STAGE_BYTES + 2 * C::A_BYTES; };
    auto B_lo = [&](int s) { return smem + (size_t)s * C::STAGE_BYTES + 2 * C::A_BYTES + C::B_BYTES; };

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int k0 = blockIdx.x * C::BM;
    const int64_t r0 = (int64_t)blockIdx.y * a.rows_per_split;
    const int64_t r1 = min(a.M, r0 + a.rows_per_split);
    const int nch = (int)((r1 - r0 + C::BR - 1) / C::BR);

    if (threadIdx.x == 0) {
        for (int s = 0; s < C::STAGES; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&split[s], 128);
            mbar_init(&empty[s], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&seg_done[b], 1);
            mbar_init(&slot_free[b], 128);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmY)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(C::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0 && nch > 0) {
            for (int c = 0; c < nch; ++c) {
                const int s = c % C::STAGES;
                if (c >= C::STAGES) mbar_wait(&empty[s], ((c / C::STAGES) - 1) & 1);
                mbar_expect_tx(&full[s], C::A_BYTES + C::B_BYTES);
                const int m = (int)(r0 + (int64_t)c * C::BR);
#pragma unroll
                for (int j = 0; j < 4; ++j) tma_load_2d(A_hi(s) + j * 4096, &tmX, k0 + 32 * j, m, &full[s]);
#pragma unroll
                for (int j = 0; j < NB; ++j) tma_load_2d(B_hi(s) + j * 4096, &tmY, 32 * j, m, &full[s]);
            }
        }
    } else if (warp == 1) {
        // D f32, A/B tf32, both MN-major (bits 15, 16), N = NP32, M = 128
        const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 15) | (1u << 16) |
                               ((uint32_t)(NP32 >> 3) << 17) | ((128u >> 4) << 24);
        for (int c = 0; c < nch; ++c) {
            const int s = c % C::STAGES;
            const int j = c / C::SEG, slot = j & 1;
            const bool first = (c % C::SEG) == 0;
            if (first && j >= 2) mbar_wait(&slot_free[slot], ((j >> 1) - 1) & 1);   // segment j-2 drained
            mbar_wait(&split[s], (c / C::STAGES) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            if (lane == 0) {
                const uint32_t d = tmem + (uint32_t)(slot * NP32);
#pragma unroll
                for (int ks = 0; ks < C::BR / 8; ++ks) {
                    const uint64_t ah = smem_desc_mn32b(A_hi(s) + ks * 1024, 4096);
                    const uint64_t al = smem_desc_mn32b(A_lo(s) + ks * 1024, 4096);
                    const uint64_t bh = smem_desc_mn32b(B_hi(s) + ks * 1024, 4096);
                    const uint64_t bl = smem_desc_mn32b(B_lo(s) + ks * 1024, 4096);
                    mma_tf32(d, al, bh, idesc, (!first || ks > 0) ? 1u : 0u);
                    mma_tf32(d, ah, bl, idesc, 1u);
                    mma_tf32(d, ah, bh, idesc, 1u);
                }
                mma_commit(&empty[s]);
                if ((c % C::SEG) == C::SEG - 1 || c == nch - 1) mma_commit(&seg_done[slot]);
            }
            __syncwarp();
        }
    } else {
        const int t = threadIdx.x - 64;
        const int q4 = warp & 3;
        float racc[NP32];
#pragma unroll
        for (int j = 0; j < NP32; ++j) racc[j] = 0.f;
        for (int c = 0; c < nch; ++c) {
            const int s = c % C::STAGES;
            mbar_wait(&full[s], (c / C::STAGES) & 1);
            // elementwise hi / lo split in place (layout preserving, conflict-free 16 B chunks)
            float4* ph = reinterpret_cast<float4*>(A_hi(s));
            float4* pl = reinterpret_cast<float4*>(A_lo(s));
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const float4 x = ph[q * 128 + t];
                const float4 h = make_float4(rna_tf32(x.x), rna_tf32(x.y), rna_tf32(x.z), rna_tf32(x.w));
                ph[q * 128 + t] = h;
                pl[q * 128 + t] = make_float4(x.x - h.x, x.y - h.y, x.z - h.z, x.w - h.w);
            }
            float4* qh = reinterpret_cast<float4*>(B_hi(s));
            float4* ql = reinterpret_cast<float4*>(B_lo(s));
#pragma unroll
            for (int q = 0; q < NB * 2; ++q) {
                const float4 x = qh[q * 128 + t];
                const float4 h = make_float4(rna_tf32(x.x), rna_tf32(x.y), rna_tf32(x.z), rna_tf32(x.w));
                qh[q * 128 + t] = h;
                ql[q * 128 + t] = make_float4(x.x - h.x, x.y - h.y, x.z - h.z, x.w - h.w);
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive(&split[s]);
            if (((c % C::SEG) == C::SEG - 1 || c == nch - 1) && c / C::SEG >= 1)
                drain_segment<NP32>(tmem, c / C::SEG - 1, q4, seg_done, slot_free, racc);
        }
        if (nch > 0) drain_segment<NP32>(tmem, (nch - 1) / C::SEG, q4, seg_done, slot_free, racc);
        // epilogue: partial[split][k0 + r][n]
        const int r = q4 * 32 + lane;
        const int64_t gk = k0 + r;
        if (gk < a.K) {
            float* prow = a.part + ((int64_t)blockIdx.y * a.K + gk) * a.N;
#pragma unroll
            for (int j = 0; j < NP32; ++j)
                if (j < a.N) prow[j] = racc[j];
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 1) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(C::TMEM_COLS));
    }
}

// ------------------------------------------------------------------------------------------------
// k_gemm_tc_tn2: dW = X^T dY with the same restructuring as k_gemm_tc2.  A = X^T (M' = 128 features k of the tile,
// K' = rows m) is K-major when each TMEM lane k holds consecutive rows m: the split warps read column k of a raw
// X tile ([32 m][128 k], plain row-major TMA box, lane-consecutive words: conflict-free), write X_hi / X_lo into
// TMEM, and the MMAs take A from there.  B = dY^T stays an MN-major shared-memory operand (SWIZZLE_128B_ATOM_32B,
// split in place into a B stage).  Raw stages (X tile + dY tile) are released right after the split, so TMA runs
// NR chunks ahead; 2 CTAs per SM.  Per-split partials [nsplit][K][N] as before (reduced in split order).
// ------------------------------------------------------------------------------------------------
template <int NP32>
struct TcTn2Cfg {
    static constexpr int BM = 128, BR = 32;                   // k tile, rows per chunk
    static constexpr int CTAS = 2;
    static constexpr uint32_t X_BYTES = BR * BM * 4;           // 16 KB raw X tile
    static constexpr uint32_t Y_BYTES = NP32 * BR * 4;         // 4 KB per 32 columns (4 KB-aligned boxes)
    static constexpr uint32_t RAW_BYTES = X_BYTES + Y_BYTES;
    static constexpr uint32_t B_BYTES = NP32 * BR * 4;
    static constexpr int NH = (256 - 2 * NP32) / 64 > 3 ? 3 : (256 - 2 * NP32) / 64;   // A stages (TMEM) = B stages
    static constexpr size_t BUDGET = (228 * 1024) / CTAS - 1024 - 1024 - 256;
    static constexpr int NR_FIT = (int)((BUDGET - (size_t)NH * 2 * B_BYTES) / RAW_BYTES);
    static constexpr int NR = NR_FIT > 8 ? 8 : NR_FIT;
    static constexpr int SEG = TC_TN_SEG;
    static constexpr uint32_t A_COL0 = 2 * NP32;
    static constexpr uint32_t TMEM_COLS = 256;
    static constexpr size_t SMEM = (size_t)NR * RAW_BYTES + (size_t)NH * 2 * B_BYTES + 1024 + 256;
    static_assert(NH >= 2 && NR >= 2, "k_gemm_tc_tn2 does not fit");
};

template <int NP32>
__global__ void __launch_bounds__(192, TcTn2Cfg<NP32>::CTAS)
    k_gemm_tc_tn2(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmY, const TcTnArgs a) {
    using C = TcTn2Cfg<NP32>;
    constexpr int NB = NP32 / 32;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t* raw_base = smem;
    uint8_t* b_base = raw_base + (size_t)C::NR * C::RAW_BYTES;
    uint64_t* bars = reinterpret_cast<uint64_t*>(b_base + (size_t)C::NH * 2 * C::B_BYTES);
    uint64_t* raw_full = bars;                   // [NR]
    uint64_t* raw_empty = raw_full + C::NR;      // [NR] (128 arrivals)
    uint64_t* split_full = raw_empty + C::NR;    // [NH] (128 arrivals)
    uint64_t* hl_empty = split_full + C::NH;     // [NH]
    uint64_t* seg_done = hl_empty + C::NH;       // [2]
    uint64_t* slot_free = seg_done + 2;          // [2] (128 arrivals)
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(slot_free + 2);
    auto RX = [&](int r) { return raw_base + (size_t)r * C::RAW_BYTES; };
    auto RY = [&](int r) { return raw_base + (size_t)r * C::RAW_BYTES + C::X_BYTES; };
    auto B_hi = [&](int h) { return b_base + (size_t)h * 2 * C::B_BYTES; };
    auto B_lo = [&](int h) { return b_base + (size_t)h * 2 * C::B_BYTES + C::B_BYTES; };

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int k0 = blockIdx.x * C::BM;
    const int64_t r0 = (int64_t)blockIdx.y * a.rows_per_split;
    const int64_t r1 = min(a.M, r0 + a.rows_per_split);
    const int nch = (int)((r1 - r0 + C::BR - 1) / C::BR);

    if (threadIdx.x == 0) {
        for (int r = 0; r < C::NR; ++r) {
            mbar_init(&raw_full[r], 1);
            mbar_init(&raw_empty[r], 128);
        }
        for (int h = 0; h < C::NH; ++h) {
            mbar_init(&split_full[h], 128);
            mbar_init(&hl_empty[h], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&seg_done[b], 1);
            mbar_init(&slot_free[b], 128);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmY)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(C::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            for (int c = 0; c < nch; ++c) {
                const int r = c % C::NR;
                if (c >= C::NR) mbar_wait(&raw_empty[r], ((c / C::NR) - 1) & 1);
                mbar_expect_tx(&raw_full[r], C::X_BYTES + C::Y_BYTES);
                const int m = (int)(r0 + (int64_t)c * C::BR);
                tma_load_2d(RX(r), &tmX, k0, m, &raw_full[r]);
#pragma unroll
                for (int j = 0; j < NB; ++j) tma_load_2d(RY(r) + j * 4096, &tmY, 32 * j, m, &raw_full[r]);
            }
        }
    } else if (warp == 1) {
        // D f32, A/B tf32, A K-major (TMEM), B MN-major (bit 16), N = NP32, M = 128
        const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 16) | ((uint32_t)(NP32 >> 3) << 17) |
                               ((128u >> 4) << 24);
        for (int c = 0; c < nch; ++c) {
            const int h = c % C::NH;
            const int j = c / C::SEG, slot = j & 1;
            const bool first = (c % C::SEG) == 0;
            if (first && j >= 2) mbar_wait(&slot_free[slot], ((j >> 1) - 1) & 1);
            mbar_wait(&split_full[h], (c / C::NH) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            if (lane == 0) {
                const uint32_t d = tmem + (uint32_t)(slot * NP32);
                const uint32_t ah = tmem + C::A_COL0 + (uint32_t)h * 64, al = ah + 32;
#pragma unroll
                for (int ks = 0; ks < C::BR / 8; ++ks) {
                    const uint64_t bh = smem_desc_mn32b(B_hi(h) + ks * 1024, 4096);
                    const uint64_t bl = smem_desc_mn32b(B_lo(h) + ks * 1024, 4096);
                    mma_tf32_ts(d, al + ks * 8, bh, idesc, (!first || ks > 0) ? 1u : 0u);
                    mma_tf32_ts(d, ah + ks * 8, bl, idesc, 1u);
                    mma_tf32_ts(d, ah + ks * 8, bh, idesc, 1u);
                }
                mma_commit(&hl_empty[h]);
                if ((c % C::SEG) == C::SEG - 1 || c == nch - 1) mma_commit(&seg_done[slot]);
            }
            __syncwarp();
        }
    } else {
        const int t = threadIdx.x - 64;
        const int q4 = warp & 3;
        const int kk = q4 * 32 + lane;                  // this thread's TMEM lane = feature k0 + kk
        float racc[NP32];
#pragma unroll
        for (int j = 0; j < NP32; ++j) racc[j] = 0.f;
        for (int c = 0; c < nch; ++c) {
            const int r = c % C::NR, h = c % C::NH;
            mbar_wait(&raw_full[r], (c / C::NR) & 1);
            const float* px = reinterpret_cast<const float*>(RX(r)) + kk;
            float xc[32];
#pragma unroll
            for (int m = 0; m < 32; ++m) xc[m] = px[m * 128];     // column kk of the [32 m][128 k] tile
            const float4* qy = reinterpret_cast<const float4*>(RY(r));
            float4 yv[NB * 2];
#pragma unroll
            for (int q = 0; q < NB * 2; ++q) yv[q] = qy[q * 128 + t];
            if (c >= C::NH) mbar_wait(&hl_empty[h], ((c / C::NH) - 1) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t ta = tmem + ((uint32_t)(q4 * 32) << 16) + C::A_COL0 + (uint32_t)h * 64;
#pragma unroll
            for (int half = 0; half < 2; ++half) {
                uint32_t hv[16], lv[16];
#pragma unroll
                for (int u = 0; u < 16; ++u) {
                    const float x = xc[16 * half + u];
                    const float hh = rna_tf32(x);
                    hv[u] = __float_as_uint(hh);
                    lv[u] = __float_as_uint(x - hh);
                }
                tmem_st16(ta + half * 16, hv);
                tmem_st16(ta + 32 + half * 16, lv);
            }
            float4* bh = reinterpret_cast<float4*>(B_hi(h));
            float4* bl = reinterpret_cast<float4*>(B_lo(h));
#pragma unroll
            for (int q = 0; q < NB * 2; ++q) {                    // layout-preserving split of the dY tile
                const float4 x = yv[q];
                const float4 hh = make_float4(rna_tf32(x.x), rna_tf32(x.y), rna_tf32(x.z), rna_tf32(x.w));
                bh[q * 128 + t] = hh;
                bl[q * 128 + t] = make_float4(x.x - hh.x, x.y - hh.y, x.z - hh.z, x.w - hh.w);
            }
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
            asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive(&split_full[h]);
            // the raw stage is released only after its values were consumed (the TMA refill is an async-proxy write;
            // arriving right after issuing the loads let refills race with loads still in flight at large M)
            mbar_arrive(&raw_empty[r]);
            if (((c % C::SEG) == C::SEG - 1 || c == nch - 1) && c / C::SEG >= 1)
                drain_segment<NP32>(tmem, c / C::SEG - 1, q4, seg_done, slot_free, racc);
        }
        if (nch > 0) drain_segment<NP32>(tmem, (nch - 1) / C::SEG, q4, seg_done, slot_free, racc);
        const int64_t gk = k0 + kk;
        if (gk < a.K) {
            float* prow = a.part + ((int64_t)blockIdx.y * a.K + gk) * a.N;
#pragma unroll
            for (int j = 0; j < NP32; ++j)
                if (j < a.N) prow[j] = racc[j];
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 1) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(C::TMEM_COLS));
    }
}

// row splits (multiples of 32 rows) so that ktiles x nsplit fills ~4 waves of 2 CTAs per SM
#ifndef TCTN_CTAS_PER_SM
#define TCTN_CTAS_PER_SM 4   // CTAs per SM the row splits aim for (measured on Reddit 602 x 64: 8 -> 0.237 ms, 4 -> 0.205, 2 -> 0.252)
#endif
static void tc_tn_geometry(int64_t M, int64_t K, int64_t& ktiles, int64_t& nsplit, int64_t& rows_per_split) {
    ktiles = (K + 127) / 128;
    int64_t want = (TCTN_CTAS_PER_SM * num_sms() + ktiles - 1) / ktiles;
    int64_t max_split = (M + 255) / 256;
    nsplit = want < max_split ? want : max_split;
    if (nsplit < 1) nsplit = 1;
    rows_per_split = (M + nsplit - 1) / nsplit;
    rows_per_split = (rows_per_split + 31) / 32 * 32;
    nsplit = (M + rows_per_split - 1) / rows_per_split;
    if (nsplit < 1) nsplit = 1;
}

size_t linear_bwd_weight_tc_part_bytes(int64_t M, int64_t K, int64_t N) {
    int64_t kt, ns, rps;
    tc_tn_geometry(M > 0 ? M : 1, K, kt, ns, rps);
    return (size_t)ns * K * N * sizeof(float);
}

template <int NP32>
static seastar_status launch_tc_tn2(const CUtensorMap& tx, const CUtensorMap& ty, const TcTnArgs& a, dim3 grid,
                                    cudaStream_t s) {
    using C = TcTn2Cfg<NP32>;
    SS_CUDA(cudaFuncSetAttribute(k_gemm_tc_tn2<NP32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::SMEM));
    k_gemm_tc_tn2<NP32><<<grid, 192, C::SMEM, s>>>(tx, ty, a);
    return check_launch("k_gemm_tc_tn2");
}

template <int NP32>
static seastar_status launch_tc_tn(const CUtensorMap& tx, const CUtensorMap& ty, const TcTnArgs& a, dim3 grid,
                                   cudaStream_t s) {
    using C = TcTnCfg<NP32>;
    // set per call: the attribute is per device, and setting it is a cheap host-side call
    SS_CUDA(cudaFuncSetAttribute(k_gemm_tc_tn<NP32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::SMEM));
    k_gemm_tc_tn<NP32><<<grid, 192, C::SMEM, s>>>(tx, ty, a);
    return check_launch("k_gemm_tc_tn");
}

// writes the per-split partials into part (linear_bwd_weight_tc_part_bytes) and returns the split
// count in *nsplit_out; SEASTAR_ERR_UNSUPPORTED (nothing launched) when the path does not apply
seastar_status linear_bwd_weight_tc(const float* X, int64_t M, int64_t K, int64_t ldx, const float* dY, int64_t N,
                                    int64_t ldy, float* part, int64_t* nsplit_out, cudaStream_t s) {
    if (getenv("SEASTAR_NO_TCGEN05") || M < 256 || K < 32 || N > 64 || (ldx % 4) != 0 || (ldy % 4) != 0 ||
        !aligned16(X) || !aligned16(dY) || M >= (1LL << 31) || K >= (1LL << 31))
        return SEASTAR_ERR_UNSUPPORTED;
    auto enc = encode_fn();
    if (!enc) return SEASTAR_ERR_UNSUPPORTED;
    CUtensorMap tx, ty;
    {
        cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)M};
        cuuint64_t strides[1] = {(cuuint64_t)ldx * sizeof(float)};
        cuuint32_t box[2] = {32, 32};
        cuuint32_t estr[2] = {1, 1};
        if (enc(&tx, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(X), dims, strides, box, estr,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
            return SEASTAR_ERR_UNSUPPORTED;
    }
    {
        cuuint64_t dims[2] = {(cuuint64_t)N, (cuuint64_t)M};
        cuuint64_t strides[1] = {(cuuint64_t)ldy * sizeof(float)};
        cuuint32_t box[2] = {32, 32};
        cuuint32_t estr[2] = {1, 1};
        if (enc(&ty, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(dY), dims, strides, box, estr,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
            return SEASTAR_ERR_UNSUPPORTED;
    }
    int64_t kt, ns, rps;
    tc_tn_geometry(M, K, kt, ns, rps);
    TcTnArgs a{M, K, N, rps, part};
    *nsplit_out = ns;
    const dim3 grid((unsigned)kt, (unsigned)ns);
    const char* v1 = getenv("SEASTAR_TC_V1");   // A/B: the r1/r2 in-place-split kernel
    if (!(v1 && v1[0] == '1')) {
        // k_gemm_tc_tn2: X as plain [32 rows][128 features] boxes (each split thread reads one feature column)
        CUtensorMap tx2;
        cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)M};
        cuuint64_t strides[1] = {(cuuint64_t)ldx * sizeof(float)};
        cuuint32_t box[2] = {128, 32};
        cuuint32_t estr[2] = {1, 1};
        if (enc(&tx2, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(X), dims, strides, box, estr,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS)
            return N <= 32 ? launch_tc_tn2<32>(tx2, ty, a, grid, s) : launch_tc_tn2<64>(tx2, ty, a, grid, s);
    }
    return N <= 32 ? launch_tc_tn<32>(tx, ty, a, grid, s) : launch_tc_tn<64>(tx, ty, a, grid, s);
}

}  // namespace seastar
