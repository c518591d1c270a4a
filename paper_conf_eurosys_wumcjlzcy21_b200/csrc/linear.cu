// linear.cu -- a4 / a11: the dense per-layer transform T = X W and its backward (the S-type
// operators the paper leaves to the DL backend; GAT's f = W h, Fig. 2).
//
// Round-1 implementation: a register-tiled fp32 SIMT GEMM specialised for the tall-skinny shapes of
// the hot path (M = #vertices up to 2e5..2e6, K = feature width, N = 16..64).  For Reddit
// (K = 602, N = 16) the kernel is HBM-bound on reading X once; the tcgen05 3xTF32 path is the
// planned replacement for the flop-heavier CoraFull/Physics shapes.
#include "common.cuh"

namespace seastar {

struct GemmArgs {
    const float* A; int64_t lda;            // [M, K]
    const float* B; int64_t ldb_k, ldb_n;   // B[k][n] = B[k*ldb_k + n*ldb_n]
    float* C; int64_t ldc;                  // [M, N]
    int64_t M, K, N;
    const float* bias; const float* row_scale; int act;
    const float* Yact; int dact;            // optional fused activation backward: C *= act'(Yact)
};

// C = row_scale * act(A B + bias).  BM x BN block tile, BK = 32, TM x TN per thread, 256 threads.
template <int BM, int BN, int TM, int TN>
__global__ void __launch_bounds__(256) k_gemm(const GemmArgs g) {
    constexpr int BK = 32;
    constexpr int TX = BN / TN;                 // threads along n
    constexpr int TY = BM / TM;                 // threads along m
    static_assert(TX * TY == 256, "thread tile");
    constexpr int A_PER = BM * BK / 256;        // A elements per thread per tile
    constexpr int B_PER = BK * BN / 256;
    __shared__ float As[BM][BK + 1];
    __shared__ __align__(16) float Bs[BK][BN];

    const int tid = threadIdx.x;
    const int tx = tid % TX, ty = tid / TX;
    const int64_t m0 = (int64_t)blockIdx.x * BM;
    const int64_t n0 = (int64_t)blockIdx.y * BN;

    float acc[TM][TN];
#pragma unroll
    for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = 0.f;

    float ra[A_PER], rb[B_PER];
    auto load_tile = [&](int64_t k0) {
#pragma unroll
        for (int i = 0; i < A_PER; ++i) {
            const int idx = tid + i * 256;
            const int kk = idx % BK, mm = idx / BK;
            const int64_t gm = m0 + mm, gk = k0 + kk;
            ra[i] = (gm < g.M && gk < g.K) ? __ldg(g.A + gm * g.lda + gk) : 0.f;
        }
#pragma unroll
        for (int i = 0; i < B_PER; ++i) {
            const int idx = tid + i * 256;
            const int nn = idx % BN, kk = idx / BN;
            const int64_t gk = k0 + kk, gn = n0 + nn;
            rb[i] = (gk < g.K && gn < g.N) ? __ldg(g.B + gk * g.ldb_k + gn * g.ldb_n) : 0.f;
        }
    };
    auto store_tile = [&]() {
#pragma unroll
        for (int i = 0; i < A_PER; ++i) {
            const int idx = tid + i * 256;
            As[idx / BK][idx % BK] = ra[i];
        }
#pragma unroll
        for (int i = 0; i < B_PER; ++i) {
            const int idx = tid + i * 256;
            Bs[idx / BN][idx % BN] = rb[i];
        }
    };

    load_tile(0);
    for (int64_t k0 = 0; k0 < g.K; k0 += BK) {
        store_tile();
        __syncthreads();
        if (k0 + BK < g.K) load_tile(k0 + BK);   // register prefetch of the next tile
#pragma unroll
        for (int kk = 0; kk < BK; ++kk) {
            float a[TM], b[TN];
#pragma unroll
            for (int i = 0; i < TM; ++i) a[i] = As[ty * TM + i][kk];
#pragma unroll
            for (int j = 0; j < TN; j += 4) {
                const float4 t = *reinterpret_cast<const float4*>(&Bs[kk][tx * TN + j]);
                b[j] = t.x; b[j + 1] = t.y; b[j + 2] = t.z; b[j + 3] = t.w;
            }
#pragma unroll
            for (int i = 0; i < TM; ++i)
#pragma unroll
                for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
        }
        __syncthreads();
    }
#pragma unroll
    for (int i = 0; i < TM; ++i) {
        const int64_t gm = m0 + ty * TM + i;
        if (gm >= g.M) continue;
        const float rs = g.row_scale ? __ldg(g.row_scale + gm) : 1.f;
#pragma unroll
        for (int j = 0; j < TN; ++j) {
            const int64_t gn = n0 + tx * TN + j;
            if (gn >= g.N) continue;
            float z = acc[i][j] + (g.bias ? __ldg(g.bias + gn) : 0.f);
            z = rs * act_apply(g.act, z);
            if (g.Yact) z *= act_grad_from_y(g.dact, __ldg(g.Yact + gm * g.ldc + gn));
            g.C[gm * g.ldc + gn] = z;
        }
    }
}

// Skinny products (K <= 64, N <= 64: the class-width layers, e.g. logits = P2 W2 and dY1 = dT2 W2^T on Reddit):
// B is staged once per persistent CTA in shared memory (zero padded to 64 x 64), a warp owns 4 rows at a time,
// lane n (and n + 32) owns output columns, A's row values are broadcast by shuffles.  Each output is the same
// fp32 FMA chain over k = 0..K-1 as k_gemm's, so the result does not depend on the kernel choice.  HBM-bound:
// A and C are streamed once (k_gemm's 128 x 64 tiles were ~8x off that bound at M = 233 k).
template <int KC, int NC>
__global__ void __launch_bounds__(256) k_gemm_skinny(const GemmArgs g) {
    __shared__ float Bs[64][64];
    for (int idx = threadIdx.x; idx < 64 * 64; idx += 256) {
        const int k = idx / 64, n = idx % 64;
        Bs[k][n] = (k < g.K && n < g.N) ? __ldg(g.B + (int64_t)k * g.ldb_k + (int64_t)n * g.ldb_n) : 0.f;
    }
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t step = (int64_t)gridDim.x * 8 * 4;
    for (int64_t m0 = ((int64_t)blockIdx.x * 8 + warp) * 4; m0 < g.M; m0 += step) {
        float a[4][KC], acc[4][NC];
#pragma unroll
        for (int r = 0; r < 4; ++r) {
#pragma unroll
            for (int c = 0; c < KC; ++c) {
                const int k = lane + 32 * c;
                a[r][c] = (m0 + r < g.M && k < g.K) ? __ldg(g.A + (m0 + r) * g.lda + k) : 0.f;
            }
#pragma unroll
            for (int c = 0; c < NC; ++c) acc[r][c] = 0.f;
        }
#pragma unroll
        for (int c = 0; c < KC; ++c) {
            const int kend = (int)(g.K - 32 * c < 32 ? g.K - 32 * c : 32);
            for (int kk = 0; kk < kend; ++kk) {
                float b[NC];
#pragma unroll
                for (int j = 0; j < NC; ++j) b[j] = Bs[32 * c + kk][lane + 32 * j];
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    const float av = __shfl_sync(0xffffffffu, a[r][c], kk);
#pragma unroll
                    for (int j = 0; j < NC; ++j) acc[r][j] = fmaf(av, b[j], acc[r][j]);
                }
            }
        }
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            const int64_t gm = m0 + r;
            if (gm >= g.M) break;
            const float rs = g.row_scale ? __ldg(g.row_scale + gm) : 1.f;
#pragma unroll
            for (int j = 0; j < NC; ++j) {
                const int64_t gn = lane + 32 * j;
                if (gn >= g.N) continue;
                float z = acc[r][j] + (g.bias ? __ldg(g.bias + gn) : 0.f);
                z = rs * act_apply(g.act, z);
                if (g.Yact) z *= act_grad_from_y(g.dact, __ldg(g.Yact + gm * g.ldc + gn));
                g.C[gm * g.ldc + gn] = z;
            }
        }
    }
}

static seastar_status launch_gemm(const GemmArgs& g, cudaStream_t s) {
    if (g.M == 0 || g.N == 0) return SEASTAR_OK;
    if (g.K <= 64 && g.N <= 64) {
        int64_t blocks = (g.M + 31) / 32;
        const int64_t cap = 8 * (int64_t)num_sms();
        if (blocks > cap) blocks = cap;
        const int kc = g.K <= 32 ? 1 : 2, nc = g.N <= 32 ? 1 : 2;
        if (kc == 1 && nc == 1) k_gemm_skinny<1, 1><<<(unsigned)blocks, 256, 0, s>>>(g);
        else if (kc == 1) k_gemm_skinny<1, 2><<<(unsigned)blocks, 256, 0, s>>>(g);
        else if (nc == 1) k_gemm_skinny<2, 1><<<(unsigned)blocks, 256, 0, s>>>(g);
        else k_gemm_skinny<2, 2><<<(unsigned)blocks, 256, 0, s>>>(g);
        return check_launch("k_gemm_skinny");
    }
    if (g.N <= 16) {
        dim3 grid((unsigned)((g.M + 255) / 256), 1);
        k_gemm<256, 16, 4, 4><<<grid, 256, 0, s>>>(g);
    } else if (g.N <= 32) {
        dim3 grid((unsigned)((g.M + 127) / 128), 1);
        k_gemm<128, 32, 4, 4><<<grid, 256, 0, s>>>(g);
    } else {
        dim3 grid((unsigned)((g.M + 127) / 128), (unsigned)((g.N + 63) / 64));
        k_gemm<128, 64, 8, 4><<<grid, 256, 0, s>>>(g);
    }
    return check_launch("k_gemm");
}

// dW partials: block (kt, split) accumulates X[rows of split, k-tile]^T dY[rows of split, :]
// into part[split][K][N].  64 k x BN n per block, 32-row smem stages.
template <int BN>
__global__ void __launch_bounds__(256) k_gemm_tn(const float* __restrict__ X, int64_t ldx,
                                                 const float* __restrict__ dY, int64_t ldy, int64_t M, int64_t K,
                                                 int64_t N, int64_t rows_per_split, float* __restrict__ part) {
    constexpr int BKT = 64, BR = 32;
    constexpr int TN = BN / 16;                   // 16 threads along n
    __shared__ __align__(16) float Xs[BR][BKT + 4];
    __shared__ __align__(16) float Ys[BR][BN];
    const int tid = threadIdx.x;
    const int tk = tid / 16, tn = tid % 16;       // 16 k-groups of 4, 16 n-groups of TN
    const int64_t k0 = (int64_t)blockIdx.x * BKT;
    const int64_t r_begin = (int64_t)blockIdx.y * rows_per_split;
    const int64_t r_end = min(M, r_begin + rows_per_split);
    float acc[4][TN];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = 0.f;
    for (int64_t r0 = r_begin; r0 < r_end; r0 += BR) {
        // X stage: 32 rows x 64 k (coalesced along k)
#pragma unroll
        for (int i = 0; i < BR * BKT / 256; ++i) {
            const int idx = tid + i * 256;
            const int rr = idx / BKT, kk = idx % BKT;
            const int64_t gr = r0 + rr, gk = k0 + kk;
            Xs[rr][kk] = (gr < r_end && gk < K) ? __ldg(X + gr * ldx + gk) : 0.f;
        }
#pragma unroll
        for (int i = 0; i < (BR * BN + 255) / 256; ++i) {
            const int idx = tid + i * 256;
            if (idx < BR * BN) {
                const int rr = idx / BN, nn = idx % BN;
                const int64_t gr = r0 + rr;
                Ys[rr][nn] = (gr < r_end && nn < N) ? __ldg(dY + gr * ldy + nn) : 0.f;
            }
        }
        __syncthreads();
#pragma unroll 8
        for (int rr = 0; rr < BR; ++rr) {
            const float4 xa = *reinterpret_cast<const float4*>(&Xs[rr][tk * 4]);
            float b[TN];
#pragma unroll
            for (int j = 0; j < TN; ++j) b[j] = Ys[rr][tn * TN + j];
            const float a[4] = {xa.x, xa.y, xa.z, xa.w};
#pragma unroll
            for (int i = 0; i < 4; ++i)
#pragma unroll
                for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
        }
        __syncthreads();
    }
    float* p = part + (int64_t)blockIdx.y * K * N;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int64_t gk = k0 + tk * 4 + i;
        if (gk >= K) continue;
#pragma unroll
        for (int j = 0; j < TN; ++j) {
            const int64_t gn = tn * TN + j;
            if (gn < N) p[gk * N + gn] = acc[i][j];
        }
    }
}

static void tn_geometry(int64_t M, int64_t K, int64_t& ktiles, int64_t& nsplit, int64_t& rows_per_split) {
    ktiles = (K + 63) / 64;
#ifndef TN_WAVES
#define TN_WAVES 2
#endif
    int64_t want = (TN_WAVES * num_sms() + ktiles - 1) / ktiles;   // ~TN_WAVES waves of blocks
    int64_t max_split = (M + 255) / 256;                    // >= 256 rows per split
    nsplit = want < max_split ? want : max_split;
    if (nsplit < 1) nsplit = 1;
    rows_per_split = (M + nsplit - 1) / nsplit;
    rows_per_split = (rows_per_split + 31) / 32 * 32;
    nsplit = rows_per_split > 0 ? (M + rows_per_split - 1) / rows_per_split : 1;
    if (nsplit < 1) nsplit = 1;
}

seastar_status colsum_impl(const float* X, int64_t M, int64_t F, int64_t ld, float* out, void* ws, size_t ws_bytes,
                           cudaStream_t s);
seastar_status linear_fwd_tc(const float* X, int64_t M, int64_t K, int64_t ldx, const float* W, int64_t N,
                             const float* bias, const float* row_scale, int act, float* Y, int64_t ldy,
                             void* ws, size_t ws_bytes, cudaStream_t s);
size_t linear_fwd_tc_workspace(int64_t K, int64_t N);
size_t colsum_ws(int64_t M, int64_t F);
size_t linear_bwd_weight_tc_part_bytes(int64_t M, int64_t K, int64_t N);
seastar_status linear_bwd_weight_tc(const float* X, int64_t M, int64_t K, int64_t ldx, const float* dY, int64_t N,
                                    int64_t ldy, float* part, int64_t* nsplit_out, cudaStream_t s);

}  // namespace seastar

using namespace seastar;

extern "C" {

size_t seastar_linear_fwd_workspace(int64_t K, int64_t Nout) { return linear_fwd_tc_workspace(K, Nout); }

seastar_status seastar_linear_fwd(const float* X, int64_t M, int64_t K, int64_t ldx, const float* W, int64_t Nout,
                                  const float* bias, const float* row_scale, seastar_act act, float* Y, int64_t ldy,
                                  void* workspace, size_t ws_bytes, seastar_stream stream) {
    SS_ARG(X && W && Y, "linear_fwd: NULL argument");
    SS_ARG(M >= 0 && K >= 1 && Nout >= 1 && ldx >= K && ldy >= Nout, "linear_fwd: bad sizes");
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "linear_fwd: bad activation");
    SS_TRY(check_device());
    // tcgen05 3xTF32 path (TMA needs ldx % 4 == 0 and a 16-byte aligned X); SIMT fp32 otherwise
    const seastar_status st =
        linear_fwd_tc(X, M, K, ldx, W, Nout, bias, row_scale, act, Y, ldy, workspace, ws_bytes, to_stream(stream));
    if (st != SEASTAR_ERR_UNSUPPORTED) return st;
    GemmArgs g{X, ldx, W, Nout, 1, Y, ldy, M, K, Nout, bias, row_scale, act, nullptr, 0};
    return launch_gemm(g, to_stream(stream));
}

seastar_status seastar_linear_bwd_data(const float* dY, int64_t M, int64_t Nout, int64_t ldy, const float* W,
                                       int64_t K, const float* row_scale, const float* Yact, seastar_act act,
                                       float* dX, int64_t ldx, seastar_stream stream) {
    SS_ARG(dY && W && dX, "linear_bwd_data: NULL argument");
    SS_ARG(M >= 0 && K >= 1 && Nout >= 1 && ldx >= K && ldy >= Nout, "linear_bwd_data: bad sizes");
    SS_TRY(check_device());
    // dX[M,K] = dY[M,Nout] W^T : inner dim Nout, B[k'][n'] = W[n'][k'] = W[n'*Nout + k']
    SS_ARG(act >= SEASTAR_ACT_NONE && act <= SEASTAR_ACT_SIGMOID, "linear_bwd_data: bad activation");
    SS_ARG((const void*)Yact != (const void*)dX || !Yact, "linear_bwd_data: Yact aliases dX");
    GemmArgs g{dY, ldy, W, 1, Nout, dX, ldx, M, Nout, K, nullptr, row_scale, SEASTAR_ACT_NONE, Yact, (int)act};
    return launch_gemm(g, to_stream(stream));
}

// dW is produced in column chunks of at most 64 outputs (the width one tcgen05 / SIMT tile covers);
// each chunk's row-split partials go through the workspace and are summed in split order
static const int64_t kBwdWChunk = 64;

size_t seastar_linear_bwd_weight_workspace(int64_t M, int64_t K, int64_t Nout) {
    const int64_t nc = Nout < kBwdWChunk ? Nout : kBwdWChunk;
    int64_t kt, ns, rps;
    tn_geometry(M > 0 ? M : 1, K, kt, ns, rps);
    size_t part = (size_t)ns * K * nc * sizeof(float);
    const size_t tc = linear_bwd_weight_tc_part_bytes(M, K, nc);
    if (tc > part) part = tc;
    return part + colsum_ws(M, Nout) + 512;
}

seastar_status seastar_linear_bwd_weight(const float* X, int64_t M, int64_t K, int64_t ldx, const float* dY,
                                         int64_t Nout, int64_t ldy, float* dW, float* db, void* workspace,
                                         size_t ws_bytes, seastar_stream stream) {
    SS_ARG(X && dY && dW && workspace, "linear_bwd_weight: NULL argument");
    SS_ARG(M >= 1 && K >= 1 && Nout >= 1 && ldx >= K && ldy >= Nout, "linear_bwd_weight: bad sizes");
    SS_ARG(ws_bytes >= seastar_linear_bwd_weight_workspace(M, K, Nout), "linear_bwd_weight: workspace too small");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    float* part = static_cast<float*>(workspace);
    for (int64_t c0 = 0; c0 < Nout; c0 += kBwdWChunk) {
        const int64_t nc = Nout - c0 < kBwdWChunk ? Nout - c0 : kBwdWChunk;
        const float* dYc = dY + c0;
        int64_t kt, ns, rps;
        // tcgen05 3xTF32 path (MN-major TMA operands); SIMT fp32 otherwise
        const seastar_status st = linear_bwd_weight_tc(X, M, K, ldx, dYc, nc, ldy, part, &ns, s);
        if (st == SEASTAR_ERR_UNSUPPORTED) {
            tn_geometry(M, K, kt, ns, rps);
            dim3 grid((unsigned)kt, (unsigned)ns);
            if (nc <= 16) k_gemm_tn<16><<<grid, 256, 0, s>>>(X, ldx, dYc, ldy, M, K, nc, rps, part);
            else if (nc <= 32) k_gemm_tn<32><<<grid, 256, 0, s>>>(X, ldx, dYc, ldy, M, K, nc, rps, part);
            else k_gemm_tn<64><<<grid, 256, 0, s>>>(X, ldx, dYc, ldy, M, K, nc, rps, part);
            SS_TRY(check_launch("k_gemm_tn"));
        } else if (st != SEASTAR_OK) {
            return st;
        }
        reduce_splits(part, ns, K * nc, K * nc, nc, Nout, dW + c0, s);
        SS_TRY(check_launch("k_reduce_splits"));
    }
    if (db) {
        size_t off = ((seastar_linear_bwd_weight_workspace(M, K, Nout) - colsum_ws(M, Nout) - 512) + 255) & ~size_t(255);
        SS_TRY(colsum_impl(dY, M, Nout, ldy, db, static_cast<char*>(workspace) + off, ws_bytes - off, s));
    }
    return SEASTAR_OK;
}

}  // extern "C"
