// misc.cu -- training-step glue kept on the GPU so the whole epoch runs in this library:
// softmax cross-entropy (mean over rows), deterministic column sums (bias gradients), axpby,
// and a flat-buffer Adam step (DGL's default training loop).
#include <math.h>

#include <algorithm>

#include "common.cuh"
#include <cmath>

namespace seastar {

static int64_t colsum_blocks(int64_t M) {
    int64_t b = 32 * num_sms();
    if (M < b * 64) b = (M + 63) / 64;
    return b < 1 ? 1 : b;
}

size_t colsum_ws(int64_t M, int64_t F) { return (size_t)colsum_blocks(M) * (size_t)F * sizeof(float) + 256; }

// stage 1: block b sums rows [b*rpb, (b+1)*rpb) of each column; CW = min(32, pow2 >= F) column lanes x 256/CW row
// lanes (all lanes busy for narrow F), fixed order.  fp64 accumulation: the bias gradients are column sums of
// (softmax - onehot) / N, which cancel to ~1/sqrt(N) of their terms' total, so fp32 chains of ~10^3 terms cost
// ~1e-5 relative (bgs-shaped db2, r2 test_gpu_fullsize)
__global__ void __launch_bounds__(256) k_colsum1(const float* __restrict__ X, int64_t M, int64_t F, int64_t ld,
                                                 int64_t rpb, int CW, float* __restrict__ part) {
    __shared__ double red[256];
    const int64_t r0 = blockIdx.x * rpb, r1 = min(M, r0 + rpb);
    const int RLN = 256 / CW;
    const int tx = threadIdx.x % CW, ty = threadIdx.x / CW;
    for (int64_t cb = 0; cb < F; cb += CW) {
        const int64_t j = cb + tx;
        double s = 0.0;
        if (j < F) {
            // four independent chains (fixed order), so four loads are in flight per thread
            double s4[4] = {0.0, 0.0, 0.0, 0.0};
            int64_t r = r0 + ty;
            for (; r + 3 * RLN < r1; r += 4 * RLN) {
                const float a0 = __ldg(X + r * ld + j), a1 = __ldg(X + (r + RLN) * ld + j);
                const float a2 = __ldg(X + (r + 2 * RLN) * ld + j), a3 = __ldg(X + (r + 3 * RLN) * ld + j);
                s4[0] += (double)a0; s4[1] += (double)a1; s4[2] += (double)a2; s4[3] += (double)a3;
            }
            for (int k = 0; r < r1; r += RLN, ++k) s4[k & 3] += (double)__ldg(X + r * ld + j);
            s = (s4[0] + s4[1]) + (s4[2] + s4[3]);
        }
        red[threadIdx.x] = s;
        __syncthreads();
        if (ty == 0 && j < F) {
            double x = 0.0;
            for (int k = 0; k < RLN; ++k) x += red[k * CW + tx];
            part[blockIdx.x * F + j] = (float)x;
        }
        __syncthreads();
    }
}

template <int WARPS>
__global__ void __launch_bounds__(32 * WARPS) k_reduce_splits(const float* __restrict__ part, int64_t nsplit,
                                                              int64_t stride, int64_t n, int64_t nc, int64_t ldo,
                                                              float* __restrict__ out) {
    __shared__ double red[WARPS][32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t i = (int64_t)blockIdx.x * 32 + lane;
    double x = 0.0;
    if (i < n) {
        int64_t b = w;
        for (; b + 3 * WARPS < nsplit; b += 4 * WARPS) {      // 4 independent loads in flight per lane
            const float a0 = __ldg(part + b * stride + i), a1 = __ldg(part + (b + WARPS) * stride + i);
            const float a2 = __ldg(part + (b + 2 * WARPS) * stride + i), a3 = __ldg(part + (b + 3 * WARPS) * stride + i);
            x += (double)a0; x += (double)a1; x += (double)a2; x += (double)a3;
        }
        for (; b < nsplit; b += WARPS) x += (double)__ldg(part + b * stride + i);
    }
    red[w][lane] = x;
    __syncthreads();
    if (w == 0 && i < n) {
        double y = 0.0;
#pragma unroll
        for (int k = 0; k < WARPS; ++k) y += red[k][lane];
        out[(i / nc) * ldo + (i % nc)] = (float)y;
    }
}

// few outputs (fewer 32-column blocks than SMs) and many splits: 32 split lanes per column instead of 8, so the
// per-lane chains are 4x shorter (the attention-projection and bias reductions: 2 blocks x 1,184 splits)
void reduce_splits(const float* part, int64_t nsplit, int64_t stride, int64_t n, int64_t nc, int64_t ldo, float* out,
                   cudaStream_t s) {
    if (n <= 0) return;
    const int64_t blocks = (n + 31) / 32;
    if (blocks < num_sms() && nsplit > 64)
        k_reduce_splits<32><<<(unsigned)blocks, 1024, 0, s>>>(part, nsplit, stride, n, nc, ldo, out);
    else
        k_reduce_splits<8><<<(unsigned)blocks, 256, 0, s>>>(part, nsplit, stride, n, nc, ldo, out);
}

seastar_status colsum_impl(const float* X, int64_t M, int64_t F, int64_t ld, float* out, void* ws, size_t ws_bytes,
                           cudaStream_t s) {
    if (ws_bytes < colsum_ws(M, F)) {
        set_error("colsum: workspace too small");
        return SEASTAR_ERR_INVALID_ARGUMENT;
    }
    if (F == 0) return SEASTAR_OK;
    const int64_t nblk = colsum_blocks(M);
    const int64_t rpb = M > 0 ? (M + nblk - 1) / nblk : 1;
    float* part = static_cast<float*>(ws);
    const int CW = F >= 32 ? 32 : pow2_ceil((int)F);
    k_colsum1<<<(unsigned)nblk, 256, 0, s>>>(X, M, F, ld, rpb, CW, part);
    reduce_splits(part, nblk, F, F, F, F, out, s);
    return check_launch("k_colsum");
}

// warp per row: loss_r = lse(z_r) - z_r[label]; dZ = (softmax - onehot) / M; per-block loss partials
__global__ void __launch_bounds__(256) k_softmax_xent(const float* __restrict__ Z, int64_t M, int64_t n_total, int C,
                                                      int64_t ldz, const int64_t* __restrict__ labels,
                                                      float* __restrict__ dZ, int64_t lddz, float* __restrict__ part) {
    __shared__ float wl[8];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t r = blockIdx.x * 8 + w;
    float loss = 0.f;
    if (r < M) {
        const float* z = Z + r * ldz;
        const int64_t lab = labels[r];
        const float inv = 1.f / (float)n_total;
        if (C <= 128) {                       // the row stays in registers: one coalesced read
            float zv[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) zv[k] = (lane + 32 * k < C) ? __ldg(z + lane + 32 * k) : -INFINITY;
            float m = fmaxf(fmaxf(zv[0], zv[1]), fmaxf(zv[2], zv[3]));
            for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
            float sum = 0.f;
#pragma unroll
            for (int k = 0; k < 4; ++k) sum += (lane + 32 * k < C) ? expf(zv[k] - m) : 0.f;
            for (int o = 16; o; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
            const float lse = m + logf(sum);
            float zl = 0.f;
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const int c = lane + 32 * k;
                if (c < C) {
                    if (dZ) dZ[r * lddz + c] = (expf(zv[k] - lse) - (c == lab ? 1.f : 0.f)) * inv;
                    if (c == lab) zl = zv[k];
                }
            }
            for (int o = 16; o; o >>= 1) zl += __shfl_xor_sync(0xffffffffu, zl, o);
            loss = lse - zl;
        } else {
            float m = -INFINITY;
            for (int c = lane; c < C; c += 32) m = fmaxf(m, __ldg(z + c));
            for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
            float sum = 0.f;
            for (int c = lane; c < C; c += 32) sum += expf(__ldg(z + c) - m);
            for (int o = 16; o; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
            const float lse = m + logf(sum);
            if (dZ)
                for (int c = lane; c < C; c += 32)
                    dZ[r * lddz + c] = (expf(__ldg(z + c) - lse) - (c == lab ? 1.f : 0.f)) * inv;
            loss = lse - __ldg(z + lab);
        }
    }
    if (lane == 0) wl[w] = loss;
    __syncthreads();
    if (threadIdx.x == 0) {
        float x = 0.f;
        for (int k = 0; k < 8; ++k) x += wl[k];
        part[blockIdx.x] = x;
    }
}

// C <= 64 (every config's class count): a warp takes 4 rows, all 8 loads issued before any reduction, so
// one memory round trip serves 4 rows (the one-row-per-warp kernel is latency-bound: 66 us at M = 233 k)
__global__ void __launch_bounds__(256) k_softmax_xent4(const float* __restrict__ Z, int64_t M, int64_t n_total, int C,
                                                       int64_t ldz, const int64_t* __restrict__ labels,
                                                       float* __restrict__ dZ, int64_t lddz, float* __restrict__ part) {
    constexpr int RPW = 4;
    __shared__ float wl[8];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t r0 = ((int64_t)blockIdx.x * 8 + w) * RPW;
    const float inv = 1.f / (float)n_total;
    float zv[RPW][2];
    int64_t lab[RPW];
#pragma unroll
    for (int i = 0; i < RPW; ++i) {
        const int64_t r = r0 + i;
        const bool ok = r < M;
        lab[i] = ok ? labels[r] : -1;
#pragma unroll
        for (int k = 0; k < 2; ++k)
            zv[i][k] = (ok && lane + 32 * k < C) ? __ldg(Z + r * ldz + lane + 32 * k) : -INFINITY;
    }
    float loss = 0.f;
#pragma unroll
    for (int i = 0; i < RPW; ++i) {
        const int64_t r = r0 + i;
        if (r >= M) break;                        // warp-uniform
        float m = fmaxf(zv[i][0], zv[i][1]);
        for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
        float sum = 0.f;
#pragma unroll
        for (int k = 0; k < 2; ++k) sum += (lane + 32 * k < C) ? expf(zv[i][k] - m) : 0.f;
        for (int o = 16; o; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
        const float lse = m + logf(sum);
        float zl = 0.f;
#pragma unroll
        for (int k = 0; k < 2; ++k) {
            const int c = lane + 32 * k;
            if (c < C) {
                if (dZ) dZ[r * lddz + c] = (expf(zv[i][k] - lse) - (c == lab[i] ? 1.f : 0.f)) * inv;
                if (c == lab[i]) zl = zv[i][k];
            }
        }
        for (int o = 16; o; o >>= 1) zl += __shfl_xor_sync(0xffffffffu, zl, o);
        loss += lse - zl;
    }
    if (lane == 0) wl[w] = loss;
    __syncthreads();
    if (threadIdx.x == 0) {
        float x = 0.f;
        for (int k = 0; k < 8; ++k) x += wl[k];
        part[blockIdx.x] = x;
    }
}

// a quad of lanes per row for narrow class counts (C <= 16; the AM R-GCN output has 1.9 M rows x 11 classes):
// lane c of the quad owns float4 chunk c of the row, so a warp reads and writes 8 consecutive rows as contiguous
// 128-bit accesses; max / sum / label logit by 2-step xor shuffles inside the quad.  The softmax itself runs in
// fp64 (exp / log of the fp32 logits): the bias gradient of the output layer is a column sum of these rows that
// cancels to ~1/sqrt(N) of its terms, and fp32 softmax rounding left it at 1.0e-5 of the fp64 oracle on the
// bgs-shaped graph (r2).  Padding columns are never written.
__global__ void __launch_bounds__(256) k_softmax_xent_q(const float* __restrict__ Z, int64_t M, int64_t n_total,
                                                        int C, int64_t ldz, const int64_t* __restrict__ labels,
                                                        float* __restrict__ dZ, int64_t lddz, float* __restrict__ part) {
    __shared__ float wl[8];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, c = lane & 3;
    const int64_t r = ((int64_t)blockIdx.x * 256 + threadIdx.x) >> 2;
    const bool ok = r < M;
    const bool mine = ok && 4 * c < C;
    double z[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
    if (mine) {
        const float4 v = ldg4(Z + r * ldz + 4 * c);
        z[0] = v.x; z[1] = v.y; z[2] = v.z; z[3] = v.w;
#pragma unroll
        for (int i = 0; i < 4; ++i)
            if (4 * c + i >= C) z[i] = -INFINITY;
    }
    const int64_t lab = ok ? labels[r] : -1;
    double m = fmax(fmax(z[0], z[1]), fmax(z[2], z[3]));
    m = fmax(m, __shfl_xor_sync(0xffffffffu, m, 1));
    m = fmax(m, __shfl_xor_sync(0xffffffffu, m, 2));
    double sum = 0.0, zl = 0.0;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int j = 4 * c + i;
        sum += (mine && j < C) ? exp(z[i] - m) : 0.0;
        zl += (mine && j == lab) ? z[i] : 0.0;
    }
    sum += __shfl_xor_sync(0xffffffffu, sum, 1);
    sum += __shfl_xor_sync(0xffffffffu, sum, 2);
    zl += __shfl_xor_sync(0xffffffffu, zl, 1);
    zl += __shfl_xor_sync(0xffffffffu, zl, 2);
    const double lse = m + log(sum);
    float loss = (ok && c == 0) ? (float)(lse - zl) : 0.f;
    if (dZ && mine) {
        const double inv = 1.0 / (double)n_total;
        float d[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) d[i] = (float)((exp(z[i] - lse) - (4 * c + i == lab ? 1.0 : 0.0)) * inv);
        float* o = dZ + r * lddz + 4 * c;
        if (4 * c + 4 <= C && (lddz % 4) == 0 && ((reinterpret_cast<uintptr_t>(dZ) & 15u) == 0)) {
            *reinterpret_cast<float4*>(o) = make_float4(d[0], d[1], d[2], d[3]);
        } else {
#pragma unroll
            for (int i = 0; i < 4; ++i)
                if (4 * c + i < C) o[i] = d[i];
        }
    }
    for (int o = 16; o; o >>= 1) loss += __shfl_xor_sync(0xffffffffu, loss, o);
    if (lane == 0) wl[w] = loss;
    __syncthreads();
    if (threadIdx.x == 0) {
        float x = 0.f;
        for (int k = 0; k < 8; ++k) x += wl[k];
        part[blockIdx.x] = x;
    }
}

__global__ void k_loss_final(const float* __restrict__ part, int64_t n, int64_t n_total, float* __restrict__ loss) {
    __shared__ double red[256];
    double x = 0.0;
    for (int64_t i = threadIdx.x; i < n; i += 256) x += (double)part[i];
    red[threadIdx.x] = x;
    __syncthreads();
    for (int o = 128; o; o >>= 1) {
        if (threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
        __syncthreads();
    }
    if (threadIdx.x == 0) *loss = (float)(red[0] / (double)n_total);
}

__global__ void k_axpby(int64_t n, float a, const float* __restrict__ x, float b, float* __restrict__ y) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) y[i] = a * x[i] + (b == 0.f ? 0.f : b * y[i]);
}

__device__ __forceinline__ void adam1(float& p, float g, float& m, float& v, float lr, float b1, float b2, float eps,
                                      float c1, float c2) {
    m = b1 * m + (1.f - b1) * g;
    v = b2 * v + (1.f - b2) * g * g;
    p -= lr * (m / c1) / (sqrtf(v / c2) + eps);
}

// grid-stride, 128-bit accesses (7 x 16 B per 4 parameters); the bias corrections are computed once per thread
__global__ void __launch_bounds__(256) k_adam(float* __restrict__ p, const float* __restrict__ g, float* __restrict__ m,
                                              float* __restrict__ v, int64_t n, float lr, float b1, float b2, float eps,
                                              const int32_t* __restrict__ step, int vec) {
    const int t = *step;
    const float c1 = 1.f - powf(b1, (float)t), c2 = 1.f - powf(b2, (float)t);
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t i0 = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t done = 0;
    if (vec) {
        const int64_t n4 = n >> 2;
        float4* p4 = reinterpret_cast<float4*>(p);
        float4* m4 = reinterpret_cast<float4*>(m);
        float4* v4 = reinterpret_cast<float4*>(v);
        const float4* g4 = reinterpret_cast<const float4*>(g);
        for (int64_t i = i0; i < n4; i += stride) {
            float4 pp = p4[i], mm = m4[i], vv = v4[i];
            const float4 gg = __ldcs(g4 + i);
            adam1(pp.x, gg.x, mm.x, vv.x, lr, b1, b2, eps, c1, c2);
            adam1(pp.y, gg.y, mm.y, vv.y, lr, b1, b2, eps, c1, c2);
            adam1(pp.z, gg.z, mm.z, vv.z, lr, b1, b2, eps, c1, c2);
            adam1(pp.w, gg.w, mm.w, vv.w, lr, b1, b2, eps, c1, c2);
            p4[i] = pp;
            __stcs(m4 + i, mm);
            __stcs(v4 + i, vv);
        }
        done = n4 << 2;
    }
    for (int64_t i = done + i0; i < n; i += stride) adam1(p[i], g[i], m[i], v[i], lr, b1, b2, eps, c1, c2);
}

__global__ void k_step_inc(int32_t* c) { *c += 1; }

// NEXT-3 dropout (reading #27): counter = global element index (sm64: common.cuh)
__global__ void __launch_bounds__(256) k_dropout(const float* X, int64_t M, uint32_t F, int64_t ldx, int64_t row0,
                                                 uint32_t thr, float scale, uint64_t seed, uint32_t site,
                                                 const int32_t* __restrict__ step, float* Y, int64_t ldy) {
    const uint32_t st = step ? (uint32_t)*step : 0u;
    const uint64_t key = sm64(seed ^ sm64(((uint64_t)site << 32) | st));
    const uint64_t n = (uint64_t)M * F;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
        const uint64_t r = n <= 0xFFFFFFFFull ? (uint64_t)((uint32_t)i / F) : i / F;
        const uint64_t f = i - r * F;
        const bool keep = (sm64(key ^ ((uint64_t)(row0 + (int64_t)r) * F + f)) >> 40) >= thr;
        const float x = X[r * ldx + f];
        Y[r * ldy + f] = keep ? x * scale : 0.f;
    }
}

}  // namespace seastar

using namespace seastar;

extern "C" {

size_t seastar_colsum_workspace(int64_t M, int64_t F) { return colsum_ws(M, F); }

seastar_status seastar_colsum(const float* X, int64_t M, int64_t F, int64_t ld, float* out, void* workspace,
                              size_t ws_bytes, seastar_stream stream) {
    SS_ARG(X && out && workspace, "colsum: NULL argument");
    SS_ARG(M >= 0 && F >= 1 && ld >= F, "colsum: bad sizes");
    SS_TRY(check_device());
    return colsum_impl(X, M, F, ld, out, workspace, ws_bytes, to_stream(stream));
}

size_t seastar_softmax_xent_workspace(int64_t M) { return (size_t)((M + 7) / 8 + 1) * sizeof(float) + 256; }

seastar_status seastar_softmax_xent(const float* Z, int64_t M, int64_t n_total, int32_t C, int64_t ldz,
                                    const int64_t* labels, float* loss, float* dZ, int64_t lddz, void* workspace,
                                    size_t ws_bytes, seastar_stream stream) {
    SS_ARG(Z && labels && loss && workspace, "softmax_xent: NULL argument");
    SS_ARG(M >= 1 && C >= 1 && ldz >= C && (!dZ || lddz >= C), "softmax_xent: bad sizes");
    SS_ARG(n_total >= M, "softmax_xent: n_total (%lld) < M (%lld)", (long long)n_total, (long long)M);
    SS_ARG(ws_bytes >= seastar_softmax_xent_workspace(M), "softmax_xent: workspace too small");
    SS_TRY(check_device());
    cudaStream_t s = to_stream(stream);
    float* part = static_cast<float*>(workspace);
    int64_t nblk;
    if (C <= 16 && ldz % 4 == 0 && aligned16(Z)) {
        nblk = (M + 63) / 64;
        k_softmax_xent_q<<<(unsigned)nblk, 256, 0, s>>>(Z, M, n_total, C, ldz, labels, dZ, lddz, part);
    } else if (C <= 64) {
        nblk = (M + 31) / 32;
        k_softmax_xent4<<<(unsigned)nblk, 256, 0, s>>>(Z, M, n_total, C, ldz, labels, dZ, lddz, part);
    } else {
        nblk = (M + 7) / 8;
        k_softmax_xent<<<(unsigned)nblk, 256, 0, s>>>(Z, M, n_total, C, ldz, labels, dZ, lddz, part);
    }
    k_loss_final<<<1, 256, 0, s>>>(part, nblk, n_total, loss);
    return check_launch("k_softmax_xent");
}

}  // extern "C"

namespace seastar {
__global__ void k_row_scale(const float* __restrict__ X, int64_t M, int64_t F, int64_t ldx,
                            const float* __restrict__ scale, float* Y, int64_t ldy) {
    const int64_t n = M * F;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = k / F, j = k % F;
        Y[i * ldy + j] = __ldg(scale + i) * X[i * ldx + j];
    }
}
}  // namespace seastar

extern "C" {

seastar_status seastar_row_scale(const float* X, int64_t M, int64_t F, int64_t ldx, const float* scale, float* Y,
                                 int64_t ldy, seastar_stream stream) {
    SS_ARG(X && scale && Y, "row_scale: NULL argument");
    SS_ARG(M >= 0 && F >= 1 && ldx >= F && ldy >= F, "row_scale: bad sizes");
    SS_ARG((void*)X != (void*)Y || ldx == ldy, "row_scale: in-place needs ldx == ldy");
    SS_TRY(check_device());
    if (M == 0) return SEASTAR_OK;
    const int64_t n = M * F;
    const int64_t blocks = std::min<int64_t>((n + 255) / 256, (int64_t)num_sms() * 16);
    k_row_scale<<<(unsigned)blocks, 256, 0, to_stream(stream)>>>(X, M, F, ldx, scale, Y, ldy);
    return check_launch("k_row_scale");
}

seastar_status seastar_axpby(int64_t n, float a, const float* x, float b, float* y, seastar_stream stream) {
    SS_ARG(x && y && n >= 0, "axpby: bad argument");
    SS_TRY(check_device());
    if (n == 0) return SEASTAR_OK;
    k_axpby<<<(unsigned)((n + 255) / 256), 256, 0, to_stream(stream)>>>(n, a, x, b, y);
    return check_launch("k_axpby");
}

seastar_status seastar_adam(float* param, const float* grad, float* m, float* v, int64_t n, float lr, float beta1,
                            float beta2, float eps, const int32_t* step, seastar_stream stream) {
    SS_ARG(param && grad && m && v && step && n >= 0, "adam: bad argument");
    SS_TRY(check_device());
    if (n == 0) return SEASTAR_OK;
    const int vec = aligned16(param) && aligned16(grad) && aligned16(m) && aligned16(v);
    int64_t blocks = ((vec ? (n + 3) / 4 : n) + 255) / 256;
    const int64_t cap = 8 * (int64_t)num_sms();
    if (blocks > cap) blocks = cap;
    if (blocks < 1) blocks = 1;
    k_adam<<<(unsigned)blocks, 256, 0, to_stream(stream)>>>(param, grad, m, v, n, lr, beta1, beta2, eps, step, vec);
    return check_launch("k_adam");
}

seastar_status seastar_dropout(const float* X, int64_t M, int64_t F, int64_t ldx, int64_t row0, float p, uint64_t seed,
                               uint32_t site, const int32_t* step, float* Y, int64_t ldy, seastar_stream stream) {
    SS_ARG(X && Y, "dropout: NULL argument");
    SS_ARG(M >= 0 && F >= 1 && F <= 0xFFFFFFFFll && ldx >= F && ldy >= F && row0 >= 0, "dropout: bad sizes");
    SS_ARG(p >= 0.f && p < 1.f, "dropout: need 0 <= p < 1 (got %g)", (double)p);
    SS_ARG(X != Y || ldx == ldy, "dropout: in place needs ldx == ldy");
    SS_TRY(check_device());
    if (M == 0) return SEASTAR_OK;
    const uint32_t thr = drop_threshold(p);
    const float scale = drop_scale(p);
    const int64_t n = M * F;
    int64_t blocks = (n + 255) / 256;
    const int64_t cap = 16 * (int64_t)num_sms();
    if (blocks > cap) blocks = cap;
    k_dropout<<<(unsigned)blocks, 256, 0, to_stream(stream)>>>(X, M, (uint32_t)F, ldx, row0, thr, scale, seed, site, step,
                                                              Y, ldy);
    return check_launch("k_dropout");
}

seastar_status seastar_step_inc(int32_t* counter, seastar_stream stream) {
    SS_ARG(counter, "step_inc: NULL");
    SS_TRY(check_device());
    k_step_inc<<<1, 1, 0, to_stream(stream)>>>(counter);
    return check_launch("k_step_inc");
}

}  // extern "C"
