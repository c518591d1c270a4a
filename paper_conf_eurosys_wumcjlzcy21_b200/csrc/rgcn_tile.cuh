// rgcn_tile.cuh -- internals shared by rgcn.cu and rgcn_tile.cu (not part of the ABI).
#pragma once
#include "common.cuh"

namespace seastar {

#ifndef RGCN_TILE_EDGES
#define RGCN_TILE_EDGES 512   // edges per tile (<= 512: one edge record per thread of the persistent kernel) (A/B knob for tools/build_variant.sh)
#endif
constexpr int kRgcnTileEdges = RGCN_TILE_EDGES;

struct RgcnTileArgs {
    const int32_t* perm; const int32_t* off; const int32_t* nbr; const int32_t* typ;
    const float* norm; const int32_t* eid; const float* norm_user;
    const int32_t* tile_row;            // IndexSet::tile_row: first / last row of each tile
    int64_t n_rows, n_edges, vbase;
    const float* table; int64_t ldt;    // gathered rows (X_all forward, dA_all for dX), ldt % 4 == 0, 16-B aligned
    const float* W;                     // [R, F_in, F_out] as the caller passed it
    int R, Fg, Fo;                      // relations, gathered width, output width (both <= 16)
    int transpose;                      // 0: forward (x W_r), 1: dX (q W_r^T)
    float* out; int64_t ldo;
    const float* bias; int act;
    const float* Yact;                  // dX only: out *= act'(Yact)
    float* part;                        // workspace: [tiles][2][16] partial sums of rows cut by tile borders
};

// the tile path takes F_in, F_out <= 16 (every R-GCN layer of the BASELINE configs); SEASTAR_RGCN_ROWS=1 selects the
// one-pass row kernel instead (A/B)
bool rgcn_tile_ok(int R, int64_t Fg, int64_t Fo);
size_t rgcn_tile_ws_bytes(int64_t n_edges);
// zero_rows_begin: the first row without edges (rows are degree-sorted, so rows [zero_rows_begin, n_rows) are empty)
seastar_status rgcn_tile_launch(const RgcnTileArgs& a, int64_t zero_rows_begin, void* ws, cudaStream_t s);

// dW over the type-major view in staged chunks (rgcn_tile.cu): part[t] = sum over task t's edges of
// norm_e X[src_e]^T dA[dst_e] (F_in, F_out <= 16)
struct RgcnDwTileArgs {
    const int32_t* src; const int32_t* dst; const int32_t* eid; const float* norm; const float* norm_user;
    const int32_t* run_off; const int32_t* task_run; int64_t n_tasks;
    const float* X; int64_t ldx; const float* dA; int64_t ldd;
    int Fin, Fout;
    float* part;                        // [n_tasks][Fin * Fout]
};
seastar_status rgcn_dw_tile_launch(const RgcnDwTileArgs& a, cudaStream_t s);

}  // namespace seastar
