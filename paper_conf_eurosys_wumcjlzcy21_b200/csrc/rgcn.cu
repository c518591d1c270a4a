// rgcn.cu -- a7 / a10: R-GCN (§6.3.5).  Placeholder until the fused kernels land.
#include "common.cuh"

using namespace seastar;

extern "C" {

seastar_status seastar_rgcn_fwd(seastar_graph g, const float* X_all, int64_t F_in, int64_t ldx, const float* W,
                                int64_t F_out, const float* norm_user, const float* bias, seastar_act act,
                                float* Y_loc, int64_t ldy, seastar_stream stream) {
    set_error("rgcn_fwd: not implemented yet");
    return SEASTAR_ERR_UNSUPPORTED;
}

size_t seastar_rgcn_bwd_workspace(seastar_graph g, int64_t F_in, int64_t F_out) { return 0; }

seastar_status seastar_rgcn_bwd(seastar_graph g, const float* X_loc, int64_t F_in, int64_t ldx, const float* dA_all,
                                int64_t F_out, int64_t ldd, const float* W, const float* norm_user, float* dX_loc,
                                float* dW, void* workspace, size_t ws_bytes, seastar_stream stream) {
    set_error("rgcn_bwd: not implemented yet");
    return SEASTAR_ERR_UNSUPPORTED;
}

}  // extern "C"
