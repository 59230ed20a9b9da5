// kernels_tile_tw16.cu — kernel T instantiations for 512-lane tiles (TW = 16 words).
#include "kernels_tile.cuh"

namespace gs {

#define TILE_DM(Q, G, CALL)                   \
    switch (dm) {                             \
        case 0: CALL(Q, G, 0); break;         \
        case 1: CALL(Q, G, 1); break;         \
        case 2: CALL(Q, G, 2); break;         \
        default: return cudaErrorInvalidValue; \
    }
#define TILE_QG(CALL)                                                                      \
    switch ((has_q ? 8 : 0) + (ng == 1 ? 0 : ng == 2 ? 1 : ng == 4 ? 2 : 7)) {             \
        case 0: TILE_DM(false, 1, CALL) break; case 1: TILE_DM(false, 2, CALL) break;      \
        case 2: TILE_DM(false, 4, CALL) break; case 8: TILE_DM(true, 1, CALL) break;       \
        case 9: TILE_DM(true, 2, CALL) break;  case 10: TILE_DM(true, 4, CALL) break;      \
        default: return cudaErrorInvalidValue;                                             \
    }

template <>
cudaError_t tile_setup_tw<16>(uint32_t ng, size_t smem, int dm, bool has_q, int* per_sm) {
    cudaError_t e = cudaSuccess;
#define PREP(Q, G, D)                                                                                     \
    e = cudaFuncSetAttribute(k_tile<16, Q, G, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); \
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_tile<16, Q, G, D>, TILE_CTA, smem)
    TILE_QG(PREP)
#undef PREP
    return e;
}

template <>
cudaError_t launch_tile_tw<16>(const TileArgs& a, uint32_t ng, uint32_t grid, size_t smem, cudaStream_t s) {
    const int dm = (int)a.desc_smem;
    const bool has_q = a.n_reg > 0;
#define LAUNCH(Q, G, D) k_tile<16, Q, G, D><<<grid, TILE_CTA, smem, s>>>(a)
    TILE_QG(LAUNCH)
#undef LAUNCH
    return cudaGetLastError();
}

}  // namespace gs
