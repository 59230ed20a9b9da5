// kernels_tile_inst.cuh — kernel T instantiations for one tile width TW: the plan-time setup
// (shared-memory attribute + occupancy) and the launch over (has registers, groups per CTA,
// descriptor mode).  Each kernels_tile_tw<TW>.cu expands GS_TILE_INSTANTIATE(TW) once, so
// the five widths compile in parallel.
#pragma once

#include "kernels_tile.cuh"

#define GS_TILE_DM(TW, Q, G, CALL)              \
    switch (dm) {                               \
        case 0: CALL(TW, Q, G, 0); break;       \
        case 1: CALL(TW, Q, G, 1); break;       \
        case 2: CALL(TW, Q, G, 2); break;       \
        default: return cudaErrorInvalidValue;  \
    }
/* programs without registers may also use narrow descriptors (mode | 4) */
#define GS_TILE_DMN(TW, G, CALL)                \
    switch (dm) {                               \
        case 0: CALL(TW, false, G, 0); break;   \
        case 1: CALL(TW, false, G, 1); break;   \
        case 2: CALL(TW, false, G, 2); break;   \
        case 4: CALL(TW, false, G, 4); break;   \
        case 5: CALL(TW, false, G, 5); break;   \
        case 6: CALL(TW, false, G, 6); break;   \
        default: return cudaErrorInvalidValue;  \
    }
#define GS_TILE_QG(TW, CALL)                                                                        \
    switch ((has_q ? 8 : 0) + (ng == 1 ? 0 : ng == 2 ? 1 : ng == 4 ? 2 : 7)) {                      \
        case 0: GS_TILE_DMN(TW, 1, CALL) break; case 1: GS_TILE_DMN(TW, 2, CALL) break;             \
        case 2: GS_TILE_DMN(TW, 4, CALL) break; case 8: GS_TILE_DM(TW, true, 1, CALL) break;        \
        case 9: GS_TILE_DM(TW, true, 2, CALL) break;  case 10: GS_TILE_DM(TW, true, 4, CALL) break; \
        default: return cudaErrorInvalidValue;                                                      \
    }
#define GS_TILE_PREP(TW, Q, G, D)                                                                        \
    e = cudaFuncSetAttribute(k_tile<TW, Q, G, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); \
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(per_sm, k_tile<TW, Q, G, D>, TILE_CTA, smem)
#define GS_TILE_LAUNCH(TW, Q, G, D) k_tile<TW, Q, G, D><<<grid, TILE_CTA, smem, s>>>(a)

#define GS_TILE_INSTANTIATE(TW)                                                                       \
    namespace gs {                                                                                    \
    template <>                                                                                       \
    cudaError_t tile_setup_tw<TW>(uint32_t ng, size_t smem, int dm, bool has_q, int* per_sm) {        \
        cudaError_t e = cudaSuccess;                                                                  \
        GS_TILE_QG(TW, GS_TILE_PREP)                                                                  \
        return e;                                                                                     \
    }                                                                                                 \
    template <>                                                                                       \
    cudaError_t launch_tile_tw<TW>(const TileArgs& a, uint32_t ng, uint32_t grid, size_t smem,        \
                                   cudaStream_t s) {                                                  \
        const int dm = (int)a.desc_smem;                                                              \
        const bool has_q = a.n_reg > 0;                                                               \
        GS_TILE_QG(TW, GS_TILE_LAUNCH)                                                                \
        return cudaGetLastError();                                                                    \
    }                                                                                                 \
    }
