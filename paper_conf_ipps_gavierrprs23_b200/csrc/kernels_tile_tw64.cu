// kernels_tile_tw64.cu — kernel T for 2048-lane tiles (TW = 64 words); see kernels_tile_inst.cuh.
#include "kernels_tile_inst.cuh"

GS_TILE_INSTANTIATE(64)
