// kernels_tile_tw32.cu — kernel T for 1024-lane tiles (TW = 32 words); see kernels_tile_inst.cuh.
#include "kernels_tile_inst.cuh"

GS_TILE_INSTANTIATE(32)
