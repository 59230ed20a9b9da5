// kernels_tile_tw16.cu — kernel T for 512-lane tiles (TW = 16 words); see kernels_tile_inst.cuh.
#include "kernels_tile_inst.cuh"

GS_TILE_INSTANTIATE(16)
