// kernels_tile_tw8.cu — kernel T for 256-lane tiles (TW = 8 words); see kernels_tile_inst.cuh.
#include "kernels_tile_inst.cuh"

GS_TILE_INSTANTIATE(8)
