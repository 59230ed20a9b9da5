// kernels_tile_tw4.cu — kernel T for 128-lane tiles (TW = 4 words); see kernels_tile_inst.cuh.
#include "kernels_tile_inst.cuh"

GS_TILE_INSTANTIATE(4)
