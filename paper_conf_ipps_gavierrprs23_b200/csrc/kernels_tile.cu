// kernels_tile.cu — kernel T dispatch: plan-time setup and launch by tile width (the
// template instantiations live in kernels_tile_tw{4,8,16,32,64}.cu).
#include "kernels_tile.cuh"

namespace gs {

static size_t lvl_bytes(uint32_t n_levels) { return (((size_t)n_levels + 1) * 4 + 15) / 16 * 16; }

size_t tile_smem_bytes(uint32_t tw, uint32_t ng, uint32_t n_slots, uint32_t n_eval, uint32_t n_levels,
                       int desc_mode, uint32_t max_width) {
    size_t b = 0, g = ((size_t)n_slots + 64) * 4 * tw;
    if (desc_mode == 1) b = (size_t)n_eval * 16 + lvl_bytes(n_levels);
    if (desc_mode == 2) {
        b = lvl_bytes(n_levels);
        g += 16 + 2 * (size_t)max_width * 16;
    }
    return b + (size_t)ng * g;
}

cudaError_t tile_setup(uint32_t tw, uint32_t ng, uint32_t n_slots, uint32_t n_eval, uint32_t n_levels,
                       int desc_smem, uint32_t max_width, uint32_t has_q, uint32_t* per_sm) {
    const size_t smem = tile_smem_bytes(tw, ng, n_slots, n_eval, n_levels, desc_smem, max_width);
    int per = 0;
    cudaError_t e;
    switch (tw) {
        case 4: e = tile_setup_tw<4>(ng, smem, desc_smem, has_q, &per); break;
        case 8: e = tile_setup_tw<8>(ng, smem, desc_smem, has_q, &per); break;
        case 16: e = tile_setup_tw<16>(ng, smem, desc_smem, has_q, &per); break;
        case 32: e = tile_setup_tw<32>(ng, smem, desc_smem, has_q, &per); break;
        case 64: e = tile_setup_tw<64>(ng, smem, desc_smem, has_q, &per); break;
        default: return cudaErrorInvalidValue;
    }
    *per_sm = (uint32_t)per;
    return e;
}

cudaError_t launch_tile(const TileArgs& a, uint32_t tw, uint32_t ng, uint32_t grid, cudaStream_t s) {
    if (a.n_tiles == 0 || a.ncycles == 0) return cudaSuccess;
    const size_t smem = tile_smem_bytes(tw, ng, a.n_slots, a.n_eval, a.n_levels, a.desc_smem, a.max_width);
    switch (tw) {
        case 4: return launch_tile_tw<4>(a, ng, grid, smem, s);
        case 8: return launch_tile_tw<8>(a, ng, grid, smem, s);
        case 16: return launch_tile_tw<16>(a, ng, grid, smem, s);
        case 32: return launch_tile_tw<32>(a, ng, grid, smem, s);
        case 64: return launch_tile_tw<64>(a, ng, grid, smem, s);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace gs
