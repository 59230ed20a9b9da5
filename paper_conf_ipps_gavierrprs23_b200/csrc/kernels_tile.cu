// kernels_tile.cu — kernel T dispatch: plan-time setup and launch by tile width (the
// template instantiations live in kernels_tile_tw{4,8,16,32,64}.cu).
#include <algorithm>

#include "kernels_tile.cuh"

namespace gs {

void tile_steps(const uint32_t* level_off, uint32_t n_levels, const GateAux* aux, uint32_t chunk,
                std::vector<uint2>& out) {
    out.clear();
    const uint32_t cap = chunk ? std::min(chunk, STEP_N_MASK) : STEP_N_MASK;
    for (uint32_t l = 0; l < n_levels; ++l)
        for (uint32_t g = level_off[l]; g < level_off[l + 1];) {
            const uint32_t k = aux ? (aux[g].k & 0xFFu) : 0u;
            uint32_t e = g + 1;                      // run of equal k (gates are k-grouped per level)
            while (e < level_off[l + 1] && e - g < cap && (!aux || (aux[e].k & 0xFFu) == k)) ++e;
            const bool end = e == level_off[l + 1];
            out.push_back(make_uint2(g, (e - g) | (k << 24) | (end ? 0x80000000u : 0u)));
            g = e;
        }
}

size_t tile_smem_bytes(uint32_t tw, uint32_t ng, uint32_t n_slots, uint32_t n_eval, uint32_t n_steps,
                       int desc_mode) {
    const size_t dbytes = (desc_mode & 4) ? 8 : 16;        // narrow descriptors: 8 bytes
    desc_mode &= 3;
    size_t b = ((size_t)n_steps + 1) / 2 * 16;
    if (desc_mode == 1) b += ((size_t)n_eval * dbytes + 15) / 16 * 16;
    const size_t g = 32 + (desc_mode == 2 ? 2 * (size_t)TILE_CHUNK * 16 : 0) + ((size_t)n_slots + 64) * 4 * tw;
    return b + (size_t)ng * g;
}

cudaError_t tile_setup(uint32_t tw, uint32_t ng, uint32_t n_slots, uint32_t n_eval, uint32_t n_steps,
                       int desc_smem, uint32_t has_q, uint32_t* per_sm) {
    const size_t smem = tile_smem_bytes(tw, ng, n_slots, n_eval, n_steps, desc_smem);
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
    const size_t smem = tile_smem_bytes(tw, ng, a.n_slots, a.n_eval, a.n_steps, a.desc_smem);
    cudaError_t e = cudaMemsetAsync(a.tile_next, 0, sizeof(unsigned int), s);   // empty the tile queue
    if (e != cudaSuccess) return e;
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
