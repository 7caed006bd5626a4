// dist.h — Z-slab decomposition of a sweep.
// Single-device for now: one slab covering the whole grid.
#pragma once
#include <cstddef>
#include <cuda_runtime.h>

namespace st35d {

struct SlabView {
    int nzb = 0;            // planes in the slab buffer (owned + ghosts)
    int zbase = 0;          // global z of buffer plane 0
    int za = 0, zb = 0;     // buffer planes this launch writes
    size_t flags_off = 0;   // offset of buffer plane 0 in the caller's flags array
    cudaStream_t stream = nullptr;
};

struct Dist {
    int nranks = 1, rank = 0;
    int z0 = 0, nzl = 0, nzb = 0, g = 0;

    void init_single(int nz) {
        nranks = 1; rank = 0; z0 = 0; nzl = nz; nzb = nz; g = 0;
    }
    void destroy() {}

    template <typename F>
    int sweep(cudaStream_t s, int /*depth*/, const void* src, void* dst, size_t /*cell_bytes*/,
              size_t /*plane_cells*/, F&& launch) {
        SlabView sv;
        sv.nzb = nzb; sv.zbase = z0 - g; sv.za = g; sv.zb = g + nzl; sv.flags_off = 0; sv.stream = s;
        return launch(src, dst, sv);
    }
};

}  // namespace st35d
