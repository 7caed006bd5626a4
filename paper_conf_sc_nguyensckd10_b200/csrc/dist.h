// dist.h — Z-slab decomposition of a sweep.
//
// The grid is cut into P slabs along Z (the streamed dimension, so a slab is
// a contiguous run of planes).  Slab r owns global planes
// [z0, z0 + nzl) (remainder planes one each to the first slabs, the flexible
// balance rule) and is stored with g = dim_T ghost planes below and above:
// buffer plane L holds global plane z0 - g + L.  A sweep of depth d needs the
// input planes [g - d, g + nzl + d): before every sweep the d planes next to
// each slab face are exchanged with the neighbouring slab (the ghosts of the
// OUTPUT of the previous sweep are never written by the kernels).
// Transports: NCCL send/recv between ranks (one process per GPU), or
// cudaMemcpyAsync between plan-owned slab buffers on one device ("loopback",
// the same exchange schedule, used to test the decomposition on one GPU).
// NCCL is dlopen'ed (the process already has torch's libnccl.so.2 loaded).
#pragma once
#include <cstddef>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>
#if ST_HAVE_NCCL
#include <nccl.h>
#endif

namespace st35d {

struct SlabView {
    int nzb = 0;                  // planes in the slab buffer (owned + ghosts)
    int zbase = 0;                // global z of buffer plane 0
    int za = 0, zb = 0;           // buffer planes this launch writes
    const uint8_t* flags = nullptr;   // LBM flags of this slab buffer (nzb planes)
    uint8_t* fl2 = nullptr;           // LBM neighbour-flag buffer of this slab (nzb planes)
    bool single = true;           // the whole grid in one buffer
    int grid_cap = 0;             // >0: leave SMs free (overlapped NCCL kernels)
    cudaStream_t stream = nullptr;
};

inline void slab_range(int nz, int P, int r, int& z0, int& nzl) {
    const int q = nz / P, rem = nz % P;
    nzl = q + (r < rem ? 1 : 0);
    z0 = r * q + (r < rem ? r : rem);
}

#if ST_HAVE_NCCL
struct NcclApi {
    void* h = nullptr;
    ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*groupStart)() = nullptr;
    ncclResult_t (*groupEnd)() = nullptr;
    const char* (*errorString)(ncclResult_t) = nullptr;
    bool load();
};
NcclApi& nccl();
#endif

struct Dist {
    enum Mode { SINGLE, NCCL, LOOPBACK } mode = SINGLE;
    int nz = 0, P = 1, rank = 0, g = 0;
    int z0 = 0, nzl = 0, nzb = 0;        // this rank's slab (NCCL) / whole grid (SINGLE)
    int nranks = 1;                       // P for NCCL, 1 otherwise (caller-visible)
#if ST_HAVE_NCCL
    ncclComm_t nccl_comm = nullptr;
#endif
    struct Slab {
        int z0 = 0, nzl = 0, nzb = 0;
        void* buf[2] = {nullptr, nullptr};
        uint8_t* flags = nullptr;
        uint8_t* fl2 = nullptr;
    };
    std::vector<Slab> slabs;              // LOOPBACK
    cudaStream_t comm = nullptr;          // ghost-exchange stream (overlapped with interior sweeps)
    cudaEvent_t ev_b = nullptr, ev_x = nullptr;
    size_t slab_cell_bytes = 0;
    int slab_ncomp = 0;

    void init_single(int nz_) {
        destroy();
        mode = SINGLE; nz = nz_; P = 1; rank = 0; g = 0; z0 = 0; nzl = nz_; nzb = nz_; nranks = 1;
    }
    void destroy();
};

}  // namespace st35d
