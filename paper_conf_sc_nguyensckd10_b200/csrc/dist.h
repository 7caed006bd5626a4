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
    int sweep = 0;                // index of the sweep (pass) this launch belongs to
    cudaStream_t stream = nullptr;
};

// One step of a rank's Z-slab sweep schedule (buffer coordinates: plane L of
// a slab buffer is global plane z0 - g + L; owned planes [g, g + nzl)).
//   EXCHANGE(src, depth): send buffer src's planes [g, g+depth) to rank-1 and
//     [g+nzl-depth, g+nzl) to rank+1, receive [g-depth, g) and
//     [g+nzl, g+nzl+depth) from them (after d levels only the slab
//     shrunk by d is valid, so d ghost planes per face feed a depth-d sweep);
//     async = 1: on the side stream, overlapped with the SWEEP steps up to WAIT
//   SWEEP(sweep, depth, src, [z_begin, z_end)): depth Jacobi steps from buffer
//     src into buffer 1-src for those output planes; grid_cap = 1: the launch
//     leaves SMs to the overlapped exchange
//   WAIT: the main stream waits for the async exchange
//   COPY: buffer 1 <- buffer 0 (an even number of sweeps left the result in 0)
struct SlabStep {
    enum Kind { EXCHANGE = 0, SWEEP = 1, WAIT = 2, COPY = 3 };
    int kind, sweep, depth, src, z_begin, z_end, async, grid_cap;
};

// The schedule: ghosts of the input, then per sweep k the
// d_{k+1} output planes next to each face first, the exchange of those
// planes for sweep k+1 started on the side stream, the interior planes
// meanwhile, and a wait before sweep k+1.  split needs every slab thicker
// than 2 d_{k+1} (nzl_min); overlap = 0 serialises exchange and sweep.
inline std::vector<SlabStep> slab_schedule(const std::vector<int>& ds, int g, int nzl, int nzl_min, bool overlap) {
    std::vector<SlabStep> v;
    if (ds.empty()) return v;
    v.push_back({SlabStep::EXCHANGE, -1, ds[0], 0, 0, 0, 0, 0});
    int cur = 0;
    for (size_t k = 0; k < ds.size(); ++k) {
        const int d = ds[k], dn = k + 1 < ds.size() ? ds[k + 1] : 0;
        const bool split = overlap && dn > 0 && nzl_min > 2 * dn;
        if (split) {
            v.push_back({SlabStep::SWEEP, (int)k, d, cur, g, g + dn, 0, 0});
            v.push_back({SlabStep::SWEEP, (int)k, d, cur, g + nzl - dn, g + nzl, 0, 0});
            v.push_back({SlabStep::EXCHANGE, (int)k, dn, 1 - cur, 0, 0, 1, 0});
            v.push_back({SlabStep::SWEEP, (int)k, d, cur, g + dn, g + nzl - dn, 0, 1});
            v.push_back({SlabStep::WAIT, (int)k, 0, 0, 0, 0, 0, 0});
        } else {
            v.push_back({SlabStep::SWEEP, (int)k, d, cur, g, g + nzl, 0, 0});
            if (dn > 0) v.push_back({SlabStep::EXCHANGE, (int)k, dn, 1 - cur, 0, 0, 0, 0});
        }
        cur ^= 1;
    }
    if (cur == 0) v.push_back({SlabStep::COPY, -1, 0, 0, 0, 0, 0, 0});
    return v;
}

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
    ncclResult_t (*commInitRankConfig)(ncclComm_t*, int, ncclUniqueId, int, ncclConfig_t*) = nullptr;
    ncclResult_t (*commGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
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
