// comm.cpp — z-slab halo exchange over NCCL (new relative to the
// paper, which runs on a single node, §6.1.2).
//
// Rank r owns global planes [z_offset, z_offset + nz_local).  Ghost planes are
// contiguous because z is the slowest axis, so each direction is one
// ncclSend/ncclRecv of depth * plane elements, with no packing.  All arrays of
// one exchange go in one ncclGroupStart/End.
#include <cuda_runtime.h>
#include <nccl.h>

#include <cstring>

#include "sf_internal.h"

static void nccl_check(ncclResult_t r, const char *what) {
    if (r != ncclSuccess)
        sf::fail(SP_E_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}

void sf_comm_unique_id_impl(void *out) {
    ncclUniqueId id;
    nccl_check(ncclGetUniqueId(&id), "ncclGetUniqueId");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    std::memcpy(out, &id, 128);
}

sp_comm *sf_comm_create_impl(const void *idp, int32_t nranks, int32_t rank) {
    sf::ensure_cuda();
    ncclUniqueId id;
    std::memcpy(&id, idp, 128);
    std::unique_ptr<sp_comm> c(new sp_comm());
    c->nranks = nranks;
    c->rank = rank;
    cudaGetDevice(&c->device);
    ncclComm_t comm;
    nccl_check(ncclCommInitRank(&comm, nranks, id, rank), "ncclCommInitRank");
    c->nccl = comm;
    cudaStream_t s;
    if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess)
        sf::fail(SP_E_CUDA, "cudaStreamCreate (comm stream)");
    c->comm_stream = s;
    return c.release();
}

void sf_comm_destroy_impl(sp_comm *c) {
    if (c->nccl) ncclCommDestroy((ncclComm_t)c->nccl);
    if (c->comm_stream) cudaStreamDestroy((cudaStream_t)c->comm_stream);
    delete c;
}

namespace sf {

void exchange(stencil_program *p, const std::vector<int> &arrays, int depth, void *stream) {
    sp_comm *c = p->comm;
    if (!c || c->nranks == 1 || arrays.empty()) return;
    for (int a : arrays)
        if (!p->ptrs[a]) fail(SP_E_STATE, "array '" + p->arrays[a].name + "' is not bound");
    const int64_t plane = p->plane;
    const int64_t nz = p->grid.nz_local;
    const int64_t oz = p->layout.origin_z;
    const size_t count = (size_t)(depth * plane);
    const ncclDataType_t dt = p->elem == 8 ? ncclFloat64 : ncclFloat32;
    const int up = c->rank + 1 < c->nranks ? c->rank + 1 : -1;
    const int dn = c->rank > 0 ? c->rank - 1 : -1;
    ncclComm_t comm = (ncclComm_t)c->nccl;
    cudaStream_t s = (cudaStream_t)stream;
    nccl_check(ncclGroupStart(), "ncclGroupStart");
    for (int a : arrays) {
        char *base = (char *)p->ptrs[a];
        auto at = [&](int64_t z) { return base + (z + oz) * plane * p->elem; };
        if (up >= 0) {
            // my top `depth` interior planes -> up's bottom ghosts; up's bottom planes -> my top ghosts
            nccl_check(ncclSend(at(nz - depth), count, dt, up, comm, s), "ncclSend");
            nccl_check(ncclRecv(at(nz), count, dt, up, comm, s), "ncclRecv");
        }
        if (dn >= 0) {
            nccl_check(ncclSend(at(0), count, dt, dn, comm, s), "ncclSend");
            nccl_check(ncclRecv(at(-depth), count, dt, dn, comm, s), "ncclRecv");
        }
    }
    nccl_check(ncclGroupEnd(), "ncclGroupEnd");
}

}  // namespace sf
