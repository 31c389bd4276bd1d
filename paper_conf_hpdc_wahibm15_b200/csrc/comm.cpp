// comm.cpp — z-slab halo exchange (new relative to the paper,
// which runs on a single node, §6.1.2).
//
// Rank r owns global planes [z_offset, z_offset + nz_local).  Ghost planes are
// contiguous because z is the slowest axis, so each direction is one transfer of
// depth * plane elements per array, with no packing.  Two transports:
//   * NCCL (one process per GPU): ncclSend/ncclRecv, all arrays of one exchange
//     in one ncclGroupStart/End;
//   * loopback (test transport): the virtual ranks of one process on one device,
//     each driven from its own host thread; a rank pulls its ghost planes from the
//     neighbours' slabs with device-to-device copies, ordered by events that the
//     ranks publish at host barriers.  It runs the executor's multi-rank schedule
//     (exchange set, interior/boundary split, events) exactly as NCCL does; only
//     the wire differs.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <chrono>
#include <atomic>
#include <thread>
#include <cstring>
#include <map>

#include "sf_internal.h"

static void nccl_check(ncclResult_t r, const char *what) {
    if (r != ncclSuccess)
        sf::fail(SP_E_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}

namespace sf {

struct LoopHub {
    int n = 0;
    std::atomic<int> arrived{0};
    std::atomic<uint64_t> gen{0};
    std::vector<stencil_program *> prog;
    std::vector<cudaEvent_t> ready, done;
    std::once_flag events_once;  // created at the first exchange (creation needs no GPU)

    // all n virtual ranks meet (spinning: the exchange issues device work between
    // barriers and a sleeping wake-up would starve the GPU); a missing rank (an
    // error on its thread) times out
    void barrier() {
        const uint64_t g = gen.load(std::memory_order_acquire);
        if (arrived.fetch_add(1, std::memory_order_acq_rel) + 1 == n) {
            arrived.store(0, std::memory_order_relaxed);
            gen.fetch_add(1, std::memory_order_acq_rel);
            return;
        }
        const auto t0 = std::chrono::steady_clock::now();
        for (uint64_t k = 1; gen.load(std::memory_order_acquire) == g; ++k) {
            if (k % 64 == 0) std::this_thread::yield();
            if (k % 4096 == 0 && std::chrono::steady_clock::now() - t0 > std::chrono::seconds(120))
                fail(SP_E_STATE, "loopback exchange: a virtual rank did not reach the exchange "
                                 "(each rank must run the same plan on its own host thread)");
        }
    }
    ~LoopHub() {
        for (cudaEvent_t e : ready) cudaEventDestroy(e);
        for (cudaEvent_t e : done) cudaEventDestroy(e);
    }
};

// Per launch, the arrays whose ghost planes must be received before it, with the
// depth below/above.  An array is exchanged once per "epoch" (the step start or a
// launch that stores it, up to the next such launch), at the largest depth any
// reader of the epoch needs; an unchanged array is not re-sent to every consumer.
// An epoch that begins at a store is exchanged before its first launch that reads
// the array beyond the slab; every step-start epoch (values final before the step:
// IN arrays, state of the previous step) is exchanged in ONE exchange in front of
// the step's first launch.  A launch never reads beyond the slab an array it
// stores (reading R11), so the epoch's value is the one every reader sees.
//
// Peer push (option xpush, several ranks): an epoch that begins at a store of a
// TEMP array is not exchanged at all; the storing launch writes the planes the
// neighbours' readers need straight into their ghost planes (peer stores over
// NVLink, or the loopback ranks' buffers), and the kernels order themselves with
// the neighbours through per-launch progress flags (codegen: xp protocol).  TEMP
// only: the caller never rebinds scratch arrays, so the neighbours' mapped
// buffers stay valid across steps.
void exchange_schedule(const stencil_program *p, Mode &m) {
    const size_t n = m.launches.size();
    const int na = (int)p->arrays.size();
    const bool push = p->opt.xpush && p->comm && p->comm->nranks > 1;
    m.xsched.assign(n, {});
    for (Launch &L : m.launches) {
        L.pushes.clear();
        L.xp = push && !L.dead;
        L.xp_dw = 0;
    }
    int first_live = -1;
    for (size_t i = 0; i < n && first_live < 0; ++i)
        if (!m.launches[i].dead) first_live = (int)i;
    std::vector<int> first(na, -1), below(na, 0), above(na, 0), writer(na, -1);
    std::vector<std::vector<int>> readers(na);
    auto flush = [&](int a) {
        if (first[a] >= 0) {
            if (push && writer[a] >= 0 && p->arrays[a].role == SP_TEMP) {
                Launch &W = m.launches[writer[a]];
                for (size_t s = 0; s < W.st.size(); ++s)
                    if (W.st[s].stored && W.st[s].out == a)
                        W.pushes.push_back({(int)s, above[a], below[a]});
                W.xp_dw = std::max({W.xp_dw, above[a], below[a]});
                for (int r : readers[a]) {
                    Launch &R = m.launches[r];
                    R.xp_dw = std::max({R.xp_dw, R.z_below, R.z_above});
                }
            } else {
                m.xsched[first[a]].push_back({a, below[a], above[a]});
            }
        }
        first[a] = -1;
        below[a] = above[a] = 0;
        readers[a].clear();
    };
    for (size_t i = 0; i < n; ++i) {
        const Launch &L = m.launches[i];
        if (L.dead) continue;
        auto read = [&](int arr, int b, int u) {
            if (!b && !u) return;
            if (first[arr] < 0) first[arr] = writer[arr] >= 0 ? (int)i : first_live;
            below[arr] = std::max(below[arr], b);
            above[arr] = std::max(above[arr], u);
            readers[arr].push_back((int)i);
        };
        for (const Input &I : L.in) read(I.arr, std::max(0, -I.qlo), std::max(0, I.ahi));
        // R2': a boxed statement evaluated on planes beyond the slab (z warm-up below,
        // lead above) loads its array's previous value there outside its box
        for (const Stage &G : L.st)
            if (G.needed && p->stmts[G.gid].boxed) read(G.out, std::max(0, -G.loff), std::max(0, G.lead));
        for (const Stage &G : L.st)
            if (G.stored) {
                flush(G.out);
                writer[G.out] = (int)i;
            }
    }
    for (int a = 0; a < na; ++a) flush(a);
    for (auto &v : m.xsched)
        std::sort(v.begin(), v.end(), [](const Mode::Xfer &x, const Mode::Xfer &y) { return x.arr < y.arr; });
    m.xsched_ok = true;
}

static void exchange_loopback(stencil_program *p, const std::vector<Mode::Xfer> &x,
                              cudaStream_t s) {
    sp_comm *c = p->comm;
    LoopHub &h = *c->hub;
    const int r = c->rank;
    std::call_once(h.events_once, [&] {
        for (int k = 0; k < h.n; ++k)
            for (auto *v : {&h.ready, &h.done}) {
                cudaEvent_t e;
                if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
                    fail(SP_E_CUDA, "cudaEventCreate");
                v->push_back(e);
            }
    });
    h.prog[r] = p;
    if (cudaEventRecord(h.ready[r], s) != cudaSuccess) fail(SP_E_CUDA, "event record");
    h.barrier();  // every rank's slab is final up to its `ready`
    const int up = r + 1 < h.n ? r + 1 : -1, dn = r > 0 ? r - 1 : -1;
    for (int nb : {up, dn})
        if (nb >= 0 && cudaStreamWaitEvent(s, h.ready[nb], 0) != cudaSuccess)
            fail(SP_E_CUDA, "stream wait");
    const int64_t nz = p->grid.nz_local;
    const size_t pb = (size_t)(p->plane * p->elem);
    for (const Mode::Xfer &t : x) {
        auto at = [&](stencil_program *q, int64_t z) {
            if (!q->ptrs[t.arr]) fail(SP_E_STATE, "array '" + q->arrays[t.arr].name + "' is not bound");
            return (char *)q->ptrs[t.arr] + (z + q->layout.origin_z) * pb;
        };
        if (up >= 0 && t.above > 0 &&
            cudaMemcpyAsync(at(p, nz), at(h.prog[up], 0), t.above * pb, cudaMemcpyDeviceToDevice, s) !=
                cudaSuccess)
            fail(SP_E_CUDA, "loopback copy");
        if (dn >= 0 && t.below > 0 &&
            cudaMemcpyAsync(at(p, -t.below), at(h.prog[dn], nz - t.below), t.below * pb,
                            cudaMemcpyDeviceToDevice, s) != cudaSuccess)
            fail(SP_E_CUDA, "loopback copy");
    }
    if (cudaEventRecord(h.done[r], s) != cudaSuccess) fail(SP_E_CUDA, "event record");
    h.barrier();
    // my interior planes stay unmodified until the neighbours have pulled them
    // (the send-completion of ncclSend)
    for (int nb : {up, dn})
        if (nb >= 0 && cudaStreamWaitEvent(s, h.done[nb], 0) != cudaSuccess)
            fail(SP_E_CUDA, "stream wait");
    h.barrier();  // no rank re-records its events before the others have waited on them
}

void exchange(stencil_program *p, const std::vector<Mode::Xfer> &x, void *stream) {
    sp_comm *c = p->comm;
    if (!c || c->nranks == 1 || x.empty()) return;
    nvtxRangePushA("stencilfuse exchange_halos");
    struct Pop { ~Pop() { nvtxRangePop(); } } pop_range;
    for (const Mode::Xfer &t : x)
        if (!p->ptrs[t.arr]) fail(SP_E_STATE, "array '" + p->arrays[t.arr].name + "' is not bound");
    if (c->hub) {
        exchange_loopback(p, x, (cudaStream_t)stream);
        return;
    }
    const int64_t plane = p->plane;
    const int64_t nz = p->grid.nz_local;
    const int64_t oz = p->layout.origin_z;
    const ncclDataType_t dt = p->elem == 8 ? ncclFloat64 : ncclFloat32;
    const int up = c->rank + 1 < c->nranks ? c->rank + 1 : -1;
    const int dn = c->rank > 0 ? c->rank - 1 : -1;
    ncclComm_t comm = (ncclComm_t)c->nccl;
    cudaStream_t s = (cudaStream_t)stream;
    nccl_check(ncclGroupStart(), "ncclGroupStart");
    for (const Mode::Xfer &t : x) {
        char *base = (char *)p->ptrs[t.arr];
        auto at = [&](int64_t z) { return base + (z + oz) * plane * p->elem; };
        // every rank runs the same schedule: the neighbour below receives `above`
        // planes into its top ghost, the one above `below` planes into its bottom ghost
        if (up >= 0) {
            if (t.below > 0) nccl_check(ncclSend(at(nz - t.below), t.below * plane, dt, up, comm, s), "ncclSend");
            if (t.above > 0) nccl_check(ncclRecv(at(nz), t.above * plane, dt, up, comm, s), "ncclRecv");
        }
        if (dn >= 0) {
            if (t.above > 0) nccl_check(ncclSend(at(0), t.above * plane, dt, dn, comm, s), "ncclSend");
            if (t.below > 0) nccl_check(ncclRecv(at(-t.below), t.below * plane, dt, dn, comm, s), "ncclRecv");
        }
    }
    nccl_check(ncclGroupEnd(), "ncclGroupEnd");
}

}  // namespace sf

void sf_comm_unique_id_impl(void *out) {
    ncclUniqueId id;
    nccl_check(ncclGetUniqueId(&id), "ncclGetUniqueId");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    std::memcpy(out, &id, 128);
}

namespace sf {
void *comm_stream(sp_comm *c) {
    if (!c->comm_stream) {
        cudaStream_t s;
        if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess)
            fail(SP_E_CUDA, "cudaStreamCreate (comm stream)");
        c->comm_stream = s;
    }
    return c->comm_stream;
}
}  // namespace sf

static cudaStream_t new_stream() {
    cudaStream_t s;
    if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess)
        sf::fail(SP_E_CUDA, "cudaStreamCreate (comm stream)");
    return s;
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
    c->comm_stream = new_stream();
    return c.release();
}

// no CUDA call here: streams and events are created at the first exchange, so a
// loopback program can be analysed and JIT-compiled on a host without a GPU
void sf_comm_create_loopback_impl(int32_t nranks, sp_comm **out) {
    auto hub = std::make_shared<sf::LoopHub>();
    hub->n = nranks;
    hub->prog.assign(nranks, nullptr);
    std::vector<std::unique_ptr<sp_comm>> cs;
    for (int r = 0; r < nranks; ++r) {
        std::unique_ptr<sp_comm> c(new sp_comm());
        c->nranks = nranks;
        c->rank = r;
        c->hub = hub;
        cs.push_back(std::move(c));
    }
    for (int r = 0; r < nranks; ++r) out[r] = cs[r].release();
}

void sf_comm_destroy_impl(sp_comm *c) {
    if (c->nccl) ncclCommDestroy((ncclComm_t)c->nccl);
    if (c->comm_stream) cudaStreamDestroy((cudaStream_t)c->comm_stream);
    delete c;
}

// CUDA IPC of a device pointer inside a cudaMalloc allocation (e.g. a torch
// tensor of the caching allocator): the handle names the whole allocation, the
// offset the pointer inside it.  A process opens each allocation once.
void sf_ipc_export_impl(const void *ptr, void *handle64, int64_t *offset) {
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "cudaIpcMemHandle_t size");
    CUdeviceptr base = 0;
    size_t size = 0;
    if (!sf::driver_mem_range(&base, &size, (CUdeviceptr)ptr))
        sf::fail(SP_E_CUDA, "cuMemGetAddressRange");
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, (void *)base) != cudaSuccess) sf::fail(SP_E_CUDA, "cudaIpcGetMemHandle");
    std::memcpy(handle64, &h, 64);
    *offset = (int64_t)((CUdeviceptr)ptr - base);
}

void *sf_ipc_open_impl(const void *handle64, int64_t offset) {
    static std::mutex mu;
    static std::map<std::string, void *> opened;
    std::lock_guard<std::mutex> lk(mu);
    std::string key((const char *)handle64, 64);
    auto it = opened.find(key);
    if (it == opened.end()) {
        cudaIpcMemHandle_t h;
        std::memcpy(&h, handle64, 64);
        void *base = nullptr;
        if (cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
            sf::fail(SP_E_CUDA, "cudaIpcOpenMemHandle");
        it = opened.emplace(key, base).first;
    }
    return (char *)it->second + offset;
}
