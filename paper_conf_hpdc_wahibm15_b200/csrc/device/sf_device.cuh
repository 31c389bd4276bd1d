// sf_device.cuh — hand-written sm_100a device primitives of the z-march kernels.
//
// Every generated group kernel (codegen.cpp) includes this header: the group
// body (statement expressions, regions, ring depths) is emitted per plan, the
// machinery below is fixed.  Inline PTX only; no CUDA headers are needed, so
// NVRTC compiles it stand-alone for -arch=sm_100a.
//
//   * TMA (cp.async.bulk.tensor.3d) stages one x-y plane of an input array over
//     the tile plus its halo into a shared-memory ring slot; an mbarrier with
//     expect_tx counts the bytes (SASS: UTMALDG / SYNCS.ARRIVE.TRANS64).
//   * Consumers wait on the slot's mbarrier phase parity (try_wait loop).
//   * Streaming stores of live-out results bypass L1.
#pragma once

typedef unsigned long long sf_u64;
typedef unsigned int sf_u32;

// 128-byte CUtensorMap, passed by value in __grid_constant__ kernel parameters
struct __align__(64) SfTmap { sf_u64 w[16]; };

__device__ __forceinline__ sf_u32 sf_smem_addr(const void *p) {
    return (sf_u32)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void sf_mbar_init(sf_u64 *bar, sf_u32 count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sf_smem_addr(bar)), "r"(count)
                 : "memory");
}

// make mbarrier initialisation visible to the async (TMA) proxy
__device__ __forceinline__ void sf_fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void sf_mbar_expect_tx(sf_u64 *bar, sf_u32 bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sf_smem_addr(bar)),
                 "r"(bytes)
                 : "memory");
}

// Phase-parity wait.  SF_SUSPEND_HINT (ns, per generated kernel) adds a suspend-time
// hint to try_wait so a waiting warp may sleep instead of re-issuing the test; off by
// default (a large hint slowed the C4 step by 35 % in round 1 measurements).
#ifndef SF_SUSPEND_HINT
#define SF_SUSPEND_HINT 0
#endif
__device__ __forceinline__ void sf_mbar_wait(sf_u64 *bar, sf_u32 parity) {
#if SF_SUSPEND_HINT
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "SF_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n\t"
        "@!P1 bra SF_WAIT_%=;\n}" ::"r"(sf_smem_addr(bar)),
        "r"(parity), "r"(SF_SUSPEND_HINT)
        : "memory");
#else
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "SF_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra SF_WAIT_%=;\n}" ::"r"(sf_smem_addr(bar)),
        "r"(parity)
        : "memory");
#endif
}

// Producer-side wait for a free ring slot with exponential nanosleep back-off (start
// `ns`, capped at 8x): the producer warp is idle most of the time, and a tight try_wait
// loop spends issue slots of its SM sub-partition (and power) the compute warps need;
// the slot is needed only PF steps later, so a sleeping producer costs no latency.
__device__ __forceinline__ void sf_mbar_wait_backoff(sf_u64 *bar, sf_u32 parity, unsigned ns) {
    unsigned t = ns;
    for (;;) {
        sf_u32 done;
        asm volatile(
            "{\n\t.reg .pred P1;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, P1;\n}" : "=r"(done) : "r"(sf_smem_addr(bar)), "r"(parity) : "memory");
        if (done) return;
        __nanosleep(t);
        t = t < 8 * ns ? 2 * t : t;
    }
}

// Producer-side wait with a suspend-time hint: try_wait suspends the thread until the phase
// completes or the hint (ns) elapses, so the idle producer issues a handful of instructions per
// step instead of a polling loop (the hint is not used for the compute warps' waits: there a
// late wake-up is on the critical path).
__device__ __forceinline__ void sf_mbar_wait_hint(sf_u64 *bar, sf_u32 parity, sf_u32 ns) {
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "SF_WAITH_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n\t"
        "@!P1 bra SF_WAITH_%=;\n}" ::"r"(sf_smem_addr(bar)),
        "r"(parity), "r"(ns)
        : "memory");
}

// consumer release of a ring slot (default .release.cta semantics)
__device__ __forceinline__ void sf_mbar_arrive(sf_u64 *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sf_smem_addr(bar)) : "memory");
}

// named barrier over the compute warps only (the producer warp never joins)
// named-barrier arrive (no wait): the compute warps' "slot free" signal to a producer
// warp blocked in bar.sync on the same id (option pbar)
__device__ __forceinline__ void sf_bar_arrive(int id, int nthreads) {
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ void sf_bar_sync(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// programmatic dependent launch: let the next group's grid start its prologue, and
// wait for the previous grid's memory operations before touching dependent data
__device__ __forceinline__ void sf_pdl_launch_dependents() {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void sf_pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

__device__ __forceinline__ void sf_prefetch_tmap(const SfTmap *m) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(m) : "memory");
}

// one plane box (x, y, z are element coordinates in the padded allocation;
// out-of-range elements are zero-filled by the TMA unit and never consumed)
__device__ __forceinline__ void sf_tma_load_3d(void *dst, const SfTmap *map, sf_u64 *bar, int x,
                                               int y, int z) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(sf_smem_addr(dst)),
        "l"(map), "r"(sf_smem_addr(bar)), "r"(x), "r"(y), "r"(z)
        : "memory");
}

// L2 prefetch of a plane box (no shared memory, no completion): raises the DRAM
// requests in flight beyond what the shared-memory rings can hold
__device__ __forceinline__ void sf_tma_prefetch_3d(const SfTmap *map, int x, int y, int z) {
    asm volatile(
        "cp.async.bulk.prefetch.tensor.3d.L2.global.tile [%0, {%1, %2, %3}];" ::"l"(map), "r"(x),
        "r"(y), "r"(z)
        : "memory");
}

// live-out stores: written once, never re-read by this launch
__device__ __forceinline__ void sf_st(double *p, double v) {
    asm volatile("st.global.L1::no_allocate.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}
__device__ __forceinline__ void sf_st(float *p, float v) {
    asm volatile("st.global.L1::no_allocate.f32 [%0], %1;" ::"l"(p), "f"(v) : "memory");
}
// 16-byte live-out stores (x-adjacent points of a register block)
__device__ __forceinline__ void sf_st_v(double *p, double2 v) {
    asm volatile("st.global.L1::no_allocate.v2.f64 [%0], {%1, %2};" ::"l"(p), "d"(v.x), "d"(v.y)
                 : "memory");
}
__device__ __forceinline__ void sf_st_v(float *p, float4 v) {
    asm volatile("st.global.L1::no_allocate.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(v.x),
                 "f"(v.y), "f"(v.z), "f"(v.w)
                 : "memory");
}

// ghost value of a point outside the global interior: predicated non-coherent
// load (no kernel writes ghost cells of the arrays it reads while it runs), 0 when
// the point is outside the allocation
__device__ __forceinline__ double sf_ldg_pred(const double *p, bool pred) {
    double v = 0.0;
    asm("{\n\t.reg .pred P1;\n\tsetp.ne.b32 P1, %2, 0;\n\t@P1 ld.global.nc.f64 %0, [%1];\n}"
        : "+d"(v) : "l"(p), "r"((int)pred));
    return v;
}
__device__ __forceinline__ float sf_ldg_pred(const float *p, bool pred) {
    float v = 0.0f;
    asm("{\n\t.reg .pred P1;\n\tsetp.ne.b32 P1, %2, 0;\n\t@P1 ld.global.nc.f32 %0, [%1];\n}"
        : "+f"(v) : "l"(p), "r"((int)pred));
    return v;
}
__device__ __forceinline__ double sf_ld(const double *p) {
    double v;
    asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ float sf_ld(const float *p) {
    float v;
    asm volatile("ld.global.nc.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}

// ---- thread-block clusters: x-halo sharing through distributed shared memory ----
// (option cluster_x; the cluster's CTAs are x-neighbouring tiles: a stage value a
// CTA needs inside its neighbour's tile is read from the neighbour's shared-memory
// ring instead of being recomputed, P:L292's reason to recompute — shared memory
// scoped to one thread block — no longer holds on sm_100a)
__device__ __forceinline__ sf_u32 sf_cluster_rank() {
    sf_u32 r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
// every thread of every CTA of the cluster (exited threads excluded)
__device__ __forceinline__ void sf_cluster_sync() {
    asm volatile("barrier.cluster.arrive.aligned;\n\tbarrier.cluster.wait.aligned;" ::: "memory");
}
// the address of the same shared-memory location in CTA `rank` of the cluster
__device__ __forceinline__ sf_u32 sf_mapa(const void *p, sf_u32 rank) {
    sf_u32 r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(sf_smem_addr(p)), "r"(rank));
    return r;
}
// arrive on an mbarrier of another CTA of the cluster; release: this thread's prior
// shared-memory writes are visible to the waiter's acquire
__device__ __forceinline__ void sf_mbar_arrive_remote(sf_u32 cluster_addr) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr)
                 : "memory");
}
__device__ __forceinline__ void sf_mbar_wait_cluster(sf_u64 *bar, sf_u32 parity) {
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "SF_CWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra SF_CWAIT_%=;\n}" ::"r"(sf_smem_addr(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ double sf_ld_dsmem(sf_u32 cluster_addr, double) {
    double v;
    asm volatile("ld.shared::cluster.f64 %0, [%1];" : "=d"(v) : "r"(cluster_addr) : "memory");
    return v;
}
__device__ __forceinline__ float sf_ld_dsmem(sf_u32 cluster_addr, float) {
    float v;
    asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(cluster_addr) : "memory");
    return v;
}

// ---- peer-push halo protocol (several ranks, option xpush) --------------------
// Signal block of a rank (64 B, device memory of that rank, mapped by its
// neighbours): u64 [0] progress published by the lower neighbour, [1] by the
// upper neighbour, [2] this rank's own progress; u32 at byte 24: CTAs done,
// byte 28: bottom end CTAs done, byte 32: top end CTAs done.
__device__ __forceinline__ sf_u64 sf_ld_volatile_u64(const sf_u64 *p) {
    sf_u64 v;
    asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ sf_u64 sf_ld_acquire_sys(const sf_u64 *p) {
    sf_u64 v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void sf_st_release_sys(sf_u64 *p, sf_u64 v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ sf_u64 sf_globaltimer() {
    sf_u64 t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
// wait until the existing neighbours have published progress >= want; a peer that
// never arrives (a rank that stopped) traps after 20 s instead of hanging the GPU
__device__ __forceinline__ void sf_xs_wait(const sf_u64 *own, bool has_dn, bool has_up, sf_u64 want) {
    const sf_u64 t0 = sf_globaltimer();
    while ((has_dn && sf_ld_acquire_sys(own + 0) < want) || (has_up && sf_ld_acquire_sys(own + 1) < want)) {
        asm volatile("nanosleep.u32 200;");
        if (sf_globaltimer() - t0 > 20000000000ull) asm volatile("trap;");
    }
    // the pushed planes were written through the generic proxy; TMA reads them
    asm volatile("fence.proxy.async.global;" ::: "memory");
}
// order of the chunks: the two slab-end chunks first (0, last), then the middle
__device__ __forceinline__ int sf_xs_chunk(int b, int n) {
    return n < 2 || b == 0 ? b : (b == 1 ? n - 1 : b - 1);
}
// end-chunk completion of one side: the last of its `total` CTAs publishes seq into
// the neighbour's slot (the whole-grid signal below publishes it again, harmlessly)
// The counters use relaxed atomics: a CTA whose stores a neighbour depends on (an
// end chunk) executed fence.sc.sys (__threadfence_system) before its increment, and
// the last CTA executes fence.sc.sys before publishing, which orders those stores
// before the publication (fence-fence synchronisation through the atomic's RMW
// chain).  A release atomic in every CTA would stall each exiting CTA's SM on a
// gpu-scope membar (measured: 23 % on a C5 group).
__device__ __forceinline__ void sf_xs_signal_side(sf_u32 *ctr, sf_u32 total, sf_u64 *slot, sf_u64 seq) {
    sf_u32 old;
    asm volatile("atom.relaxed.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(ctr) : "memory");
    if (old != total - 1) return;
    asm volatile("st.relaxed.gpu.global.u32 [%0], 0;" ::"l"(ctr) : "memory");
    asm volatile("fence.sc.sys;" ::: "memory");
    sf_st_release_sys(slot, seq);
}
// CTA completion; the last CTA of the grid publishes seq (own progress and both
// neighbours' "from" slots) after a system-scope fence
__device__ __forceinline__ void sf_xs_signal(sf_u32 *ctr, sf_u32 total, sf_u64 *self, sf_u64 *dn,
                                             sf_u64 *up, sf_u64 seq) {
    sf_u32 old;
    asm volatile("atom.relaxed.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(ctr) : "memory");
    if (old != total - 1) return;
    asm volatile("st.relaxed.gpu.global.u32 [%0], 0;" ::"l"(ctr) : "memory");
    asm volatile("fence.sc.sys;" ::: "memory");
    asm volatile("st.volatile.global.u64 [%0], %1;" ::"l"(self), "l"(seq) : "memory");
    if (dn) sf_st_release_sys(dn + 1, seq);  // I am the lower neighbour's upper neighbour
    if (up) sf_st_release_sys(up + 0, seq);
}
