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

// consumer release of a ring slot (default .release.cta semantics)
__device__ __forceinline__ void sf_mbar_arrive(sf_u64 *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sf_smem_addr(bar)) : "memory");
}

// named barrier over the compute warps only (the producer warp never joins)
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
// load (ghost cells are never written), 0 when the point is outside the allocation
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
