// sf_device_check.cu — AOT (nvcc, sm_100a) self-check of the device primitives.
//
// Built by build.py with `nvcc -gencode arch=compute_100a,code=sm_100a`; never
// loaded at run time.  It instantiates every primitive of sf_device.cuh in one
// small TMA ring kernel so a toolchain or PTX regression fails the build, and
// its SASS shows the Blackwell instructions the generated kernels rely on
// (UTMALDG, SYNCS.* for mbarriers).
#include "sf_device.cuh"

extern "C" __global__ void __launch_bounds__(128)
    sf_device_check(const __grid_constant__ SfTmap tm, double *out, int planes) {
    extern __shared__ __align__(128) unsigned char smem[];
    double *ring = (double *)smem;
    sf_u64 *bar = (sf_u64 *)(smem + 2 * 32 * 8 * 8);
    if (threadIdx.x == 0) {
        sf_mbar_init(&bar[0], 1);
        sf_mbar_init(&bar[1], 1);
        sf_fence_mbar_init();
        sf_prefetch_tmap(&tm);
    }
    __syncthreads();
    double acc = 0;
    for (int q = 0; q < planes; ++q) {
        if (threadIdx.x == 0) {
            sf_mbar_expect_tx(&bar[q & 1], 32 * 8 * 8);
            sf_tma_load_3d(ring + (q & 1) * 256, &tm, &bar[q & 1], 0, 0, q);
        }
        sf_mbar_wait(&bar[q & 1], (q >> 1) & 1);
        acc += ring[(q & 1) * 256 + threadIdx.x] + sf_ld(out + threadIdx.x);
        __syncthreads();
    }
    sf_st(out + blockIdx.x * 128 + threadIdx.x, acc);
}

// the peer-push protocol primitives (wait on the neighbours, last-CTA signal)
extern "C" __global__ void __launch_bounds__(32)
    sf_device_check_xs(sf_u64 *sig, sf_u64 *dn, sf_u64 *up, double *peer, double v) {
    const sf_u64 seq = sf_ld_volatile_u64(sig + 2) + 1;
    if (threadIdx.x == 0) sf_xs_wait(sig, dn != nullptr, up != nullptr, seq - 1);
    __syncthreads();
    sf_st(peer + threadIdx.x, v);
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) sf_xs_signal((sf_u32 *)(sig + 3), gridDim.x, sig + 2, dn, up, seq);
}
