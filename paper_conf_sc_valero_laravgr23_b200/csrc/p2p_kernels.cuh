// p2p_kernels.cuh -- device-side ordering of the P2P halo transport (host TU only:
// non-template kernels, so exactly one translation unit may include this).
#pragma once
#include "mrlbm_kernels.cuh"

namespace mr {

// ------------------------------------------------------------ P2P transport synchronisation
// Per handle, a device word array sync[4]: [0] pushes completed by this rank,
// [1] / [2] pushes completed by the lower / upper neighbour (written by them,
// through peer memory).  Before a step's boundary layers a rank waits until
// both neighbours have completed as many pushes as itself: then its ghost
// planes hold their latest layers (read after write) and they have finished
// the step that last read the ghost planes it is about to overwrite (write
// after read).  Device-side counters, so the sequence is graph-capturable.
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer_ns()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__global__ void p2p_wait_kernel(unsigned long long *sync, int need_lo, int need_hi, int *err)
{
    if (*(volatile int *)err) return; // already failed: no further 30 s waits (mrlbm_sync reports it)
    const unsigned long long target = sync[0];
    const unsigned long long t0 = globaltimer_ns();
    while ((need_lo && ld_acquire_sys(&sync[1]) < target) || (need_hi && ld_acquire_sys(&sync[2]) < target)) {
        __nanosleep(256);
        if (globaltimer_ns() - t0 > 30ull * 1000000000ull) { // a neighbour stopped: report, do not hang
            atomicExch(err, 2);
            return;
        }
    }
}

__global__ void p2p_signal_kernel(unsigned long long *sync, unsigned long long *lo_sync, unsigned long long *hi_sync,
                                  const int *err)
{
    // after a timed-out wait this rank's boundary layers used stale ghosts: stop
    // signalling, so the neighbours time out (and report) instead of reading them
    if (*(volatile const int *)err) return;
    __threadfence_system();
    const unsigned long long c = sync[0] + 1;
    sync[0] = c;
    if (lo_sync) st_release_sys(&lo_sync[2], c); // this rank is its lower neighbour's upper neighbour
    if (hi_sync) st_release_sys(&hi_sync[1], c);
}

} // namespace mr
