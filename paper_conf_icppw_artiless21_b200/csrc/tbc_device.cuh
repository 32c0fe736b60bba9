// tbc_device.cuh -- device-side memory-model and cache-policy helpers shared by the
// persistent kernels of libturbobc (product code; shares nothing with oracle/).
#pragma once
#include <cstdint>

namespace tbc {

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// tid.x through a volatile move: values derived from it cannot be rematerialised from S2R, so the
// compiler keeps them in registers (see k_bcb)
__device__ __forceinline__ unsigned tid_opaque() {
    unsigned t;
    asm volatile("mov.u32 %0, %%tid.x;" : "=r"(t));
    return t;
}

__device__ __forceinline__ void fence_acq_rel() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// streaming read of graph indices: read-only for the whole kernel, L1 no-allocate, L2 evict-first
__device__ __forceinline__ int ld_stream(const int32_t *ptr, uint64_t pol) {
    int v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(ptr), "l"(pol));
    return v;
}

__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long *p) {
    return *(volatile const unsigned long long *)p;
}

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

#ifndef TBC_WATCHDOG_S
#define TBC_WATCHDOG_S 20
#endif
constexpr unsigned long long kWatchdogNs = TBC_WATCHDOG_S * 1000ull * 1000 * 1000;  // at one barrier (sanitizer builds: longer)

}  // namespace tbc
