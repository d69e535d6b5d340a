// device_util.cuh -- small device helpers shared by the tile kernels
// (apply.cu, blocked.cu).  Internal to libsvb200.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/sv.h"

namespace svb {
namespace dev {

__device__ __forceinline__ uint64_t insert_zeros(uint64_t x, const int* pos, int npos) {
#pragma unroll
    for (int b = 0; b < SV_MAX_FUSED; ++b) {
        if (b < npos) {
            const int p = pos[b];
            const uint64_t lo = x & ((1ull << p) - 1ull);
            x = ((x >> p) << (p + 1)) | lo;
        }
    }
    return x;
}

// Shared/global accesses are volatile PTX so that ptxas keeps their order
// (it otherwise sinks stores and re-issues loads under register pressure).
__device__ __forceinline__ void st_stream(float4* p, float4 v) {
    asm volatile("st.global.cs.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
                 : "memory");
}
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ float4 lds4(uint32_t a) {
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts4(uint32_t a, float4 v) {
    asm volatile("st.shared.v4.f32 [%0], {%1,%2,%3,%4};" ::"r"(a), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}
__device__ __forceinline__ float2 lds2(uint32_t a) {
    float2 v;
    asm volatile("ld.shared.v2.f32 {%0,%1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts2(uint32_t a, float2 v) {
    asm volatile("st.shared.v2.f32 [%0], {%1,%2};" ::"r"(a), "f"(v.x), "f"(v.y) : "memory");
}

__device__ __forceinline__ uint32_t swizzle(uint32_t t, const uint32_t* swz) {
    return t ^ ((__popc(t & swz[0]) & 1) << 1) ^ ((__popc(t & swz[1]) & 1) << 2) ^ ((__popc(t & swz[2]) & 1) << 3);
}

__device__ __forceinline__ void cp_async16(uint32_t saddr, const void* g) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(saddr), "l"(g) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

}  // namespace dev
}  // namespace svb
