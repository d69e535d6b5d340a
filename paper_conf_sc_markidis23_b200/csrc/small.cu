// small.cu -- whole-circuit kernel for states that fit in shared memory
// (n <= 13: 2^13 x 8 B = 64 KB).  SURVEY.md §7.2 hard part 6: a 12-qubit
// circuit (BASELINE config 1) is launch-bound -- 121 separate launches of a
// 32 KB state cost ~5 us each.  Here ONE CTA loads the state into shared
// memory, applies every fused gate of the circuit in order (the same group
// transform as apply.cu: gather the 2^k members, y = M a in the
// 3-multiplication form, scatter), with a block barrier
// between gates, and writes the state back.  Matrices for all gates are
// uploaded once per circuit (row a4).
#include <cuda_runtime.h>

#include <cstring>

#include "kernels.h"

namespace svb {

namespace {

__device__ __forceinline__ uint32_t ins_zero32(uint32_t x, const int* pos, int k) {
    for (int b = 0; b < k; ++b) {
        const int p = pos[b];
        x = ((x >> p) << (p + 1)) | (x & ((1u << p) - 1u));
    }
    return x;
}

constexpr int kSmallThreads = 256;

// One fused gate on the shared-memory state: every group's members are
// gathered into registers, transformed (Gauss 3-multiplication form with the
// planes P = Re m, S = Re m + Im m, Q = Im m - Re m) and scattered back.
template <int K>
__device__ __forceinline__ void small_gate(float2* st, int n, const int* q, const float* P, const float* S,
                                           const float* Q) {
    constexpr int D = 1 << K;
    uint32_t off[D];
#pragma unroll
    for (int c = 0; c < D; ++c) {
        uint32_t o = 0;
#pragma unroll
        for (int b = 0; b < K; ++b)
            if ((c >> b) & 1) o |= 1u << q[b];
        off[c] = o;
    }
    const uint32_t ngroups = (1u << n) >> K;
    for (uint32_t grp = threadIdx.x; grp < ngroups; grp += blockDim.x) {
        const uint32_t base = ins_zero32(grp, q, K);
        float2 a[D];
        float s[D];
#pragma unroll
        for (int c = 0; c < D; ++c) {
            a[c] = st[base | off[c]];
            s[c] = a[c].x + a[c].y;
        }
#pragma unroll 1
        for (int r = 0; r < D; ++r) {
            float A = 0.f, B = 0.f, C = 0.f;
#pragma unroll
            for (int c = 0; c < D; ++c) {
                A = fmaf(P[r * D + c], s[c], A);
                B = fmaf(S[r * D + c], a[c].y, B);
                C = fmaf(Q[r * D + c], a[c].x, C);
            }
            st[base | off[r]] = make_float2(A - B, A + C);
        }
    }
}

__global__ void __launch_bounds__(kSmallThreads) small_circuit_kernel(float2* __restrict__ psi, int n, int ngates,
                                                                      const SmallGateDesc* __restrict__ gates,
                                                                      const float2* __restrict__ mats) {
    extern __shared__ float4 ssm[];
    float2* st = reinterpret_cast<float2*>(ssm);
    const uint32_t dim = 1u << n;
    float* P = reinterpret_cast<float*>(st + dim);  // 3 planes of up to 64 x 64
    float* S = P + 4096;
    float* Q = S + 4096;
    for (uint32_t i = threadIdx.x; i < dim; i += blockDim.x) st[i] = psi[i];
    for (int gi = 0; gi < ngates; ++gi) {
        const SmallGateDesc g = gates[gi];
        const int k = g.k, D = 1 << k;
        const float2* m = mats + g.mat_off;
        __syncthreads();  // previous gate done with the planes and the state
        for (int e = threadIdx.x; e < D * D; e += blockDim.x) {
            const float2 v = m[e];
            P[e] = v.x;
            S[e] = v.x + v.y;
            Q[e] = v.y - v.x;
        }
        __syncthreads();
        switch (k) {
            case 1: small_gate<1>(st, n, g.q, P, S, Q); break;
            case 2: small_gate<2>(st, n, g.q, P, S, Q); break;
            case 3: small_gate<3>(st, n, g.q, P, S, Q); break;
            case 4: small_gate<4>(st, n, g.q, P, S, Q); break;
            case 5: small_gate<5>(st, n, g.q, P, S, Q); break;
            default: small_gate<6>(st, n, g.q, P, S, Q); break;
        }
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < dim; i += blockDim.x) psi[i] = st[i];
}

}  // namespace

size_t small_circuit_smem(int n) { return ((size_t)8 << n) + 3 * 4096 * sizeof(float); }

cudaError_t launch_small_circuit(float2* psi, int n, int ngates, const SmallGateDesc* gates_dev,
                                 const float2* mats_dev, cudaStream_t st) {
    const size_t smem = small_circuit_smem(n);
    cudaError_t e = cudaFuncSetAttribute(small_circuit_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    small_circuit_kernel<<<1, kSmallThreads, smem, st>>>(psi, n, ngates, gates_dev, mats_dev);
    return cudaGetLastError();
}

}  // namespace svb
