// blocked.cu -- cache-blocked multi-gate passes.
//
// Related work [12] applies several gates per memory pass;
// the paper's own smem remedy (L94-96) keeps a block of the state on chip.
// A pass loads a tile -- the 2^T amplitudes that share every bit outside a
// qubit set S (|S| = T, S contains the low qubits 0..4 so runs stay >= 256 B)
// -- into shared memory, applies EVERY fused gate of the pass (all their
// qubits are in S) one after another inside the tile, and writes it back:
// one HBM read + write for many gates.  The sequence of qubit sets comes from
// the S4 planner run with "local" = the tile's T slots (planner.cpp); a
// "remap" is only a change of S for the next pass -- the state never moves.
// Per gate the group transform is the one of apply.cu (gather the 2^k
// members, Gauss 3-multiplication y = M a, scatter).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "device_util.cuh"
#include "kernels.h"

namespace svb {

namespace {

using namespace dev;

constexpr int kPassThreads = 256;

struct alignas(16) PassParams {
    float planes[kPassPlaneFloats];  // Gauss planes P, S, Q of every gate (first: 16 B aligned)
    float2* psi;
    uint64_t n_tiles;
    int T, r, nH;
    int Hpos[32];
    int upt;
    uint64_t goff[64];
    uint32_t soff[64];
    uint32_t swz[3];
    int ngates;
    PassGate gates[kPassMaxGates];
};

template <int K>
__device__ __forceinline__ uint32_t ins_zeros_k(uint32_t x, const int* pos) {
#pragma unroll
    for (int b = 0; b < K; ++b) {
        const int q = pos[b];
        x = ((x >> q) << (q + 1)) | (x & ((1u << q) - 1u));
    }
    return x;
}

// One gate on the tile, two groups per thread (like apply.cu's GPT = 2):
//  * tile bit 0 not a gate bit: a 16 B word holds the same member of the
//    neighbouring groups (t, t+1);
//  * tile bit 0 a gate bit (PAIR): a 16 B word holds members 2j, 2j+1 of one
//    group and the thread's second group differs in the lowest non-gate bit.
// Gauss 3-multiplication rows; matrix planes are warp-uniform constant-bank
// loads.  The pass swizzle (bits 1..3 ^= bits 4..6) keeps bit 0 in place.
template <int K, bool PAIR>
__device__ __forceinline__ void pass_gate(uint32_t sbuf, int T, const PassGate& g, const float* planes,
                                          const uint32_t* swz) {
    constexpr int D = 1 << K;
    const float* P = planes + g.poff;
    const float* S = P + D * D;
    const float* Q = S + D * D;
    int zpos[K];
#pragma unroll
    for (int b = 0; b < K; ++b) zpos[b] = g.pos[b];
    constexpr int NL = PAIR ? D / 2 : D;
    uint32_t loc[NL];
#pragma unroll
    for (int m = 0; m < NL; ++m) {
        const int mm = PAIR ? 2 * m : m;
        uint32_t o = 0;
#pragma unroll
        for (int b = 0; b < K; ++b)
            if ((mm >> b) & 1) o |= 1u << zpos[b];
        loc[m] = swizzle(o, swz);
    }
    // PAIR: the second group sets the lowest non-gate tile bit
    uint32_t sec = 0;
    if (PAIR) {
        uint32_t gm = 0;
#pragma unroll
        for (int b = 0; b < K; ++b) gm |= 1u << zpos[b];
        sec = swizzle((~gm) & (gm + 1), swz);  // lowest zero bit of the gate mask
    }
    const uint32_t npairs = 1u << (T - K - 1);
    for (uint32_t gi = threadIdx.x; gi < npairs; gi += blockDim.x) {
        const uint32_t pb = swizzle(ins_zeros_k<K>(gi << 1, zpos), swz);
        float2 a0[D], a1[D];
        if constexpr (PAIR) {
#pragma unroll
            for (int j = 0; j < D / 2; ++j) {
                const float4 v0 = lds4(sbuf + ((pb ^ loc[j]) << 3));
                const float4 v1 = lds4(sbuf + ((pb ^ sec ^ loc[j]) << 3));
                a0[2 * j] = make_float2(v0.x, v0.y);
                a0[2 * j + 1] = make_float2(v0.z, v0.w);
                a1[2 * j] = make_float2(v1.x, v1.y);
                a1[2 * j + 1] = make_float2(v1.z, v1.w);
            }
        } else {
#pragma unroll
            for (int c = 0; c < D; ++c) {
                const float4 v = lds4(sbuf + ((pb ^ loc[c]) << 3));
                a0[c] = make_float2(v.x, v.y);
                a1[c] = make_float2(v.z, v.w);
            }
        }
        float s0[D], s1[D];
#pragma unroll
        for (int c = 0; c < D; ++c) {
            s0[c] = a0[c].x + a0[c].y;
            s1[c] = a1[c].x + a1[c].y;
        }
#pragma unroll 1
        for (int r = 0; r < D; r += (PAIR ? 2 : 1)) {
            float2 y0[2], y1[2];
#pragma unroll
            for (int i = 0; i < (PAIR ? 2 : 1); ++i) {
                float A0 = 0.f, B0 = 0.f, C0 = 0.f, A1 = 0.f, B1 = 0.f, C1 = 0.f;
#pragma unroll
                for (int c = 0; c < D; ++c) {
                    const float pp = P[(r + i) * D + c], ss = S[(r + i) * D + c], qq = Q[(r + i) * D + c];
                    A0 = fmaf(pp, s0[c], A0);
                    A1 = fmaf(pp, s1[c], A1);
                    B0 = fmaf(ss, a0[c].y, B0);
                    B1 = fmaf(ss, a1[c].y, B1);
                    C0 = fmaf(qq, a0[c].x, C0);
                    C1 = fmaf(qq, a1[c].x, C1);
                }
                y0[i] = make_float2(A0 - B0, A0 + C0);
                y1[i] = make_float2(A1 - B1, A1 + C1);
            }
            if constexpr (PAIR) {
                sts4(sbuf + ((pb ^ loc[r >> 1]) << 3), make_float4(y0[0].x, y0[0].y, y0[1].x, y0[1].y));
                sts4(sbuf + ((pb ^ sec ^ loc[r >> 1]) << 3), make_float4(y1[0].x, y1[0].y, y1[1].x, y1[1].y));
            } else {
                sts4(sbuf + ((pb ^ loc[r]) << 3), make_float4(y0[0].x, y0[0].y, y1[0].x, y1[0].y));
            }
        }
    }
}

__global__ void __launch_bounds__(kPassThreads) apply_pass(const __grid_constant__ PassParams p) {
    extern __shared__ float4 bsm[];
    const uint32_t tile_bytes = 8u << p.T;
    const uint32_t s0 = smem_addr(bsm);
    const uint32_t t0 = 2u * threadIdx.x;
    const uint32_t rmask = (1u << p.r) - 1u;
    uint64_t dthr = t0 & rmask;
    {
        const uint32_t h = t0 >> p.r;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1u) dthr += 1ull << p.Hpos[b];
    }
    const uint32_t sthr = swizzle(t0, p.swz);
    auto tbase = [&](uint64_t u) {
        // insert zeros at the H positions (ascending) into u << r
        uint64_t x = u << p.r;
        for (int b = 0; b < p.nH; ++b) {
            const int q = p.Hpos[b];
            x = ((x >> q) << (q + 1)) | (x & ((1ull << q) - 1ull));
        }
        return x;
    };
    auto load = [&](uint64_t u, uint32_t sbuf) {
        const float2* g = p.psi + tbase(u) + dthr;
        for (int i = 0; i < p.upt; ++i) cp_async16(sbuf + ((sthr ^ p.soff[i]) << 3), g + p.goff[i]);
    };
    auto store = [&](uint64_t u, uint32_t sbuf) {
        float2* g = p.psi + tbase(u) + dthr;
        for (int i = 0; i < p.upt; ++i)
            st_stream(reinterpret_cast<float4*>(g + p.goff[i]), lds4(sbuf + ((sthr ^ p.soff[i]) << 3)));
    };
    uint64_t u = blockIdx.x;
    if (u < p.n_tiles) load(u, s0);
    cp_async_commit();
    for (int it = 0; u < p.n_tiles; u += gridDim.x, ++it) {
        const uint32_t cur = s0 + (uint32_t)(it & 1) * tile_bytes;
        const uint32_t nxt = s0 + (uint32_t)((it + 1) & 1) * tile_bytes;
        const uint64_t un = u + gridDim.x;
        __syncthreads();
        if (un < p.n_tiles) load(un, nxt);
        cp_async_commit();
        cp_async_wait1();
        __syncthreads();
        for (int gi = 0; gi < p.ngates; ++gi) {
            const PassGate& g = p.gates[gi];
            const bool pair = g.pos[0] == 0;
            switch (g.k * 2 + (pair ? 1 : 0)) {
                case 2: pass_gate<1, false>(cur, p.T, g, p.planes, p.swz); break;
                case 3: pass_gate<1, true>(cur, p.T, g, p.planes, p.swz); break;
                case 4: pass_gate<2, false>(cur, p.T, g, p.planes, p.swz); break;
                case 5: pass_gate<2, true>(cur, p.T, g, p.planes, p.swz); break;
                case 6: pass_gate<3, false>(cur, p.T, g, p.planes, p.swz); break;
                case 7: pass_gate<3, true>(cur, p.T, g, p.planes, p.swz); break;
                case 8: pass_gate<4, false>(cur, p.T, g, p.planes, p.swz); break;
                default: pass_gate<4, true>(cur, p.T, g, p.planes, p.swz); break;
            }
            __syncthreads();
        }
        store(u, cur);
    }
}

int pass_sms() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

}  // namespace

void plan_pass_tile(PassDesc& pd) {
    // S ascending; runs = longest prefix {0..r-1}
    std::sort(pd.S.begin(), pd.S.end());
    int r = 0;
    while (r < (int)pd.S.size() && pd.S[r] == r) ++r;
    pd.r = r;
}

cudaError_t launch_pass(float2* psi, int n, const PassDesc& pd, cudaStream_t st) {
    static_assert(sizeof(PassParams) <= 32764, "pass params exceed the kernel parameter space");
    PassParams* pp = new PassParams;  // large: keep off the host stack
    PassParams& p = *pp;
    std::memset(&p, 0, sizeof(p));
    const int T = (int)pd.S.size();
    p.psi = psi;
    p.T = T;
    p.r = pd.r;
    p.nH = 0;
    for (int i = pd.r; i < T; ++i) p.Hpos[p.nH++] = pd.S[i];
    // bank swizzle: bits 1..3 ^= bits 4..6 (fixed per pass; T >= 7)
    p.swz[0] = 1u << 4;
    p.swz[1] = 1u << 5;
    p.swz[2] = 1u << 6;
    auto sw = [&](uint32_t t) {
        return t ^ ((__builtin_popcount(t & p.swz[0]) & 1) << 1) ^ ((__builtin_popcount(t & p.swz[1]) & 1) << 2) ^
               ((__builtin_popcount(t & p.swz[2]) & 1) << 3);
    };
    auto dep = [&](uint64_t t) {
        uint64_t g = t & ((1ull << p.r) - 1);
        const uint64_t h = t >> p.r;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1) g += 1ull << p.Hpos[b];
        return g;
    };
    const uint32_t units = 1u << (T - 1);
    const uint32_t nthr = std::min<uint32_t>(kPassThreads, units);
    p.upt = (int)(units / nthr);
    for (int i = 0; i < p.upt; ++i) {
        p.goff[i] = dep(2ull * nthr * i);
        p.soff[i] = sw(2u * nthr * i);
    }
    p.ngates = (int)pd.gates.size();
    for (int i = 0; i < p.ngates; ++i) p.gates[i] = pd.gates[i];
    std::memcpy(p.planes, pd.planes.data(), pd.planes.size() * sizeof(float));
    p.n_tiles = 1ull << (n - T);
    const size_t smem = 2 * ((size_t)8 << T);
    cudaError_t e = cudaFuncSetAttribute(apply_pass, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) {
        const int per_sm = std::max(1, (int)((227 * 1024) / (smem + 1024)));
        const uint64_t grid = std::min<uint64_t>(p.n_tiles, (uint64_t)pass_sms() * per_sm);
        apply_pass<<<(unsigned)grid, nthr, smem, st>>>(p);
        e = cudaGetLastError();
    }
    delete pp;
    return e;
}

}  // namespace svb
