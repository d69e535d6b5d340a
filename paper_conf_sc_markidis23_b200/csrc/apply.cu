// apply.cu -- the hot path: in-place application of one fused k-qubit gate
// (k = 1..6) to a complex64 state shard.
//
// What is computed (§2.2, Figs. 3-4): for each of the
// 2^(n-k) groups -- base index with zero bits at the gate's qubits -- gather
// a_c = psi[base | sum_b c_b 2^{q_b}], compute y = M a (2^k x 2^k complex
// matvec, fp32 FMA) and scatter y back in place.  Per amplitude the
// algorithmic cost is 16 B of HBM traffic and 8*2^k - 2 flop (L82: "14 FLOPs
// and 16 B" for k = 1).
//
// Two kernel classes, as in the paper's design (L110-112: ApplyGateH /
// ApplyGateL), both built on one B200 tile engine:
//  * a persistent CTA streams "tiles" -- the 2^|H| contiguous runs of 2^r
//    amplitudes (H = gate qubits >= r) that together hold complete groups --
//    from HBM into shared memory with 16 B cp.async copies (no register
//    staging, so every copy of a tile is in flight at once), double-buffered
//    so the next tile loads while the current one is transformed;
//  * the groups are transformed in place in shared memory (L94-96: "temporary
//    arrays ... in shared memory"), then streamed back with 16 B stores;
//  * apply_high: no gate qubit in {1,2,3}; runs are whole 128 B lines and no
//    swizzle is needed.  apply_low: a gate qubit in {1,2,3} puts partners
//    inside one 128 B line; a per-gate XOR swizzle of the shared-memory
//    layout keeps the group gathers bank-conflict free.
// The fused matrix (k <= 5) travels in the kernel parameters
// (__grid_constant__), so the unrolled FMAs read it from the constant bank;
// k = 6 (32 KB) is staged in shared memory once per CTA.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "kernels.h"

namespace svb {

namespace {

constexpr int kThreads = 256;

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

// y += m * a (complex), 4 FFMA.
__device__ __forceinline__ void cmac(float2& y, const float2 m, const float2 a) {
    y.x = fmaf(m.x, a.x, y.x);
    y.x = fmaf(-m.y, a.y, y.x);
    y.y = fmaf(m.x, a.y, y.y);
    y.y = fmaf(m.y, a.x, y.y);
}

template <int K>
struct MatStore {
    float2 m[1 << K][1 << K];
};
template <>
struct MatStore<6> {  // 32 KB: does not fit the 32764 B parameter space
    const float2* dev;
};

template <int K>
__device__ __forceinline__ float2 mat_elem(const MatStore<K>& M, const float2* sm, int r, int c) {
    return M.m[r][c];
}
template <>
__device__ __forceinline__ float2 mat_elem<6>(const MatStore<6>&, const float2* sm, int r, int c) {
    return sm[r * 64 + c];
}

// Rows unrolled fully for k <= 4 (matrix from the constant bank as FFMA
// operands); k = 5/6 loop over rows to bound code size.
template <int K>
struct RowUnroll {
    static constexpr int value = (K <= 4) ? (1 << K) : 1;
    static constexpr int half = (K <= 4) ? (1 << (K - 1)) : 1;
};

// ------------------------------------------------------------------ kernels
// One tile per CTA iteration: the 2^nH runs of 2^r contiguous amplitudes that
// share every bit outside {0..r-1} u H (H = gate qubits >= r).  The tile holds
// complete groups, so the gate is applied entirely inside shared memory.
template <int K>
struct TileParams {
    float2* psi;
    uint64_t n_tiles;
    int T, r;                          // tile bits, run bits
    int nH;
    int Hpos[SV_MAX_FUSED];            // gate qubits >= r (ascending, global positions)
    uint64_t offH[1 << SV_MAX_FUSED];  // amplitude offset of run h (deposit of h into Hpos)
    int nzt;
    int ztpos[SV_MAX_FUSED];           // tile-local gate bit positions, ascending
    uint32_t swz[3];                   // phys bit (i+1) ^= parity(t & swz[i])
    uint32_t loc[1 << K];              // swizzled tile offsets of the gathers
    MatStore<K> M;
};

__device__ __forceinline__ uint32_t swizzle(uint32_t t, const uint32_t* swz) {
    return t ^ ((__popc(t & swz[0]) & 1) << 1) ^ ((__popc(t & swz[1]) & 1) << 2) ^ ((__popc(t & swz[2]) & 1) << 3);
}

__device__ __forceinline__ void cp_async16(uint32_t saddr, const void* g) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(saddr), "l"(g) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }

constexpr int kStages = 2;

// Issue the asynchronous global->shared copies of tile u (16 B per lane,
// swizzled destination; consecutive lanes read consecutive 16 B of a run).
template <int K>
__device__ __forceinline__ void tile_load(const TileParams<K>& p, uint64_t u, uint32_t sbuf) {
    const uint64_t tbase = insert_zeros(u << p.r, p.Hpos, p.nH);
    const uint32_t units = 1u << (p.T - 1);
    const uint32_t rmask = (1u << p.r) - 1u;
    for (uint32_t v = threadIdx.x; v < units; v += blockDim.x) {
        const uint32_t t = v << 1;
        const uint64_t g = tbase + p.offH[t >> p.r] + (t & rmask);
        cp_async16(sbuf + (swizzle(t, p.swz) << 3), p.psi + g);
    }
}

template <int K>
__device__ __forceinline__ void tile_store(const TileParams<K>& p, uint64_t u, uint32_t sbuf) {
    const uint64_t tbase = insert_zeros(u << p.r, p.Hpos, p.nH);
    const uint32_t units = 1u << (p.T - 1);
    const uint32_t rmask = (1u << p.r) - 1u;
    for (uint32_t v = threadIdx.x; v < units; v += blockDim.x) {
        const uint32_t t = v << 1;
        const uint64_t g = tbase + p.offH[t >> p.r] + (t & rmask);
        st_stream(reinterpret_cast<float4*>(p.psi + g), lds4(sbuf + (swizzle(t, p.swz) << 3)));
    }
}

// y = M a for every group of the tile, in place in shared memory.
// PAIR: qubit 0 is a gate qubit -> 16 B gathers hold members 2j, 2j+1.
template <int K, bool PAIR>
__device__ __forceinline__ void tile_compute(const TileParams<K>& p, uint32_t sbuf, const float2* sm) {
    constexpr int D = 1 << K;
    const uint32_t ngroups = 1u << (p.T - K);
    for (uint32_t gidx = threadIdx.x; gidx < ngroups; gidx += blockDim.x) {
        const uint32_t bt = (uint32_t)insert_zeros(gidx, p.ztpos, p.nzt);
        const uint32_t pb = swizzle(bt, p.swz);
        if constexpr (PAIR) {
            float4 v[D / 2];
#pragma unroll
            for (int j = 0; j < D / 2; ++j) v[j] = lds4(sbuf + ((pb ^ p.loc[j]) << 3));
#pragma unroll RowUnroll<K>::half
            for (int r2 = 0; r2 < D / 2; ++r2) {
                float2 y0 = make_float2(0.f, 0.f), y1 = make_float2(0.f, 0.f);
#pragma unroll
                for (int c = 0; c < D; ++c) {
                    const float2 a = (c & 1) ? make_float2(v[c >> 1].z, v[c >> 1].w)
                                             : make_float2(v[c >> 1].x, v[c >> 1].y);
                    cmac(y0, mat_elem<K>(p.M, sm, 2 * r2, c), a);
                    cmac(y1, mat_elem<K>(p.M, sm, 2 * r2 + 1, c), a);
                }
                sts4(sbuf + ((pb ^ p.loc[r2]) << 3), make_float4(y0.x, y0.y, y1.x, y1.y));
            }
        } else {
            float2 v[D];
#pragma unroll
            for (int j = 0; j < D; ++j) v[j] = lds2(sbuf + ((pb ^ p.loc[j]) << 3));
#pragma unroll RowUnroll<K>::value
            for (int r = 0; r < D; ++r) {
                float2 y = make_float2(0.f, 0.f);
#pragma unroll
                for (int c = 0; c < D; ++c) cmac(y, mat_elem<K>(p.M, sm, r, c), v[c]);
                sts2(sbuf + ((pb ^ p.loc[r]) << 3), y);
            }
        }
    }
}

// Persistent, double-buffered: the copies of tile i+1 are in flight while
// tile i is transformed and written back.
template <int K, bool PAIR>
__device__ __forceinline__ void tile_loop(const TileParams<K>& p) {
    extern __shared__ float4 dsm[];
    const uint32_t tile_bytes = 8u << p.T;
    const uint32_t s0 = smem_addr(dsm);
    const float2* sm = nullptr;
    if constexpr (K == 6) {
        float2* smat = reinterpret_cast<float2*>(reinterpret_cast<char*>(dsm) + kStages * tile_bytes);
        for (int i = threadIdx.x; i < 64 * 64; i += blockDim.x) smat[i] = p.M.dev[i];
        sm = smat;
        __syncthreads();
    }
    uint64_t u = blockIdx.x;
    if (u < p.n_tiles) tile_load<K>(p, u, s0);
    cp_async_commit();
    for (int it = 0; u < p.n_tiles; u += gridDim.x, ++it) {
        const uint32_t cur = s0 + (uint32_t)(it & 1) * tile_bytes;
        const uint32_t nxt = s0 + (uint32_t)((it + 1) & 1) * tile_bytes;
        const uint64_t un = u + gridDim.x;
        __syncthreads();  // buffer `nxt` was drained by the previous iteration's store
        if (un < p.n_tiles) tile_load<K>(p, un, nxt);
        cp_async_commit();
        cp_async_wait1();  // this thread's copies of tile u have landed
        __syncthreads();   // ... and everyone else's
        tile_compute<K, PAIR>(p, cur, sm);
        __syncthreads();
        tile_store<K>(p, u, cur);
    }
}

// The paper's two kernel classes (L110-112).  Same tile engine; "high" gates
// (no qubit in {1,2,3}) need no swizzle and have runs of >= 16 amplitudes
// per member, "low" gates carry their partners inside a 128 B line.
template <int K, bool PAIR>
__global__ void __launch_bounds__(kThreads) apply_high(const __grid_constant__ TileParams<K> p) {
    tile_loop<K, PAIR>(p);
}
template <int K, bool PAIR>
__global__ void __launch_bounds__(kThreads) apply_low(const __grid_constant__ TileParams<K> p) {
    tile_loop<K, PAIR>(p);
}

int g_num_sms = 0;
int num_sms() {
    if (g_num_sms == 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
        if (g_num_sms <= 0) g_num_sms = 148;
    }
    return g_num_sms;
}

template <int K>
void fill_matrix(MatStore<K>& M, const ApplyDesc& d) {
    std::memcpy(M.m, d.m.data(), sizeof(M.m));
}
template <>
void fill_matrix<6>(MatStore<6>& M, const ApplyDesc& d) {
    M.dev = d.dev_m;
}

template <int K>
cudaError_t launch_tile_k(float2* psi, int n, const ApplyDesc& d, cudaStream_t st) {
    TileParams<K> p;
    std::memset(&p, 0, sizeof(p));
    p.psi = psi;
    fill_matrix<K>(p.M, d);
    p.T = d.T;
    p.r = d.r;
    const bool pair = d.q[0] == 0;
    // tile-local gate positions
    int tl[SV_MAX_FUSED];
    for (int b = 0; b < K; ++b) {
        if (d.q[b] < p.r) {
            tl[b] = d.q[b];
        } else {
            tl[b] = p.r + p.nH;
            p.Hpos[p.nH++] = d.q[b];
        }
    }
    for (int h = 0; h < (1 << p.nH); ++h) {
        uint64_t o = 0;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1) o |= 1ull << p.Hpos[b];
        p.offH[h] = o;
    }
    p.nzt = K;
    for (int b = 0; b < K; ++b) p.ztpos[b] = tl[b];
    // swizzle: the lanes of one shared-memory phase run over the lowest W
    // non-gate tile bits; each gate bit f in {1,2,3} (fixed within a gather)
    // is XORed with one of those lane bits >= 4, so the W lanes hit W distinct
    // 8/16 B bank slots.  Linear over GF(2), so phys(base ^ off) = phys(base) ^ phys(off).
    uint32_t gmask = 0;
    for (int b = 0; b < K; ++b) gmask |= 1u << tl[b];
    const int W = pair ? 3 : 4;
    int hl[8], nhl = 0, nl = 0;
    for (int t = 0; t < p.T && nl < W; ++t)
        if (!((gmask >> t) & 1)) {
            ++nl;
            if (t >= 4) hl[nhl++] = t;
        }
    int j = 0;
    for (int f = 1; f <= 3; ++f)
        if (((gmask >> f) & 1) && j < nhl) p.swz[f - 1] = 1u << hl[j++];
    auto sw = [&](uint32_t t) {
        return t ^ ((__builtin_popcount(t & p.swz[0]) & 1) << 1) ^ ((__builtin_popcount(t & p.swz[1]) & 1) << 2) ^
               ((__builtin_popcount(t & p.swz[2]) & 1) << 3);
    };
    const int ng = pair ? (1 << (K - 1)) : (1 << K);
    for (int m = 0; m < ng; ++m) {
        const int mm = pair ? (m << 1) : m;
        uint32_t o = 0;
        for (int b = 0; b < K; ++b)
            if ((mm >> b) & 1) o |= 1u << tl[b];
        p.loc[m] = sw(o);
    }
    p.n_tiles = 1ull << (n - p.T);
    size_t smem = (size_t)kStages * ((size_t)8 << p.T);
    if (K == 6) smem += 64 * 64 * 8;
    const int per_sm = std::max(1, (int)((220 * 1024) / (smem + 1024)));
    const uint64_t grid = std::max<uint64_t>(1, std::min<uint64_t>(p.n_tiles, (uint64_t)num_sms() * per_sm));
    auto go = [&](auto kern) -> cudaError_t {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        kern<<<(unsigned)grid, kThreads, smem, st>>>(p);
        return cudaGetLastError();
    };
    if (d.high) return pair ? go(apply_high<K, true>) : go(apply_high<K, false>);
    return pair ? go(apply_low<K, true>) : go(apply_low<K, false>);
}

}  // namespace

void plan_apply(int n, ApplyDesc& d) {
    uint64_t gm = 0;
    for (int b = 0; b < d.k; ++b) gm |= 1ull << d.q[b];
    d.high = (gm & kLowMask) == 0;
    // tile: runs of >= 16 amplitudes (128 B); grow the run until the tile
    // reaches the target size (32 KB for k <= 4).
    const int target = std::min(n, d.k <= 4 ? 12 : 13);
    auto tile_bits = [&](int rr) {
        int t = rr;
        for (int b = 0; b < d.k; ++b)
            if (d.q[b] >= rr) ++t;
        return t;
    };
    int r = std::min(n, 4);
    while (r < n && tile_bits(r) < target) ++r;
    d.r = r;
    d.T = tile_bits(r);
}

cudaError_t launch_apply(float2* psi, int n, const ApplyDesc& d, cudaStream_t st) {
    switch (d.k) {
        case 1: return launch_tile_k<1>(psi, n, d, st);
        case 2: return launch_tile_k<2>(psi, n, d, st);
        case 3: return launch_tile_k<3>(psi, n, d, st);
        case 4: return launch_tile_k<4>(psi, n, d, st);
        case 5: return launch_tile_k<5>(psi, n, d, st);
        case 6: return launch_tile_k<6>(psi, n, d, st);
    }
    return cudaErrorInvalidValue;
}

}  // namespace svb
