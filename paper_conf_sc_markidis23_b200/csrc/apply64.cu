// apply64.cu -- complex128 (fp64) state kernels.
//
// PAPER.md L191 (§5, Fig. 8): qsim compiled for double precision is 1.8-2x
// slower than single precision with no substantial state differences.  The
// same method at 16 B per amplitude: the fused-gate apply (
// 16 -> 32 B of HBM traffic and 8*2^k - 2 fp64 flop per amplitude), |0..0>
// init, amplitude gather and the sampler's fixed-point weights.
//
// Apply: the tile engine of apply.cu with 16 B amplitudes -- persistent CTAs
// stream tiles of 2^11 amplitudes (32 KB: 2^|H| runs of >= 8 amplitudes) with
// cp.async, double-buffered; one group per thread is gathered from shared
// memory (per-gate XOR swizzle of amplitude bits 0..2 keeps the 8-lane LDS.128
// phases conflict-free), transformed with the Gauss 3-multiplication form in
// fp64 and scattered back.  Matrix planes travel in the kernel parameters.
// k = 6 (apply64_k6_kernel): a group's 64 inputs do not fit in registers, so
// the 8 warps of a CTA split the 64 output rows (8 each) of the 32 groups of
// a 2^11-amplitude tile (lane = group), read the inputs from the shared-memory
// tile and the (transposed) planes from shared memory (warp-wide broadcasts),
// and write the outputs to a second tile buffer that is then stored.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "device_util.cuh"
#include "kernels.h"

namespace svb {

namespace {

using namespace dev;

constexpr int kT64 = 11;  // tile bits (2^11 x 16 B = 32 KB)

template <int K>
struct Mat64 {
    alignas(16) double P[1 << K][1 << K];
    alignas(16) double S[1 << K][1 << K];
    alignas(16) double Q[1 << K][1 << K];
};
template <>
struct Mat64<6> {
    const double* dev;  // planes P, S, Q (3 x 4096 doubles)
};

template <int K>
struct alignas(16) Tile64Params {
    Mat64<K> M;
    double2* psi;
    uint64_t n_tiles;
    int T, r, nH;
    int Hpos[SV_MAX_FUSED];
    int nzt;
    int ztpos[SV_MAX_FUSED];
    uint32_t swz[3];  // phys bit i ^= parity(t & swz[i]), i = 0..2
    int upt;
    uint64_t goff[64];
    uint32_t soff[64];
    uint32_t loc[1 << K];
};

__device__ __forceinline__ uint32_t swz64(uint32_t t, const uint32_t* s) {
    return t ^ (__popc(t & s[0]) & 1) ^ ((__popc(t & s[1]) & 1) << 1) ^ ((__popc(t & s[2]) & 1) << 2);
}
__device__ __forceinline__ double2 ldsd(uint32_t a) {
    double2 v;
    asm volatile("ld.shared.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(a));
    return v;
}
__device__ __forceinline__ void stsd(uint32_t a, double2 v) {
    asm volatile("st.shared.v2.f64 [%0], {%1,%2};" ::"r"(a), "d"(v.x), "d"(v.y) : "memory");
}
__device__ __forceinline__ void stgd(double2* p, double2 v) {
    asm volatile("st.global.cs.v2.f64 [%0], {%1,%2};" ::"l"(p), "d"(v.x), "d"(v.y) : "memory");
}

template <int K>
__device__ __forceinline__ double mP(const Mat64<K>& M, const double*, int r, int c) { return M.P[r][c]; }
template <int K>
__device__ __forceinline__ double mS(const Mat64<K>& M, const double*, int r, int c) { return M.S[r][c]; }
template <int K>
__device__ __forceinline__ double mQ(const Mat64<K>& M, const double*, int r, int c) { return M.Q[r][c]; }
template <>
__device__ __forceinline__ double mP<6>(const Mat64<6>&, const double* sm, int r, int c) { return sm[r * 64 + c]; }
template <>
__device__ __forceinline__ double mS<6>(const Mat64<6>&, const double* sm, int r, int c) { return sm[4096 + r * 64 + c]; }
template <>
__device__ __forceinline__ double mQ<6>(const Mat64<6>&, const double* sm, int r, int c) { return sm[8192 + r * 64 + c]; }

template <int K>
__global__ void __launch_bounds__(256) apply64_kernel(const __grid_constant__ Tile64Params<K> p) {
    constexpr int D = 1 << K;
    constexpr int STAGES = (K == 6) ? 1 : 2;
    extern __shared__ double2 dsm64[];
    const uint32_t tile_bytes = 16u << p.T;
    const uint32_t s0 = smem_addr(dsm64);
    const double* sm = nullptr;
    if constexpr (K == 6) {
        double* m = reinterpret_cast<double*>(reinterpret_cast<char*>(dsm64) + STAGES * tile_bytes);
        for (int i = threadIdx.x; i < 3 * 4096; i += blockDim.x) m[i] = p.M.dev[i];
        sm = m;
        __syncthreads();
    }
    const uint32_t t0 = threadIdx.x;
    const uint32_t rmask = (1u << p.r) - 1u;
    uint64_t dthr = t0 & rmask;
    {
        const uint32_t h = t0 >> p.r;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1u) dthr += 1ull << p.Hpos[b];
    }
    const uint32_t sthr = swz64(t0, p.swz);
    auto load = [&](uint64_t u, uint32_t sbuf) {
        const double2* g = p.psi + insert_zeros(u << p.r, p.Hpos, p.nH) + dthr;
        for (int i = 0; i < p.upt; ++i) cp_async16(sbuf + ((sthr ^ p.soff[i]) << 4), g + p.goff[i]);
    };
    auto store = [&](uint64_t u, uint32_t sbuf) {
        double2* g = p.psi + insert_zeros(u << p.r, p.Hpos, p.nH) + dthr;
        for (int i = 0; i < p.upt; ++i) stgd(g + p.goff[i], ldsd(sbuf + ((sthr ^ p.soff[i]) << 4)));
    };
    auto compute = [&](uint32_t sbuf) {
        const uint32_t ngroups = 1u << (p.T - K);
        for (uint32_t gi = threadIdx.x; gi < ngroups; gi += blockDim.x) {
            const uint32_t pb = swz64((uint32_t)insert_zeros(gi, p.ztpos, p.nzt), p.swz);
            double2 a[D];
            double s[D];
#pragma unroll
            for (int c = 0; c < D; ++c) {
                a[c] = ldsd(sbuf + ((pb ^ p.loc[c]) << 4));
                s[c] = a[c].x + a[c].y;
            }
#pragma unroll 1
            for (int r = 0; r < D; ++r) {
                double A = 0.0, B = 0.0, C = 0.0;
#pragma unroll
                for (int c = 0; c < D; ++c) {
                    A = fma(mP<K>(p.M, sm, r, c), s[c], A);
                    B = fma(mS<K>(p.M, sm, r, c), a[c].y, B);
                    C = fma(mQ<K>(p.M, sm, r, c), a[c].x, C);
                }
                stsd(sbuf + ((pb ^ p.loc[r]) << 4), make_double2(A - B, A + C));
            }
        }
    };
    uint64_t u = blockIdx.x;
    if constexpr (STAGES == 2) {
        if (u < p.n_tiles) load(u, s0);
        cp_async_commit();
        for (int it = 0; u < p.n_tiles; u += gridDim.x, ++it) {
            const uint32_t cur = s0 + (uint32_t)(it & 1) * tile_bytes;
            const uint32_t nxt = s0 + (uint32_t)((it + 1) & 1) * tile_bytes;
            __syncthreads();
            if (u + gridDim.x < p.n_tiles) load(u + gridDim.x, nxt);
            cp_async_commit();
            cp_async_wait1();
            __syncthreads();
            compute(cur);
            __syncthreads();
            store(u, cur);
        }
    } else {
        for (; u < p.n_tiles; u += gridDim.x) {
            __syncthreads();
            load(u, s0);
            cp_async_commit();
            cp_async_wait0();
            __syncthreads();
            compute(s0);
            __syncthreads();
            store(u, s0);
        }
    }
}

__global__ void __launch_bounds__(256) apply64_k6_kernel(const __grid_constant__ Tile64Params<6> p) {
    extern __shared__ double2 dsm64[];
    const uint32_t tile_bytes = 16u << p.T;
    const uint32_t s_in = smem_addr(dsm64), s_out = s_in + tile_bytes;
    // planes transposed: pl[(plane * 64 + c) * 64 + r]
    double* pl = reinterpret_cast<double*>(reinterpret_cast<char*>(dsm64) + 2 * tile_bytes);
    for (int i = threadIdx.x; i < 3 * 4096; i += blockDim.x) {
        const int plane = i >> 12, r = (i >> 6) & 63, c = i & 63;
        pl[(plane * 64 + c) * 64 + r] = p.M.dev[i];
    }
    __syncthreads();
    const uint32_t t0 = threadIdx.x;
    const uint32_t rmask = (1u << p.r) - 1u;
    uint64_t dthr = t0 & rmask;
    {
        const uint32_t h = t0 >> p.r;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1u) dthr += 1ull << p.Hpos[b];
    }
    const uint32_t sthr = swz64(t0, p.swz);
    const uint32_t g = threadIdx.x & 31u, r0 = (threadIdx.x >> 5) * 8u;  // lane = group, warp = 8 rows
    const uint32_t pb = swz64((uint32_t)insert_zeros(g, p.ztpos, p.nzt), p.swz);
    uint64_t u = blockIdx.x;
    if (u < p.n_tiles) {
        const double2* gp = p.psi + insert_zeros(u << p.r, p.Hpos, p.nH) + dthr;
        for (int i = 0; i < p.upt; ++i) cp_async16(s_in + ((sthr ^ p.soff[i]) << 4), gp + p.goff[i]);
    }
    cp_async_commit();
    for (; u < p.n_tiles; u += gridDim.x) {
        cp_async_wait0();
        __syncthreads();
        double A[8], B[8], C[8];
#pragma unroll
        for (int rr = 0; rr < 8; ++rr) A[rr] = B[rr] = C[rr] = 0.0;
#pragma unroll 2
        for (int c = 0; c < 64; ++c) {
            const double2 a = ldsd(s_in + ((pb ^ p.loc[c]) << 4));
            const double sc = a.x + a.y;
            const double2* P = reinterpret_cast<const double2*>(pl + (0 * 64 + c) * 64 + r0);
            const double2* S = reinterpret_cast<const double2*>(pl + (1 * 64 + c) * 64 + r0);
            const double2* Q = reinterpret_cast<const double2*>(pl + (2 * 64 + c) * 64 + r0);
#pragma unroll
            for (int h = 0; h < 4; ++h) {
                const double2 pp = P[h], ss = S[h], qq = Q[h];
                A[2 * h] = fma(pp.x, sc, A[2 * h]);
                A[2 * h + 1] = fma(pp.y, sc, A[2 * h + 1]);
                B[2 * h] = fma(ss.x, a.y, B[2 * h]);
                B[2 * h + 1] = fma(ss.y, a.y, B[2 * h + 1]);
                C[2 * h] = fma(qq.x, a.x, C[2 * h]);
                C[2 * h + 1] = fma(qq.y, a.x, C[2 * h + 1]);
            }
        }
#pragma unroll
        for (int rr = 0; rr < 8; ++rr)
            stsd(s_out + ((pb ^ p.loc[r0 + rr]) << 4), make_double2(A[rr] - B[rr], A[rr] + C[rr]));
        __syncthreads();  // the input tile is free, the output tile complete
        const uint64_t un = u + gridDim.x;
        if (un < p.n_tiles) {
            const double2* gp = p.psi + insert_zeros(un << p.r, p.Hpos, p.nH) + dthr;
            for (int i = 0; i < p.upt; ++i) cp_async16(s_in + ((sthr ^ p.soff[i]) << 4), gp + p.goff[i]);
        }
        cp_async_commit();
        double2* gs = p.psi + insert_zeros(u << p.r, p.Hpos, p.nH) + dthr;
        for (int i = 0; i < p.upt; ++i) stgd(gs + p.goff[i], ldsd(s_out + ((sthr ^ p.soff[i]) << 4)));
    }
    cp_async_wait0();
}

// Tiny states: one thread per group, direct global accesses.
__global__ void apply64_small_kernel(double2* psi, int n, int k, const int* q_dev, const double* planes) {
    const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (g >= (1ull << (n - k))) return;
    const int D = 1 << k;
    int q[SV_MAX_FUSED];
    for (int b = 0; b < k; ++b) q[b] = q_dev[b];
    const uint64_t base = insert_zeros(g, q, k);
    double2 a[64];
    uint64_t off[64];
    for (int c = 0; c < D; ++c) {
        uint64_t o = 0;
        for (int b = 0; b < k; ++b)
            if ((c >> b) & 1) o |= 1ull << q[b];
        off[c] = base | o;
        a[c] = psi[off[c]];
    }
    double2 y[64];
    for (int r = 0; r < D; ++r) {
        double A = 0.0, B = 0.0, C = 0.0;
        for (int c = 0; c < D; ++c) {
            A = fma(planes[r * D + c], a[c].x + a[c].y, A);
            B = fma(planes[D * D + r * D + c], a[c].y, B);
            C = fma(planes[2 * D * D + r * D + c], a[c].x, C);
        }
        y[r] = make_double2(A - B, A + C);
    }
    for (int r = 0; r < D; ++r) psi[off[r]] = y[r];
}

int sms64() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

template <int K>
cudaError_t launch64_k(double2* psi, int n, const Apply64Desc& d, cudaStream_t st) {
    constexpr int D = 1 << K;
    Tile64Params<K> p;
    std::memset(&p, 0, sizeof(p));
    p.psi = psi;
    if constexpr (K <= 5) {
        for (int r = 0; r < D; ++r)
            for (int c = 0; c < D; ++c) {
                const cd m = d.m[(size_t)r * D + c];
                p.M.P[r][c] = m.real();
                p.M.S[r][c] = m.real() + m.imag();
                p.M.Q[r][c] = m.imag() - m.real();
            }
    } else {
        p.M.dev = d.dev_planes;
    }
    // tile: runs of >= 8 amplitudes (128 B), grown to 2^11 amplitudes
    const int T = std::min(n, kT64);
    auto tile_bits = [&](int rr) {
        int t = rr;
        for (int b = 0; b < K; ++b)
            if (d.q[b] >= rr) ++t;
        return t;
    };
    int r = std::min(n, 3);
    while (r < n && tile_bits(r) < T) ++r;
    p.r = r;
    p.T = tile_bits(r);
    int tl[SV_MAX_FUSED];
    for (int b = 0; b < K; ++b) {
        if (d.q[b] < r) tl[b] = d.q[b];
        else {
            tl[b] = r + p.nH;
            p.Hpos[p.nH++] = d.q[b];
        }
    }
    p.nzt = K;
    uint32_t gmask = 0;
    for (int b = 0; b < K; ++b) {
        p.ztpos[b] = tl[b];
        gmask |= 1u << tl[b];
    }
    // lanes of an 8-lane LDS.128 phase run over the lowest 3 non-gate bits;
    // each gate bit in {0,1,2} is XORed with one of those lane bits >= 3
    std::vector<int> lane, hl;
    for (int t = 0; t < p.T && (int)lane.size() < 3; ++t)
        if (!((gmask >> t) & 1)) lane.push_back(t);
    for (int t : lane)
        if (t >= 3) hl.push_back(t);
    size_t jh = 0;
    for (int f = 0; f <= 2; ++f)
        if (((gmask >> f) & 1) && jh < hl.size()) p.swz[f] = 1u << hl[jh++];
    auto sw = [&](uint32_t t) {
        return t ^ (__builtin_popcount(t & p.swz[0]) & 1) ^ ((__builtin_popcount(t & p.swz[1]) & 1) << 1) ^
               ((__builtin_popcount(t & p.swz[2]) & 1) << 2);
    };
    auto dep = [&](uint64_t t) {
        uint64_t g = t & ((1ull << p.r) - 1);
        const uint64_t h = t >> p.r;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1) g += 1ull << p.Hpos[b];
        return g;
    };
    for (int m = 0; m < D; ++m) {
        uint32_t o = 0;
        for (int b = 0; b < K; ++b)
            if ((m >> b) & 1) o |= 1u << tl[b];
        p.loc[m] = sw(o);
    }
    const uint32_t units = 1u << p.T;
    const uint32_t ngroups = 1u << (p.T - K);
    // k = 6: 256 threads (8 warps x 8 output rows, lane = group) on 32 groups
    const uint32_t nthr = K == 6 ? 256u : std::min<uint32_t>(256, ngroups);
    if (K == 6 ? ngroups != 32 : (nthr < 32 || units / nthr > 64)) return cudaErrorNotSupported;  // small kernel
    p.upt = (int)(units / nthr);
    for (int i = 0; i < p.upt; ++i) {
        p.goff[i] = dep((uint64_t)nthr * i);
        p.soff[i] = sw(nthr * (uint32_t)i);
    }
    p.n_tiles = 1ull << (n - p.T);
    // two tile buffers: double-buffered input (k <= 5) or input + output (k = 6)
    size_t smem = 2 * ((size_t)16 << p.T) + (K == 6 ? 3 * 4096 * 8 : 0);
    const void* kern = nullptr;
    if constexpr (K == 6)
        kern = (const void*)apply64_k6_kernel;
    else
        kern = (const void*)apply64_kernel<K>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const int per_sm = std::max(1, (int)((227 * 1024) / (smem + 1024)));
    const uint64_t grid = std::min<uint64_t>(p.n_tiles, (uint64_t)sms64() * per_sm);
    if constexpr (K == 6)
        apply64_k6_kernel<<<(unsigned)grid, nthr, smem, st>>>(p);
    else
        apply64_kernel<K><<<(unsigned)grid, nthr, smem, st>>>(p);
    return cudaGetLastError();
}

__global__ void reset64_kernel(double2* psi, uint64_t n, int one) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
        psi[i] = make_double2((one && i == 0) ? 1.0 : 0.0, 0.0);
}

// exact in-place swap of local index bits a < b (pure moves): the element
// with bit a = 1, bit b = 0 trades places with its partner (a = 0, b = 1)
__global__ void swap_bits64_kernel(double2* psi, uint64_t n_pairs, int a, int b) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < n_pairs; w += stride) {
        // insert a 0 at a and at b, then set bit a
        uint64_t i = w;
        i = ((i >> a) << (a + 1)) | (i & ((1ull << a) - 1ull));
        i = ((i >> b) << (b + 1)) | (i & ((1ull << b) - 1ull));
        const uint64_t x = i | (1ull << a), y = i | (1ull << b);
        const double2 vx = psi[x], vy = psi[y];
        psi[x] = vy;
        psi[y] = vx;
    }
}

__global__ void gather64_kernel(const double2* psi, const uint64_t* phys, uint64_t count, double2* out) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < count) out[i] = psi[phys[i]];
}

}  // namespace

void pack_planes64(const Apply64Desc& d, double* out) {
    const int D = 1 << d.k;
    for (int i = 0; i < D * D; ++i) {
        out[i] = d.m[i].real();
        out[D * D + i] = d.m[i].real() + d.m[i].imag();
        out[2 * D * D + i] = d.m[i].imag() - d.m[i].real();
    }
}

cudaError_t launch_apply64(double2* psi, int n, const Apply64Desc& d, cudaStream_t st) {
    cudaError_t e = cudaErrorNotSupported;
    switch (d.k) {
        case 1: e = launch64_k<1>(psi, n, d, st); break;
        case 2: e = launch64_k<2>(psi, n, d, st); break;
        case 3: e = launch64_k<3>(psi, n, d, st); break;
        case 4: e = launch64_k<4>(psi, n, d, st); break;
        case 5: e = launch64_k<5>(psi, n, d, st); break;
        case 6:
            if (!d.dev_planes) return cudaErrorInvalidValue;
            e = launch64_k<6>(psi, n, d, st);
            break;
    }
    if (e != cudaErrorNotSupported) return e;
    // small states: per-group kernel with planes and qubits in device scratch
    if (!d.small_scratch) return cudaErrorInvalidValue;
    const uint64_t ng = 1ull << (n - d.k);
    apply64_small_kernel<<<(unsigned)((ng + 127) / 128), 128, 0, st>>>(
        psi, n, d.k, reinterpret_cast<const int*>(d.small_scratch), d.dev_planes);
    return cudaGetLastError();
}

cudaError_t launch_reset64(double2* psi, uint64_t n_amps, bool one, cudaStream_t st) {
    const uint64_t blocks = std::min<uint64_t>((n_amps + 255) / 256, (uint64_t)sms64() * 16);
    reset64_kernel<<<(unsigned)std::max<uint64_t>(blocks, 1), 256, 0, st>>>(psi, n_amps, one ? 1 : 0);
    return cudaGetLastError();
}

cudaError_t launch_swap_bits64(double2* psi, int l, int a, int b, cudaStream_t st) {
    if (a == b) return cudaSuccess;
    if (a > b) std::swap(a, b);
    const uint64_t n_pairs = 1ull << (l - 2);
    const uint64_t blocks = std::min<uint64_t>((n_pairs + 255) / 256, (uint64_t)sms64() * 16);
    swap_bits64_kernel<<<(unsigned)std::max<uint64_t>(blocks, 1), 256, 0, st>>>(psi, n_pairs, a, b);
    return cudaGetLastError();
}

cudaError_t launch_gather64(const double2* psi, const uint64_t* phys, uint64_t count, double2* out,
                            cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    gather64_kernel<<<(unsigned)((count + 255) / 256), 256, 0, st>>>(psi, phys, count, out);
    return cudaGetLastError();
}

}  // namespace svb
