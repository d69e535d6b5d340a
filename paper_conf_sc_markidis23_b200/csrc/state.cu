// state.cu -- state-space kernels: |0..0> init (row a0), amplitude gather
// (row a9), the fixed-point sampler (row a8) and the shard exchange (row a7).
//
// PAPER.md L131-132 (§3): the state space sets states, gets amplitudes,
// reduces and samples "to generate measurement outcomes".  The sampler is
// the integer reading S5: w_i = floor(p_i * 2^62) with p_i
// formed in fp64 from the complex64 parts (both products exact), exact uint64
// bin sums and prefix sums, t_s = (splitmix64#(s+1)(seed) * T) >> 64,
// out[s] = min{ i : C_i > t_s }.  Integer sums make the result independent
// of the reduction order, block size or shard split.
#include <cuda_runtime.h>

#include <algorithm>

#include "kernels.h"

namespace svb {

namespace {

int sms() {
    static int n = 0;
    if (n == 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

unsigned grid_cap(uint64_t items, int threads, int per_sm = 16) {
    uint64_t need = (items + threads - 1) / threads;
    uint64_t cap = (uint64_t)sms() * per_sm;
    return (unsigned)std::max<uint64_t>(1, std::min(need, cap));
}

__global__ void reset_kernel(float4* psi4, uint64_t n_units, float2* psi, uint64_t n_amps, int one) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_units; i += stride) __stcs(psi4 + i, z);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (n_amps & 1) psi[n_amps - 1] = make_float2(0.f, 0.f);
        if (one) psi[0] = make_float2(1.f, 0.f);
    }
}

__global__ void gather_kernel(const float2* psi, const uint64_t* phys, const int32_t* owner, int shard,
                              uint64_t count, float2* out) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < count && (owner == nullptr || owner[i] == shard)) out[i] = psi[phys[i]];
}

__device__ __forceinline__ uint64_t weight(float2 a) {
    const double re = (double)a.x, im = (double)a.y;
    const double p = __fma_rn(re, re, im * im);  // re*re and im*im are exact in fp64
    return __double2ull_rz(p * 0x1p62);           // floor for p >= 0 (exact scaling)
}

// complex128 states: p = fl(fl(re*re) + fl(im*im)) with explicit roundings
// (no FMA contraction), the reading R5 shared with oracle/sample.py.
__device__ __forceinline__ uint64_t weight(double2 a) {
    const double p = __dadd_rn(__dmul_rn(a.x, a.x), __dmul_rn(a.y, a.y));
    return __double2ull_rz(p * 0x1p62);
}

// kAmpsPerLane = 2 consecutive amplitudes per lane (8 lanes per 16-amplitude bin)
__device__ __forceinline__ void load_lane_w(const float2* psi, uint64_t i0, uint64_t& w) {
    const float4 u = __ldcs(reinterpret_cast<const float4*>(psi + i0));
    w = weight(make_float2(u.x, u.y)) + weight(make_float2(u.z, u.w));
}
__device__ __forceinline__ void load_lane_w(const double2* psi, uint64_t i0, uint64_t& w) {
    w = weight(__ldcs(psi + i0)) + weight(__ldcs(psi + i0 + 1));
}

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    return v;
}

// 8 lanes per 16-amplitude bin, 2 amplitudes per lane.
constexpr int kAmpsPerLane = (1 << kSampleBinBits) / 8;
static_assert(kAmpsPerLane == 2, "bin_weights_kernel loads 2 amplitudes per lane");
template <class E>
__global__ void bin_weights_kernel(const E* __restrict__ psi, uint64_t n_amps, uint64_t* __restrict__ bins,
                                   uint64_t n_bins) {
    const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint64_t nthr = (uint64_t)gridDim.x * blockDim.x;  // multiple of 32
    const int sub = threadIdx.x & 7;
    const uint64_t full_bins = n_amps >> kSampleBinBits;  // bins with all 16 amplitudes
    // warp-uniform loop (4 bins per warp per trip) so the shuffles see all lanes
    for (uint64_t b0 = (tid >> 5) << 2; b0 < n_bins; b0 += (nthr >> 5) << 2) {
        const uint64_t b = b0 + ((threadIdx.x & 31) >> 3);
        uint64_t w = 0;
        const uint64_t i0 = (b << kSampleBinBits) + kAmpsPerLane * sub;
        if (b < full_bins) {
            load_lane_w(psi, i0, w);
        } else if (b < n_bins) {
            for (int j = 0; j < kAmpsPerLane; ++j)
                if (i0 + j < n_amps) w += weight(psi[i0 + j]);
        }
        w += __shfl_xor_sync(0xffffffffu, w, 1);
        w += __shfl_xor_sync(0xffffffffu, w, 2);
        w += __shfl_xor_sync(0xffffffffu, w, 4);
        if (sub == 0 && b < n_bins) bins[b] = w;
    }
}

// ---- inclusive scan of uint64 (exact), 1024 threads x 4 elements per block
constexpr int kScanThreads = 1024;
constexpr int kScanPer = 4;
constexpr uint64_t kScanBlock = (uint64_t)kScanThreads * kScanPer;

__device__ uint64_t block_exclusive_scan(uint64_t v, uint64_t* sh_warp, uint64_t& total) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint64_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) sh_warp[wid] = x;
    __syncthreads();
    if (wid == 0) {
        uint64_t s = (lane < (int)(blockDim.x >> 5)) ? sh_warp[lane] : 0ull;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint64_t y = __shfl_up_sync(0xffffffffu, s, o);
            if (lane >= o) s += y;
        }
        sh_warp[lane] = s;  // inclusive warp totals
    }
    __syncthreads();
    total = sh_warp[(blockDim.x >> 5) - 1];
    const uint64_t before = (wid > 0) ? sh_warp[wid - 1] : 0ull;
    __syncthreads();
    return before + x - v;
}

__global__ void scan_reduce_kernel(const uint64_t* data, uint64_t count, uint64_t* block_sums) {
    __shared__ uint64_t sh[32];
    const uint64_t base = (uint64_t)blockIdx.x * kScanBlock;
    uint64_t s = 0;
    for (int j = 0; j < kScanPer; ++j) {
        const uint64_t i = base + (uint64_t)j * kScanThreads + threadIdx.x;
        if (i < count) s += data[i];
    }
    uint64_t total;
    block_exclusive_scan(s, sh, total);
    if (threadIdx.x == 0) block_sums[blockIdx.x] = total;
}

__global__ void scan_apply_kernel(uint64_t* data, uint64_t count, const uint64_t* block_prefix /* inclusive */) {
    __shared__ uint64_t sh[32];
    const uint64_t base = (uint64_t)blockIdx.x * kScanBlock + (uint64_t)threadIdx.x * kScanPer;
    uint64_t v[kScanPer];
    uint64_t s = 0;
    for (int j = 0; j < kScanPer; ++j) {
        const uint64_t i = base + j;
        v[j] = (i < count) ? data[i] : 0ull;
        s += v[j];
    }
    uint64_t total;
    uint64_t ex = block_exclusive_scan(s, sh, total);
    if (blockIdx.x > 0 && block_prefix) ex += block_prefix[blockIdx.x - 1];
    for (int j = 0; j < kScanPer; ++j) {
        ex += v[j];
        const uint64_t i = base + j;
        if (i < count) data[i] = ex;
    }
}

__device__ __forceinline__ uint64_t splitmix64_at(uint64_t seed, uint64_t s) {
    uint64_t z = seed + (s + 1ull) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

template <class E>
__global__ void sample_resolve_kernel(const E* __restrict__ psi, const uint64_t* __restrict__ cum,
                                      uint64_t n_bins, const uint64_t* range_lo_dev, const uint64_t* total_dev,
                                      uint64_t seed, uint64_t n_samples, uint64_t index_base, uint64_t n_amps,
                                      uint64_t* out, uint64_t* status) {
    const uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n_samples) return;
    const uint64_t T = *total_dev;
    // S5 validity (checked here so that sampling needs no host round trip):
    // a zero total or sum |c|^2 >= 3.99 (uint64 overflow risk) yields no
    // sample -- every output is UINT64_MAX and the status word is set
    if (T == 0 || (double)T >= 3.99 * 4611686018427387904.0) {
        out[s] = ~0ull;
        if (s == 0 && status) *status = T == 0 ? 1ull : 2ull;
        return;
    }
    const uint64_t lo = range_lo_dev ? *range_lo_dev : 0ull;
    const uint64_t local_total = cum[n_bins - 1];
    const uint64_t t = __umul64hi(splitmix64_at(seed, s), T);
    if (t < lo || t - lo >= local_total) return;
    const uint64_t tl = t - lo;
    // first bin with cum[b] > tl
    uint64_t a = 0, b = n_bins - 1;
    while (a < b) {
        const uint64_t mid = (a + b) >> 1;
        if (cum[mid] > tl) b = mid;
        else a = mid + 1;
    }
    uint64_t acc = (a > 0) ? cum[a - 1] : 0ull;
    const uint64_t i0 = a << kSampleBinBits;
    uint64_t idx = i0;
    for (int j = 0; j < (1 << kSampleBinBits) && i0 + j < n_amps; ++j) {
        acc += weight(psi[i0 + j]);
        if (acc > tl) {
            idx = i0 + j;
            break;
        }
    }
    out[s] = index_base + idx;
}

// ---- shard exchange -----------------------------------------------------------
struct XParams {
    float2* const* shards;
    int world, d0, d1, l, s;
    int P[8], p[8];
    int ps[8];     // local positions p_j sorted ascending
    int pj[8];     // pj[t] = j of the t-th smallest position
};

// Shard d swaps, for every chunk c != c_d, its chunk c with chunk c_d of
// shard e (e = d with device bits (P_j - l) := c_j, c_d = d's device bits);
// the 2^(l-s) elements x of a chunk pair are split in halves: the lower shard
// of the pair swaps x < half, the other x >= half, so P ranks share the work
// evenly and every element pair is swapped exactly once.  Work item w of
// shard d enumerates only the elements it swaps: (chunk index, x in its half);
// VEC: all p_j >= 1, so x is handled in pairs of neighbouring amplitudes (16 B).
template <bool VEC>
__global__ void exchange_kernel(const __grid_constant__ XParams xp) {
    const int l = xp.l, s = xp.s;
    const int hb = l - s - 1 - (VEC ? 1 : 0);  // bits of the per-chunk work index
    const uint64_t per_chunk = 1ull << hb;
    const uint64_t per_shard = per_chunk * (uint64_t)((1 << s) - 1);
    const uint64_t total = per_shard * (uint64_t)(xp.d1 - xp.d0);
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t half = 1ull << (l - s - 1);
    for (uint64_t gw = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; gw < total; gw += stride) {
        const int d = xp.d0 + (int)(gw / per_shard);
        const uint64_t w = gw % per_shard;
        uint32_t cd = 0;
        for (int j = 0; j < s; ++j) cd |= (uint32_t)((d >> (xp.P[j] - l)) & 1) << j;
        uint32_t c = (uint32_t)(w >> hb);
        if (c >= cd) ++c;  // skip the self chunk
        int e = d;
        for (int j = 0; j < s; ++j) {
            const int gb = xp.P[j] - l;
            e = (e & ~(1 << gb)) | (int)(((c >> j) & 1u) << gb);
        }
        uint64_t x = (w & (per_chunk - 1)) << (VEC ? 1 : 0);
        if (d > e) x += half;
        uint64_t za = x, zb = x;
        for (int t = 0; t < s; ++t) {
            const int q = xp.ps[t];
            const uint64_t lo_a = za & ((1ull << q) - 1ull), lo_b = zb & ((1ull << q) - 1ull);
            za = ((za >> q) << (q + 1)) | ((uint64_t)((c >> xp.pj[t]) & 1u) << q) | lo_a;
            zb = ((zb >> q) << (q + 1)) | ((uint64_t)((cd >> xp.pj[t]) & 1u) << q) | lo_b;
        }
        float2* A = xp.shards[d];
        float2* B = xp.shards[e];
        if constexpr (VEC) {
            float4* pa = reinterpret_cast<float4*>(A + za);
            float4* pb = reinterpret_cast<float4*>(B + zb);
            const float4 va = *pa, vb = *pb;
            *pa = vb;
            *pb = va;
        } else {
            const float2 va = A[za], vb = B[zb];
            A[za] = vb;
            B[zb] = va;
        }
    }
}

}  // namespace

cudaError_t launch_reset(float2* psi, uint64_t n_amps, bool one, cudaStream_t st) {
    const uint64_t units = n_amps >> 1;
    reset_kernel<<<grid_cap(std::max<uint64_t>(units, 1), 256), 256, 0, st>>>(reinterpret_cast<float4*>(psi), units,
                                                                               psi, n_amps, one ? 1 : 0);
    return cudaGetLastError();
}

cudaError_t launch_gather(const float2* psi, const uint64_t* phys, const int32_t* owner, int shard, uint64_t count,
                          float2* out, cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    gather_kernel<<<(unsigned)((count + 255) / 256), 256, 0, st>>>(psi, phys, owner, shard, count, out);
    return cudaGetLastError();
}

cudaError_t launch_bin_weights(const void* psi, bool fp64, uint64_t n_amps, uint64_t* bins, cudaStream_t st) {
    const uint64_t n_bins = (n_amps + (1u << kSampleBinBits) - 1) >> kSampleBinBits;
    // whole warps per loop trip (the 8-lane shuffles need all lanes)
    if (fp64)
        bin_weights_kernel<double2><<<grid_cap(n_bins * 8, 256, 16), 256, 0, st>>>((const double2*)psi, n_amps, bins,
                                                                                     n_bins);
    else
        bin_weights_kernel<float2><<<grid_cap(n_bins * 8, 256, 16), 256, 0, st>>>((const float2*)psi, n_amps, bins,
                                                                                    n_bins);
    return cudaGetLastError();
}

size_t scan_scratch_elems(uint64_t count) {
    size_t total = 0;
    uint64_t c = count;
    while (c > kScanBlock) {
        c = (c + kScanBlock - 1) / kScanBlock;
        total += c;
    }
    return total + 1;
}

cudaError_t launch_inclusive_scan(uint64_t* data, uint64_t count, uint64_t* scratch, cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    if (count <= kScanBlock) {
        scan_apply_kernel<<<1, kScanThreads, 0, st>>>(data, count, nullptr);
        return cudaGetLastError();
    }
    const uint64_t nblocks = (count + kScanBlock - 1) / kScanBlock;
    uint64_t* sums = scratch;
    scan_reduce_kernel<<<(unsigned)nblocks, kScanThreads, 0, st>>>(data, count, sums);
    cudaError_t e = launch_inclusive_scan(sums, nblocks, scratch + nblocks, st);
    if (e != cudaSuccess) return e;
    scan_apply_kernel<<<(unsigned)nblocks, kScanThreads, 0, st>>>(data, count, sums);
    return cudaGetLastError();
}

cudaError_t launch_sample_resolve(const void* psi, bool fp64, uint64_t n_amps, const uint64_t* cum_bins,
                                  uint64_t n_bins, const uint64_t* range_lo_dev, const uint64_t* total_dev,
                                  uint64_t seed, uint64_t n_samples, uint64_t index_base, uint64_t* out,
                                  uint64_t* status, cudaStream_t st) {
    if (n_samples == 0) return cudaSuccess;
    if (fp64)
        sample_resolve_kernel<double2><<<(unsigned)((n_samples + 255) / 256), 256, 0, st>>>(
            (const double2*)psi, cum_bins, n_bins, range_lo_dev, total_dev, seed, n_samples, index_base, n_amps, out,
            status);
    else
        sample_resolve_kernel<float2><<<(unsigned)((n_samples + 255) / 256), 256, 0, st>>>(
            (const float2*)psi, cum_bins, n_bins, range_lo_dev, total_dev, seed, n_samples, index_base, n_amps, out,
            status);
    return cudaGetLastError();
}

cudaError_t launch_exchange(float2* const* shards_dev, int world, int me, const ExchangeDesc& x, cudaStream_t st) {
    XParams p;
    p.shards = shards_dev;
    p.world = world;
    p.d0 = (me < 0) ? 0 : me;
    p.d1 = (me < 0) ? world : me + 1;
    p.l = x.l;
    p.s = x.s;
    for (int j = 0; j < 8; ++j) {
        p.P[j] = x.P[j];
        p.p[j] = x.p[j];
        p.pj[j] = j;
    }
    std::sort(p.pj, p.pj + x.s, [&](int a, int b) { return x.p[a] < x.p[b]; });
    for (int t = 0; t < x.s; ++t) p.ps[t] = x.p[p.pj[t]];
    bool vec = x.l - x.s - 1 >= 1;
    for (int j = 0; j < x.s; ++j)
        if (x.p[j] < 1) vec = false;
    const uint64_t total = ((uint64_t)(p.d1 - p.d0) * (((1ull << x.s) - 1) << (x.l - x.s - 1))) >> (vec ? 1 : 0);
    if (vec) exchange_kernel<true><<<grid_cap(total, 256, 16), 256, 0, st>>>(p);
    else exchange_kernel<false><<<grid_cap(total, 256, 16), 256, 0, st>>>(p);
    return cudaGetLastError();
}

}  // namespace svb

namespace svb {

namespace {

__global__ void shard_offsets_kernel(const uint64_t* const* totals_src, const int32_t* sigma, int world,
                                     uint64_t* lo, uint64_t* total) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    uint64_t tot = 0;
    for (int d = 0; d < world; ++d) tot += *totals_src[d];
    for (int d = 0; d < world; ++d) {
        uint64_t acc = 0;
        for (int e = 0; e < world; ++e)
            if (sigma[e] < sigma[d]) acc += *totals_src[e];
        lo[d] = acc;
    }
    *total = tot;
}

__global__ void merge_min_kernel(const uint64_t* const* src, int world, uint64_t count, uint64_t* out) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride) {
        uint64_t m = ~0ull;
        for (int r = 0; r < world; ++r) {
            const uint64_t v = src[r][i];
            m = v < m ? v : m;
        }
        out[i] = m;
    }
}

// flags_dev[r] = rank r's flag array (world words).  Thread j signals rank j
// (writes epoch into flags[j][me]), then thread 0.. waits for own flags.
__global__ void barrier_kernel(uint64_t* const* flags, int world, int me, uint64_t epoch) {
    __threadfence_system();
    const int j = threadIdx.x;
    if (j < world) {
        volatile uint64_t* dst = flags[j] + me;
        *dst = epoch;
    }
    __threadfence_system();
    if (j < world) {
        volatile uint64_t* mine = flags[me] + j;
        while (*mine < epoch) {
        }
    }
    __threadfence_system();
    __syncthreads();
}

}  // namespace

cudaError_t launch_shard_offsets(const uint64_t* const* totals_src_dev, const int32_t* sigma_dev, int world,
                                 uint64_t* lo_dev, uint64_t* total_dev, cudaStream_t st) {
    shard_offsets_kernel<<<1, 32, 0, st>>>(totals_src_dev, sigma_dev, world, lo_dev, total_dev);
    return cudaGetLastError();
}

cudaError_t launch_merge_min(const uint64_t* const* src_dev, int world, uint64_t count, uint64_t* out,
                             cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    merge_min_kernel<<<grid_cap(count, 256), 256, 0, st>>>(src_dev, world, count, out);
    return cudaGetLastError();
}

cudaError_t launch_barrier(uint64_t* const* flags_dev, int world, int me, uint64_t epoch, cudaStream_t st) {
    barrier_kernel<<<1, 64, 0, st>>>(flags_dev, world, me, epoch);
    return cudaGetLastError();
}

}  // namespace svb
