// blocked.cu -- cache-blocked multi-gate passes.
//
// Related work [12] applies several gates per memory pass;
// the paper's own smem remedy (L94-96) keeps a block of the state on chip.
// A pass loads a tile -- the 2^T amplitudes that share every bit outside a
// qubit set S (|S| = T, S contains qubits 0..3 so runs stay >= 128 B) -- applies
// EVERY fused gate of the pass (all their qubits are in S) inside the tile,
// and writes it back: one HBM read + write for many gates.  Passes are formed
// on the host (build_passes in sv_api.cpp, reading R7); the state
// never moves -- a pass only chooses which amplitudes share a tile.
//
// Two kernels:
//  * apply_rpass (default, gates with k <= 2): the gates of a pass run in
//    register phases -- each thread holds 32 amplitudes of the tile in
//    registers and applies every gate whose qubits lie in the phase's 5 tile
//    positions (plus CZ-like gates anywhere), one shared-memory exchange and
//    barrier per phase;
//  * apply_pass (k = 3, 4; opt-in): one sweep of the shared-memory tile per
//    gate (gather the 2^k members, Gauss 3-multiplication y = M a, scatter).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "device_util.cuh"
#include "kernels.h"

// Build options (compile-time; A/B variants via build.py --variant):
#ifndef SVB_RP_M
#define SVB_RP_M 5  // log2 amplitudes per thread (4: 16 per thread, measured slower)
#endif
#ifndef SVB_RP_ENABLE
#define SVB_RP_ENABLE 1  // register-blocked passes (0: shared-memory pass kernel only)
#endif
#ifndef SVB_RP_F2
#define SVB_RP_F2 1  // packed FFMA2 complex MACs
#endif
#ifndef SVB_RP_DIRECT
#define SVB_RP_DIRECT 1  // last phase stores registers straight to HBM when coalesced
#endif
#ifndef SVB_RP_CZBONUS
#define SVB_RP_CZBONUS 1  // phase planning: prefer register sets holding both qubits of CZ-like gates
#endif
#ifndef SVB_RP_DLOAD
#define SVB_RP_DLOAD 0  // first phase loads registers straight from HBM
#endif
#ifndef SVB_RP_EARLY
#define SVB_RP_EARLY 1  // next tile's load issued before the last phase's gates
#endif
#ifndef SVB_RP_DEBUG
#define SVB_RP_DEBUG 0  // print phase plans to stderr
#endif

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

}  // namespace

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

namespace {


// ------------------------------------------------ register-blocked passes
// apply_rpass<M, F2>: the same tiles and tile loop, but a gate is not one sweep
// of the shared-memory tile.  The pass's gates (k <= 2) are grouped into
// PHASES (host, plan_phases): sets of gates whose tile positions fit in a set
// R of M positions, gates moved forward only past gates on disjoint qubits
// (they commute).  In a phase every thread gathers the 2^M amplitudes whose
// tile index varies over R (its other tile bits are fixed by the thread
// index), applies all the phase's gates to them in registers -- a gate on
// register bits MASK is a compile-time-indexed 2^k x 2^k complex matvec over
// the 2^M / 2^k groups, each matrix element loaded once per gate -- and
// scatters them back: one barrier per phase instead of one per gate.
// Addresses are XOR-linear: slot = tbase ^ roff[j], swizzled on the host with
// a fold swizzle (16 B chunk bits 1..3 ^= the XOR of tile bits 4..6, 7..9,
// ...) and the thread -> position order chosen so that each quarter-warp
// (LDS.128) / half-warp (LDS.64) gather is conflict-free.
constexpr int kRpMatFloats = kRpMaxGates * 64;  // 4 floats per element, k <= 2

struct RpPhase {
    uint32_t roff[32];  // byte offsets of register index j (swizzled)
    uint32_t tbw[10];   // byte offset contributed by thread-index bit i (swizzled)
    uint16_t g0, g1;    // gates [g0, g1) in launch order
    uint32_t b0;        // tile bit 0 is register bit 0: 16 B gathers
};

struct alignas(16) RpassParams {
    float mats[kRpMatFloats];
    float2* psi;
    uint64_t n_tiles;
    int T, r, nH, nph, tbits;
    int Hpos[32];
    uint64_t goff[16];
    uint32_t soff[16];
    uint32_t gcode[kRpMaxGates];  // register mask (bits 0..4) | kind << 5 | matrix float offset << 8
    // direct store: the last phase writes its registers straight to HBM
    // (16 B pairs; tile bit 0 in registers, tile bits 1..3 on lanes 0..2 so
    // each quarter-warp writes one 128 B run) instead of through the tile
    int direct;
    uint64_t dgoff[32];   // amplitude offset of register pair j (16 B) / register j (8 B layout)
    uint64_t dgtbw[10];   // amplitude offset of thread-index bit i
    // direct load: the first phase reads its registers straight from HBM
    // (same layout condition; one tile buffer only) instead of via the tile
    int dload;
    int early;  // direct store: issue the next tile's load before the last phase's gates
    int zinit;  // the state is |0...0>: nothing is loaded, phase 0 starts from zeros
    int zone;   // ... and this shard holds amplitude 0 (= 1, tile 0, thread 0, register 0)
    uint64_t lgoff[16];
    uint64_t lgtbw[10];
    RpPhase ph[kRpMaxPhases];
};

__host__ __device__ constexpr int pdep5(int v, int mask) {
    int r = 0, b = 0;
    for (int i = 0; i < 5; ++i)
        if ((mask >> i) & 1) {
            if ((v >> b) & 1) r |= 1 << i;
            ++b;
        }
    return r;
}
__host__ __device__ constexpr int popc5(int m) { return (m & 1) + ((m >> 1) & 1) + ((m >> 2) & 1) + ((m >> 3) & 1) + ((m >> 4) & 1); }

__device__ __forceinline__ void st_stream2(float2* p, float2 v) {
    asm volatile("st.global.cs.v2.f32 [%0], {%1,%2};" ::"l"(p), "f"(v.x), "f"(v.y) : "memory");
}
__device__ __forceinline__ float4 ld_stream(const float4* p) {
    float4 v;
    asm volatile("ld.global.cs.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}

// packed fp32 pair FMA (FFMA2): d = a * b + c per lane
__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
    unsigned long long d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;"
        : "=l"(d)
        : "l"(*reinterpret_cast<unsigned long long*>(&a)), "l"(*reinterpret_cast<unsigned long long*>(&b)),
          "l"(*reinterpret_cast<unsigned long long*>(&c)));
    return *reinterpret_cast<float2*>(&d);
}

// Matrix element e of a gate is stored as 4 floats (mr, mr, -mi, mi).
// F2: complex MAC y += m x as two packed FFMA2, y += (mr, mr) (xr, xi) and
// y += (-mi, mi) (xi, xr) (ptxas encodes the swapped pair as an operand
// modifier; both matrix pairs come straight from uniform registers,
// LDCU.64).  Otherwise four FFMA.
#ifndef SVB_RP_G
#define SVB_RP_G 1  // groups transformed together (1 measured 0.8 % faster than 2 or 4 at T = 13)
#endif
template <int M, int MASK, bool F2>
__device__ __forceinline__ void reg_gate(float2 (&a)[1 << M], const float* __restrict__ mf) {
    constexpr int K = popc5(MASK);
    constexpr int D = 1 << K;
    constexpr int REST = ((1 << M) - 1) & ~MASK;
    constexpr int NG = (1 << M) / D;
    constexpr int G = SVB_RP_G < NG ? SVB_RP_G : NG;
    float4 m[D * D];
#pragma unroll
    for (int i = 0; i < D * D; ++i) m[i] = reinterpret_cast<const float4*>(mf)[i];
#pragma unroll
    for (int g0 = 0; g0 < NG; g0 += G) {
        float2 x[G][D];
#pragma unroll
        for (int h = 0; h < G; ++h)
#pragma unroll
            for (int c = 0; c < D; ++c) x[h][c] = a[pdep5(g0 + h, REST) | pdep5(c, MASK)];
#pragma unroll
        for (int rr = 0; rr < D; ++rr) {
            float2 y[G];
#pragma unroll
            for (int h = 0; h < G; ++h) {
                if constexpr (F2) {
                    y[h] = make_float2(0.f, 0.f);
                } else {
                    y[h] = make_float2(m[rr * D].x * x[h][0].x, m[rr * D].x * x[h][0].y);
                    y[h].x = fmaf(m[rr * D].z, x[h][0].y, y[h].x);
                    y[h].y = fmaf(m[rr * D].w, x[h][0].x, y[h].y);
                }
            }
#pragma unroll
            for (int c = F2 ? 0 : 1; c < D; ++c) {
                const float4 mc = m[rr * D + c];
#pragma unroll
                for (int h = 0; h < G; ++h) {
                    if constexpr (F2) {
                        y[h] = ffma2(make_float2(mc.x, mc.y), x[h][c], y[h]);
                        y[h] = ffma2(make_float2(mc.z, mc.w), make_float2(x[h][c].y, x[h][c].x), y[h]);
                    } else {
                        y[h].x = fmaf(mc.x, x[h][c].x, y[h].x);
                        y[h].x = fmaf(mc.z, x[h][c].y, y[h].x);
                        y[h].y = fmaf(mc.x, x[h][c].y, y[h].y);
                        y[h].y = fmaf(mc.w, x[h][c].x, y[h].y);
                    }
                }
            }
#pragma unroll
            for (int h = 0; h < G; ++h) a[pdep5(g0 + h, REST) | pdep5(rr, MASK)] = y[h];
        }
    }
}

__host__ __device__ constexpr int pext5(int v, int mask) {
    int r = 0, b = 0;
    for (int i = 0; i < 5; ++i)
        if ((mask >> i) & 1) {
            if ((v >> i) & 1) r |= 1 << b;
            ++b;
        }
    return r;
}

// Diagonal gate on register bits MASK: a[j] *= d[e(j)], entries stored like
// matrix elements (dr, dr, -di, di); one complex product = two FFMA2.
template <int M, int MASK>
__device__ __forceinline__ void reg_diag(float2 (&a)[1 << M], const float* __restrict__ mf) {
    constexpr int D = 1 << popc5(MASK);
#pragma unroll
    for (int i = 0; i < D; ++i) {
        const float4 e = reinterpret_cast<const float4*>(mf)[i];
#pragma unroll
        for (int j = 0; j < (1 << M); ++j) {
            if (pext5(j, MASK) != i) continue;
            const float2 x = a[j];
            a[j] = ffma2(make_float2(e.z, e.w), make_float2(x.y, x.x), ffma2(make_float2(e.x, e.y), x, make_float2(0.f, 0.f)));
        }
    }
}

// CZ-like gate (diag(1, 1, 1, -1)): sign flips only.  Its qubits need not be
// register bits: MASK holds the ones that are, and `tp` (per thread) tells
// whether the thread-index bits holding the others are all 1.
template <int M, int MASK>
__device__ __forceinline__ void reg_cz(float2 (&a)[1 << M], bool tp) {
#pragma unroll
    for (int j = 0; j < (1 << M); ++j)
        if ((j & MASK) == MASK) {
            if (popc5(MASK) == 2 || tp) a[j] = make_float2(-a[j].x, -a[j].y);
        }
}

template <int M, bool F2>
__device__ __forceinline__ void reg_gate_dispatch(uint32_t code, float2 (&a)[1 << M], const float* mf) {
    // code = register mask (bits 0..4) | kind << 5 (0 dense, 1 diagonal, 2 CZ-like)
    //        | dense/diagonal: matrix float offset << 8; CZ: thread-index mask << 8.
    // Balanced compare trees on the (warp-uniform) code: a switch becomes a
    // BRX jump table on a vector register, and the matrices then load with
    // LDC into vector registers instead of uniform registers
    const int mask = code & 31, kind = (code >> 5) & 3;
    if constexpr (M == 4) {
        if (kind == 0) {
            if (mask < 6) {
                if (mask < 3) {
                    if (mask < 2) {
                        reg_gate<4, 1, F2>(a, mf);
                    } else {
                        reg_gate<4, 2, F2>(a, mf);
                    }
                } else {
                    if (mask < 4) {
                        reg_gate<4, 3, F2>(a, mf);
                    } else {
                        if (mask < 5) {
                            reg_gate<4, 4, F2>(a, mf);
                        } else {
                            reg_gate<4, 5, F2>(a, mf);
                        }
                    }
                }
            } else {
                if (mask < 9) {
                    if (mask < 8) {
                        reg_gate<4, 6, F2>(a, mf);
                    } else {
                        reg_gate<4, 8, F2>(a, mf);
                    }
                } else {
                    if (mask < 10) {
                        reg_gate<4, 9, F2>(a, mf);
                    } else {
                        if (mask < 12) {
                            reg_gate<4, 10, F2>(a, mf);
                        } else {
                            reg_gate<4, 12, F2>(a, mf);
                        }
                    }
                }
            }
        } else if (kind == 1) {
            if (mask < 6) {
                if (mask < 3) {
                    if (mask < 2) {
                        reg_diag<4, 1>(a, mf);
                    } else {
                        reg_diag<4, 2>(a, mf);
                    }
                } else {
                    if (mask < 4) {
                        reg_diag<4, 3>(a, mf);
                    } else {
                        if (mask < 5) {
                            reg_diag<4, 4>(a, mf);
                        } else {
                            reg_diag<4, 5>(a, mf);
                        }
                    }
                }
            } else {
                if (mask < 9) {
                    if (mask < 8) {
                        reg_diag<4, 6>(a, mf);
                    } else {
                        reg_diag<4, 8>(a, mf);
                    }
                } else {
                    if (mask < 10) {
                        reg_diag<4, 9>(a, mf);
                    } else {
                        if (mask < 12) {
                            reg_diag<4, 10>(a, mf);
                        } else {
                            reg_diag<4, 12>(a, mf);
                        }
                    }
                }
            }
        } else {
            const uint32_t tm = code >> 8;
            const bool tp = (threadIdx.x & tm) == tm;
            if (mask < 5) {
                if (mask < 2) {
                    if (mask < 1) {
                        reg_cz<4, 0>(a, tp);
                    } else {
                        reg_cz<4, 1>(a, tp);
                    }
                } else {
                    if (mask < 3) {
                        reg_cz<4, 2>(a, tp);
                    } else {
                        if (mask < 4) {
                            reg_cz<4, 3>(a, tp);
                        } else {
                            reg_cz<4, 4>(a, tp);
                        }
                    }
                }
            } else {
                if (mask < 9) {
                    if (mask < 6) {
                        reg_cz<4, 5>(a, tp);
                    } else {
                        if (mask < 8) {
                            reg_cz<4, 6>(a, tp);
                        } else {
                            reg_cz<4, 8>(a, tp);
                        }
                    }
                } else {
                    if (mask < 10) {
                        reg_cz<4, 9>(a, tp);
                    } else {
                        if (mask < 12) {
                            reg_cz<4, 10>(a, tp);
                        } else {
                            reg_cz<4, 12>(a, tp);
                        }
                    }
                }
            }
        }
    } else {
        if (kind == 0) {
            if (mask < 9) {
                if (mask < 4) {
                    if (mask < 2) {
                        reg_gate<5, 1, F2>(a, mf);
                    } else {
                        if (mask < 3) {
                            reg_gate<5, 2, F2>(a, mf);
                        } else {
                            reg_gate<5, 3, F2>(a, mf);
                        }
                    }
                } else {
                    if (mask < 6) {
                        if (mask < 5) {
                            reg_gate<5, 4, F2>(a, mf);
                        } else {
                            reg_gate<5, 5, F2>(a, mf);
                        }
                    } else {
                        if (mask < 8) {
                            reg_gate<5, 6, F2>(a, mf);
                        } else {
                            reg_gate<5, 8, F2>(a, mf);
                        }
                    }
                }
            } else {
                if (mask < 17) {
                    if (mask < 12) {
                        if (mask < 10) {
                            reg_gate<5, 9, F2>(a, mf);
                        } else {
                            reg_gate<5, 10, F2>(a, mf);
                        }
                    } else {
                        if (mask < 16) {
                            reg_gate<5, 12, F2>(a, mf);
                        } else {
                            reg_gate<5, 16, F2>(a, mf);
                        }
                    }
                } else {
                    if (mask < 20) {
                        if (mask < 18) {
                            reg_gate<5, 17, F2>(a, mf);
                        } else {
                            reg_gate<5, 18, F2>(a, mf);
                        }
                    } else {
                        if (mask < 24) {
                            reg_gate<5, 20, F2>(a, mf);
                        } else {
                            reg_gate<5, 24, F2>(a, mf);
                        }
                    }
                }
            }
        } else if (kind == 1) {
            if (mask < 9) {
                if (mask < 4) {
                    if (mask < 2) {
                        reg_diag<5, 1>(a, mf);
                    } else {
                        if (mask < 3) {
                            reg_diag<5, 2>(a, mf);
                        } else {
                            reg_diag<5, 3>(a, mf);
                        }
                    }
                } else {
                    if (mask < 6) {
                        if (mask < 5) {
                            reg_diag<5, 4>(a, mf);
                        } else {
                            reg_diag<5, 5>(a, mf);
                        }
                    } else {
                        if (mask < 8) {
                            reg_diag<5, 6>(a, mf);
                        } else {
                            reg_diag<5, 8>(a, mf);
                        }
                    }
                }
            } else {
                if (mask < 17) {
                    if (mask < 12) {
                        if (mask < 10) {
                            reg_diag<5, 9>(a, mf);
                        } else {
                            reg_diag<5, 10>(a, mf);
                        }
                    } else {
                        if (mask < 16) {
                            reg_diag<5, 12>(a, mf);
                        } else {
                            reg_diag<5, 16>(a, mf);
                        }
                    }
                } else {
                    if (mask < 20) {
                        if (mask < 18) {
                            reg_diag<5, 17>(a, mf);
                        } else {
                            reg_diag<5, 18>(a, mf);
                        }
                    } else {
                        if (mask < 24) {
                            reg_diag<5, 20>(a, mf);
                        } else {
                            reg_diag<5, 24>(a, mf);
                        }
                    }
                }
            }
        } else {
            const uint32_t tm = code >> 8;
            const bool tp = (threadIdx.x & tm) == tm;
            if (mask < 9) {
                if (mask < 4) {
                    if (mask < 2) {
                        if (mask < 1) {
                            reg_cz<5, 0>(a, tp);
                        } else {
                            reg_cz<5, 1>(a, tp);
                        }
                    } else {
                        if (mask < 3) {
                            reg_cz<5, 2>(a, tp);
                        } else {
                            reg_cz<5, 3>(a, tp);
                        }
                    }
                } else {
                    if (mask < 6) {
                        if (mask < 5) {
                            reg_cz<5, 4>(a, tp);
                        } else {
                            reg_cz<5, 5>(a, tp);
                        }
                    } else {
                        if (mask < 8) {
                            reg_cz<5, 6>(a, tp);
                        } else {
                            reg_cz<5, 8>(a, tp);
                        }
                    }
                }
            } else {
                if (mask < 17) {
                    if (mask < 12) {
                        if (mask < 10) {
                            reg_cz<5, 9>(a, tp);
                        } else {
                            reg_cz<5, 10>(a, tp);
                        }
                    } else {
                        if (mask < 16) {
                            reg_cz<5, 12>(a, tp);
                        } else {
                            reg_cz<5, 16>(a, tp);
                        }
                    }
                } else {
                    if (mask < 20) {
                        if (mask < 18) {
                            reg_cz<5, 17>(a, tp);
                        } else {
                            reg_cz<5, 18>(a, tp);
                        }
                    } else {
                        if (mask < 24) {
                            reg_cz<5, 20>(a, tp);
                        } else {
                            reg_cz<5, 24>(a, tp);
                        }
                    }
                }
            }
        }
    }
}

#ifndef SVB_RP_STAGES
#define SVB_RP_STAGES 1  // tile buffers per CTA (1: four CTAs per SM at T = 12 measured faster than 2 with three)
#endif
#ifndef SVB_RP_MAXREG5
#define SVB_RP_MAXREG5 128
#endif
#ifndef SVB_RP_PF
#define SVB_RP_PF 0  // L2 prefetch distance in tiles (0: off; 1 and 2 measured 5 % slower at 30q D14)
#endif
__device__ __forceinline__ void prefetch_l2(const void* g) { asm volatile("prefetch.global.L2 [%0];" ::"l"(g)); }
template <int M, bool F2>
__global__ void __launch_bounds__(M == 4 ? 512 : 256) __maxnreg__(M == 4 ? 80 : SVB_RP_MAXREG5) apply_rpass(const __grid_constant__ RpassParams p) {
    constexpr int NA = 1 << M;   // amplitudes per thread
    constexpr int UPT = NA / 2;  // 16 B load/store units per thread
    extern __shared__ float4 rsm[];
    const uint32_t tile_bytes = 8u << p.T;
    const uint32_t s0 = smem_addr(rsm);
    const uint32_t t0 = 2u * threadIdx.x;
    const uint32_t rmask = (1u << p.r) - 1u;
    uint64_t dthr = t0 & rmask;
    {
        const uint32_t h = t0 >> p.r;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1u) dthr += 1ull << p.Hpos[b];
    }
    // unit i of this thread: tile index t0 + 2*nthr*i; its smem byte offset
    // is fold(t0) ^ soff[i] (the fold swizzle is XOR-linear)
    uint32_t sthr = 0;
    {
        uint32_t f = 0;
        for (int q = 4; q < p.T; ++q)
            if ((t0 >> q) & 1u) f ^= 1u << (1 + (q - 4) % 3);
        sthr = (t0 ^ f) << 3;
    }
    auto tbase = [&](uint64_t u) {
        uint64_t x = u << p.r;
        for (int b = 0; b < p.nH; ++b) {
            const int q = p.Hpos[b];
            x = ((x >> q) << (q + 1)) | (x & ((1ull << q) - 1ull));
        }
        return x;
    };
    auto load = [&](const float2* g, uint32_t sbuf) {
#pragma unroll
        for (int i = 0; i < UPT; ++i) cp_async16(sbuf + (sthr ^ p.soff[i]), g + p.goff[i]);
    };
    auto store = [&](float2* g, uint32_t sbuf) {
#pragma unroll
        for (int i = 0; i < UPT; ++i) st_stream(reinterpret_cast<float4*>(g + p.goff[i]), lds4(sbuf + (sthr ^ p.soff[i])));
    };
    uint64_t dgthr = 0, lgthr = 0;
    for (int i = 0; i < p.tbits; ++i)
        if ((threadIdx.x >> i) & 1u) {
            dgthr += p.dgtbw[i];
            lgthr += p.lgtbw[i];
        }
    uint64_t u = blockIdx.x;
    const float2* gcur = nullptr;
    const float2* gtile = nullptr;
    if (u < p.n_tiles) {
        gtile = p.psi + tbase(u);
        gcur = gtile + dthr;
        if (!p.dload && !p.zinit) load(gcur, s0);
    }
    cp_async_commit();
    for (int it = 0; u < p.n_tiles; u += gridDim.x, ++it) {
        const uint32_t cur = s0 + (SVB_RP_STAGES == 2 ? (uint32_t)(it & 1) * tile_bytes : 0u);
        const uint32_t nxt = s0 + (SVB_RP_STAGES == 2 ? (uint32_t)((it + 1) & 1) * tile_bytes : 0u);
        const uint64_t un = u + gridDim.x;
        const float2* gnext = nullptr;
        const float2* gtile_next = nullptr;
        if (un < p.n_tiles) {
            gtile_next = p.psi + tbase(un);
            gnext = gtile_next + dthr;
        }
        if constexpr (SVB_RP_PF > 0) {
            // pull a later tile into L2 while this one is transformed, so that
            // HBM reads stay in flight across the phases (8 threads cover one
            // 128 B line: runs are >= 16 amplitudes)
            const uint64_t up = u + (uint64_t)SVB_RP_PF * gridDim.x;
            if (up < p.n_tiles && !p.zinit && (threadIdx.x & 7u) == 0) {
                const float2* g = p.psi + tbase(up) + dthr;
#pragma unroll
                for (int i = 0; i < UPT; ++i) prefetch_l2(g + p.goff[i]);
            }
        }
        if constexpr (SVB_RP_STAGES == 2) {
            __syncthreads();  // buffer `nxt` drained by the previous store
            if (gnext && !p.zinit) load(gnext, nxt);
            cp_async_commit();
            cp_async_wait1();
        } else {
            cp_async_wait0();
        }
        __syncthreads();
        for (int ph = 0; ph < p.nph; ++ph) {
            const RpPhase& P = p.ph[ph];
            uint32_t tb = 0;
            for (int i = 0; i < p.tbits; ++i)
                if ((threadIdx.x >> i) & 1u) tb ^= P.tbw[i];
            float2 a[NA];
            if (ph == 0 && p.zinit) {
#pragma unroll
                for (int j = 0; j < NA; ++j) a[j] = make_float2(0.f, 0.f);
                if (p.zone && u == 0 && threadIdx.x == 0) a[0].x = 1.f;
            } else if (ph == 0 && p.dload) {
                const float2* g = gtile + lgthr;
#pragma unroll
                for (int j = 0; j < NA / 2; ++j) {
                    const float4 v = ld_stream(reinterpret_cast<const float4*>(g + p.lgoff[j]));
                    a[2 * j] = make_float2(v.x, v.y);
                    a[2 * j + 1] = make_float2(v.z, v.w);
                }
            } else if (P.b0) {
#pragma unroll
                for (int j = 0; j < NA / 2; ++j) {
                    const float4 v = lds4(cur + (tb ^ P.roff[2 * j]));
                    a[2 * j] = make_float2(v.x, v.y);
                    a[2 * j + 1] = make_float2(v.z, v.w);
                }
            } else {
#pragma unroll
                for (int j = 0; j < NA; ++j) a[j] = lds2(cur + (tb ^ P.roff[j]));
            }
            const bool early = SVB_RP_STAGES == 1 && ph == p.nph - 1 && p.direct && !p.dload && !p.zinit && p.early;
            if (early) {
                // the last phase keeps its amplitudes in registers and stores
                // them straight to HBM: once every thread has gathered, the
                // tile buffer is free -- start the next tile's load now so it
                // overlaps this phase's gates
                __syncthreads();
                if (gnext) load(gnext, cur);
                cp_async_commit();
            }
            for (int gi = P.g0; gi < P.g1; ++gi) {
                const uint32_t code = p.gcode[gi];
                reg_gate_dispatch<M, F2>(code, a, p.mats + (code >> 8));
            }
            if (ph == p.nph - 1 && p.direct) {
                float2* g = const_cast<float2*>(gtile) + dgthr;
                if (P.b0) {
#pragma unroll
                    for (int j = 0; j < NA / 2; ++j)
                        st_stream(reinterpret_cast<float4*>(g + p.dgoff[j]),
                                  make_float4(a[2 * j].x, a[2 * j].y, a[2 * j + 1].x, a[2 * j + 1].y));
                } else {
                    // tile bits 0..3 on lanes 0..3: each half-warp writes one 128 B run
#pragma unroll
                    for (int j = 0; j < NA; ++j) st_stream2(g + p.dgoff[j], a[j]);
                }
                break;  // the next iteration's first barrier guards `cur`
            }
            if (P.b0) {
#pragma unroll
                for (int j = 0; j < NA / 2; ++j)
                    sts4(cur + (tb ^ P.roff[2 * j]), make_float4(a[2 * j].x, a[2 * j].y, a[2 * j + 1].x, a[2 * j + 1].y));
            } else {
#pragma unroll
                for (int j = 0; j < NA; ++j) sts2(cur + (tb ^ P.roff[j]), a[j]);
            }
            __syncthreads();
        }
        if (!p.direct) store(const_cast<float2*>(gcur), cur);
        if constexpr (SVB_RP_STAGES == 1) {
            if (!p.dload && !p.zinit && !(p.direct && p.early)) {
                __syncthreads();  // every thread is done with the tile buffer
                if (gnext) load(gnext, cur);
                cp_async_commit();
            }
        }
        gcur = gnext;
        gtile = gtile_next;
    }
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

// ---------------------------------------------- register-blocked pass (host)
namespace svb {

uint32_t fold_swz(uint32_t t, int T) {
    uint32_t f = 0;
    for (int q = 4; q < T; ++q)
        if ((t >> q) & 1u) f ^= 1u << (1 + (q - 4) % 3);
    return t ^ f;
}
// 16 B chunk bank bit (0..2) that tile position q moves under the fold swizzle
int bank_class(int q) { return q == 0 ? -1 : (q <= 3 ? q - 1 : (q - 4) % 3); }

uint32_t deposit(uint32_t v, const std::vector<int>& pos) {
    uint32_t x = 0;
    for (size_t b = 0; b < pos.size(); ++b)
        if ((v >> b) & 1u) x |= 1u << pos[b];
    return x;
}

int rpass_m() { return SVB_RP_M; }

// 0 dense, 1 diagonal, 2 CZ-like (diag(1, 1, 1, -1)), exact in fp32
int gate_kind(const PassDesc& pd, const PassGate& pg) {
    if (pg.kind >= 0) return pg.kind;
    const int D = 1 << pg.k;
    const float* mg = pd.mats.data() + pg.moff;  // (re, im) row-major
    bool diag = true, cz = pg.k == 2;
    for (int r = 0; r < D; ++r)
        for (int c = 0; c < D; ++c) {
            const float re = mg[2 * (r * D + c)], im = mg[2 * (r * D + c) + 1];
            if (r != c && (re != 0.f || im != 0.f)) diag = cz = false;
            if (r == c && (im != 0.f || re != (r == D - 1 ? -1.f : 1.f))) cz = false;
        }
    return cz ? 2 : diag ? 1 : 0;
}

// Phases of gates [g0, g1): each phase takes, in order, every remaining gate
// whose positions fit in the phase's M-set and that does not touch a position
// of a gate skipped before it (so it only moves past gates it commutes with).
std::vector<RpPhaseHost> plan_phases(const PassDesc& pd, size_t g0, size_t g1, int M, bool wide) {
    const int T = (int)pd.S.size();
    std::vector<RpPhaseHost> out;
    std::vector<int> rem;
    for (size_t g = g0; g < g1; ++g) rem.push_back((int)g);
    std::vector<uint32_t> gm(pd.gates.size(), 0);
    for (size_t g = g0; g < g1; ++g)
        for (int b = 0; b < pd.gates[g].k; ++b) gm[g] |= 1u << pd.gates[g].pos[b];
    auto gmask = [&](int g) { return gm[g]; };
    // CZ-like gates run in any layout (their qubits may be thread bits)
    std::vector<char> anyl(pd.gates.size(), 0);
    for (size_t g = g0; g < g1; ++g) anyl[g] = gate_kind(pd, pd.gates[g]) == 2;
    while (!rem.empty()) {
        RpPhaseHost ph;
        // R = the M-subset of tile positions that lets the most remaining
        // gates run in this phase (a gate runs if its positions are in R and
        // it touches no position of a gate skipped before it); ties prefer
        // tile bit 0 in R (16 B gathers), then R free of bits 1..3 (lanes
        // 0..2 = bits 1..3: direct-store layout)
        uint32_t used = 0;
        int best = -1;
        // remaining gates as flat arrays (the subset loop below is the hot spot)
        std::vector<uint32_t> rm(rem.size());
        std::vector<char> ra(rem.size());
        for (size_t i = 0; i < rem.size(); ++i) {
            rm[i] = gm[rem[i]];
            ra[i] = anyl[rem[i]];
        }
        const size_t nr = rem.size();
        for (uint32_t R = (1u << M) - 1u; R < (1u << T);) {
            int cnt = 0, czin = 0;
            uint32_t blocked = 0;
            for (size_t i = 0; i < nr; ++i) {
                const uint32_t m = rm[i];
                if (!(m & blocked) && (ra[i] || !(m & ~R))) {
                    ++cnt;
                    czin += ra[i] && !(m & ~R);
                } else {
                    blocked |= m;
                }
            }
            // wide (16 B complex128 amplitudes): ties prefer R free of bits
            // 0..2 (lanes 0..2 = bits 0..2: conflict-free, direct-store layout).
            // complex64: ties prefer more CZ-like gates with both qubits in R
            // (sign bookkeeping in the pass kernels instead of FMUL2s by a
            // per-thread sign), then tile bit 0 in R, then the direct layout
            const int score = wide ? 4 * cnt + ((R & 0x7u) ? 0 : 1)
                                   : 64 * cnt + 4 * std::min(czin, 15) * SVB_RP_CZBONUS + ((R & 1u) ? 2 : 0) +
                                         ((R & 0xEu) ? 0 : 1);
            if (score > best) {
                best = score;
                used = R;
            }
            const uint32_t c = R & (0u - R), r = R + c;  // next subset of the same size (Gosper)
            R = (((r ^ R) >> 2) / c) | r;
        }
        {
            uint32_t blocked = 0;
            std::vector<int> keep;
            for (int g : rem) {
                const uint32_t m = gmask(g);
                if (!(m & blocked) && (anyl[g] || !(m & ~used))) {
                    ph.gates.push_back(g);
                } else {
                    blocked |= m;
                    keep.push_back(g);
                }
            }
            rem.swap(keep);
        }
        for (int q = 0; q < T; ++q)
            if ((used >> q) & 1u) ph.R.push_back(q);
        ph.b0 = !wide && (used & 1u) != 0;
        if (wide) {
            // 16 B per amplitude: the first 3 lanes (a quarter-warp of LDS.128)
            // must move distinct chunk bits under the wide fold swizzle
            // (class q % 3), lowest positions first
            std::vector<int> rest, lanes;
            for (int q = 0; q < T; ++q)
                if (!((used >> q) & 1u)) rest.push_back(q);
            int have = 0;
            for (size_t i = 0; i < rest.size() && have != 7;) {
                const int c = rest[i] % 3;
                if (!((have >> c) & 1)) {
                    have |= 1 << c;
                    lanes.push_back(rest[i]);
                    rest.erase(rest.begin() + (long)i);
                } else {
                    ++i;
                }
            }
            lanes.insert(lanes.end(), rest.begin(), rest.end());
            ph.lanes = lanes;
            out.push_back(ph);
            continue;
        }
        // lanes: the first lanes of a quarter- (16 B) / half-warp (8 B) must
        // move distinct bank bits
        std::vector<int> rest;
        for (int q = 0; q < T; ++q)
            if (!((used >> q) & 1u)) rest.push_back(q);
        std::vector<int> lanes;
        if (!ph.b0) {
            lanes.push_back(0);
            rest.erase(rest.begin());
        }
        int have = 0;
        for (size_t i = 0; i < rest.size() && have != 7;) {
            const int c = bank_class(rest[i]);
            if (c >= 0 && !((have >> c) & 1)) {
                have |= 1 << c;
                lanes.push_back(rest[i]);
                rest.erase(rest.begin() + (long)i);
            } else {
                ++i;
            }
        }
        lanes.insert(lanes.end(), rest.begin(), rest.end());
        ph.lanes = lanes;
        out.push_back(ph);
    }
    return out;
}

std::vector<std::pair<size_t, size_t>> rpass_chunks(const PassDesc& pd, int M, bool wide) {
    std::vector<std::pair<size_t, size_t>> out;
    const size_t ng = pd.gates.size();
    size_t g0 = 0;
    while (g0 < ng) {
        size_t g1 = std::min(ng, g0 + (size_t)kRpMaxGates);
        if ((int)plan_phases(pd, g0, g1, M, wide).size() > kRpMaxPhases) {
            // the first kRpMaxPhases phases hold a prefix of the gates only if
            // no gate was moved past a later phase: re-plan a shorter prefix
            size_t cut = g1;
            do {
                cut = g0 + (cut - g0) / 2;
            } while ((int)plan_phases(pd, g0, cut, M, wide).size() > kRpMaxPhases);
            g1 = cut;
        }
        out.push_back({g0, g1});
        g0 = g1;
    }
    return out;
}

namespace {

// worst bank-conflict degree of a phase's gathers (warp 0, every register j)
int phase_conflicts(const RpPhaseHost& ph, int T, int M) {
    int worst = 1;
    for (uint32_t j = 0; j < (1u << M); j += ph.b0 ? 2 : 1) {
        const int group = ph.b0 ? 8 : 16;
        for (int l0 = 0; l0 < 32; l0 += group) {
            int cnt[16] = {0};
            for (int l = l0; l < l0 + group; ++l) {
                const uint32_t slot = fold_swz(deposit(j, ph.R) | deposit((uint32_t)l, ph.lanes), T);
                const int bank = ph.b0 ? (int)((slot >> 1) & 7) : (int)(slot & 15);
                worst = std::max(worst, ++cnt[bank]);
            }
        }
    }
    return worst;
}

template <int M, bool F2>
cudaError_t launch_rpass_m(float2* psi, int n, const PassDesc& pd, cudaStream_t st, bool zinit, bool zone, int slot) {
    const float* mats = pd.mats_shard.empty() ? pd.mats.data() : pd.mats_shard[slot].data();
    const int T = (int)pd.S.size();
    const uint32_t nthr = 1u << (T - M);
    const size_t smem = SVB_RP_STAGES * ((size_t)8 << T);
    cudaError_t e = cudaFuncSetAttribute(apply_rpass<M, F2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    static int per_sm_cache[16] = {0};
    if (!per_sm_cache[T]) {
        int nb = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, apply_rpass<M, F2>, (int)nthr, smem);
        if (e != cudaSuccess) return e;
        per_sm_cache[T] = std::max(1, nb);
    }
    RpassParams* pp = new RpassParams;
    RpassParams& p = *pp;
    std::memset(&p, 0, sizeof(p));
    p.psi = psi;
    p.T = T;
    p.r = pd.r;
    p.nH = 0;
    for (int i = pd.r; i < T; ++i) p.Hpos[p.nH++] = pd.S[i];
    p.tbits = T - M;
    auto dep = [&](uint64_t t) {
        uint64_t g = t & ((1ull << p.r) - 1);
        const uint64_t h = t >> p.r;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1) g += 1ull << p.Hpos[b];
        return g;
    };
    for (int i = 0; i < (1 << (M - 1)); ++i) {
        p.goff[i] = dep(2ull * nthr * i);
        p.soff[i] = fold_swz(2u * nthr * i, T) << 3;
    }
    p.n_tiles = 1ull << (n - T);
    const uint64_t grid = std::min<uint64_t>(p.n_tiles, (uint64_t)pass_sms() * per_sm_cache[T]);
    // gates in chunks that fit the parameter block (one launch each)
    for (const auto& ch : rpass_chunks(pd, M)) {
        if (e != cudaSuccess) break;
        const size_t g0 = ch.first, g1 = ch.second;
        auto phs = plan_phases(pd, g0, g1, M);
        p.nph = (int)phs.size();
        uint32_t moff = 0;
        int li = 0;
        for (int i = 0; i < p.nph; ++i) {
            const RpPhaseHost& h = phs[i];
            RpPhase& P = p.ph[i];
            P.g0 = (uint16_t)li;
            P.b0 = h.b0 ? 1u : 0u;
            for (uint32_t j = 0; j < (1u << M); ++j) P.roff[j] = fold_swz(deposit(j, h.R), T) << 3;
            for (int b = 0; b < p.tbits; ++b) P.tbw[b] = fold_swz(1u << h.lanes[b], T) << 3;
            for (int g : h.gates) {
                const PassGate& pg = pd.gates[g];
                const int D = 1 << pg.k;
                const float* mg = mats + pg.moff;  // (re, im) row-major
                const int kind = gate_kind(pd, pg);
                const int ne = kind == 1 ? D : kind == 2 ? 0 : D * D;
                for (int e2 = 0; e2 < ne; ++e2) {
                    const int src = kind == 1 ? e2 * D + e2 : e2;
                    const float mr = mg[2 * src], mi = mg[2 * src + 1];
                    p.mats[moff + 4 * e2 + 0] = mr;
                    p.mats[moff + 4 * e2 + 1] = mr;
                    p.mats[moff + 4 * e2 + 2] = -mi;
                    p.mats[moff + 4 * e2 + 3] = mi;
                }
                uint32_t mask = 0, tmask = 0;
                for (int b = 0; b < pg.k; ++b) {
                    const auto it = std::find(h.R.begin(), h.R.end(), pg.pos[b]);
                    if (it != h.R.end()) mask |= 1u << (int)(it - h.R.begin());
                    else tmask |= 1u << (int)(std::find(h.lanes.begin(), h.lanes.end(), pg.pos[b]) - h.lanes.begin());
                }
                p.gcode[li++] = mask | ((uint32_t)kind << 5) | ((kind == 2 ? tmask : moff) << 8);
                moff += 4 * ne;
            }
            P.g1 = (uint16_t)li;
        }
        if (SVB_RP_DEBUG) {
            int w = 1;
            for (auto& x : phs) w = std::max(w, phase_conflicts(x, T, M));
            int nb0 = 0;
            for (auto& x : phs) nb0 += x.b0;
            fprintf(stderr, "rpass T=%d M=%d gates=%zu phases=%d b0=%d worst_conflict=%d S=", T, M, g1 - g0, p.nph, nb0, w);
            for (int q : pd.S) fprintf(stderr, "%d,", q);
            fprintf(stderr, "\n");
        }
        {
            auto coalesced = [](const RpPhaseHost& h) {
                return h.b0 && h.lanes.size() >= 3 && h.lanes[0] == 1 && h.lanes[1] == 2 && h.lanes[2] == 3;
            };
            auto coalesced8 = [](const RpPhaseHost& h) {
                return !h.b0 && h.lanes.size() >= 4 && h.lanes[0] == 0 && h.lanes[1] == 1 && h.lanes[2] == 2 &&
                       h.lanes[3] == 3;
            };
            const RpPhaseHost& lp = phs.back();
            p.direct = SVB_RP_DIRECT && (coalesced(lp) || coalesced8(lp));
            if (p.direct) {
                if (lp.b0)
                    for (int j = 0; j < (1 << (M - 1)); ++j) p.dgoff[j] = dep(deposit(2u * j, lp.R));
                else
                    for (int j = 0; j < (1 << M); ++j) p.dgoff[j] = dep(deposit((uint32_t)j, lp.R));
                for (int b = 0; b < p.tbits; ++b) p.dgtbw[b] = dep(1ull << lp.lanes[b]);
            }
            const RpPhaseHost& fp = phs.front();
            // measured 1.5 % slower on 30q F=1 (the load latency is no longer
            // hidden behind the other CTAs' phases): build option SVB_RP_DLOAD=1
            p.dload = SVB_RP_DLOAD && SVB_RP_STAGES == 1 && coalesced(fp);
            p.early = SVB_RP_EARLY;
            p.zinit = zinit && g0 == 0;  // only the first launch of a split pass starts from |0...0>
            p.zone = zone ? 1 : 0;
            if (p.dload) {
                for (int j = 0; j < (1 << (M - 1)); ++j) p.lgoff[j] = dep(deposit(2u * j, fp.R));
                for (int b = 0; b < p.tbits; ++b) p.lgtbw[b] = dep(1ull << fp.lanes[b]);
            }
        }
        if (SVB_RP_DEBUG) fprintf(stderr, "   direct=%d dload=%d\n", p.direct, p.dload);
        apply_rpass<M, F2><<<(unsigned)grid, nthr, smem, st>>>(p);
        e = cudaGetLastError();
    }
    delete pp;
    return e;
}

}  // namespace

bool rpass_supported(const PassDesc& pd) {
    if (!SVB_RP_ENABLE) return false;
    const int T = (int)pd.S.size();
    if (T < 10 || T > 14 || pd.r < 1) return false;  // 14: pass-specialised kernels only
    for (auto& g : pd.gates)
        if (g.k > 2) return false;
    return true;
}

uint64_t rpass_fma_per_amp(const PassDesc& pd) {
    uint64_t f = 0;
    for (auto& g : pd.gates) {
        const int kind = gate_kind(pd, g);
        f += kind == 0 ? 4ull << g.k : kind == 1 ? 4 : 0;
    }
    return f;
}

void rpass_phase_plan(const PassDesc& pd, std::vector<std::vector<int>>& R, std::vector<std::vector<int>>& gates) {
    auto ph = plan_phases(pd, 0, pd.gates.size(), rpass_m());
    R.clear();
    gates.clear();
    for (auto& x : ph) {
        R.push_back(x.R);
        gates.push_back(x.gates);
    }
}

void rpass_plan_stats(const PassDesc& pd, int* n_phases, int* worst_conflict) {
    const int M = rpass_m();
    auto ph = plan_phases(pd, 0, pd.gates.size(), M);
    int w = 1;
    for (auto& x : ph) w = std::max(w, phase_conflicts(x, (int)pd.S.size(), M));
    if (n_phases) *n_phases = (int)ph.size();
    if (worst_conflict) *worst_conflict = w;
}

cudaError_t launch_rpass(float2* psi, int n, const PassDesc& pd, cudaStream_t st, bool zinit, bool zone, int slot) {
    static_assert(sizeof(RpassParams) <= 32764, "rpass params exceed the kernel parameter space");
    constexpr bool f2 = SVB_RP_F2 != 0;
    if (pd.S.size() > 13) return cudaErrorInvalidValue;  // 14-qubit tiles: pass-specialised kernels only
    if (rpass_m() == 5) return f2 ? launch_rpass_m<5, true>(psi, n, pd, st, zinit, zone, slot) : launch_rpass_m<5, false>(psi, n, pd, st, zinit, zone, slot);
    return f2 ? launch_rpass_m<4, true>(psi, n, pd, st, zinit, zone, slot) : launch_rpass_m<4, false>(psi, n, pd, st, zinit, zone, slot);
}

}  // namespace svb
