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
#include <cuda.h>  // CUtensorMap (the encoder is fetched with cudaGetDriverEntryPoint)
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>

#include "device_util.cuh"
#include "kernels.h"

// Build options (compile-time; A/B variants via build.py --variant):
#ifndef SVB_TF32X3
#define SVB_TF32X3 0  // TF32x3 tensor-core path (biased): quarantined, off
#endif
#ifndef SVB_WS
#define SVB_WS 1  // bulk/tensor-copy (warp-specialised) tile loop
#endif
#ifndef SVB_WS_UNSWZ
#define SVB_WS_UNSWZ -1  // low gates on the bulk-copy loop: -1 conflict model, 0 never, 1 always
#endif
#ifndef SVB_SWZ128
#define SVB_SWZ128 1  // allow the TMA 128 B swizzle layout
#endif
#ifndef SVB_WS_MINRUN
#define SVB_WS_MINRUN 2048u  // shortest run (bytes) moved by per-run bulk copies
#endif
#ifndef SVB_TMAP
#define SVB_TMAP -1  // tensor-map tile copies: -1 auto, 0 never, 1 always
#endif

namespace svb {

namespace {

using namespace dev;


// y += m * a (complex), 4 FFMA.
__device__ __forceinline__ void cmac(float2& y, const float2 m, const float2 a) {
    y.x = fmaf(m.x, a.x, y.x);
    y.x = fmaf(-m.y, a.y, y.x);
    y.y = fmaf(m.x, a.y, y.y);
    y.y = fmaf(m.y, a.x, y.y);
}

// Fused matrix as three real planes for the 3-multiplication complex product
// (Gauss): with m = p + iq and a = x + iy,
//   A = sum_c p_c (x_c + y_c),  B = sum_c (p_c + q_c) y_c,  C = sum_c (q_c - p_c) x_c,
//   Re y = A - B,  Im y = A + C.
// 3 FMAs per complex multiply-add instead of 4 (k <= 5, planes in the kernel
// parameters).  k = 6 keeps the plain 4-FMA form with the matrix in shared
// memory (3 planes of 64 x 64 would not fit next to the tile).
template <int K>
struct MatStore {
    alignas(16) float P[1 << K][1 << K];
    alignas(16) float S[1 << K][1 << K];
    alignas(16) float Q[1 << K][1 << K];
    float2 cm[1 << K][1 << K];  // complex64 matrix (tensor-core path builds its B operand from it)
};
template <>
struct MatStore<6> {  // 32 KB complex: does not fit the 32764 B parameter space
    const float2* dev;
};

#ifndef SV_ROWS
#define SV_ROWS 1  // output rows per (non-unrolled) row-loop iteration
#endif
#ifndef SVB_WS_STAGES
#define SVB_WS_STAGES 2  // SIMT bulk-copy loop: tile buffers
#endif
#ifndef SVB_SMEM_PLANES
#define SVB_SMEM_PLANES 1  // dense k = 2, 3 SIMT: Gauss planes read from shared memory (LDS.128)
#endif

// ------------------------------------------------------------------ kernels
// A tile is the set of 2^nH runs of 2^r contiguous amplitudes that share
// every bit outside {0..r-1} u H (H = gate qubits >= r); it holds complete
// groups, so the gate is applied entirely inside shared memory.  Tile index
// t (0 <= t < 2^T) maps to the global offset dep(t) = (t mod 2^r) + deposit of
// (t >> r) into H, and to the swizzled shared-memory slot phys(t); both maps
// are additive/XOR-linear over disjoint bits, so per-unit offsets are
// precomputed on the host and a thread adds/XORs them to its own base.
template <int K>
struct alignas(64) TileParams {
    MatStore<K> M;                     // first: 16 B aligned in the constant bank (LDCU.128)
    float2* psi;
    uint64_t n_tiles;
    int T, r;                          // tile bits, run bits
    int nH;
    int Hpos[SV_MAX_FUSED];            // gate qubits >= r (ascending, global positions)
    int nzt;
    int ztpos[SV_MAX_FUSED];           // tile-local gate bit positions, ascending
    uint32_t zthigh[SV_MAX_FUSED];     // ~0u << ztpos[b]
    uint32_t swz[3];                   // phys bit (i+1) ^= parity(t & swz[i])
    int nZ;                            // tile-base zero insertions: H and control qubits, ascending
    uint64_t Zhigh[2 * SV_MAX_FUSED];  // ~0 << Zpos[b]: inserting a zero at q is x += x & (~0 << q)
    uint64_t ones;                     // control qubits forced to 1 in the tile base
    int upt;                           // 16-byte units per thread per tile
    int iters;                         // compute iterations per thread per tile
    uint64_t goff[64];                 // 8 * dep(2 * nthreads * i)  (bytes)
    uint32_t soff[64];                 // phys(2 * nthreads * i)
    uint32_t loc[1 << K];              // phys offsets of the gathers (members / member pairs)
    uint32_t gsec;                     // phys offset of the second group of a pair (PAIR, 2 groups)
    const uint8_t* wi8;                // tensor-core int8 path: W slices + column exponents (device)
    uint64_t roff[64];                 // bulk-copy path: byte offset of run j (dep(j << r))
    int trank;                         // tensor-copy path: rank (0 = per-run bulk copies)
    int tstart[5], tbits[5];           // dim d covers index bits [tstart[d], tstart[d] + tbits[d])
    int tnx;                           // gate qubits left out of the box: 2^tnx copies per tile
    int txpos[SV_MAX_FUSED];           // their positions (ascending)
    CUtensorMap tmap;                  // tensor map of the state for this gate's tile shape
    // monomial matrices (one nonzero per row: permutations, diagonals, identity)
    int mono;
    uint32_t mloc[1 << K];             // phys offset of member r (output slot of row r)
    uint32_t ploc[1 << K];             // phys offset of the source member of row r
    float2 mdiag[1 << K];              // the nonzero of row r
};

// Swizzled shared-memory slot of tile-local group index g: zeros inserted at
// the K gate positions (ascending; inserting a zero at q is x += x & (~0 << q))
// -- 2 instructions per position in 32-bit arithmetic.
template <int K>
__device__ __forceinline__ uint32_t slot_of(const TileParams<K>& p, uint32_t g) {
#pragma unroll
    for (int b = 0; b < K; ++b) g += g & p.zthigh[b];
    return swizzle(g, p.swz);
}

// Gauss form of output rows [r0, r0 + R) for one group (s[c] = x_c + y_c).
// The row loop of the callers is NOT unrolled: each iteration is a scheduling
// fence, so ptxas cannot interleave all rows (which needs 6 accumulators per
// row live at once and spills at k >= 4).  Matrix operands are warp-uniform
// constant-bank loads (LDCU) feeding FFMA uniform-register operands.
template <int K, int R>
__device__ __forceinline__ void gauss_block(const MatStore<K>& M, int r0, const float2* a, const float* s, float2* y) {
    constexpr int D = 1 << K;
#pragma unroll
    for (int i = 0; i < R; ++i) {
        float A = 0.f, B = 0.f, C = 0.f;
#pragma unroll
        for (int c = 0; c < D; ++c) {
            A = fmaf(M.P[r0 + i][c], s[c], A);
            B = fmaf(M.S[r0 + i][c], a[c].y, B);
            C = fmaf(M.Q[r0 + i][c], a[c].x, C);
        }
        y[i] = make_float2(A - B, A + C);
    }
}

template <int K, int R>
__device__ __forceinline__ void gauss_block2(const MatStore<K>& M, int r0, const float2* a0, const float* s0,
                                             const float2* a1, const float* s1, float2* y0, float2* y1,
                                             uint32_t splanes = 0) {
    constexpr int D = 1 << K;
#pragma unroll
    for (int i = 0; i < R; ++i) {
        float A0 = 0.f, B0 = 0.f, C0 = 0.f, A1 = 0.f, B1 = 0.f, C1 = 0.f;
#if SVB_SMEM_PLANES
        if constexpr (D >= 4 && D <= 8) {
            // planes staged in shared memory: one broadcast LDS.128 per 4 operands
            // (the constant-bank path issues LDCU.64, twice as many loads)
            const uint32_t rowP = splanes + 4u * (uint32_t)((r0 + i) * D);
#pragma unroll
            for (int c4 = 0; c4 < D / 4; ++c4) {
                const float4 pv = lds4(rowP + 16u * c4);
                const float4 sv = lds4(rowP + 4u * D * D + 16u * c4);
                const float4 qv = lds4(rowP + 8u * D * D + 16u * c4);
                const float pp[4] = {pv.x, pv.y, pv.z, pv.w}, ss[4] = {sv.x, sv.y, sv.z, sv.w},
                            qq[4] = {qv.x, qv.y, qv.z, qv.w};
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int c = 4 * c4 + j;
                    A0 = fmaf(pp[j], s0[c], A0);
                    A1 = fmaf(pp[j], s1[c], A1);
                    B0 = fmaf(ss[j], a0[c].y, B0);
                    B1 = fmaf(ss[j], a1[c].y, B1);
                    C0 = fmaf(qq[j], a0[c].x, C0);
                    C1 = fmaf(qq[j], a1[c].x, C1);
                }
            }
            y0[i] = make_float2(A0 - B0, A0 + C0);
            y1[i] = make_float2(A1 - B1, A1 + C1);
            continue;
        }
#endif
        (void)splanes;
#pragma unroll
        for (int c = 0; c < D; ++c) {
            const float p = M.P[r0 + i][c], sq = M.S[r0 + i][c], q = M.Q[r0 + i][c];
            A0 = fmaf(p, s0[c], A0);
            A1 = fmaf(p, s1[c], A1);
            B0 = fmaf(sq, a0[c].y, B0);
            B1 = fmaf(sq, a1[c].y, B1);
            C0 = fmaf(q, a0[c].x, C0);
            C1 = fmaf(q, a1[c].x, C1);
        }
        y0[i] = make_float2(A0 - B0, A0 + C0);
        y1[i] = make_float2(A1 - B1, A1 + C1);
    }
}

// One group, rows one by one (small-state fallback).
template <int K, class Emit>
__device__ __forceinline__ void gauss_rows(const MatStore<K>& M, const float2* a, Emit&& emit) {
    constexpr int D = 1 << K;
    float s[D];
#pragma unroll
    for (int c = 0; c < D; ++c) s[c] = a[c].x + a[c].y;
#pragma unroll 1
    for (int r = 0; r < D; ++r) {
        float2 y;
        gauss_block<K, 1>(M, r, a, s, &y);
        emit(r, y);
    }
}

// GPT (groups per thread) = 2 for k <= 4, else 1.  PAIR: tile bit 0 is a gate
// bit, so a 16 B shared-memory word holds members 2j, 2j+1 of one group;
// otherwise (GPT = 2) it holds the same member of two neighbouring groups.
// y_r = m_r * a_{perm(r)}: exact for entries in {+-1, +-i} (identity,
// permutation and CZ-like matrices).  All sources are read before any output
// is written (in place).
__device__ __forceinline__ float2 cmul(float2 m, float2 a) {
    return make_float2(fmaf(m.x, a.x, -(m.y * a.y)), fmaf(m.x, a.y, m.y * a.x));
}

template <int K, bool PAIR>
__device__ __forceinline__ void tile_compute_mono(const TileParams<K>& p, uint32_t sbuf, uint32_t pb0,
                                                  uint32_t nt = blockDim.x) {
    constexpr int D = 1 << K;
    constexpr int GPT = (K <= 4) ? 2 : 1;
    for (int j = 0; j < p.iters; ++j) {
        const uint32_t gidx = threadIdx.x + (uint32_t)j * nt;
        if constexpr (GPT == 2 && !PAIR) {
            const uint32_t pb = j == 0 ? pb0 : slot_of<K>(p, gidx << 1);
            float4 v[D];
#pragma unroll
            for (int r = 0; r < D; ++r) v[r] = lds4(sbuf + ((pb ^ p.ploc[r]) << 3));
#pragma unroll
            for (int r = 0; r < D; ++r) {
                const float2 y0 = cmul(p.mdiag[r], make_float2(v[r].x, v[r].y));
                const float2 y1 = cmul(p.mdiag[r], make_float2(v[r].z, v[r].w));
                sts4(sbuf + ((pb ^ p.mloc[r]) << 3), make_float4(y0.x, y0.y, y1.x, y1.y));
            }
        } else {
            const uint32_t pb = j == 0 ? pb0 : (GPT == 2) ? slot_of<K>(p, gidx << 1) : slot_of<K>(p, gidx);
#pragma unroll
            for (int gg = 0; gg < GPT; ++gg) {
                const uint32_t b = gg ? (pb ^ p.gsec) : pb;
                float2 v[D];
#pragma unroll
                for (int r = 0; r < D; ++r) v[r] = lds2(sbuf + ((b ^ p.ploc[r]) << 3));
#pragma unroll
                for (int r = 0; r < D; ++r) sts2(sbuf + ((b ^ p.mloc[r]) << 3), cmul(p.mdiag[r], v[r]));
            }
        }
    }
}

template <int K, bool PAIR>
__device__ __forceinline__ void tile_compute(const TileParams<K>& p, uint32_t sbuf, const float2* smat, uint32_t pb0,
                                             uint32_t splanes, uint32_t nt = blockDim.x) {
    constexpr int D = 1 << K;
    constexpr int GPT = (K <= 4) ? 2 : 1;
    for (int j = 0; j < p.iters; ++j) {
        const uint32_t gidx = threadIdx.x + (uint32_t)j * nt;
        if constexpr (GPT == 2) {
            const uint32_t pb = j == 0 ? pb0 : slot_of<K>(p, gidx << 1);
            float2 a0[D], a1[D];
            float s0[D], s1[D];
            if constexpr (PAIR) {
#pragma unroll
                for (int jj = 0; jj < D / 2; ++jj) {
                    const float4 v0 = lds4(sbuf + ((pb ^ p.loc[jj]) << 3));
                    const float4 v1 = lds4(sbuf + ((pb ^ p.gsec ^ p.loc[jj]) << 3));
                    a0[2 * jj] = make_float2(v0.x, v0.y);
                    a0[2 * jj + 1] = make_float2(v0.z, v0.w);
                    a1[2 * jj] = make_float2(v1.x, v1.y);
                    a1[2 * jj + 1] = make_float2(v1.z, v1.w);
                }
            } else {
#pragma unroll
                for (int c = 0; c < D; ++c) {
                    const float4 v = lds4(sbuf + ((pb ^ p.loc[c]) << 3));
                    a0[c] = make_float2(v.x, v.y);
                    a1[c] = make_float2(v.z, v.w);
                }
            }
#pragma unroll
            for (int c = 0; c < D; ++c) {
                s0[c] = a0[c].x + a0[c].y;
                s1[c] = a1[c].x + a1[c].y;
            }
            if constexpr (PAIR) {
#pragma unroll 1
                for (int r2 = 0; r2 < D / 2; ++r2) {
                    float2 y0[2], y1[2];
                    gauss_block2<K, 2>(p.M, 2 * r2, a0, s0, a1, s1, y0, y1, splanes);
                    sts4(sbuf + ((pb ^ p.loc[r2]) << 3), make_float4(y0[0].x, y0[0].y, y0[1].x, y0[1].y));
                    sts4(sbuf + ((pb ^ p.gsec ^ p.loc[r2]) << 3), make_float4(y1[0].x, y1[0].y, y1[1].x, y1[1].y));
                }
            } else {
#pragma unroll 1
                for (int r = 0; r < D; r += SV_ROWS) {
                    float2 y0[SV_ROWS], y1[SV_ROWS];
                    gauss_block2<K, SV_ROWS>(p.M, r, a0, s0, a1, s1, y0, y1, splanes);
#pragma unroll
                    for (int i = 0; i < SV_ROWS; ++i)
                        sts4(sbuf + ((pb ^ p.loc[r + i]) << 3), make_float4(y0[i].x, y0[i].y, y1[i].x, y1[i].y));
                }
            }
        } else {
            const uint32_t pb = j == 0 ? pb0 : slot_of<K>(p, gidx);
            float2 a[D];
            if constexpr (PAIR) {
#pragma unroll
                for (int jj = 0; jj < D / 2; ++jj) {
                    const float4 v = lds4(sbuf + ((pb ^ p.loc[jj]) << 3));
                    a[2 * jj] = make_float2(v.x, v.y);
                    a[2 * jj + 1] = make_float2(v.z, v.w);
                }
            } else {
#pragma unroll
                for (int c = 0; c < D; ++c) a[c] = lds2(sbuf + ((pb ^ p.loc[c]) << 3));
            }
            if constexpr (K <= 5) {
                float s[D];
#pragma unroll
                for (int c = 0; c < D; ++c) s[c] = a[c].x + a[c].y;
                if constexpr (PAIR) {
#pragma unroll 1
                    for (int r2 = 0; r2 < D / 2; ++r2) {
                        float2 y[2];
                        gauss_block<K, 2>(p.M, 2 * r2, a, s, y);
                        sts4(sbuf + ((pb ^ p.loc[r2]) << 3), make_float4(y[0].x, y[0].y, y[1].x, y[1].y));
                    }
                } else {
#pragma unroll 1
                    for (int r = 0; r < D; ++r) {
                        float2 y;
                        gauss_block<K, 1>(p.M, r, a, s, &y);
                        sts2(sbuf + ((pb ^ p.loc[r]) << 3), y);
                    }
                }
            } else {
                // k = 6: rows in a loop, matrix rows broadcast from shared memory
#pragma unroll 1
                for (int r2 = 0; r2 < D / 2; ++r2) {
                    float2 y0 = make_float2(0.f, 0.f), y1 = make_float2(0.f, 0.f);
                    const float4* m0 = reinterpret_cast<const float4*>(smat + (2 * r2) * D);
                    const float4* m1 = reinterpret_cast<const float4*>(smat + (2 * r2 + 1) * D);
#pragma unroll
                    for (int c2 = 0; c2 < D / 2; ++c2) {
                        const float4 u0 = m0[c2], u1 = m1[c2];
                        cmac(y0, make_float2(u0.x, u0.y), a[2 * c2]);
                        cmac(y0, make_float2(u0.z, u0.w), a[2 * c2 + 1]);
                        cmac(y1, make_float2(u1.x, u1.y), a[2 * c2]);
                        cmac(y1, make_float2(u1.z, u1.w), a[2 * c2 + 1]);
                    }
                    if constexpr (PAIR) {
                        sts4(sbuf + ((pb ^ p.loc[r2]) << 3), make_float4(y0.x, y0.y, y1.x, y1.y));
                    } else {
                        sts2(sbuf + ((pb ^ p.loc[2 * r2]) << 3), y0);
                        sts2(sbuf + ((pb ^ p.loc[2 * r2 + 1]) << 3), y1);
                    }
                }
            }
        }
    }
}

// ------------------------------------------------------------- tensor cores
// Dense k = 4, 5 gates on tcgen05 (TF32 x3 split for fp32 accuracy).  The
// apply is the contraction Out[g][n] = sum_kk In[g][kk] W[kk][n] over the
// groups g of a tile: In = a group's amplitudes as 2^(k+1) reals (re, im by
// member), W = real expansion of the fused matrix
//   W[(c,re)][(r,re)] = Re M_rc, W[(c,im)][(r,re)] = -Im M_rc,
//   W[(c,re)][(r,im)] = Im M_rc, W[(c,im)][(r,im)] =  Re M_rc.
// x = hi + lo with hi = rna_tf32(x), lo = rna_tf32(x - hi) on both operands,
// In.W = hi.Whi + hi.Wlo + lo.Whi (dropped lo.lo < 2^-22 relative).
// Operand A (In) lives in TMEM (one lane per group: thread i of the CTA owns
// TMEM lane i), written with tcgen05.st by the thread that gathered the
// group from the swizzled shared-memory tile; operand B (W) is in shared
// memory in the canonical K-major SWIZZLE_NONE layout; D accumulates in TMEM.
template <int K>
struct TcShape {
    static constexpr int D = 1 << K;
    static constexpr int KR = 2 * D;                // MMA K (real inputs)
    static constexpr int N = 2 * D;                 // MMA N (real outputs)
    static constexpr int MB = (1 << (12 - K)) / 128;  // M-blocks (128 groups) per 2^12 tile
    static constexpr int KB = KR / 8;               // tf32 MMA K-steps
    static constexpr uint32_t SBO_B = (KR / 4) * 128;
    static constexpr uint32_t W_BYTES = N * KR * 4;
    static constexpr int A_COLS = 2 * KR * MB;      // hi + lo per M-block
    static constexpr int COLS = A_COLS + N * MB;
    static constexpr int ALLOC = COLS <= 32 ? 32 : COLS <= 64 ? 64 : COLS <= 128 ? 128 : COLS <= 256 ? 256 : 512;
};

__device__ __forceinline__ float tf32_rna(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return __uint_as_float(r);
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tmem_st8(uint32_t taddr, const float* v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr),
                 "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])),
                 "r"(__float_as_uint(v[3])), "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])),
                 "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7]))
                 : "memory");
}
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t* v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t* v) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t* v) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr));
}

// UMMA shared-memory descriptor: K-major SWIZZLE_NONE, version 1 (sm_100).
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}
// Instruction descriptor: D f32, A/B tf32, K-major, M = 128, N.
__host__ __device__ constexpr uint32_t umma_idesc_tf32(int N) {
    return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}
__device__ __forceinline__ void mma_tf32_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t bdesc, uint32_t idesc,
                                            uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}\n" ::"r"(d_tmem),
        "r"(a_tmem), "l"(bdesc), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred done;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 done, [%0], %1;\n\t"
        "@!done bra WAIT_%=;\n\t}\n" ::"r"(bar),
        "r"(parity)
        : "memory");
}

struct TcState {
    uint32_t tmem, sW, bar, phase;
};

// One-time per CTA: B operand (W hi/lo) in shared memory, mbarrier, TMEM.
template <int K>
__device__ __forceinline__ TcState tc_setup(const TileParams<K>& p, uint32_t sW, uint32_t sBar, uint32_t sSlot) {
    using S = TcShape<K>;
    for (int e = threadIdx.x; e < S::N * S::KR; e += blockDim.x) {
        const int n = e / S::KR, kk = e % S::KR;
        const int r = n >> 1, ni = n & 1, c = kk >> 1, ki = kk & 1;
        const float2 m = p.M.cm[r][c];
        const float v = (ni == 0) ? (ki == 0 ? m.x : -m.y) : (ki == 0 ? m.y : m.x);
        const float hi = tf32_rna(v), lo = tf32_rna(v - hi);
        const uint32_t off =
            (uint32_t)(n >> 3) * S::SBO_B + (uint32_t)(kk >> 2) * 128u + (uint32_t)(n & 7) * 16u + (uint32_t)(kk & 3) * 4u;
        asm volatile("st.shared.f32 [%0], %1;" ::"r"(sW + off), "f"(hi) : "memory");
        asm volatile("st.shared.f32 [%0], %1;" ::"r"(sW + S::W_BYTES + off), "f"(lo) : "memory");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sBar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if ((threadIdx.x >> 5) == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(sSlot), "n"(S::ALLOC)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    TcState t;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(t.tmem) : "r"(sSlot) : "memory");
    t.sW = sW;
    t.bar = sBar;
    t.phase = 0;
    return t;
}

template <int K>
__device__ __forceinline__ void tc_teardown(const TcState& t) {
    using S = TcShape<K>;
    tc_fence_before();
    __syncthreads();
    if ((threadIdx.x >> 5) == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(t.tmem), "n"(S::ALLOC) : "memory");
}

template <int K, bool PAIR>
__device__ __forceinline__ void tile_compute_tc(const TileParams<K>& p, uint32_t sbuf, TcState& t) {
    using S = TcShape<K>;
    constexpr int D = S::D;
    const uint32_t lane_base = (uint32_t)((threadIdx.x >> 5) * 32) << 16;  // this warp's TMEM lane quarter
    // split: gather this thread's group(s), tf32 hi/lo into TMEM
#pragma unroll
    for (int mb = 0; mb < S::MB; ++mb) {
        const uint32_t g = (uint32_t)mb * 128u + threadIdx.x;
        const uint32_t pb = slot_of<K>(p, g);
        const uint32_t thi = t.tmem + lane_base + (uint32_t)(mb * 2 * S::KR);
        const uint32_t tlo = thi + (uint32_t)S::KR;
#pragma unroll
        for (int q = 0; q < D / 4; ++q) {  // 4 members = 8 reals = one st.x8
            float x[8];
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int j = 2 * q + h;  // member pair (2j, 2j+1)
                if constexpr (PAIR) {
                    const float4 v = lds4(sbuf + ((pb ^ p.loc[j]) << 3));
                    x[4 * h] = v.x; x[4 * h + 1] = v.y; x[4 * h + 2] = v.z; x[4 * h + 3] = v.w;
                } else {
                    const float2 u = lds2(sbuf + ((pb ^ p.loc[2 * j]) << 3));
                    const float2 w = lds2(sbuf + ((pb ^ p.loc[2 * j + 1]) << 3));
                    x[4 * h] = u.x; x[4 * h + 1] = u.y; x[4 * h + 2] = w.x; x[4 * h + 3] = w.y;
                }
            }
            float hi[8], lo[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) {
                hi[e] = tf32_rna(x[e]);
                lo[e] = tf32_rna(x[e] - hi[e]);
            }
            tmem_st8(thi + (uint32_t)(8 * q), hi);
            tmem_st8(tlo + (uint32_t)(8 * q), lo);
}
    }
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (threadIdx.x == 0) {
        constexpr uint32_t idesc = umma_idesc_tf32(S::N);
#pragma unroll
        for (int mb = 0; mb < S::MB; ++mb) {
            const uint32_t d = t.tmem + (uint32_t)(S::A_COLS + mb * S::N);
            const uint32_t ahi = t.tmem + (uint32_t)(mb * 2 * S::KR), alo = ahi + (uint32_t)S::KR;
#pragma unroll
            for (int kb = 0; kb < S::KB; ++kb) {
                const uint64_t bhi = umma_desc(t.sW + (uint32_t)kb * 256u, 128, S::SBO_B);
                const uint64_t blo = umma_desc(t.sW + S::W_BYTES + (uint32_t)kb * 256u, 128, S::SBO_B);
                mma_tf32_ts(d, ahi + (uint32_t)(8 * kb), bhi, idesc, kb > 0 ? 1u : 0u);
                mma_tf32_ts(d, ahi + (uint32_t)(8 * kb), blo, idesc, 1u);
                mma_tf32_ts(d, alo + (uint32_t)(8 * kb), bhi, idesc, 1u);
            }
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(t.bar)
                     : "memory");
    }
    mbar_wait(t.bar, t.phase);
    t.phase ^= 1u;
    tc_fence_after();
    // epilogue: outputs back into the swizzled tile (same slots as the inputs)
#pragma unroll
    for (int mb = 0; mb < S::MB; ++mb) {
        const uint32_t g = (uint32_t)mb * 128u + threadIdx.x;
        const uint32_t pb = slot_of<K>(p, g);
#pragma unroll
        for (int c0 = 0; c0 < S::N; c0 += 32) {
            uint32_t v[32];
            tmem_ld32(t.tmem + lane_base + (uint32_t)(S::A_COLS + mb * S::N + c0), v);
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
            for (int i = 0; i < 8; ++i) {  // 8 member pairs of this 32-column chunk
                const int j = c0 / 4 + i;
                const float4 o = make_float4(__uint_as_float(v[4 * i]), __uint_as_float(v[4 * i + 1]),
                                             __uint_as_float(v[4 * i + 2]), __uint_as_float(v[4 * i + 3]));
                if constexpr (PAIR) {
                    sts4(sbuf + ((pb ^ p.loc[j]) << 3), o);
                } else {
                    sts2(sbuf + ((pb ^ p.loc[2 * j]) << 3), make_float2(o.x, o.y));
                    sts2(sbuf + ((pb ^ p.loc[2 * j + 1]) << 3), make_float2(o.z, o.w));
                }
            }
        }
    }
    tc_fence_before();
}

// ------------------------------------------ tensor cores, exact accumulation
// The TF32 path above is biased (its accumulation truncates toward zero).
// Here the contraction Out = In . W runs on tcgen05.mma.kind::i8 with exact
// s32 accumulation: every real input of a group row is scaled by a
// power-of-two row scale 2^(22 - e_r) to an integer |xi| <= 2^22 written in
// balanced signed base-256 digits
//   xi = a0 2^16 + a1 2^8 + a2     (a1, a2 in [-128, 127], |a0| <= 65),
// every column n of W likewise with 2^(22 - f_n) into b0, b1, b2, and
//   sum_kk xi wi ~= 2^16 (S32 2^16 + S24 2^8 + S16),
//   S32 = a0.b0, S24 = a0.b1 + a1.b0, S16 = a0.b2 + a1.b1 + a2.b0
// (6 int8 MMAs per K-step of 32).  The dropped cross terms (a1.b2, a2.b1,
// a2.b2) are below 2^-21 of the row x column scale and zero-mean (balanced
// digits), so no bias.  The three s32 sums are exact; they are combined in
// int64, converted to fp32 with a single correctly rounded conversion and
// scaled by 2^(e_r + f_n - 28) (exact).
// Operand A (slices) and B (W slices) live in shared memory in the K-major
// SWIZZLE_NONE canonical layout (core matrix 8 rows x 16 B), D in TMEM.
__host__ __device__ constexpr int tci_threads(int K) { return K == 6 ? 512 : 256; }
// Accumulators: S32, S24, S16 (+ S8 = a1 b2 + a2 b1).  Without S8 the
// dropped products correlate with the output through the state's own middle
// digit and leave a per-gate norm change of random sign (DESIGN.md §11:
// -1.1e-6 over a 23-gate k = 6 circuit, 1.3e-7 over 25 k = 5 gates); S8 costs
// 2 MMAs per K-step, one more TMEM load per column group and ~1 instruction
// per output (+7 % at k = 4, 5, +13 % at k = 6).  k = 6 keeps S8.
__host__ __device__ constexpr int tci_nacc(int K) {
#ifdef SVB_TCI_NACC4
    return 4 + 0 * K;
#else
    return K == 6 ? 4 : 3;
#endif
}
// Output scale 2^(e + f - 2 SH) split as 2^(e - SH) 2^(f - SH): tt is
// sum xi wi / 2^16 with three accumulators (SH = 14), / 2^8 with four (SH = 18).
__host__ __device__ constexpr int tci_shift(int K) { return tci_nacc(K) == 4 ? 18 : 14; }

template <int K>
struct TciShape {
    static constexpr int D = 1 << K;
    static constexpr int KR = 2 * D;                  // MMA K (reals per group)
    static constexpr int N = 2 * D;                   // MMA N
    static constexpr int T = K == 6 ? 13 : 12;        // tile bits
    static constexpr int MB = (1 << (T - K)) / 128;   // M-blocks of 128 groups per tile
    static constexpr int TPR = K == 6 ? 4 : 2;        // threads per MMA row (k = 6: 1 CTA/SM -> 16 warps)
    static constexpr int THREADS = 128 * TPR;
    static_assert(THREADS == tci_threads(K), "thread count");
    // The A slices are written into the current tile buffer once its
    // amplitudes are in registers (the MMA is complete before the epilogue
    // writes the outputs there): 3 x 128 MB KR bytes <= 3/4 of the tile.
    static constexpr bool A_IN_TILE = true;
    // k <= 5: three tile buffers (store of tile i-1 overlaps the MMAs of tile
    // i, load of tile i+2 in flight); k = 6 (64 KB tiles): two.
    static constexpr int STAGES = K == 6 ? 2 : 3;
    static constexpr int KS = KR / 32;                // int8 MMA K-steps (K = 32)
    static constexpr uint32_t SBO = KR * 8;           // byte distance between row octets (KR/16 chunks x 128 B)
    static constexpr uint32_t A_SLICE = 128u * MB * KR;  // bytes of one A slice
    static constexpr uint32_t B_SLICE = (uint32_t)N * KR;
    static constexpr uint32_t ROWMAX = 4 * 128 * MB * 4;  // part-row maxima exchange (TPR <= 4)
    static constexpr uint32_t SMEM = (A_IN_TILE ? 0u : 3 * A_SLICE) + 3 * B_SLICE + N * 4 + ROWMAX + 64;
    static constexpr int NACC = tci_nacc(K);          // S32, S24, S16 (, S8)
    static constexpr int COLS = NACC * N * MB;
    static constexpr int ALLOC = COLS <= 32 ? 32 : COLS <= 64 ? 64 : COLS <= 128 ? 128 : COLS <= 256 ? 256 : 512;
};

__host__ __device__ constexpr uint32_t umma_idesc_i8(int N, bool a_signed, bool b_signed) {
    return (2u << 4) | ((a_signed ? 1u : 0u) << 7) | ((b_signed ? 1u : 0u) << 10) | ((uint32_t)(N >> 3) << 17) |
           ((uint32_t)(128 >> 4) << 24);
}
__device__ __forceinline__ void mma_i8_ss(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc)
        : "memory");
}


struct TciState {
    uint32_t tmem, sA, sB, sF, sM, bar, phase;
};

template <int K>
__device__ __forceinline__ TciState tci_setup(const TileParams<K>& p, uint32_t sBase) {
    using S = TciShape<K>;
    TciState t;
    t.sA = sBase;
    t.sB = sBase + (S::A_IN_TILE ? 0u : 3 * S::A_SLICE);
    t.sF = t.sB + 3 * S::B_SLICE;
    t.sM = t.sF + S::N * 4;
    t.bar = t.sM + S::ROWMAX;
    const uint32_t slot = t.bar + 8;
    // B slices (canonical layout, prepared on the host) + column exponents
    const uint4* src = reinterpret_cast<const uint4*>(p.wi8);
    for (uint32_t i = threadIdx.x; i < (3 * S::B_SLICE + S::N * 4) / 16; i += blockDim.x) {
        const uint4 v = src[i];
        asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(t.sB + 16 * i), "r"(v.x), "r"(v.y), "r"(v.z),
                     "r"(v.w)
                     : "memory");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(t.bar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if ((threadIdx.x >> 5) == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(slot), "n"(S::ALLOC)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(t.tmem) : "r"(slot) : "memory");
    t.phase = 0;
    return t;
}

template <int K>
__device__ __forceinline__ void tci_teardown(const TciState& t) {
    using S = TciShape<K>;
    tc_fence_before();
    __syncthreads();
    if ((threadIdx.x >> 5) == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(t.tmem), "n"(S::ALLOC) : "memory");
}

// 16 reals -> one 16 B chunk of each of the three slices.
// v = x * scale + 1.5 * 2^23 rounds x * scale to the nearest integer xi
// (|xi| <= 2^22) and leaves bits(v) = 0x4B400000 + xi.  The balanced digits
// are d2 = low byte of xi, d1 = byte 1 of xi + 2^7, d0 = byte 2 of
// xi + 2^15 + 2^7, i.e. bytes of bits(v) plus constants (the additions only
// carry upward, so the low bytes of 0x4B400000 + ... are those of xi + ...).
__device__ __forceinline__ void slice16(const float* x, float scale, uint4& s0, uint4& s1, uint4& s2) {
    uint32_t w0[4], w1[4], w2[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        uint32_t b2[4], b1[4], b0[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
            const uint32_t v = __float_as_uint(fmaf(x[4 * q + e], scale, 12582912.0f));
            b2[e] = v;
            b1[e] = v + 128u;
            b0[e] = v + (32896u - 0x400000u);
        }
        w2[q] = __byte_perm(__byte_perm(b2[0], b2[1], 0x0040), __byte_perm(b2[2], b2[3], 0x0040), 0x5410);
        w1[q] = __byte_perm(__byte_perm(b1[0], b1[1], 0x0051), __byte_perm(b1[2], b1[3], 0x0051), 0x5410);
        w0[q] = __byte_perm(__byte_perm(b0[0], b0[1], 0x0062), __byte_perm(b0[2], b0[3], 0x0062), 0x5410);
    }
    s0 = make_uint4(w0[0], w0[1], w0[2], w0[3]);
    s1 = make_uint4(w1[0], w1[1], w1[2], w1[3]);
    s2 = make_uint4(w2[0], w2[1], w2[2], w2[3]);
}

__device__ __forceinline__ void sts128u(uint32_t a, uint4 v) {
    asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

// TPR threads per MMA row (128 TPR threads; TPR = 2 for k <= 5 -- 4 measured
// slower there -- and 4 for k = 6): thread part p = threadIdx.x / 128
// of row r = threadIdx.x % 128 gathers and slices members [p D/TPR,
// (p+1) D/TPR) and later combines output columns [p N/TPR, (p+1) N/TPR);
// warps w and w + 4j read the same TMEM lane quarter (w % 4).
template <int MB>
struct TciRows {
    float srow[MB];    // 2^(e - 14) per M-block row
};

// Phys (swizzled) slot of this thread's group row in M-block mb: the same
// for every tile, computed once per kernel.
template <int K>
__device__ __forceinline__ void tci_slots(const TileParams<K>& p, uint32_t (&pbs)[TciShape<K>::MB]) {
#pragma unroll
    for (int mb = 0; mb < TciShape<K>::MB; ++mb) {
        const uint32_t g = (uint32_t)mb * 128u + (threadIdx.x & 127u);
        pbs[mb] = slot_of<K>(p, g);
    }
}

// Phase A: gather, slice, issue the MMAs (asynchronous; completion is
// signalled on t.bar).
// Barrier among the MMA/compute threads only: in the warp-specialised loop
// (WS) a producer warp does not take part (named barrier 1).
template <int K, bool WS>
__device__ __forceinline__ void tci_sync() {
    if constexpr (WS) asm volatile("bar.sync 1, %0;" ::"n"(TciShape<K>::THREADS) : "memory");
    else __syncthreads();
}

template <int K, bool PAIR, bool WS = false>
__device__ __forceinline__ void tci_phase_a(const TileParams<K>& p, uint32_t sbuf, TciState& t,
                                            TciRows<TciShape<K>::MB>& rw, const uint32_t (&pbs)[TciShape<K>::MB]) {
    using S = TciShape<K>;
    constexpr int TPR = S::TPR;
    constexpr int D = S::D;
    const uint32_t sA = S::A_IN_TILE ? sbuf : t.sA;
    constexpr int HM = D / TPR;   // members per thread
    constexpr int RPT = 2 * HM;   // reals per thread (8 or 16)
    static_assert(RPT == 8 || RPT % 16 == 0, "slice granularity");
    const int part = threadIdx.x >> 7;
    const uint32_t row = threadIdx.x & 127u;
    float x[S::MB][RPT];
    // 1a. gather this thread's part of the row, publish the part maximum
#pragma unroll
    for (int mb = 0; mb < S::MB; ++mb) {
        const uint32_t pb = pbs[mb];
#pragma unroll
        for (int j = 0; j < HM / 2; ++j) {
            const int jj = part * (HM / 2) + j;  // member pair (2jj, 2jj+1)
            if constexpr (PAIR) {
                const float4 v = lds4(sbuf + ((pb ^ p.loc[jj]) << 3));
                x[mb][4 * j] = v.x; x[mb][4 * j + 1] = v.y; x[mb][4 * j + 2] = v.z; x[mb][4 * j + 3] = v.w;
            } else {
                const float2 u = lds2(sbuf + ((pb ^ p.loc[2 * jj]) << 3));
                const float2 w = lds2(sbuf + ((pb ^ p.loc[2 * jj + 1]) << 3));
                x[mb][4 * j] = u.x; x[mb][4 * j + 1] = u.y; x[mb][4 * j + 2] = w.x; x[mb][4 * j + 3] = w.y;
            }
        }
        float mx = 0.f;
#pragma unroll
        for (int i = 0; i < RPT; ++i) mx = fmaxf(mx, fabsf(x[mb][i]));
        asm volatile("st.shared.f32 [%0], %1;" ::"r"(t.sM + 4u * ((uint32_t)mb * (128u * TPR) + threadIdx.x)), "f"(mx)
                     : "memory");
    }
    tci_sync<K, WS>();
    // 1b. row scale 2^(22 - e) with max|x| < 2^e; slice into A (shared memory)
#pragma unroll
    for (int mb = 0; mb < S::MB; ++mb) {
        float mx = 0.f;
#pragma unroll
        for (int q = 0; q < TPR; ++q) {
            float m;
            asm volatile("ld.shared.f32 %0, [%1];"
                         : "=f"(m)
                         : "r"(t.sM + 4u * ((uint32_t)mb * (128u * TPR) + (uint32_t)q * 128u + row)));
            mx = fmaxf(mx, m);
        }
        const int e = max(((int)(__float_as_uint(mx) >> 23) & 0xFF) - 126, -100);  // mx < 2^e
        rw.srow[mb] = __uint_as_float((uint32_t)(127 + e - tci_shift(K)) << 23);      // 2^(e - SH)
        const float scale = __uint_as_float((uint32_t)(127 + 22 - e) << 23);
        const uint32_t rbase = (uint32_t)mb * 128u * S::KR + (row >> 3) * S::SBO + (row & 7) * 16u;
        if constexpr (RPT == 8) {
            uint4 s0, s1, s2;
            float xx[16];
#pragma unroll
            for (int i = 0; i < 8; ++i) { xx[i] = x[mb][i]; xx[8 + i] = 0.f; }
            slice16(xx, scale, s0, s1, s2);
            const uint32_t a = sA + rbase + (uint32_t)(part >> 1) * 128u + (uint32_t)(part & 1) * 8u;
            asm volatile("st.shared.v2.u32 [%0], {%1,%2};" ::"r"(a), "r"(s0.x), "r"(s0.y) : "memory");
            asm volatile("st.shared.v2.u32 [%0], {%1,%2};" ::"r"(a + S::A_SLICE), "r"(s1.x), "r"(s1.y) : "memory");
            asm volatile("st.shared.v2.u32 [%0], {%1,%2};" ::"r"(a + 2 * S::A_SLICE), "r"(s2.x), "r"(s2.y)
                         : "memory");
        } else {
#pragma unroll
            for (int c = 0; c < RPT / 16; ++c) {  // 16 reals per chunk
                uint4 s0, s1, s2;
                slice16(x[mb] + 16 * c, scale, s0, s1, s2);
                const uint32_t a = sA + rbase + (uint32_t)(part * (RPT / 16) + c) * 128u;
                sts128u(a, s0);
                sts128u(a + S::A_SLICE, s1);
                sts128u(a + 2 * S::A_SLICE, s2);
            }
        }
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    tci_sync<K, WS>();
    tc_fence_after();
    // 2. six int8 MMAs per K-step into three exact s32 accumulators
    if (threadIdx.x == 0) {
        constexpr uint32_t i_ss = umma_idesc_i8(S::N, true, true);
#pragma unroll
        for (int mb = 0; mb < S::MB; ++mb) {
            const uint32_t d0 = t.tmem + (uint32_t)(mb * S::NACC * S::N);
            const uint32_t d32 = d0, d24 = d0 + S::N, d16 = d0 + 2 * S::N, d8 = d0 + 3 * S::N;
            (void)d8;
#pragma unroll
            for (int ks = 0; ks < S::KS; ++ks) {
                const uint32_t ao = sA + (uint32_t)mb * 128u * S::KR + (uint32_t)ks * 256u;
                const uint32_t bo = t.sB + (uint32_t)ks * 256u;
                const uint64_t a0 = umma_desc(ao, 128, S::SBO), a1 = umma_desc(ao + S::A_SLICE, 128, S::SBO),
                               a2 = umma_desc(ao + 2 * S::A_SLICE, 128, S::SBO);
                const uint64_t b0 = umma_desc(bo, 128, S::SBO), b1 = umma_desc(bo + S::B_SLICE, 128, S::SBO),
                               b2 = umma_desc(bo + 2 * S::B_SLICE, 128, S::SBO);
                const uint32_t acc = ks > 0 ? 1u : 0u;
                mma_i8_ss(d32, a0, b0, i_ss, acc);
                mma_i8_ss(d24, a0, b1, i_ss, acc);
                mma_i8_ss(d24, a1, b0, i_ss, 1u);
                mma_i8_ss(d16, a0, b2, i_ss, acc);
                mma_i8_ss(d16, a1, b1, i_ss, 1u);
                mma_i8_ss(d16, a2, b0, i_ss, 1u);
                if constexpr (S::NACC == 4) {
                    mma_i8_ss(d8, a1, b2, i_ss, acc);
                    mma_i8_ss(d8, a2, b1, i_ss, 1u);
                }
            }
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(t.bar)
                     : "memory");
    }
}

// Phase B: wait for the MMAs, exact recombination of this thread's columns
// (one rounding), outputs written back into the tile.
template <int K, bool PAIR, bool WS = false>
__device__ __forceinline__ void tci_phase_b(const TileParams<K>& p, uint32_t sbuf, TciState& t,
                                            const TciRows<TciShape<K>::MB>& rw, const uint32_t (&pbs)[TciShape<K>::MB]) {
    using S = TciShape<K>;
    constexpr int TPR = S::TPR;
    constexpr int NPT = S::N / TPR;
    constexpr int CW = K == 6 ? 8 : 16;  // columns per TMEM-load round (16 at k = 6 measured slower)
    const int part = threadIdx.x >> 7;
    const uint32_t lane_base = (uint32_t)(((threadIdx.x >> 5) & 3) * 32) << 16;
    mbar_wait(t.bar, t.phase);
    t.phase ^= 1u;
    tc_fence_after();
    // 3. exact recombination of this thread's columns, one rounding
#pragma unroll
    for (int mb = 0; mb < S::MB; ++mb) {
        const uint32_t pb = pbs[mb];
        const uint32_t d0 = t.tmem + lane_base + (uint32_t)(mb * S::NACC * S::N);
#pragma unroll 1
        for (int c0 = part * NPT; c0 < (part + 1) * NPT; c0 += CW) {
            uint32_t v32[CW], v24[CW], v16[CW], v8[S::NACC == 4 ? CW : 1];
            if constexpr (CW == 16) {
                tmem_ld16(d0 + (uint32_t)c0, v32);
                tmem_ld16(d0 + (uint32_t)(S::N + c0), v24);
                tmem_ld16(d0 + (uint32_t)(2 * S::N + c0), v16);
                if constexpr (S::NACC == 4) tmem_ld16(d0 + (uint32_t)(3 * S::N + c0), v8);
            } else {
                tmem_ld8(d0 + (uint32_t)c0, v32);
                tmem_ld8(d0 + (uint32_t)(S::N + c0), v24);
                tmem_ld8(d0 + (uint32_t)(2 * S::N + c0), v16);
                if constexpr (S::NACC == 4) tmem_ld8(d0 + (uint32_t)(3 * S::N + c0), v8);
            }
            float fc[CW];
#pragma unroll
            for (int q = 0; q < CW / 4; ++q)
                asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];"
                             : "=f"(fc[4 * q]), "=f"(fc[4 * q + 1]), "=f"(fc[4 * q + 2]), "=f"(fc[4 * q + 3])
                             : "r"(t.sF + 4u * (uint32_t)(c0 + 4 * q)));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
            float o[CW];
#pragma unroll
            for (int i = 0; i < CW; ++i) {
                // exact integer combination (|S24 2^8 + S16| < 2^30), ONE
                // correctly rounded int64 -> fp32 conversion, then the exact
                // power-of-two scaling 2^(e - 14) 2^(f - 14) (each factor normal)
                if constexpr (S::NACC == 4) {
                    // |S32 2^8 + S24| < 2^28, |S16 2^8 + S8| < 2^31
                    const int hi = (int)v32[i] * 256 + (int)v24[i];
                    const int lo = (int)v16[i] * 256 + (int)v8[i];
                    const long long tt = (long long)hi * 65536ll + (long long)lo;
                    o[i] = __ll2float_rn(tt) * rw.srow[mb] * fc[i];
                } else {
                    const int lo = (int)v24[i] * 256 + (int)v16[i];
                    const long long tt = (long long)(int)v32[i] * 65536ll + (long long)lo;
                    o[i] = __ll2float_rn(tt) * rw.srow[mb] * fc[i];
                }
            }
#pragma unroll
            for (int i = 0; i < CW / 4; ++i) {
                const int j = c0 / 4 + i;
                if constexpr (PAIR) {
                    sts4(sbuf + ((pb ^ p.loc[j]) << 3), make_float4(o[4 * i], o[4 * i + 1], o[4 * i + 2], o[4 * i + 3]));
                } else {
                    sts2(sbuf + ((pb ^ p.loc[2 * j]) << 3), make_float2(o[4 * i], o[4 * i + 1]));
                    sts2(sbuf + ((pb ^ p.loc[2 * j + 1]) << 3), make_float2(o[4 * i + 2], o[4 * i + 3]));
                }
            }
        }
    }
    tc_fence_before();
}

template <int K, bool PAIR>
__device__ __forceinline__ void tile_compute_tci(const TileParams<K>& p, uint32_t sbuf, TciState& t,
                                                 const uint32_t (&pbs)[TciShape<K>::MB]) {
    TciRows<TciShape<K>::MB> rw;
    tci_phase_a<K, PAIR>(p, sbuf, t, rw, pbs);
    tci_phase_b<K, PAIR>(p, sbuf, t, rw, pbs);
}

// Persistent loop over tiles.  STAGES = 2: the copies of tile i+1 are in
// flight while tile i is transformed and written back.
// Global index of tile u's first amplitude: zeros at the tile's high gate
// qubits and at the control qubits, then the controls set to 1.
template <int K>
__device__ __forceinline__ uint64_t tile_base(const TileParams<K>& p, uint64_t u) {
    uint64_t x = u << p.r;
    for (int b = 0; b < p.nZ; ++b) x += x & p.Zhigh[b];  // ascending positions: shift bits >= q up by one
    return x | p.ones;
}

template <int K, bool PAIR, int MODE, int STAGES>
__device__ __forceinline__ void tile_loop(const TileParams<K>& p) {
    extern __shared__ float4 dsm[];
    const uint32_t tile_bytes = 8u << p.T;
    const uint32_t s0 = smem_addr(dsm);
    const float2* smat = nullptr;
    uint32_t splanes = 0;
#if SVB_SMEM_PLANES
    // k = 2, 3 only: at k = 4 it measured 19 % slower (3.70 vs 3.12 ms; the
    // LDCU operands feed the FFMAs without occupying vector registers)
    if constexpr (MODE == 0 && K >= 2 && K <= 3) {
        // Gauss planes P, S, Q (3 x 2^k x 2^k fp32) after the tile buffers
        constexpr int DD = (1 << K) * (1 << K);
        float* sp = reinterpret_cast<float*>(reinterpret_cast<char*>(dsm) + STAGES * tile_bytes);
        for (int i = threadIdx.x; i < DD; i += blockDim.x) {
            sp[i] = (&p.M.P[0][0])[i];
            sp[DD + i] = (&p.M.S[0][0])[i];
            sp[2 * DD + i] = (&p.M.Q[0][0])[i];
        }
        splanes = s0 + STAGES * tile_bytes;
        __syncthreads();
    }
#endif
    if constexpr (K == 6 && MODE != 3) {
        float2* sm = reinterpret_cast<float2*>(reinterpret_cast<char*>(dsm) + STAGES * tile_bytes);
        for (int i = threadIdx.x; i < 64 * 64; i += blockDim.x) sm[i] = p.M.dev[i];
        smat = sm;
        __syncthreads();
    }
    // slot of this thread's first group (the same in every tile)
    const uint32_t pb0 = slot_of<K>(p, K <= 4 ? (threadIdx.x << 1) : threadIdx.x);
    TciState tis{};
    uint32_t tslot[MODE == 3 ? TciShape<K>::MB : 1];
    if constexpr (MODE == 3) {
        tis = tci_setup<K>(p, s0 + STAGES * tile_bytes);
        tci_slots<K>(p, tslot);
    }
    TcState tcs{};
    if constexpr (MODE == 2 && K <= 5) {
        const uint32_t sW = s0 + STAGES * tile_bytes;
        const uint32_t sBar = sW + 2 * TcShape<K>::W_BYTES;
        tcs = tc_setup<K>(p, sW, sBar, sBar + 8);
    }
    // per-thread bases of the unit maps (t = 2*tid + 2*nthreads*i)
    const uint32_t t0 = 2u * threadIdx.x;
    const uint32_t rmask = (1u << p.r) - 1u;
    uint64_t dthr = t0 & rmask;
    {
        const uint32_t h = t0 >> p.r;
        for (int b = 0; b < p.nH; ++b)
            if ((h >> b) & 1u) dthr += 1ull << p.Hpos[b];
    }
    const uint32_t sthr = swizzle(t0, p.swz);
    const int upt = p.upt;
    // byte address of this thread's first unit of tile u (computed once per
    // tile: the same address serves the load and the store)
    auto gaddr = [&](uint64_t u) { return reinterpret_cast<const char*>(p.psi + tile_base(p, u) + dthr); };
    auto load = [&](const char* g, uint32_t sbuf) {
        for (int i = 0; i < upt; ++i)
            cp_async16(sbuf + ((sthr ^ p.soff[i]) << 3), reinterpret_cast<const float2*>(g + p.goff[i]));
    };
    auto store = [&](const char* g, uint32_t sbuf) {
        for (int i = 0; i < upt; ++i)
            st_stream(reinterpret_cast<float4*>(const_cast<char*>(g) + p.goff[i]), lds4(sbuf + ((sthr ^ p.soff[i]) << 3)));
    };
    uint64_t u = blockIdx.x;
    if constexpr (MODE == 3 && STAGES == 3) {
        // Three buffers, tile i in buf[i % 3]:
        //   wait load(i) | phase A(i): gather, slice, issue MMAs |
        //   store(i-1) while the MMAs run | load(i+2) into the drained buffer |
        //   phase B(i): wait MMAs, epilogue into buf[i % 3]
        const uint64_t G = gridDim.x;
        // global addresses / buffers of tiles it-1 (prv), it (cur), it+1 (nxt)
        const char* gprv = nullptr;
        const char* gcur = nullptr;
        const char* gnxt = nullptr;
        uint32_t bprv = s0 + 2 * tile_bytes, bcur = s0, bnxt = s0 + tile_bytes;
        if (u < p.n_tiles) {
            gcur = gaddr(u);
            load(gcur, bcur);
        }
        cp_async_commit();
        if (u + G < p.n_tiles) {
            gnxt = gaddr(u + G);
            load(gnxt, bnxt);
        }
        cp_async_commit();
        for (int it = 0; u < p.n_tiles; u += G, ++it) {
            cp_async_wait1();  // this thread's copies of tile it have landed
            __syncthreads();   // ... and everyone else's; epilogue(it-1) writes are visible
            TciRows<TciShape<K>::MB> rw;
            tci_phase_a<K, PAIR>(p, bcur, tis, rw, tslot);
            if (it > 0) store(gprv, bprv);
            __syncthreads();  // buffer of tile it-1 drained
            const uint64_t u2 = u + 2 * G;
            const char* gnew = nullptr;
            if (u2 < p.n_tiles) {
                gnew = gaddr(u2);
                load(gnew, bprv);
            }
            cp_async_commit();
            tci_phase_b<K, PAIR>(p, bcur, tis, rw, tslot);
            const uint32_t bfree = bprv;
            gprv = gcur; bprv = bcur;
            gcur = gnxt; bcur = bnxt;
            gnxt = gnew; bnxt = bfree;
        }
        __syncthreads();  // last epilogue complete
        if (u != blockIdx.x) store(gprv, bprv);
        cp_async_wait0();
        tci_teardown<K>(tis);
    } else if constexpr (STAGES == 2) {
        const char* gcur = nullptr;
        if (u < p.n_tiles) {
            gcur = gaddr(u);
            load(gcur, s0);
        }
        cp_async_commit();
        for (int it = 0; u < p.n_tiles; u += gridDim.x, ++it) {
            const uint32_t cur = s0 + (uint32_t)(it & 1) * tile_bytes;
            const uint32_t nxt = s0 + (uint32_t)((it + 1) & 1) * tile_bytes;
            const uint64_t un = u + gridDim.x;
            const char* gnext = nullptr;
            __syncthreads();  // buffer `nxt` was drained by the previous iteration's store
            if (un < p.n_tiles) {
                gnext = gaddr(un);
                load(gnext, nxt);
            }
            cp_async_commit();
            cp_async_wait1();  // this thread's copies of tile u have landed
            __syncthreads();   // ... and everyone else's
            if constexpr (MODE == 1) tile_compute_mono<K, PAIR>(p, cur, pb0);
            else if constexpr (MODE == 2 && K <= 5) tile_compute_tc<K, PAIR>(p, cur, tcs);
            else if constexpr (MODE == 3) tile_compute_tci<K, PAIR>(p, cur, tis, tslot);
            else tile_compute<K, PAIR>(p, cur, smat, pb0, splanes);
            __syncthreads();
            store(gcur, cur);
            gcur = gnext;
        }
        if constexpr (MODE == 2 && K <= 5) tc_teardown<K>(tcs);
        if constexpr (MODE == 3) tci_teardown<K>(tis);
    } else {
        for (; u < p.n_tiles; u += gridDim.x) {
            __syncthreads();
            const char* g = gaddr(u);
            load(g, s0);
            cp_async_commit();
            cp_async_wait0();
            __syncthreads();
            if constexpr (MODE == 1) tile_compute_mono<K, PAIR>(p, s0, pb0);
            else tile_compute<K, PAIR>(p, s0, smat, pb0, splanes);
            __syncthreads();
            store(g, s0);
        }
    }
}

// ------------------------------------- tensor cores, bulk-copy pipeline
// For gates with no qubit in {1,2,3} the shared-memory tile is unswizzled
// (slot = tile index), so each of its 2^nH runs of 2^r contiguous amplitudes
// is one contiguous block in HBM and in shared memory: the tile moves with
// 2^nH bulk copies (cp.async.bulk, the TMA engine's non-tensor copy) issued
// by ONE producer thread instead of 16 B copies from every thread.  A
// producer warp (warp THREADS/32) streams tiles into NB buffers (mbarrier
// full[b], transaction-counted) and, once the compute threads have written a
// tile's outputs (mbarrier done[b]), bulk-stores it and refills the buffer;
// the compute threads only gather/slice, issue the MMAs and run the
// epilogue, so a tile's store and the next loads overlap its neighbours'
// compute.
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_load(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                 "l"(src), "r"(bytes), "r"(bar)
                 : "memory");
}
__device__ __forceinline__ void bulk_store(void* dst, uint32_t src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src), "r"(bytes)
                 : "memory");
}
// Tensor copies (rank 2..5): coordinates c[d] in elements of 8 B.
__device__ __forceinline__ void tensor_load(int rank, uint32_t dst, const void* tmap, const int* c, uint32_t bar) {
    const uint64_t m = reinterpret_cast<uint64_t>(tmap);
    switch (rank) {
        case 2:
            asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                         ::"r"(dst), "l"(m), "r"(c[0]), "r"(c[1]), "r"(bar) : "memory");
            break;
        case 3:
            asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                         ::"r"(dst), "l"(m), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(bar) : "memory");
            break;
        case 4:
            asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
                         ::"r"(dst), "l"(m), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "r"(bar) : "memory");
            break;
        default:
            asm volatile("cp.async.bulk.tensor.5d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                         ::"r"(dst), "l"(m), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "r"(c[4]), "r"(bar) : "memory");
            break;
    }
}
__device__ __forceinline__ void tensor_store(int rank, const void* tmap, const int* c, uint32_t src) {
    const uint64_t m = reinterpret_cast<uint64_t>(tmap);
    switch (rank) {
        case 2:
            asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];"
                         ::"l"(m), "r"(src), "r"(c[0]), "r"(c[1]) : "memory");
            break;
        case 3:
            asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];"
                         ::"l"(m), "r"(src), "r"(c[0]), "r"(c[1]), "r"(c[2]) : "memory");
            break;
        case 4:
            asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5}], [%1];"
                         ::"l"(m), "r"(src), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]) : "memory");
            break;
        default:
            asm volatile("cp.async.bulk.tensor.5d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5, %6}], [%1];"
                         ::"l"(m), "r"(src), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "r"(c[4]) : "memory");
            break;
    }
}
template <int K>
__device__ __forceinline__ void tensor_coords(const TileParams<K>& p, uint64_t base, int* c) {
#pragma unroll
    for (int d = 0; d < 5; ++d)
        c[d] = d < p.trank ? (int)((base >> p.tstart[d]) & ((1ull << p.tbits[d]) - 1ull)) : 0;
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// Warp-specialised tile loop (bulk copies).  Shared memory: NB tile buffers,
// then the mode's area (k = 2, 3 Gauss planes / tensor-core state), then
// 2 NB mbarriers.  The first NT threads compute; warp NT/32 is the producer.
template <int K, int MODE>
__host__ __device__ constexpr uint32_t ws_mode_bytes() {
    if constexpr (MODE == 3) return TciShape<K>::SMEM;
    else if constexpr (MODE == 0 && K >= 2 && K <= 3) return 3u * 4u << (2 * K);
    else return 0u;
}
template <int K, int MODE>
__host__ __device__ constexpr int ws_stages() {
    if constexpr (MODE == 3) return TciShape<K>::STAGES;
    else return SVB_WS_STAGES;
}

template <int K, bool PAIR, int MODE>
__device__ __forceinline__ void ws_loop(const TileParams<K>& p) {
    constexpr int NB = ws_stages<K, MODE>();
    extern __shared__ float4 dsm[];
    const uint32_t NT = blockDim.x - 32u;  // compute threads
    const uint32_t tile_bytes = 8u << p.T;
    const uint32_t s0 = (smem_addr(dsm) + 1023u) & ~1023u;  // the 128 B swizzle repeats every 1 KB
    const uint32_t sarea = s0 + NB * tile_bytes;
    const uint32_t fullb = sarea + ws_mode_bytes<K, MODE>();  // NB x 8 B
    const uint32_t doneb = fullb + 8u * NB;                   // NB x 8 B
    if (threadIdx.x == 0) {
        for (int b = 0; b < NB; ++b) {
            mbar_init(fullb + 8u * b, 1);
            mbar_init(doneb + 8u * b, 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    uint32_t splanes = 0;
    if constexpr (MODE == 0 && K >= 2 && K <= 3) {
        constexpr int DD = (1 << K) * (1 << K);
        float* sp = reinterpret_cast<float*>(reinterpret_cast<char*>(dsm) + (s0 - smem_addr(dsm)) + NB * tile_bytes);
        for (int i = threadIdx.x; i < DD; i += blockDim.x) {
            sp[i] = (&p.M.P[0][0])[i];
            sp[DD + i] = (&p.M.S[0][0])[i];
            sp[2 * DD + i] = (&p.M.Q[0][0])[i];
        }
        splanes = sarea;
    }
    TciState tis{};
    if constexpr (MODE == 3) tis = tci_setup<K>(p, sarea);  // __syncthreads inside
    else __syncthreads();
    const uint64_t G = gridDim.x;
    if (threadIdx.x >= NT) {
        // producer warp: its 32 lanes issue the runs' bulk copies round-robin
        // (runs can be as small as 1 KB; one thread alone measured slower)
        const uint32_t lane = threadIdx.x - NT;
        const uint32_t nrun = 1u << p.nH, rbytes = 8u << p.r;
        if (p.trank > 0) {
            // one tensor copy per tile (loads) / per tile (stores)
            if (lane == 0) {
                const uint32_t nops = 1u << p.tnx, obytes = tile_bytes >> p.tnx;
                auto xoff = [&](uint32_t o) {  // o's bits at the gate qubits left out of the box
                    uint64_t x = 0;
                    for (int e = 0; e < p.tnx; ++e) x |= (uint64_t)((o >> e) & 1u) << p.txpos[e];
                    return x;
                };
                auto store_tile = [&](uint64_t base, uint32_t sb) {
                    int c[5];
                    for (uint32_t o = 0; o < nops; ++o) {
                        tensor_coords(p, base | xoff(o), c);
                        tensor_store(p.trank, &p.tmap, c, sb + o * obytes);
                    }
                    bulk_commit();
                };
                uint64_t gbase[NB];
                int i = 0;
                for (uint64_t u = blockIdx.x; u < p.n_tiles; u += G, ++i) {
                    const int b = i % NB;
                    const uint32_t sb = s0 + (uint32_t)b * tile_bytes;
                    if (i >= NB) {
                        mbar_wait(doneb + 8u * b, (uint32_t)(i / NB - 1) & 1u);
                        store_tile(gbase[b], sb);
                        bulk_wait_read0();
                    }
                    gbase[b] = tile_base(p, u);
                    mbar_expect_tx(fullb + 8u * b, tile_bytes);
                    for (uint32_t o = 0; o < nops; ++o) {
                        int c[5];
                        tensor_coords(p, gbase[b] | xoff(o), c);
                        tensor_load(p.trank, sb + o * obytes, &p.tmap, c, fullb + 8u * b);
                    }
                }
                for (int t = i > NB ? i - NB : 0; t < i; ++t) {
                    const int b = t % NB;
                    mbar_wait(doneb + 8u * b, (uint32_t)(t / NB) & 1u);
                    store_tile(gbase[b], s0 + (uint32_t)b * tile_bytes);
                }
                bulk_wait0();
            }
        } else {
        char* gb[NB];
        int i = 0;
        for (uint64_t u = blockIdx.x; u < p.n_tiles; u += G, ++i) {
            const int b = i % NB;
            const uint32_t sb = s0 + (uint32_t)b * tile_bytes;
            if (i >= NB) {
                mbar_wait(doneb + 8u * b, (uint32_t)(i / NB - 1) & 1u);
                for (uint32_t j = lane; j < nrun; j += 32) bulk_store(gb[b] + p.roff[j], sb + j * rbytes, rbytes);
                bulk_commit();
                bulk_wait_read0();
                __syncwarp();
            }
            gb[b] = reinterpret_cast<char*>(p.psi + tile_base(p, u));
            if (lane == 0) mbar_expect_tx(fullb + 8u * b, tile_bytes);
            __syncwarp();
            for (uint32_t j = lane; j < nrun; j += 32) bulk_load(sb + j * rbytes, gb[b] + p.roff[j], rbytes, fullb + 8u * b);
        }
        for (int t = i > NB ? i - NB : 0; t < i; ++t) {
            const int b = t % NB;
            mbar_wait(doneb + 8u * b, (uint32_t)(t / NB) & 1u);
            for (uint32_t j = lane; j < nrun; j += 32)
                bulk_store(gb[b] + p.roff[j], s0 + (uint32_t)b * tile_bytes + j * rbytes, rbytes);
            bulk_commit();
        }
        bulk_wait0();
        }
    } else {
        uint32_t tslot[MODE == 3 ? TciShape<K>::MB : 1];
        if constexpr (MODE == 3) tci_slots<K>(p, tslot);
        const uint32_t pb0 = slot_of<K>(p, K <= 4 ? (threadIdx.x << 1) : threadIdx.x);
        int i = 0;
        for (uint64_t u = blockIdx.x; u < p.n_tiles; u += G, ++i) {
            const int b = i % NB;
            const uint32_t sb = s0 + (uint32_t)b * tile_bytes;
            mbar_wait(fullb + 8u * b, (uint32_t)(i / NB) & 1u);
            if constexpr (MODE == 3) {
                TciRows<TciShape<K>::MB> rw;
                tci_phase_a<K, PAIR, true>(p, sb, tis, rw, tslot);
                tci_phase_b<K, PAIR, true>(p, sb, tis, rw, tslot);
            } else if constexpr (MODE == 1) {
                tile_compute_mono<K, PAIR>(p, sb, pb0, NT);
            } else {
                tile_compute<K, PAIR>(p, sb, nullptr, pb0, splanes, NT);
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // outputs -> async proxy (bulk store)
            asm volatile("bar.sync 1, %0;" ::"r"(NT) : "memory");
            if (threadIdx.x == 0) mbar_arrive(doneb + 8u * b);
        }
    }
    if constexpr (MODE == 3) tci_teardown<K>(tis);
}

template <int K, bool PAIR>
__global__ void __launch_bounds__(TciShape<K>::THREADS + 32, K == 6 ? 1 : 2) apply_tci_ws(const __grid_constant__ TileParams<K> p) {
    ws_loop<K, PAIR, 3>(p);
}
template <int K, bool PAIR, bool MONO>
__global__ void __launch_bounds__(256 + 32) apply_high_ws(const __grid_constant__ TileParams<K> p) {
    ws_loop<K, PAIR, MONO ? 1 : 0>(p);
}

__host__ __device__ constexpr int stages_for(int K) { return K == 6 ? 1 : 2; }

// The paper's two kernel classes (L110-112).  Same tile engine; "high" gates
// (no qubit in {1,2,3}) need no swizzle and read whole 128 B lines per
// member, "low" gates carry partners inside one 128 B line.
// MONO: the matrix has one nonzero per row (permutation x diagonal) -> the
// exact y_r = m_r a_perm(r) path, a separate instantiation so the dense path
// carries no branch.  apply_tc: dense k = 4, 5 on the tensor cores.
template <int K, bool PAIR, bool MONO>
__global__ void __launch_bounds__(256) apply_high(const __grid_constant__ TileParams<K> p) {
    tile_loop<K, PAIR, MONO ? 1 : 0, stages_for(K)>(p);
}
template <int K, bool PAIR, bool MONO>
__global__ void __launch_bounds__(256) apply_low(const __grid_constant__ TileParams<K> p) {
    tile_loop<K, PAIR, MONO ? 1 : 0, stages_for(K)>(p);
}
template <int K, bool PAIR>
__global__ void __launch_bounds__(128, 1) apply_tc(const __grid_constant__ TileParams<K> p) {
    tile_loop<K, PAIR, 2, 2>(p);
}
template <int K, bool PAIR>
__global__ void __launch_bounds__(TciShape<K>::THREADS, K == 6 ? 1 : 2) apply_tci(const __grid_constant__ TileParams<K> p) {
    tile_loop<K, PAIR, 3, TciShape<K>::STAGES>(p);
}

// Tiny states (fewer amplitudes than one tile can split into thread work):
// one thread per group, direct global accesses.  Only used when n is small.
template <int K>
struct SmallParams {
    float2* psi;
    uint64_t n_groups;
    int q[SV_MAX_FUSED];
    int nz;                        // gate + control qubits, ascending (zero insertion)
    int zpos[2 * SV_MAX_FUSED];
    uint64_t ones;                 // control qubits set to 1
    MatStore<K> M;
};
template <int K>
__global__ void __launch_bounds__(256) apply_small(const __grid_constant__ SmallParams<K> p) {
    constexpr int D = 1 << K;
    const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (g >= p.n_groups) return;
    uint64_t base = g;
    for (int b = 0; b < p.nz; ++b) {
        const int q = p.zpos[b];
        base = ((base >> q) << (q + 1)) | (base & ((1ull << q) - 1ull));
    }
    base |= p.ones;
    uint64_t off[D];
    float2 a[D];
#pragma unroll
    for (int c = 0; c < D; ++c) {
        uint64_t o = 0;
#pragma unroll
        for (int b = 0; b < K; ++b)
            if ((c >> b) & 1) o |= 1ull << p.q[b];
        off[c] = base | o;
        a[c] = p.psi[off[c]];
    }
    if constexpr (K <= 5) {
        gauss_rows<K>(p.M, a, [&](int r, float2 y) { p.psi[off[r]] = y; });
    } else {
        float2 y[D];
        for (int r = 0; r < D; ++r) {
            float2 acc = make_float2(0.f, 0.f);
            for (int c = 0; c < D; ++c) cmac(acc, p.M.dev[r * D + c], a[c]);
            y[r] = acc;
        }
        for (int r = 0; r < D; ++r) p.psi[off[r]] = y[r];
    }
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
    constexpr int D = 1 << K;
    for (int r = 0; r < D; ++r)
        for (int c = 0; c < D; ++c) {
            const cf m = d.m[(size_t)r * D + c];
            M.P[r][c] = m.real();
            M.S[r][c] = m.real() + m.imag();
            M.Q[r][c] = m.imag() - m.real();
            M.cm[r][c] = make_float2(m.real(), m.imag());
        }
}
template <>
void fill_matrix<6>(MatStore<6>& M, const ApplyDesc& d) {
    M.dev = d.dev_m;
}

// Tensor map of the state for a tile of 2^nH runs of 2^r amplitudes (run j
// at dep(j << r)).  Dimension 0 covers index bits [0, H_0) with a box of 2^r
// (the run); every maximal group of consecutive gate qubits H_g..H_g+m-1
// opens a dimension covering bits [H_g, next group) with a box of 2^m (the
// gate bits are its low bits, the tile base supplies the rest as the
// coordinate).  The box is then exactly the tile in tile-index order, and
// one tensor copy moves a whole tile (runs longer than 256 amplitudes take
// two dimensions; groups beyond rank 5 are iterated: 2^nx copies per tile).
// rank = 0 when it does not fit or the driver has no encoder: per-run copies.
using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn tensor_map_encoder() {
    static EncodeTiledFn fn = []() -> EncodeTiledFn {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            return nullptr;
        return reinterpret_cast<EncodeTiledFn>(f);
    }();
    return fn;
}
void encode_tile_map(CUtensorMap& map, int& rank, int* tstart, int* tbits, int& nx, int* xpos, float2* psi, int n,
                     int r, const int* H, int nH, bool swz128) {
    rank = 0;
    nx = 0;
    // dimension(s) of the run: [0, c) and, for r > c, [c, H_0) with a box of 2^(r-c); c = 8
    // (256 amplitudes, the box limit), or 4 (128 B rows) with the 128 B swizzle
    const int c = swz128 ? 4 : 8;
    if (r > c + 8 || (swz128 && r < c)) return;
    int start[12], hbits[12], nd = 0;
    start[nd] = 0;
    hbits[nd] = std::min(r, c);
    ++nd;
    if (r > c) {
        start[nd] = c;
        hbits[nd] = r - c;
        ++nd;
    }
    int gfirst[SV_MAX_FUSED + 1], ng = 0;  // first H index of each group of consecutive gate qubits
    for (int b = 0; b < nH; ++b)
        if (b == 0 || H[b] != H[b - 1] + 1) gfirst[ng++] = b;
    gfirst[ng] = nH;
    const int keep = std::min(ng, 5 - nd);  // groups with their own dimension
    for (int g = 0; g < keep; ++g) {
        start[nd] = H[gfirst[g]];
        hbits[nd] = gfirst[g + 1] - gfirst[g];
        ++nd;
    }
    for (int b = gfirst[keep]; b < nH; ++b) xpos[nx++] = H[b];  // the rest: one copy per combination
    if (nx > 4) return;
    cuuint64_t gdim[5], gstride[4];
    cuuint32_t box[5], estr[5];
    for (int d = 0; d < nd; ++d) {
        const int end = d + 1 < nd ? start[d + 1] : n;
        const int bits = end - start[d];
        if (bits > 31 || bits < hbits[d] || hbits[d] > 8) {
            nx = 0;
            return;
        }
        gdim[d] = 1ull << bits;
        box[d] = 1u << hbits[d];
        estr[d] = 1;
        if (d > 0) gstride[d - 1] = 8ull << start[d];
        tstart[d] = start[d];
        tbits[d] = bits;
    }
    EncodeTiledFn enc = tensor_map_encoder();
    if (!enc || enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, (cuuint32_t)nd, psi, gdim, gstride, box, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, swz128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                    CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
        nx = 0;
        return;
    }
    rank = nd;
}

// Bank-conflict factor (wavefronts / ideal) of the group gathers of warp 0 for
// a tile laid out with XOR swizzle swz (phys bit i+1 ^= parity(t & swz[i])): 16 B words are served per quarter warp, 8 B per
// half warp; a phase costs as many wavefronts as the most distinct words in
// one bank group.  gpt = 2: lane t gathers the group pair (2t, 2t+1) (or,
// PAIR, groups 2t and its partner at bit ng0); gpt = 1: lane t one group.
double gather_conflicts(int K, int gpt, bool pair, const int* tl, int ng0, const uint32_t* swz) {
    auto phys = [&](uint32_t t) {
        return t ^ ((__builtin_popcount(t & swz[0]) & 1) << 1) ^ ((__builtin_popcount(t & swz[1]) & 1) << 2) ^
               ((__builtin_popcount(t & swz[2]) & 1) << 3);
    };
    auto slot = [&](uint32_t g) {
        for (int b = 0; b < K; ++b) g += g & (~0u << tl[b]);
        return g;
    };
    auto locf = [&](int mm) {
        uint32_t o = 0;
        for (int b = 0; b < K; ++b)
            if ((mm >> b) & 1) o |= 1u << tl[b];
        return o;
    };
    int wf = 0, ideal = 0;
    auto count = [&](const uint32_t* addr, int bytes) {
        const int lpp = 128 / bytes;
        for (int ph = 0; ph < 32; ph += lpp) {
            int worst = 0;
            for (int bank = 0; bank < lpp; ++bank) {
                uint32_t seen[32];
                int ns = 0;
                for (int l = ph; l < ph + lpp; ++l) {
                    if ((int)((addr[l] / bytes) % lpp) != bank) continue;
                    bool dup = false;
                    for (int s = 0; s < ns; ++s) dup |= seen[s] == addr[l];
                    if (!dup) seen[ns++] = addr[l];
                }
                worst = std::max(worst, ns);
            }
            wf += worst;
            ++ideal;
        }
    };
    const int D = 1 << K;
    uint32_t a[32];
    if (gpt == 2) {
        for (int m = 0; m < (pair ? D / 2 : D); ++m)
            for (int h = 0; h < (pair ? 2 : 1); ++h) {
                for (int t = 0; t < 32; ++t)
                    a[t] = 8u * phys(slot(2u * t) ^ (h ? (1u << ng0) : 0u) ^ locf(pair ? 2 * m : m));
                count(a, 16);
            }
    } else {
        for (int m = 0; m < (pair ? D / 2 : D); ++m) {
            for (int t = 0; t < 32; ++t) a[t] = 8u * phys(slot((uint32_t)t) ^ locf(pair ? 2 * m : m));
            count(a, pair ? 16 : 8);
        }
    }
    return ideal ? (double)wf / ideal : 1.0;
}

template <int K>
cudaError_t launch_tile_k(float2* psi, int n, const ApplyDesc& d, cudaStream_t st) {
    constexpr int GPT = (K <= 4) ? 2 : 1;
    TileParams<K> p;
    std::memset(&p, 0, sizeof(p));
    p.psi = psi;
    fill_matrix<K>(p.M, d);
    p.T = d.T;
    p.r = d.r;
    const bool pair = d.q[0] == 0;
    int tl[SV_MAX_FUSED];  // tile-local gate positions
    for (int b = 0; b < K; ++b) {
        if (d.q[b] < p.r) {
            tl[b] = d.q[b];
        } else {
            tl[b] = p.r + p.nH;
            p.Hpos[p.nH++] = d.q[b];
        }
    }
    p.nzt = K;
    for (int b = 0; b < K; ++b) {
        p.ztpos[b] = tl[b];
        p.zthigh[b] = ~0u << tl[b];
    }
    uint32_t gmask = 0;
    for (int b = 0; b < K; ++b) gmask |= 1u << tl[b];
    int ng[32], nng = 0;  // non-gate tile bits, ascending
    for (int t = 0; t < p.T; ++t)
        if (!((gmask >> t) & 1)) ng[nng++] = t;
    // Bank-conflict-free gathers: one shared-memory phase is 8 lanes of 16 B
    // (or 16 lanes of 8 B when GPT = 1 and bit 0 is free).  Lanes run over the
    // non-gate bits `lane`; every bit in {1,2,3} that is fixed within one gather
    // (a gate bit, or the pair-of-groups bit) is XORed with one lane bit >= 4.
    const int gpt = d.tc ? 1 : GPT;
    std::vector<int> lane;
    uint32_t fixed = gmask;
    if (gpt == 2) {
        // ng[0] selects the group of the pair (bit 0 when free -> inside the 16 B word)
        if (pair) fixed |= 1u << ng[0];
        for (int i = 1; i < nng && (int)lane.size() < 3; ++i) lane.push_back(ng[i]);
    } else {
        const int W = pair ? 3 : 4;
        for (int i = 0; i < nng && (int)lane.size() < W; ++i) lane.push_back(ng[i]);
    }
    std::vector<int> hl;
    for (int t : lane)
        if (t >= 4) hl.push_back(t);
    size_t jh = 0;
    for (int f = 1; f <= 3; ++f)
        if (((fixed >> f) & 1) && jh < hl.size()) p.swz[f - 1] = 1u << hl[jh++];
    // Bulk-copy (warp-specialised) loop.  A bulk copy cannot apply the 16 B XOR
    // swizzle of the 16 B-copy loop, so its tiles are either unswizzled or
    // laid out with the TMA's 128 B swizzle (16 B chunk bits 1..3 ^= amplitude
    // bits 4..6, tensor copies only).  Gates with no qubit in {1,2,3} need no
    // swizzle; for the others the layout with fewer bank conflicts on the group
    // gathers is taken (host model, gather_conflicts) when it is at most 2-way
    // (tensor cores) / 4-way (SIMT) conflicted -- measured at 30 qubits
    // (DESIGN.md §11): 2-way always beats the swizzled 16 B-copy loop, 4-way
    // breaks even on SIMT k = 4 and loses on the k = 6 tensor-core path,
    // 8-way loses badly.  k = 3 SIMT keeps the 16 B-copy loop (0.7 % faster).
    bool ws = false, swz128 = false;
    {
        static const uint32_t kNone[3] = {0u, 0u, 0u}, k128[3] = {1u << 4, 1u << 5, 1u << 6};
        const bool natural = p.swz[0] == 0 && p.swz[1] == 0 && p.swz[2] == 0;
        const bool simt = !d.tc && K <= 5 && K != 3;
        const bool eligible = SVB_WS && p.nH <= 6 && (simt || d.tci);
        const bool force = SVB_WS_UNSWZ == 1, never = SVB_WS_UNSWZ == 0;
        double cf = 1.0;
        if (eligible && !natural) {
            cf = gather_conflicts(K, gpt, pair, tl, ng[0], kNone);
            const double c128 = gather_conflicts(K, gpt, pair, tl, ng[0], k128);
            // SIMT: the fewer conflicts win; tensor cores: unswizzled whenever it is
            // at most 2-way (its >= 2 KB runs can use per-run bulk copies, which
            // measured faster there than tensor copies: k = 5 2.86 vs 2.96 ms)
            const bool better = d.tci ? (cf > 2.0 && c128 <= 2.0) : c128 < cf;
            if (better && SVB_SWZ128) {
                swz128 = true;
                cf = c128;
            }
        }
        const bool low_ok = (simt && K != 5 && cf <= 4.0) || (d.tci && cf <= 2.0);
        if (eligible && (natural || (!never && (low_ok || force)))) {
            // runs of <= 2 KB (and every k = 6 tensor-core tile) move as tensor
            // copies (encode_tile_map): per-run bulk copies of 1 KB runs measured
            // 10-40 % slower, of 2 KB runs 8 % slower inside a circuit; tensor
            // copies of >= 4 KB runs 1-3 % slower than per-run bulk copies
            const uint32_t minrun = SVB_WS_MINRUN;
            const bool tmap = swz128 || (SVB_TMAP >= 0 ? SVB_TMAP == 1 : (p.r <= 8 || (d.tci && K == 6) || (gpt == 2 && pair)));
            if (tmap)
                encode_tile_map(p.tmap, p.trank, p.tstart, p.tbits, p.tnx, p.txpos, psi, n, p.r, p.Hpos, p.nH, swz128);
            ws = swz128 ? p.trank > 0 : ((8u << p.r) >= minrun || p.trank > 0);
        }
        if (!ws) {
            swz128 = false;
            p.trank = 0;
        } else {
            for (int i = 0; i < 3; ++i) p.swz[i] = swz128 ? k128[i] : 0u;
        }
    }
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
    const int nloc = pair ? (1 << (K - 1)) : (1 << K);
    for (int m = 0; m < nloc; ++m) {
        const int mm = pair ? (m << 1) : m;
        uint32_t o = 0;
        for (int b = 0; b < K; ++b)
            if ((mm >> b) & 1) o |= 1u << tl[b];
        p.loc[m] = sw(o);
    }
    if (gpt == 2 && pair) p.gsec = sw(1u << ng[0]);
    {
        // monomial detection on the complex64 matrix (exact zeros)
        constexpr int D = 1 << K;
        int src[D];
        bool mono = true;
        uint64_t used = 0;
        for (int r = 0; r < D && mono; ++r) {
            int cnt = 0;
            for (int c = 0; c < D; ++c) {
                const cf m = d.m[(size_t)r * D + c];
                if (m.real() != 0.f || m.imag() != 0.f) {
                    ++cnt;
                    src[r] = c;
                }
            }
            if (cnt != 1 || ((used >> src[r]) & 1)) mono = false;
            else used |= 1ull << src[r];
        }
        p.mono = mono ? 1 : 0;
        if (mono) {
            for (int r = 0; r < D; ++r) {
                uint32_t o = 0, oc = 0;
                for (int b = 0; b < K; ++b) {
                    if ((r >> b) & 1) o |= 1u << tl[b];
                    if ((src[r] >> b) & 1) oc |= 1u << tl[b];
                }
                p.mloc[r] = sw(o);
                p.ploc[r] = sw(oc);
                const cf m = d.m[(size_t)r * D + src[r]];
                p.mdiag[r] = make_float2(m.real(), m.imag());
            }
        }
    }
    // threads: one (GPT = 1) or two (GPT = 2) groups each per compute step
    const int wbits = p.T - K - (gpt == 2 ? 1 : 0);
    const uint32_t work = wbits >= 0 ? (1u << wbits) : 0u;
    const uint32_t nthr = d.tc ? (d.tci ? tci_threads(K) : 128u) : std::min<uint32_t>(256, std::max<uint32_t>(32, work));
    p.iters = (int)std::max<uint32_t>(1, work / nthr);
    const uint32_t units = 1u << (p.T - 1);
    p.upt = (int)(units / nthr);
    if (p.T < K + (gpt == 2 ? 1 : 0) || work < 32 || p.upt < 1 || p.upt > 64 || (work < nthr && !d.tci)) {
        SmallParams<K> sp;
        std::memset(&sp, 0, sizeof(sp));
        sp.psi = psi;
        sp.n_groups = 1ull << (n - K - d.nc);
        for (int b = 0; b < K; ++b) sp.q[b] = d.q[b];
        std::vector<int> z(d.q, d.q + K);
        for (int c = 0; c < d.nc; ++c) {
            z.push_back(d.cq[c]);
            sp.ones |= 1ull << d.cq[c];
        }
        std::sort(z.begin(), z.end());
        sp.nz = (int)z.size();
        for (size_t i = 0; i < z.size(); ++i) sp.zpos[i] = z[i];
        fill_matrix<K>(sp.M, d);
        apply_small<K><<<(unsigned)((sp.n_groups + 255) / 256), 256, 0, st>>>(sp);
        return cudaGetLastError();
    }
    for (int i = 0; i < p.upt; ++i) {
        p.goff[i] = 8ull * dep(2ull * nthr * i);
        p.soff[i] = sw(2u * nthr * i);
    }
    {
        std::vector<int> z(p.Hpos, p.Hpos + p.nH);
        for (int c = 0; c < d.nc; ++c) {
            z.push_back(d.cq[c]);
            p.ones |= 1ull << d.cq[c];
        }
        std::sort(z.begin(), z.end());
        p.nZ = (int)z.size();
        for (size_t i = 0; i < z.size(); ++i) p.Zhigh[i] = ~0ull << z[i];
    }
    p.n_tiles = 1ull << (n - p.T - d.nc);
    int STG = d.tc ? 2 : stages_for(K);
    if constexpr (K >= 4) {
        if (d.tci) STG = TciShape<K>::STAGES;
    }
    size_t smem = (size_t)STG * ((size_t)8 << p.T);
    if (K == 6 && !d.tci) smem += 64 * 64 * 8;
#if SVB_SMEM_PLANES
    if (K >= 2 && K <= 3 && !d.tc && !p.mono) smem += (size_t)3 * 4 << (2 * K);
#endif
    if constexpr (K >= 4) {
        if (d.tci) smem += TciShape<K>::SMEM;
    }
    // bulk-copy loop: run offsets, and its shared memory (tiles, mode area, mbarriers)
    if (ws) {
        for (uint32_t j = 0; j < (1u << p.nH); ++j) p.roff[j] = 8ull * dep((uint64_t)j << p.r);
        const int nb = d.tci ? STG : SVB_WS_STAGES;
        smem = (size_t)nb * ((size_t)8 << p.T) + 16u * nb + 1024u;  // + alignment of the tiles to 1 KB
        if constexpr (K >= 4) {
            if (d.tci) smem += TciShape<K>::SMEM;
        }
        if (!d.tci && !p.mono && K >= 2 && K <= 3) smem += (size_t)3 * 4 << (2 * K);
    }
    if constexpr (K == 4 || K == 5) {
        if (d.tc && !d.tci) smem += 2 * TcShape<K>::W_BYTES + 64;
    }
    const int per_sm_smem = std::max(1, (int)((227 * 1024) / (smem + 1024)));
    const uint64_t grid = std::max<uint64_t>(1, std::min<uint64_t>(p.n_tiles, (uint64_t)num_sms() * per_sm_smem));
    auto go = [&](auto kern, uint32_t threads = 0) -> cudaError_t {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        kern<<<(unsigned)grid, threads ? threads : nthr, smem, st>>>(p);
        return cudaGetLastError();
    };
    if constexpr (K >= 4) {
        if (d.tci) {
            if (p.T != TciShape<K>::T) return cudaErrorInvalidConfiguration;
            p.wi8 = d.dev_wi8;
            if (ws) return pair ? go(apply_tci_ws<K, true>, nthr + 32) : go(apply_tci_ws<K, false>, nthr + 32);
            return pair ? go(apply_tci<K, true>) : go(apply_tci<K, false>);
        }
    }
#if SVB_TF32X3
    if constexpr (K == 4 || K == 5) {
        if (d.tc) {
            if (p.T != 12) return cudaErrorInvalidConfiguration;
            return pair ? go(apply_tc<K, true>) : go(apply_tc<K, false>);
        }
    }
#else
    if (d.tc) return cudaErrorInvalidConfiguration;  // only the int8 path is built
#endif
    if constexpr (K <= 5) {
        if (ws) {
            if (p.mono) return pair ? go(apply_high_ws<K, true, true>, nthr + 32) : go(apply_high_ws<K, false, true>, nthr + 32);
            return pair ? go(apply_high_ws<K, true, false>, nthr + 32) : go(apply_high_ws<K, false, false>, nthr + 32);
        }
    }
    if (p.mono) {
        if (d.high) return pair ? go(apply_high<K, true, true>) : go(apply_high<K, false, true>);
        return pair ? go(apply_low<K, true, true>) : go(apply_low<K, false, true>);
    }
    if (d.high) return pair ? go(apply_high<K, true, false>) : go(apply_high<K, false, false>);
    return pair ? go(apply_low<K, true, false>) : go(apply_low<K, false, false>);
}

}  // namespace

size_t wi8_bytes(int k) {
    const int D = 1 << k, KR = 2 * D, N = 2 * D;
    return (size_t)3 * N * KR + (size_t)N * 4;
}

void pack_wi8(const ApplyDesc& d, uint8_t* out) {
    const int D = 1 << d.k, KR = 2 * D, N = 2 * D;
    const uint32_t SBO = KR * 8, BS = (uint32_t)N * KR;
    std::memset(out, 0, wi8_bytes(d.k));
    float* fcol = reinterpret_cast<float*>(out + 3 * BS);
    const bool have64 = d.m64.size() == d.m.size();
    for (int n = 0; n < N; ++n) {
        const int r = n >> 1, ni = n & 1;
        double w[128];
        double mx = 0.0;
        for (int kk = 0; kk < KR; ++kk) {
            const int c = kk >> 1, ki = kk & 1;
            const std::complex<double> m =
                have64 ? d.m64[(size_t)r * D + c] : std::complex<double>(d.m[(size_t)r * D + c]);
            w[kk] = (ni == 0) ? (ki == 0 ? m.real() : -m.imag()) : (ki == 0 ? m.imag() : m.real());
            mx = std::max(mx, std::fabs(w[kk]));
        }
        int f = 0;
        std::frexp(mx, &f);  // mx < 2^f
        f = std::max(f, -100);
        fcol[n] = std::ldexp(1.0f, f - tci_shift(d.k));  // column half of the output scale
        // Round to 22-bit integers, then match the column's exact squared norm:
        // plain rounding changes each column norm by ~2^-23, and for a unitary
        // that is a systematic per-gate change of the state norm (DESIGN.md
        // §11: ~1e-8 per apply, 1.8e-6 of fidelity over a 30-qubit circuit).
        // Flipping the rounding direction of an entry (it stays within one
        // unit of its exact value) changes the integer sum of squares by
        // 2|wi| +- 1; entries are visited from the largest down, so the
        // residual ends near the smallest entries' granularity.
        int64_t wi[128];
        double sx[128];
        double target = 0.0, cur = 0.0;
        for (int kk = 0; kk < KR; ++kk) {
            sx[kk] = std::ldexp(w[kk], 22 - f);
            wi[kk] = (int64_t)std::nearbyint(sx[kk]);
            target += sx[kk] * sx[kk];
            cur += (double)wi[kk] * (double)wi[kk];
        }
        int order[128];
        for (int kk = 0; kk < KR; ++kk) order[kk] = kk;
        std::sort(order, order + KR, [&](int a, int b) { return std::llabs(wi[a]) > std::llabs(wi[b]); });
        for (int i = 0; i < KR; ++i) {
            const int kk = order[i];
            const double delta = target - cur;
            const int64_t s = (sx[kk] > (double)wi[kk]) ? 1 : -1;  // the other rounding direction
            if (std::fabs(sx[kk] - (double)(wi[kk] + s)) >= 1.0) continue;
            const double change = (double)(2 * wi[kk] * s + 1);
            if (std::fabs(delta - change) < std::fabs(delta)) {
                wi[kk] += s;
                cur += change;
            }
        }
        for (int kk = 0; kk < KR; ++kk) {
            const int32_t v = (int32_t)wi[kk];
            // balanced signed base-256 digits (as the kernel slices the state)
            const int32_t d2 = (int32_t)(int8_t)(v & 0xFF);
            const int32_t r1 = (v - d2) >> 8;
            const int32_t d1 = (int32_t)(int8_t)(r1 & 0xFF);
            const int32_t d0 = (r1 - d1) >> 8;
            const uint32_t off = (uint32_t)(n >> 3) * SBO + (uint32_t)(kk >> 4) * 128u + (uint32_t)(n & 7) * 16u +
                                 (uint32_t)(kk & 15);
            out[off] = (uint8_t)(d0 & 0xFF);
            out[BS + off] = (uint8_t)(d1 & 0xFF);
            out[2 * BS + off] = (uint8_t)(d2 & 0xFF);
        }
    }
}

bool tc_supported(int n_local, const ApplyDesc& d) {
    return ((d.k == 4 || d.k == 5) && n_local >= 13) || (d.k == 6 && n_local >= 14);
}

void plan_apply(int n, ApplyDesc& d) {
    {
        const int D = 1 << d.k;
        uint64_t used = 0;
        bool mono = (int)d.m.size() == D * D;
        for (int r = 0; r < D && mono; ++r) {
            int cnt = 0, src = -1;
            for (int c = 0; c < D; ++c) {
                const cf m = d.m[(size_t)r * D + c];
                if (m.real() != 0.f || m.imag() != 0.f) {
                    ++cnt;
                    src = c;
                }
            }
            if (cnt != 1 || ((used >> src) & 1)) mono = false;
            else used |= 1ull << src;
        }
        d.mono = mono;
        // Tensor cores for dense gates; d.tc_mode (sv_set_option
        // SV_OPT_APPLY_PATH) selects the path:
        //   3 (auto, default): k = 5, 6 on the exact int8-slice tensor-core path
        //     (SIMT k = 5, 6 are FP32-issue bound), k <= 4 SIMT (HBM-bound or
        //     close to it);
        //   2: the int8 path for k = 4..6;   0: SIMT only;
        //   1: TF32x3 for k = 4, 5 -- quarantined: its accumulation truncates
        //     toward zero, shrinking the norm by ~4u / ~7u per apply (DESIGN.md
        //     §11), so it exists only in builds with -DSVB_TF32X3=1.
        const int tc_mode = (d.tc_mode == 1 && !SVB_TF32X3) ? 0 : d.tc_mode;
        const bool want = (tc_mode == 1 && d.k <= 5) || tc_mode == 2 || (tc_mode == 3 && d.k >= 5);
        d.tc = !mono && want && d.nc == 0 && tc_supported(n, d);
        d.tci = d.tc && tc_mode != 1;
    }
    uint64_t gm = 0;
    for (int b = 0; b < d.k; ++b) gm |= 1ull << d.q[b];
    d.high = (gm & kLowMask) == 0;
    // tile: runs of >= 16 amplitudes (128 B); grow the run until the tile
    // reaches the target size (32 KB for k <= 4).
    const int target = std::min(n, d.k <= 5 ? 12 : (d.tci ? 13 : 14));
    auto tile_bits = [&](int rr) {
        int t = rr;
        for (int b = 0; b < d.k; ++b)
            if (d.q[b] >= rr) ++t;
        return t;
    };
    int minc = n;
    for (int c = 0; c < d.nc; ++c) minc = std::min(minc, d.cq[c]);
    const int nfree = n - d.nc;  // qubits a tile may span
    int r = std::min(std::min(nfree, 4), minc);
    while (r < n && r < minc && tile_bits(r) < std::min(target, nfree)) ++r;
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
