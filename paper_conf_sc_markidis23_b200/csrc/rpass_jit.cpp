// rpass_jit.cpp -- pass-specialised register-blocked kernels (SURVEY.md §8f
// NEXT-2; related work [12]: several gates per memory pass).
//
// The generic apply_rpass kernel (blocked.cu) reads its phase plan from the
// kernel parameters and dispatches every gate through a compare tree on a
// gate code.  ncu on a 20-gate pass of the 30q RQC (profiles/r2_*) put only
// 42 % of its instructions in the FFMA2 complex MACs: the per-gate dispatch,
// the per-phase address tables and the uniform-datapath chains between them
// cost as much issue time as the math.  Here the same plan -- the phases
// (register positions R, lane positions, 16 B or 8 B gathers), every gate's
// kind and register mask, every shared-memory and global offset -- is
// written out as straight-line PTX for one launch chunk and assembled for
// sm_100a by the driver's JIT (ptxas: ~0.1-0.3 s per kernel; going through
// CUDA C++ and NVVM took 15-130 s) when the circuit is created; only the matrices,
// the state pointer and the tile count remain launch parameters, so circuits
// with the same structure share kernels (process-wide cache keyed by the
// PTX text).
//
// The arithmetic is the generic kernel's, operation for operation (the same
// FFMA2 sequence per complex MAC, the same order over columns), so both
// produce bit-identical states; tests/test_gpu_jit.py checks that.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstring>
#include <map>
#include <mutex>
#include <sstream>
#include <thread>

#include "kernels.h"

#ifndef SVB_JIT_SECTOR_DIRECT
#define SVB_JIT_SECTOR_DIRECT 1  // direct stores also for 32 B-sector layouts of the last phase
#endif
#ifndef SVB_JIT_ANY_DIRECT
#define SVB_JIT_ANY_DIRECT 0  // the last phase always stores straight to HBM, any layout (measured: 30q 23.5 -> 27.2 ms: scattered 8/16 B stores)
#endif
#ifndef SVB_JIT_M
#define SVB_JIT_M 5  // log2 amplitudes per thread of the complex64 pass kernels (4: 16 per thread, 64 registers)
#endif
#ifndef SVB_JIT_M64
#define SVB_JIT_M64 5  // log2 amplitudes per thread of the complex128 pass kernels for 13-qubit tiles (32: 256 threads,
                       // <= 255 registers; 30q D14 59.3 -> 54.4 ms); 12-qubit and smaller tiles keep 16 per thread
#endif
#ifndef SVB_JIT_M14
#define SVB_JIT_M14 6  // ... for 14-qubit tiles: 64 per thread (256 threads, <= 255 registers, 8 warps per SM)
#endif
#ifndef SVB_JIT_P0_M
#define SVB_JIT_P0_M 5  // the compute-bound product-state first pass keeps 32 per thread (16 warps per SM: 30q 21.52 -> 21.0 ms)
#endif
#ifndef SVB_JIT_BINS_M
#define SVB_JIT_BINS_M 0  // nonzero: log2 amplitudes per thread of the circuit's last pass (it writes the bins)
#endif
#ifndef SVB_JIT_M14_RUN
#define SVB_JIT_M14_RUN 4  // ... when the tile's runs are >= 2^this amplitudes
#endif
#ifndef SVB_JIT_RING
#define SVB_JIT_RING 0  // two warp groups over three tile buffers per CTA (loads 1.5 tiles ahead)
#endif
#ifndef SVB_JIT_DB
#define SVB_JIT_DB 0  // two tile buffers per CTA: the next tile loads during the whole current tile
#endif
#ifndef SVB_JIT_CZFOLD
#define SVB_JIT_CZFOLD 1  // CZ sign flips on register bits as pending signs: 1 materialised at the phase end; 2 also folded into each register's last write (no change on the RQC: no sign is pending at a phase end)
#endif
#ifndef SVB_JIT_PL
#define SVB_JIT_PL 0  // three quarters of the next tile land in a spare buffer during the whole current tile
#endif
#ifndef SVB_JIT_L2PF
#define SVB_JIT_L2PF 0  // tile loads with an L2 prefetch-size hint: 1 = 128 B, 2 = 256 B (the neighbouring tile's run)
#endif
#ifndef SVB_JIT_PF
#define SVB_JIT_PF 0  // L2 bulk prefetch of the next tile at the top of each tile (pass kernels)
#endif

namespace svb {

struct RpJitKernel {
    std::string key;  // chunk_key (cache key)
    std::string src;  // PTX
    int nthr = 0;
    int T = 0;
    size_t smem = 0;
    size_t param_bytes = 0;  // sizeof(JP) of the generated kernel
    size_t nm = 0;           // float4 matrix slots
    std::mutex mu;           // guards the lazy module load
    cudaLibrary_t lib = nullptr;
    cudaKernel_t kern = nullptr;
    int blocks_per_sm = 0;
    uint64_t dev_mask = 0;   // devices on which the smem attribute is set
};

namespace {
// log2 amplitudes per thread of a pass kernel: 16 (complex128); 64 for
// 14-qubit complex64 tiles without dense two-qubit gates (fewer phases per
// pass: 30q D14 24.8 -> 23.7 ms; with dense 4 x 4 matvecs, e.g. fSim, the
// 8 warps of such a CTA stall on the FFMA2 chains: Sycamore 30q 0.114 ->
// 0.156 s); else 32 (the generic kernel's, so the two stay bit-identical)
// The 64-amplitude form only for tiles of runs >= 2^SVB_JIT_M14_RUN
// amplitudes (A/B, round 2: 30q D14 with 128 B runs 24.8 -> 23.7 ms; 32q
// D20 with 64 B runs 137.5 -> 142.5 ms, with 128 B runs unchanged)
// A two-qubit gate with exactly one nonzero per row and column (e.g.
// fSim(pi/2, phi), iSWAP, SWAP with phases): out_r = m_r a_perm[r] (reading
// R11, two-qubit monomial form).  complex64 pass kernels with SV_OPT_PASS_SPEC.
bool monomial2(const PassDesc& pd, const PassGate& pg, int perm[4], std::complex<double> m[4]) {
    if (!pd.spec || pd.wide || pg.k != 2 || gate_kind(pd, pg) != 0 || pd.mats64.size() < pg.moff + 32) return false;
    const double* M = pd.mats64.data() + pg.moff;
    double big = 0;
    for (int e = 0; e < 16; ++e) big = std::max(big, std::abs(std::complex<double>(M[2 * e], M[2 * e + 1])));
    const double tiny = 1e-9 * big;
    int used = 0;
    for (int r = 0; r < 4; ++r) {
        int c0 = -1;
        for (int c = 0; c < 4; ++c)
            if (std::abs(std::complex<double>(M[2 * (4 * r + c)], M[2 * (4 * r + c) + 1])) > tiny) {
                if (c0 >= 0) return false;
                c0 = c;
            }
        if (c0 < 0 || ((used >> c0) & 1)) return false;
        used |= 1 << c0;
        perm[r] = c0;
        m[r] = std::complex<double>(M[2 * (4 * r + c0)], M[2 * (4 * r + c0) + 1]);
    }
    return true;
}
int jit_m(const PassDesc& pd) {
    if (pd.wide) return pd.S.size() >= 13 ? SVB_JIT_M64 : 4;
    if (pd.S.size() < 14 || pd.r < SVB_JIT_M14_RUN) return SVB_JIT_M;
    int perm[4];
    std::complex<double> m[4];
    for (const auto& g : pd.gates)
        if (g.k == 2 && gate_kind(pd, g) == 0 && !monomial2(pd, g, perm, m)) return SVB_JIT_M;
    if (SVB_JIT_P0_M && !pd.pinit_v.empty()) return SVB_JIT_P0_M;  // product-state first pass
    if (SVB_JIT_BINS_M && pd.bins) return SVB_JIT_BINS_M;  // the last pass (sampler bins)
    return SVB_JIT_M14;
}

std::mutex g_cache_mu;
std::map<std::string, std::shared_ptr<RpJitKernel>> g_cache;
std::atomic<uint64_t> g_compiled{0}, g_hits{0};
std::atomic<uint64_t> g_compile_ns{0};

constexpr int popc(uint32_t m) { return __builtin_popcount(m); }
uint32_t pdep(uint32_t v, uint32_t mask) {
    uint32_t r = 0, b = 0;
    for (int i = 0; i < 32; ++i)
        if ((mask >> i) & 1u) {
            if ((v >> b) & 1u) r |= 1u << i;
            ++b;
        }
    return r;
}
uint32_t pext(uint32_t v, uint32_t mask) {
    uint32_t r = 0, b = 0;
    for (int i = 0; i < 32; ++i)
        if ((mask >> i) & 1u) {
            if ((v >> i) & 1u) r |= 1u << b;
            ++b;
        }
    return r;
}

// global amplitude offset (within the tile's base) of tile index t
struct TileMap {
    int r = 0;
    std::vector<int> H;  // tile positions >= r -> qubit
    uint64_t dep(uint64_t t) const {
        uint64_t g = t & ((1ull << r) - 1ull);
        const uint64_t h = t >> r;
        for (size_t b = 0; b < H.size(); ++b)
            if ((h >> b) & 1ull) g += 1ull << H[b];
        return g;
    }
};

// ---------------------------------------------------------------------------
// Structured one-qubit gates (reading R11).  A one-qubit matrix U
// whose rows are multiples of (1, i^p) -- U = diag(u00, u10) [[1, i^p0],
// [1, i^p1]], the "row form" of H, sqrt(X), sqrt(Y), T sqrt(X), T sqrt(Y) --
// or whose columns are multiples of (1, i^k) -- U = [[1, 1], [i^k0, i^k1]]
// diag(u00, u01), the "column form" of H T -- or a diagonal one, runs as c B
// with c = u00 taken out: B's products with 1 and i^p are sign and re/im
// choices in fp32 additions (2 FADDs per output amplitude where a dense 2 x 2
// takes 8 FMAs), its other factors complex multiplies (4 operations).  The
// product C of the c's of a pass is multiplied in once by the pass's first
// chunk: into the start state (|0...0> start), a generic gate's matrix, the
// multipliers of a row-form gate, or explicitly.  Exact in real arithmetic;
// in fp32 only the rounding differs from the dense product.
using cd = std::complex<double>;
struct GSpec {
    int cls = 0;                  // 0 generic, 1 row form, 2 column form, 3 one-qubit diagonal, 4 two-qubit monomial
    int p[2] = {0, 0};            // row: out_r = s_r (a0 + i^p[r] a1); column: out1 = i^p[0] a0 + i^p[1] mu a1
    int q[2] = {0, 0};            // s_r = i^q[r] when unit[r]
    bool unit[2] = {true, true};  // diagonal: s_r multiplies the amplitudes with the gate bit = r
    cd s[2] = {1.0, 1.0};         // the non-unit s_r
    cd mu = 1.0;                  // column form: out0 = a0 + mu a1
    cd c = 1.0;                   // the scalar taken out
    int perm[4] = {0, 1, 2, 3};   // monomial: out_r = m_r a_perm[r], m_r = i^mq[r] when munit[r]
    int mq[4] = {0, 0, 0, 0};
    bool munit[4] = {true, true, true, true};
    cd ms[4] = {1.0, 1.0, 1.0, 1.0};
};
cd ipow(int q) {
    static const cd u[4] = {cd(1, 0), cd(0, 1), cd(-1, 0), cd(0, -1)};
    return u[q & 3];
}
bool unit_exp(cd z, int& e) {
    static const cd u[4] = {cd(1, 0), cd(0, 1), cd(-1, 0), cd(0, -1)};
    for (int k = 0; k < 4; ++k)
        if (std::abs(z - u[k]) <= 1e-9) {
            e = k;
            return true;
        }
    return false;
}
GSpec classify(const PassDesc& pd, const PassGate& pg) {
    GSpec g;
    if (pg.k == 2) {
        cd m[4];
        if (!monomial2(pd, pg, g.perm, m)) return g;
        g.cls = 4;
        for (int r = 0; r < 4; ++r)
            if (!unit_exp(m[r], g.mq[r])) {
                g.munit[r] = false;
                g.ms[r] = m[r];
            }
        return g;
    }
    if (!pd.spec || pg.k != 1 || pd.mats64.size() < pg.moff + 8) return g;
    const int kind = gate_kind(pd, pg);
    const double* m = pd.mats64.data() + pg.moff;
    const cd u00(m[0], m[1]), u01(m[2], m[3]), u10(m[4], m[5]), u11(m[6], m[7]);
    const double big = std::max(std::max(std::abs(u00), std::abs(u01)), std::max(std::abs(u10), std::abs(u11)));
    const double tiny = 1e-9 * big;
    if (kind == 1) {
        if (std::abs(u00) <= tiny) return g;
        g.cls = 3;
        g.c = u00;
        if (!unit_exp(u11 / u00, g.q[1])) {
            g.unit[1] = false;
            g.s[1] = u11 / u00;
        }
        return g;
    }
    if (kind != 0) return g;
    if (std::abs(u00) > tiny && std::abs(u10) > tiny && unit_exp(u01 / u00, g.p[0]) && unit_exp(u11 / u10, g.p[1])) {
        g.cls = 1;
        g.c = u00;
        if (!unit_exp(u10 / u00, g.q[1])) {
            g.unit[1] = false;
            g.s[1] = u10 / u00;
        }
        return g;
    }
    GSpec h;
    if (std::abs(u00) > tiny && std::abs(u01) > tiny && unit_exp(u10 / u00, h.p[0]) && unit_exp(u11 / u01, h.p[1])) {
        h.cls = 2;
        h.c = u00;
        h.mu = u01 / u00;
        return h;
    }
    return GSpec{};
}
// The gates of a pass classified, and how the launch chunk [g0, g1) applies
// the pass scalar C (chunk 0 only): mode 1 start state, 2 folded into the
// generic gate `fold`, 3 into the multipliers of the structured gate `fold`,
// 4 explicit multiply after the chunk's last phase.
struct ChunkSpec {
    std::vector<GSpec> g;
    cd C = 1.0;
    int mode = 0;
    int fold = -1;
};
ChunkSpec chunk_spec(const PassDesc& pd, size_t g0, size_t g1, bool zinit) {
    ChunkSpec cs;
    cs.g.resize(pd.gates.size());
    if (!pd.spec) return cs;
    bool any = false;
    for (size_t i = 0; i < pd.gates.size(); ++i) {
        cs.g[i] = classify(pd, pd.gates[i]);
        cs.C *= cs.g[i].c;
        any = any || cs.g[i].cls != 0;
    }
    if (g0 != 0 || !any) return cs;
    if (zinit) {
        cs.mode = 1;
        return cs;
    }
    for (size_t i = g0; i < g1; ++i)
        if (cs.g[i].cls == 0 && gate_kind(pd, pd.gates[i]) != 2) {
            cs.mode = 2;
            cs.fold = (int)i;
            return cs;
        }
    // a row-form gate: +1 operation per amplitude when its row 1 already
    // has a multiplier, +2 otherwise; a diagonal with one: +2
    for (int pass = 0; pass < 3; ++pass)
        for (size_t i = g0; i < g1; ++i) {
            GSpec& x = cs.g[i];
            const bool ok = pass == 0 ? x.cls == 1 && !x.unit[1] : pass == 1 ? x.cls == 1 : x.cls == 3 && !x.unit[1];
            if (!ok) continue;
            for (int r = 0; r < 2; ++r) {
                if (x.unit[r]) x.s[r] = ipow(x.q[r]);
                x.s[r] *= cs.C;
                x.unit[r] = false;
            }
            cs.mode = 3;
            cs.fold = (int)i;
            return cs;
        }
    cs.mode = 4;
    return cs;
}

// Launch chunks of a pass: tiles up to 13 qubits as the generic kernel's
// (rpass_chunks: <= 64 gates, <= 48 phases; bit-identical states), 14-qubit
// tiles up to kJitPassMaxGates gates and 96 phases with at most 1800 matrix
// slots of 16 B (the parameter space, 32 KB)
std::vector<RpPhaseHost> phases_cached(const PassDesc& pd, size_t g0, size_t g1, int M, bool wide);
std::vector<std::pair<size_t, size_t>> jit_chunks(const PassDesc& pd) {
    const int M = jit_m(pd);
    if (pd.S.size() < 14) return rpass_chunks(pd, M, pd.wide);
    std::vector<std::pair<size_t, size_t>> out;
    const size_t ng = pd.gates.size();
    auto slots = [&](size_t g) {
        const int kind = gate_kind(pd, pd.gates[g]), k = pd.gates[g].k;
        return kind == 2 ? 0u : kind == 1 ? (1u << k) : (1u << (2 * k));
    };
    size_t g0 = 0;
    while (g0 < ng) {
        size_t g1 = g0, sl = 0;
        while (g1 < ng && g1 - g0 < (size_t)kJitPassMaxGates && sl + slots(g1) <= 1800) sl += slots(g1++);
        while ((int)phases_cached(pd, g0, g1, M, pd.wide).size() > 96) g1 = g0 + (g1 - g0) / 2;
        out.push_back({g0, g1});
        g0 = g1;
    }
    return out;
}

// PTX text builder: amplitudes live in %a0..%a31 (one .b64 = packed
// (re, im) complex64 each), rewritten in place; ptxas renames them.
struct Ptx {
    std::ostringstream o;
    int nr = 0, nrd = 0, np = 0;
    std::string r32() { return "%r" + std::to_string(nr++); }
    std::string r64() { return "%rd" + std::to_string(nrd++); }
    std::string pr() { return "%p" + std::to_string(np++); }
    template <class... A>
    void op(const A&... a) {
        o << "\t";
        (o << ... << a);
        o << ";\n";
    }
};

// global address "[base+off]" operand (PTX offsets are 32-bit signed)
std::string gaddr(Ptx& P, const std::string& base, uint64_t off) {
    if (off == 0) return "[" + base + "]";
    if (off < (1ull << 31)) return "[" + base + "+" + std::to_string(off) + "]";
    const std::string t = P.r64();
    P.op("add.s64 ", t, ", ", base, ", ", off);
    return "[" + t + "]";
}

// tile base byte offset = bit-deposit of the tile index u into the qubit
// positions outside S (runs of consecutive free positions), times 8
void emit_tbase(Ptx& P, const std::vector<int>& S, int n_local, const std::string& u, const std::string& out) {
    std::vector<char> in(64, 0);
    for (int q : S) in[q] = 1;
    P.op("mov.b64 ", out, ", 0");
    int b = 0;  // next bit of u
    for (int q = 0; q < n_local;) {
        if (in[q]) {
            ++q;
            continue;
        }
        int e = q;
        while (e < n_local && !in[e]) ++e;
        const int L = e - q;
        const std::string t = P.r64();
        // (u >> b) & (2^L - 1)) << (q + 3)
        if (q + 3 >= b) P.op("shl.b64 ", t, ", ", u, ", ", q + 3 - b);
        else P.op("shr.u64 ", t, ", ", u, ", ", b - q - 3);
        const uint64_t mask = (L >= 61 ? ~0ull : ((1ull << L) - 1ull)) << (q + 3);
        P.op("and.b64 ", t, ", ", t, ", ", mask);
        P.op("or.b64 ", out, ", ", out, ", ", t);
        b += L;
        q = e;
    }
}

// Structural key of a launch chunk: everything the PTX text depends on
// (tile, state size, flags and every gate's size, positions and kind).
std::string chunk_key(const PassDesc& pd, int n_local, size_t g0, size_t g1, bool zinit) {
    std::string k;
    k.reserve(16 + 8 * (g1 - g0));
    auto put = [&](int v) {
        k += std::to_string(v);
        k += ',';
    };
    if (pd.wide) k += "w,";
    put(jit_m(pd));
    put(n_local);
    put(pd.r);
    put(zinit ? 1 : 0);
    put(zinit && !pd.pinit_v.empty() ? 1 : 0);
    put(pd.bins && g1 == pd.gates.size() ? 1 : 0);
    for (int q : pd.S) put(q);
    k += '|';
    const ChunkSpec cs = chunk_spec(pd, g0, g1, zinit);
    for (size_t g = g0; g < g1; ++g) {
        const PassGate& pg = pd.gates[g];
        put(pg.k * 16 + gate_kind(pd, pg));
        for (int b = 0; b < pg.k; ++b) put(pg.pos[b]);
        const GSpec& x = cs.g[g];
        if (x.cls) k += 's';
        if (x.cls == 4)
            for (int r = 0; r < 4; ++r) put(x.perm[r] + 4 * x.mq[r] + (x.munit[r] ? 16 : 0));
        if (x.cls) put(64 * x.cls + 16 * x.p[0] + 4 * x.p[1] + x.q[0] * 256 + x.q[1] * 1024 + (x.unit[0] ? 4096 : 0) +
                       (x.unit[1] ? 8192 : 0));
    }
    if (cs.mode) {
        k += 'm';
        put(cs.mode);
        put(cs.fold);
    }
    return k;
}

// Phase plans by chunk structure (plan_phases searches every M-subset of
// the tile positions per phase: the dominant host cost of creating a
// circuit; circuits of the same structure reuse the plan)
std::mutex g_phase_mu;
std::map<std::string, std::vector<RpPhaseHost>> g_phase_cache;
std::vector<RpPhaseHost> phases_cached(const PassDesc& pd, size_t g0, size_t g1, int M, bool wide) {
    const std::string key = chunk_key(pd, 0, g0, g1, false) + "#" + std::to_string(M) + (wide ? "w" : "");
    {
        std::lock_guard<std::mutex> lk(g_phase_mu);
        auto it = g_phase_cache.find(key);
        if (it != g_phase_cache.end()) return it->second;
    }
    std::vector<RpPhaseHost> ph = plan_phases(pd, g0, g1, M, wide);
    std::lock_guard<std::mutex> lk(g_phase_mu);
    if (g_phase_cache.size() > 4096) g_phase_cache.clear();
    g_phase_cache[key] = ph;
    return ph;
}

// PTX of one launch chunk [g0, g1) of pass pd; nm receives the number of
// float4 matrix slots, mats their values (launch order).  emit == false:
// only nm and mats (the PTX is cached under chunk_key).
std::string gen_chunk(const PassDesc& pd, int n_local, size_t g0, size_t g1, bool zinit, size_t& nm,
                      std::vector<float>& mats, bool emit = true, const std::vector<float>* msrc = nullptr) {
    const std::vector<float>& pmats = msrc ? *msrc : pd.mats;
    const int M = jit_m(pd), NA = 1 << M, UPT = 1 << (M - 1);
    const int T = (int)pd.S.size();
    const int tbits = T - M;
    const uint32_t nthr = 1u << tbits;
    TileMap tm;
    tm.r = pd.r;
    for (int i = pd.r; i < T; ++i) tm.H.push_back(pd.S[i]);
    const auto phs = phases_cached(pd, g0, g1, M, false);
    const int nph = (int)phs.size();
    auto coalesced = [](const RpPhaseHost& h) {
        return h.b0 && h.lanes.size() >= 3 && h.lanes[0] == 1 && h.lanes[1] == 2 && h.lanes[2] == 3;
    };
    auto coalesced8 = [](const RpPhaseHost& h) {
        return !h.b0 && h.lanes.size() >= 4 && h.lanes[0] == 0 && h.lanes[1] == 1 && h.lanes[2] == 2 && h.lanes[3] == 3;
    };
    const RpPhaseHost& lp = phs.back();
    // direct store of the last phase's registers: full 128 B runs per quarter-
    // (16 B) / half-warp (8 B), or -- SVB_JIT_SECTOR_DIRECT -- full 32 B
    // sectors per lane pair / quad (the L2 merges the sectors of a line before
    // write-back; the whole tile is written by this CTA)
    auto sector = [](const RpPhaseHost& h) {
        return h.b0 ? (h.lanes.size() >= 1 && h.lanes[0] == 1)
                    : (h.lanes.size() >= 2 && h.lanes[0] == 0 && h.lanes[1] == 1);
    };
    const bool direct = coalesced(lp) || coalesced8(lp) || (SVB_JIT_SECTOR_DIRECT && sector(lp)) || SVB_JIT_ANY_DIRECT;
    const bool early = direct && !zinit;
    // sampling bin weights (the last launch of a circuit's last pass): 16-
    // amplitude bins = tile bits 0..3, reduced over the lanes that hold them
    const bool bins = pd.bins && g1 == pd.gates.size() && pd.r >= kSampleBinBits;
    // ring (SVB_JIT_RING): two warp groups per CTA, each on its own tiles,
    // over three tile buffers; the group that releases buffer b (its last
    // read of tile k) loads tile k + 3 (the other group's) into it, tracked by
    // an mbarrier -- loads are issued one and a half tiles ahead
    const bool ring = SVB_JIT_RING != 0;
    // double buffering (SVB_JIT_DB): tile u computes in buffer %cur while
    // tile u + grid loads into %alt; the last phase frees %cur and loads
    // tile u + 2 grid into it
    const bool db = SVB_JIT_DB && !ring && !zinit;
    // pre-landing (SVB_JIT_PL): the tile buffer is only free between the
    // last phase's gather and the next tile's first gather, so a single
    // buffer leaves HBM idle during all earlier phases.  A spare buffer of
    // 3/4 tile takes quarters 0..2 (top two tile bits) of the next tile,
    // issued right after this tile's first gather; quarter 3 lands in the
    // tile buffer once the last phase has read it.  The first gather of a
    // tile reads quarters 0..2 from the spare buffer (same swizzle).
    const bool pl = SVB_JIT_PL && !ring && !db && !zinit && M >= 3;
    const uint32_t tile_bytes = 8u << T;
    // matrix slots first (their count fixes the parameter layout)
    mats.clear();
    const ChunkSpec cs = chunk_spec(pd, g0, g1, zinit);
    // structured-gate multiplier slot: (sr, sr, si, si)
    auto put_s = [&](cd z) {
        mats.push_back((float)z.real());
        mats.push_back((float)z.real());
        mats.push_back((float)z.imag());
        mats.push_back((float)z.imag());
    };
    std::vector<size_t> gbase(pd.gates.size(), 0);
    for (int ph = 0; ph < nph; ++ph)
        for (int g : phs[ph].gates) {
            const PassGate& pg = pd.gates[g];
            const int kind = gate_kind(pd, pg);
            const GSpec& x = cs.g[g];
            gbase[g] = mats.size() / 4;
            if (x.cls == 2) {
                put_s(x.mu);
                continue;
            }
            if (x.cls == 4) {
                for (int r = 0; r < 4; ++r)
                    if (!x.munit[r]) put_s(x.ms[r]);
                continue;
            }
            if (x.cls) {
                for (int r = 0; r < 2; ++r)
                    if (!x.unit[r]) put_s(x.s[r]);
                continue;
            }
            if (kind == 2) continue;
            const int D = 1 << pg.k;
            const float* mg = pmats.data() + pg.moff;
            const cd f = cs.mode == 2 && g == cs.fold ? cs.C : cd(1.0);
            const int ne = kind == 1 ? D : D * D;
            for (int e = 0; e < ne; ++e) {
                const int src = kind == 1 ? e * D + e : e;
                float mr = mg[2 * src], mi = mg[2 * src + 1];
                if (f != cd(1.0)) {
                    const cd z = cd(mr, mi) * f;
                    mr = (float)z.real();
                    mi = (float)z.imag();
                }
                mats.push_back(mr);
                mats.push_back(mr);
                mats.push_back(-mi);
                mats.push_back(mi);
            }
        }
    // the pass scalar as the start amplitude (|0...0> start without the
    // product state) or for the explicit multiply
    size_t cslot = 0;
    if (cs.mode == 1 && pd.pinit_v.empty()) {  // (C re, C im, 0, 0): the start amplitude
        cslot = mats.size() / 4;
        mats.push_back((float)cs.C.real());
        mats.push_back((float)cs.C.imag());
        mats.push_back(0.f);
        mats.push_back(0.f);
    } else if (cs.mode == 4) {
        cslot = mats.size() / 4;
        put_s(cs.C);
    }
    // product-state start: register factors of phase 0 (32 slots) and the
    // two vectors of every lane position (2 slots per thread bit)
    const bool pinit = zinit && !pd.pinit_v.empty();
    size_t reg0 = 0, lane0 = 0;
    if (pinit) {
        auto put = [&](std::complex<double> z) {
            mats.push_back((float)z.real());
            mats.push_back((float)z.real());
            mats.push_back((float)-z.imag());
            mats.push_back((float)z.imag());
        };
        const RpPhaseHost& P0 = phs[0];
        reg0 = mats.size() / 4;
        for (uint32_t j = 0; j < (uint32_t)NA; ++j) {
            std::complex<double> z = cs.mode == 1 ? cs.C : cd(1.0);
            for (int b = 0; b < M; ++b) z *= pd.pinit_v[2 * P0.R[b] + ((j >> b) & 1u)];
            put(z);
        }
        lane0 = mats.size() / 4;
        for (int b = 0; b < tbits; ++b) {
            put(pd.pinit_v[2 * P0.lanes[b]]);
            put(pd.pinit_v[2 * P0.lanes[b] + 1]);
        }
    }
    nm = mats.size() / 4;
    // parameter tail (rpj_jit_tail): psi, n_tiles, zone, h1, tabA, tabB
    const size_t off_psi = std::max<size_t>(nm, 1) * 16, off_nt = off_psi + 8, off_zone = off_psi + 16,
                 off_h1 = off_psi + 20, off_ta = off_psi + 24, off_tb = off_psi + 32, off_bins = off_psi + 40;
    const size_t pbytes = off_psi + 48;
    if (!emit) return std::string();

    Ptx P;
    // S5 weight floor(fl(re^2 + im^2) 2^62) of the packed amplitude a (the
    // products are exact in fp64, so the FMA form equals state.cu weight()),
    // into acc (first: set, else add)
    auto wadd = [&](const std::string& a, bool first) {
        P.op("mov.b64 {%lo, %hi}, ", a);
        P.op("cvt.f64.f32 %dre, %lo");
        P.op("cvt.f64.f32 %dim, %hi");
        P.op("mul.rn.f64 %dp, %dim, %dim");
        P.op("fma.rn.f64 %dp, %dre, %dre, %dp");
        P.op("mul.rn.f64 %dp, %dp, 0d43D0000000000000");  // 2^62
        if (first) {
            P.op("cvt.rzi.u64.f64 %w, %dp");
        } else {
            P.op("cvt.rzi.u64.f64 %wt, %dp");
            P.op("add.u64 %w, %w, %wt");
        }
    };
    // sum over the lane bits `lbits` (exact uint64 butterfly), then the lane
    // whose bits there are 0 (%p_bw) stores the bin of the slot at `addr`
    auto wstore = [&](const std::vector<int>& lbits, const std::string& addr) {
        for (int b : lbits) {
            P.op("mov.b64 {%wl, %wh}, %w");
            P.op("shfl.sync.bfly.b32 %wl2, %wl, ", 1 << b, ", 31, -1");
            P.op("shfl.sync.bfly.b32 %wh2, %wh, ", 1 << b, ", 31, -1");
            P.op("mov.b64 %wt, {%wl2, %wh2}");
            P.op("add.u64 %w, %w, %wt");
        }
        P.op("sub.s64 %bo, ", addr, ", %psi");
        P.op("shr.u64 %bo, %bo, 4");
        P.op("add.s64 %bo, %bo, %bins");
        P.op("@%p_bw st.global.u64 [%bo], %w");
    };
    auto gaddr_reg = [&](const std::string& base, uint64_t off) {  // base + off into a register
        const std::string t = P.r64();
        P.op("add.s64 ", t, ", ", base, ", ", off);
        return t;
    };
    // ---- structured gates (GSpec), on packed amplitudes: i^k X is a swap
    // and per-lane negations that ptxas folds into the FADD2 / FFMA2 operand
    // modifiers (.LO_HI, .NP, -), so out = i^q (a0 + i^p a1) is one FADD2 and
    // a complex multiply s t = sr t + si (i t) one FMUL2 + one FFMA2
    // pending signs (SVB_JIT_CZFOLD, structured path only: with
    // SV_OPT_PASS_SPEC 0 the kernels stay bit-identical to the generic one,
    // which a negated zero would break): register j holds sgn[j] ? -a_j : a_j.
    // A CZ on two register bits only flips them; structured gates take the
    // sign difference of their inputs into the rotation exponent (i^2 = -1)
    // and pass the first input's sign on; dense gates whose inputs disagree
    // materialise them first; every register is materialised at the end of
    // the phase (FMUL2 by -1 where still pending).
    std::vector<int> sgn(NA, 0);
    auto materialize = [&](uint32_t j) {
        if (!sgn[j]) return;
        P.op("mul.rn.f32x2 %a", j, ", %a", j, ", %mneg1");
        sgn[j] = 0;
    };
    // SVB_JIT_CZFOLD 2: a dry run of the phase records each register's last
    // write (write events numbered in emission order) and its final pending
    // sign; the real run negates that write instead (a rotation by i^2 in the
    // operand modifiers: no extra instruction) when the sign would be pending
    bool dry = false;
    int wev = 0;
    std::vector<int> lastw(NA, -1), need(NA, 0);
    auto fold_out = [&](uint32_t j) -> bool {  // a foldable write of register j
        const int e = wev++;
        if (dry || SVB_JIT_CZFOLD < 2) {
            lastw[j] = e;
            return false;
        }
        return e == lastw[j] && need[j];
    };
    auto note_write = [&](uint32_t j) {  // a write that cannot take the sign
        const int e = wev++;
        if (dry) lastw[j] = e;
    };
    int nrot = 0;
    auto rot = [&](const std::string& X, int k) -> std::string {
        k &= 3;
        if (k == 0) return X;
        const std::string t = "%rt" + std::to_string(nrot++ % 8);
        P.op("mov.b64 {%rlo, %rhi}, ", X);
        if (k == 1) {
            P.op("neg.f32 %rnh, %rhi");
            P.op("mov.b64 ", t, ", {%rnh, %rlo}");
        } else if (k == 2) {
            P.op("neg.f32 %rnl, %rlo");
            P.op("neg.f32 %rnh, %rhi");
            P.op("mov.b64 ", t, ", {%rnl, %rnh}");
        } else {
            P.op("neg.f32 %rnl, %rlo");
            P.op("mov.b64 ", t, ", {%rhi, %rnl}");
        }
        return t;
    };
    // d = i^q (A + i^p B)
    auto plin = [&](const std::string& d, int q, int p, const std::string& A, const std::string& B) {
        const std::string x = rot(A, q), y = rot(B, p + q);
        P.op("add.rn.f32x2 ", d, ", ", x, ", ", y);
    };
    // d = s t (neg: -s t), s from slot (sr, sr, si, si); d may alias t
    auto pmul = [&](const std::string& d, const std::string& t, size_t slot, bool neg = false) {
        P.op("ld.param.v2.b64 {%qsr, %qsi}, [rpj_param_0+", 16 * slot, "]");
        P.op("mul.rn.f32x2 %py, ", rot(t, neg ? 2 : 0), ", %qsr");
        const std::string it = rot(t, neg ? 3 : 1);
        P.op("fma.rn.f32x2 ", d, ", ", it, ", %qsi, %py");
    };
    auto emit_spec = [&](const GSpec& x, uint32_t mask, size_t base) {
        if (x.cls == 4) {  // two-qubit monomial: out_r = m_r a_perm[r] (copies, rotations, multiplies)
            size_t slr[4];
            size_t nxt = base;
            for (int r = 0; r < 4; ++r) slr[r] = x.munit[r] ? 0 : nxt++;
            const uint32_t rest = ((1u << M) - 1u) & ~mask;
            for (uint32_t gi = 0; gi < (uint32_t)NA / 4; ++gi) {
                const uint32_t b0 = pdep(gi, rest);
                int s_in[4];
                for (int c = 0; c < 4; ++c) s_in[c] = sgn[b0 | pdep(c, mask)];
                for (int r = 0; r < 4; ++r) sgn[b0 | pdep(r, mask)] = s_in[x.perm[r]];
                for (int c = 0; c < 4; ++c) P.op("mov.b64 %x", c, ", %a", b0 | pdep(c, mask));
                for (int r = 0; r < 4; ++r) {
                    const uint32_t jr = b0 | pdep(r, mask);
                    const std::string d = "%a" + std::to_string(jr);
                    const std::string src = "%x" + std::to_string(x.perm[r]);
                    const bool ng = fold_out(jr);
                    if (ng) sgn[jr] ^= 1;
                    if (!x.munit[r]) {
                        pmul(d, src, slr[r], ng);
                    } else if ((x.mq[r] + (ng ? 2 : 0)) & 3) {
                        const std::string t = rot(src, x.mq[r] + (ng ? 2 : 0));
                        P.op("mul.rn.f32x2 ", d, ", ", t, ", %pone");
                    } else {
                        P.op("mov.b64 ", d, ", ", src);
                    }
                }
            }
            return;
        }
        size_t sl[2] = {base, base};
        if (!x.unit[0]) sl[1] = base + 1;
        if (x.cls == 3) {  // diagonal: s_r on the amplitudes whose gate bit is r
            for (uint32_t j = 0; j < (uint32_t)NA; ++j) {
                const int r = (j & mask) ? 1 : 0;
                const std::string a = "%a" + std::to_string(j);
                if (!x.unit[r]) {
                    const bool ng = fold_out(j);
                    if (ng) sgn[j] ^= 1;
                    pmul(a, a, sl[r], ng);
                } else if (x.q[r]) {  // i^q a (one FMUL2 by 1 carries the rotation)
                    const bool ng = fold_out(j);
                    if (ng) sgn[j] ^= 1;
                    const std::string t = rot(a, x.q[r] + (ng ? 2 : 0));
                    P.op("mul.rn.f32x2 ", a, ", ", t, ", %pone");
                }
            }
            return;
        }
        for (uint32_t j0 = 0; j0 < (uint32_t)NA; ++j0) {
            if (j0 & mask) continue;
            const uint32_t j1 = j0 | mask;
            const std::string a0 = "%a" + std::to_string(j0), a1 = "%a" + std::to_string(j1);
            // stored a1 = (-1)^(sgn1 - sgn0) relative to a0: a rotation by i^2
            const int dz = (sgn[j0] ^ sgn[j1]) ? 2 : 0;
            sgn[j1] = sgn[j0];  // both outputs carry the first input's sign
            const bool n0 = fold_out(j0), n1 = fold_out(j1);
            if (n0) sgn[j0] ^= 1;
            if (n1) sgn[j1] ^= 1;
            const int z[2] = {n0 ? 2 : 0, n1 ? 2 : 0};
            if (x.cls == 2) {  // out0 = a0 + mu a1, out1 = i^p0 a0 + i^p1 (mu a1)
                pmul("%pt", a1, sl[0]);
                plin("%po0", z[0], dz, a0, "%pt");
                const std::string u = rot(a0, x.p[0] + z[1]), v = rot("%pt", x.p[1] + dz + z[1]);
                P.op("add.rn.f32x2 %po1, ", u, ", ", v);
            } else {  // row form: out_r = s_r (a0 + i^p_r a1)
                for (int r = 0; r < 2; ++r) {
                    const std::string d = "%po" + std::to_string(r);
                    if (x.unit[r]) {
                        plin(d, x.q[r] + z[r], x.p[r] + dz, a0, a1);
                    } else {
                        plin("%pt", 0, x.p[r] + dz, a0, a1);
                        pmul(d, "%pt", sl[r], z[r] != 0);
                    }
                }
            }
            P.op("mov.b64 ", a0, ", %po0");
            P.op("mov.b64 ", a1, ", %po1");
        }
    };
    // ---- prologue: thread constants
    P.op("mov.u32 %t_id, %tid.x");
    P.op("mov.u32 %rsm0, rsm");
    P.op("mov.u32 %cur, rsm");
    if (ring) {
        P.op("shr.u32 %grp, %t_id, ", tbits);
        P.op("and.b32 %t_id, %t_id, ", nthr - 1);  // thread index within the group
        P.op("add.u32 %bid, %grp, 1");
    }
    P.op("mov.b64 %dthr, 0");
    P.op("mov.b32 %sthr, 0");
    if (direct) P.op("mov.b64 %dg, 0");
    for (int b = 0; b < tbits; ++b) {
        const std::string t = P.r32(), q = P.pr();
        P.op("and.b32 ", t, ", %t_id, ", 1u << b);
        P.op("setp.ne.u32 ", q, ", ", t, ", 0");
        const uint32_t t2 = 2u << b;  // unit 0 of the thread: tile index 2 tid
        P.op("@", q, " add.s64 %dthr, %dthr, ", 8 * tm.dep(t2));
        P.op("@", q, " xor.b32 %sthr, %sthr, ", fold_swz(t2, T) << 3);
        if (direct) P.op("@", q, " add.s64 %dg, %dg, ", 8 * tm.dep(1ull << lp.lanes[b]));
    }
    if (pinit) {
        // thread factor: product of the lane vectors selected by the thread index
        P.op("mov.b64 %tf, 1065353216");  // (1.0f, 0.0f)
        for (int b = 0; b < tbits; ++b) {
            const std::string t = P.r32(), q = P.pr();
            P.op("and.b32 ", t, ", %t_id, ", 1u << b);
            P.op("setp.ne.u32 ", q, ", ", t, ", 0");
            P.op("ld.param.v2.b64 {%ml, %mh}, [rpj_param_0+", 16 * (lane0 + 2 * b), "]");
            P.op("ld.param.v2.b64 {%x0, %x1}, [rpj_param_0+", 16 * (lane0 + 2 * b + 1), "]");
            P.op("selp.b64 %ml, %x0, %ml, ", q);
            P.op("selp.b64 %mh, %x1, %mh, ", q);
            P.op("mov.b64 {%lo, %hi}, %tf");
            P.op("mov.b64 %xs0, {%hi, %lo}");
            P.op("fma.rn.f32x2 %y, %ml, %tf, %zero");
            P.op("fma.rn.f32x2 %tf, %mh, %xs0, %y");
        }
        P.op("ld.param.u32 %h1, [rpj_param_0+", off_h1, "]");
        P.op("ld.param.u64 %tabA, [rpj_param_0+", off_ta, "]");
        P.op("ld.param.u64 %tabB, [rpj_param_0+", off_tb, "]");
    }
    P.op("ld.param.u64 %psi, [rpj_param_0+", off_psi, "]");
    P.op("ld.param.u64 %ntiles, [rpj_param_0+", off_nt, "]");
    P.op("ld.param.u32 %zone, [rpj_param_0+", off_zone, "]");
    // bin layout: the last phase's register / lane bits that hold tile bits
    // 0..3 (direct store), or the write-back units (tile bit 0 = the pair,
    // bits 1..3 = lane bits 0..2)
    uint32_t bin_regs = 0;
    std::vector<int> bin_lanes;
    if (direct) {
        for (int j = 0; j < M; ++j)
            if (lp.R[j] < 4) bin_regs |= 1u << j;
        for (int b = 0; b < tbits; ++b)
            if (lp.lanes[b] < 4) bin_lanes.push_back(b);
    } else {
        bin_lanes = {0, 1, 2};
    }
    if (bins) {
        P.op("ld.param.u64 %bins, [rpj_param_0+", off_bins, "]");
        uint32_t lm = 0;
        for (int b : bin_lanes) lm |= 1u << b;
        P.op("and.b32 %r_c, %t_id, ", lm);
        P.op("setp.eq.u32 %p_bw, %r_c, 0");
    }
    P.op("mov.u32 %r_c, %ctaid.x");
    P.op("cvt.u64.u32 %u, %r_c");
    P.op("mov.u32 %r_c, %nctaid.x");
    P.op("cvt.u64.u32 %grid, %r_c");
    // quarters: bit q of `qmask` loads the units whose top two tile bits
    // are q (unit i: tile index 2 (tid + nthr i), top bits = i >> (M - 3));
    // with pre-landing quarters 0..2 go to the spare buffer
    auto loadtile = [&](const std::string& g, const std::string& pred, const std::string& base = "%cur",
                        unsigned qmask = 15u) {
        for (int i = 0; i < UPT; ++i) {
            const int quarter = i >> (M - 3);
            if (!((qmask >> quarter) & 1u)) continue;
            const std::string sa = P.r32();
            P.op("xor.b32 ", sa, ", %sthr, ", fold_swz(2u * nthr * i, T) << 3);
            P.op("add.s32 ", sa, ", ", sa, ", ", pl && quarter < 3 ? std::string("%spr") : base);
            const std::string ga = gaddr(P, g, 8 * tm.dep(2ull * nthr * i));
            P.op(pred, "cp.async.cg.shared.global", SVB_JIT_L2PF == 1 ? ".L2::128B" : SVB_JIT_L2PF == 2 ? ".L2::256B" : "",
                 " [", sa, "], ", ga, ", 16");
        }
    };
    const std::string gbar = ring ? "bar.sync %bid, " + std::to_string(nthr) : std::string("bar.sync 0");
    if (ring) {
        // mbarriers full[0..2] after the three buffers; initial loads: group 0
        // tiles 0 and 2, group 1 tile 1 (tile k of this CTA -> buffer k mod 3)
        P.op("add.u32 %mb0, %rsm0, ", 3 * tile_bytes);
        P.op("setp.eq.u32 %p_z, %t_id, 0");
        P.op("setp.eq.and.u32 %p_z, %grp, 0, %p_z");
        for (int b = 0; b < 3; ++b) {
            P.op("add.u32 %fb, %mb0, ", 8 * b);
            P.op("@%p_z mbarrier.init.shared.b64 [%fb], ", nthr);
        }
        P.op("fence.mbarrier_init.release.cluster");
        P.op("bar.sync 0");
        if (!zinit)
            for (int k0 = 0; k0 < 3; ++k0) {
                const std::string q = P.pr();
                P.op("add.s64 %un, %u, ", 0);
                for (int t = 0; t < k0; ++t) P.op("add.s64 %un, %un, %grid");
                P.op("setp.lt.u64 ", q, ", %un, %ntiles");
                P.op("setp.eq.and.u32 ", q, ", %grp, ", k0 % 2, ", ", q);
                P.op("@!", q, " bra $INIT", k0);
                emit_tbase(P, pd.S, n_local, "%un", "%tbo");
                P.op("add.s64 %gnext, %psi, %tbo");
                P.op("add.s64 %gnext, %gnext, %dthr");
                P.op("add.u32 %cur, %rsm0, ", k0 * tile_bytes);
                loadtile("%gnext", "");
                P.op("add.u32 %fb, %mb0, ", 8 * k0);
                P.op("cp.async.mbarrier.arrive.noinc.shared.b64 [%fb]");
                P.o << "$INIT" << k0 << ":\n";
            }
        // this group's first tile: k = grp
        P.op("cvt.u64.u32 %rdk, %grp");
        P.op("mul.lo.u64 %rdk, %rdk, %grid");
        P.op("add.s64 %u, %u, %rdk");
        P.op("mov.u32 %kk, %grp");
        P.op("mov.u32 %bb, %grp");
        P.op("setp.ge.u64 %p_out, %u, %ntiles");
        P.op("@%p_out bra $DONE");
    } else {
        P.op("setp.ge.u64 %p_out, %u, %ntiles");
        P.op("@%p_out bra $DONE");
        emit_tbase(P, pd.S, n_local, "%u", "%tbo");
        P.op("add.s64 %gtile, %psi, %tbo");
        P.op("add.s64 %gcur, %gtile, %dthr");
        if (pl) P.op("add.u32 %spr, %rsm0, ", tile_bytes);
        if (!zinit) loadtile("%gcur", "");
        P.op("cp.async.commit_group");
        if (db) {  // the second tile into the other buffer
            P.op("add.u32 %alt, %rsm0, ", tile_bytes);
            P.op("add.s64 %un, %u, %grid");
            P.op("setp.lt.u64 %p_next, %un, %ntiles");
            emit_tbase(P, pd.S, n_local, "%un", "%tbo");
            P.op("add.s64 %gnext, %psi, %tbo");
            P.op("add.s64 %gnext, %gnext, %dthr");
            loadtile("%gnext", "@%p_next ", "%alt");
            P.op("cp.async.commit_group");
        }
    }
    P.o << "$LOOP:\n";
    if (ring) {
        // this tile: buffer bb, full[bb]; the tile 3 ahead (other group) goes
        // into the same buffer once this group is done reading it
        P.op("mul.lo.u32 %r_c, %bb, ", tile_bytes);
        P.op("add.u32 %cur, %rsm0, %r_c");
        P.op("shl.b32 %r_c, %bb, 3");
        P.op("add.u32 %fb, %mb0, %r_c");
        emit_tbase(P, pd.S, n_local, "%u", "%tbo");
        P.op("add.s64 %gtile, %psi, %tbo");
        P.op("add.s64 %gcur, %gtile, %dthr");
        P.op("add.s64 %un, %u, %grid");
        P.op("add.s64 %un, %un, %grid");
        P.op("add.s64 %un, %un, %grid");  // u + 3 grid
        P.op("setp.lt.u64 %p_next, %un, %ntiles");
        emit_tbase(P, pd.S, n_local, "%un", "%tbo");
        P.op("add.s64 %gtile_next, %psi, %tbo");
        P.op("add.s64 %gnext, %gtile_next, %dthr");
        // wait for this tile: load mode phase (k / 3) & 1; zinit: buffer free
        // (released by tile k - 3) for k >= 3
        P.op("div.u32 %r_c, %kk, 3");
        if (zinit) {
            P.op("setp.ge.u32 %p_w, %kk, 3");
            P.op("@!%p_w bra $READY");
            P.op("sub.u32 %r_c, %r_c, 1");
        }
        P.op("and.b32 %par, %r_c, 1");
        P.o << "$WAIT:\n";
        P.op("mbarrier.try_wait.parity.shared.b64 %p_w, [%fb], %par");
        P.op("@!%p_w bra $WAIT");
        P.o << "$READY:\n";
    } else if (db) {
        // this tile's addresses, and the tile two ahead (loaded into %cur
        // once this tile's last phase has read it)
        emit_tbase(P, pd.S, n_local, "%u", "%tbo");
        P.op("add.s64 %gtile, %psi, %tbo");
        P.op("add.s64 %gcur, %gtile, %dthr");
        P.op("add.s64 %un, %u, %grid");
        P.op("add.s64 %un, %un, %grid");
        P.op("setp.lt.u64 %p_next, %un, %ntiles");
        emit_tbase(P, pd.S, n_local, "%un", "%tbo");
        P.op("add.s64 %gnext, %psi, %tbo");
        P.op("add.s64 %gnext, %gnext, %dthr");
    } else {
        P.op("add.s64 %un, %u, %grid");
        P.op("setp.lt.u64 %p_next, %un, %ntiles");
        emit_tbase(P, pd.S, n_local, "%un", "%tbo");
        P.op("add.s64 %gtile_next, %psi, %tbo");
        P.op("add.s64 %gnext, %gtile_next, %dthr");
    }
    if (SVB_JIT_PF && !zinit) {
        // pull the next tile's runs into L2 now (one bulk prefetch per run,
        // spread over the threads), so the cp.async of the early load finds
        // them there instead of waiting for HBM
        const int runs = 1 << (T - pd.r);
        const uint32_t rb = 8u << pd.r;
        for (int i = 0; i < (runs + (int)nthr - 1) / (int)nthr; ++i) {
            const std::string t = P.r32(), q = P.pr(), a = P.r64(), o = P.r64();
            // run index j = tid + nthr * i -> tile index j << r
            P.op("add.u32 ", t, ", %t_id, ", nthr * i);
            P.op("setp.lt.u32 ", q, ", ", t, ", ", runs);
            P.op("and.pred ", q, ", ", q, ", %p_next");
            // offset: deposit of the run index into H (the tile's positions >= r)
            P.op("mov.b64 ", o, ", 0");
            for (size_t b = 0; b < tm.H.size(); ++b) {
                const std::string tt = P.r32(), qq = P.pr();
                P.op("and.b32 ", tt, ", ", t, ", ", 1u << b);
                P.op("setp.ne.u32 ", qq, ", ", tt, ", 0");
                P.op("@", qq, " add.s64 ", o, ", ", o, ", ", 8ull << tm.H[b]);
            }
            P.op("add.s64 ", a, ", %gtile_next, ", o);
            P.op("@", q, " cp.async.bulk.prefetch.L2.global [", a, "], ", rb);
        }
    }
    if (!ring) {
        P.op(db ? "cp.async.wait_group 1" : "cp.async.wait_group 0");  // db: the newest group is the next tile
        P.op("bar.sync 0");
    }
    // ring: release buffer bb (this group is done reading it): load the tile
    // three ahead into it, or in zinit mode just mark it free
    auto release = [&]() {
        P.op(gbar);
        if (zinit) {
            P.op("mbarrier.arrive.shared.b64 %rdk, [%fb]");
        } else {
            loadtile("%gnext", "@%p_next ");
            P.op("@%p_next cp.async.mbarrier.arrive.noinc.shared.b64 [%fb]");
        }
    };
    // ---- phases
    for (int ph = 0; ph < nph; ++ph) {
        const RpPhaseHost& Ph = phs[ph];
        const bool last = ph == nph - 1;
        P.o << "\t// phase " << ph << ": R = {";
        for (int q : Ph.R) P.o << q << ",";
        P.o << "}, " << Ph.gates.size() << " gates\n";
        P.op("mov.b32 %tb, 0");
        for (int b = 0; b < tbits; ++b) {
            const std::string t = P.r32(), q = P.pr();
            P.op("and.b32 ", t, ", %t_id, ", 1u << b);
            P.op("setp.ne.u32 ", q, ", ", t, ", 0");
            P.op("@", q, " xor.b32 %tb, %tb, ", fold_swz(1u << Ph.lanes[b], T) << 3);
        }
        // pre-landed first gather: the base of an amplitude depends on its
        // quarter = (lane part of the top tile bits) | (register part);
        // one base per register part, chosen per thread
        const bool plg = pl && ph == 0;
        uint32_t qreg_mask = 0;  // register bits (of j) that are top tile bits -> quarter bit
        if (plg) {
            P.op("mov.b32 %qt, 0");
            for (int b = 0; b < tbits; ++b)
                if (Ph.lanes[b] >= T - 2) {
                    const std::string t = P.r32(), q = P.pr();
                    P.op("and.b32 ", t, ", %t_id, ", 1u << b);
                    P.op("setp.ne.u32 ", q, ", ", t, ", 0");
                    P.op("@", q, " or.b32 %qt, %qt, ", 1u << (Ph.lanes[b] - (T - 2)));
                }
            for (int v = 0; v < 4; ++v) {
                bool ok = true;  // v must be reachable from register bits
                for (int qb = 0; qb < 2; ++qb)
                    if (((v >> qb) & 1) && std::find(Ph.R.begin(), Ph.R.end(), T - 2 + qb) == Ph.R.end()) ok = false;
                if (!ok) continue;
                const std::string t = P.r32(), q = P.pr();
                P.op("or.b32 ", t, ", %qt, ", v);
                P.op("setp.eq.u32 ", q, ", ", t, ", 3");
                P.op("selp.b32 %pb", v, ", %cur, %spr, ", q);
            }
            for (int b = 0; b < M; ++b)
                if (Ph.R[b] >= T - 2) qreg_mask |= 1u << b;
        }
        auto saddr = [&](uint32_t j, bool gather = false) {
            const std::string t = P.r32();
            P.op("xor.b32 ", t, ", %tb, ", fold_swz(deposit(j, Ph.R), T) << 3);
            if (plg && gather) {
                const uint32_t v = deposit(j & qreg_mask, Ph.R) >> (T - 2);
                P.op("add.s32 ", t, ", ", t, ", %pb", v);
            } else {
                P.op("add.s32 ", t, ", ", t, ", %cur");
            }
            return t;
        };
        if (ph == 0 && pinit) {
            // tile factor from the two tables, times the thread factor
            P.op("cvt.u64.u32 %rdA, %h1");
            P.op("mov.b64 %rdB, 1");
            P.op("shl.b64 %rdB, %rdB, %h1");
            P.op("sub.s64 %rdB, %rdB, 1");
            P.op("and.b64 %rdB, %u, %rdB");
            P.op("shl.b64 %rdB, %rdB, 3");
            P.op("add.s64 %rdB, %tabA, %rdB");
            P.op("ld.global.nc.b64 %x0, [%rdB]");
            P.op("shr.u64 %rdB, %u, %h1");
            P.op("shl.b64 %rdB, %rdB, 3");
            P.op("add.s64 %rdB, %tabB, %rdB");
            P.op("ld.global.nc.b64 %x1, [%rdB]");
            auto cmul = [&](const std::string& a, const std::string& b, const std::string& out) {  // out = a * b
                P.op("mov.b64 {%lo, %hi}, ", b);
                P.op("neg.f32 %nhi, %hi");
                P.op("mov.b64 %ml, {%lo, %lo}");
                P.op("mov.b64 %mh, {%nhi, %hi}");
                P.op("mov.b64 {%lo, %hi}, ", a);
                P.op("mov.b64 %xs0, {%hi, %lo}");
                P.op("fma.rn.f32x2 %y, %ml, ", a, ", %zero");
                P.op("fma.rn.f32x2 ", out, ", %mh, %xs0, %y");
            };
            cmul("%x0", "%x1", "%x2");
            cmul("%x2", "%tf", "%x3");
            P.op("mov.b64 {%lo, %hi}, %x3");
            P.op("mov.b64 %xs1, {%hi, %lo}");
            for (int j = 0; j < NA; ++j) {
                P.op("ld.param.v2.b64 {%ml, %mh}, [rpj_param_0+", 16 * (reg0 + j), "]");
                P.op("fma.rn.f32x2 %y, %ml, %x3, %zero");
                P.op("fma.rn.f32x2 %a", j, ", %mh, %xs1, %y");
            }
        } else if (ph == 0 && zinit) {
            for (int j = 0; j < NA; ++j) P.op("mov.b64 %a", j, ", 0");
            // amplitude 0 = 1 (tile 0, thread 0, register 0) on the shard that holds it
            P.op("setp.ne.u32 %p_z, %zone, 0");
            P.op("setp.eq.and.u64 %p_z, %u, 0, %p_z");
            P.op("setp.eq.and.u32 %p_z, %t_id, 0, %p_z");
            if (cs.mode == 1 && !pinit)  // (C re, C im)
                P.op("@%p_z ld.param.b64 %a0, [rpj_param_0+", 16 * cslot, "]");
            else
                P.op("@%p_z mov.b64 %a0, 1065353216");  // (1.0f, 0.0f)
        } else if (Ph.b0) {
            for (int j = 0; j < NA / 2; ++j) {
                const std::string a = saddr(2u * j, true);
                P.op("ld.shared.v2.b64 {%a", 2 * j, ", %a", 2 * j + 1, "}, [", a, "]");
            }
        } else {
            for (int j = 0; j < NA; ++j) {
                const std::string a = saddr((uint32_t)j, true);
                P.op("ld.shared.b64 %a", j, ", [", a, "]");
            }
        }
        if (plg) {
            // every thread has read the spare buffer (and quarter 3 of the
            // tile buffer, which this phase's scatter overwrites): quarters
            // 0..2 of the next tile land during the rest of this tile
            P.op("bar.sync 0");
            loadtile("%gnext", "@%p_next ", "%cur", 7u);
            P.op("cp.async.commit_group");
        }
        if (ring && last && direct) {
            release();
        } else if (last && early) {
            // tile buffer free: the next tile's load overlaps this phase's gates
            if (!plg) P.op("bar.sync 0");
            loadtile("%gnext", "@%p_next ", "%cur", pl ? 8u : 15u);
            P.op("cp.async.commit_group");
        }
        auto gates_body = [&]() {
        for (int g : Ph.gates) {
                const PassGate& pg = pd.gates[g];
                const int kind = gate_kind(pd, pg);
                uint32_t mask = 0, tmask = 0;
                for (int b = 0; b < pg.k; ++b) {
                    const auto it = std::find(Ph.R.begin(), Ph.R.end(), pg.pos[b]);
                    if (it != Ph.R.end()) mask |= 1u << (int)(it - Ph.R.begin());
                    else tmask |= 1u << (int)(std::find(Ph.lanes.begin(), Ph.lanes.end(), pg.pos[b]) - Ph.lanes.begin());
                }
                const int D = 1 << pg.k;
                P.o << "\t// gate " << g << ": k=" << pg.k << " kind=" << kind << " mask=" << mask << " tmask=" << tmask
                    << " cls=" << cs.g[g].cls << "\n";
                if (cs.g[g].cls) {
                    emit_spec(cs.g[g], mask, gbase[g]);
                    continue;
                }
                if (kind == 2) {  // CZ-like: sign flips of both halves
                    // one FMUL2 per flipped amplitude (2 LOP3s as an xor), by -1
                    // or, when a qubit is a thread bit, by this thread's sign
                    std::string sg = "%mneg1";
                    if (popc(mask) != 2) {
                        const std::string t = P.r32(), q = P.pr();
                        P.op("and.b32 ", t, ", %t_id, ", tmask);
                        P.op("setp.eq.u32 ", q, ", ", t, ", ", tmask);
                        P.op("selp.b64 %csg, %mneg1, %pone, ", q);
                        sg = "%csg";
                    }
                    for (uint32_t j = 0; j < (uint32_t)NA; ++j)
                        if ((j & mask) == mask) {
                            if (SVB_JIT_CZFOLD && pd.spec && popc(mask) == 2) {
                                sgn[j] ^= 1;
                            } else {
                                const bool ng = fold_out(j);
                                if (ng) sgn[j] ^= 1;
                                const std::string a = "%a" + std::to_string(j);
                                P.op("mul.rn.f32x2 ", a, ", ", ng ? rot(a, 2) : a, ", ", sg);
                            }
                        }
                    continue;
                }
                const size_t base = gbase[g];
                auto mload = [&](size_t e) {  // (mr, mr) -> %ml, (-mi, mi) -> %mh
                    P.op("ld.param.v2.b64 {%ml, %mh}, [rpj_param_0+", 16 * e, "]");
                };
                auto swp = [&](const std::string& x, const std::string& out) {
                    P.op("mov.b64 {%lo, %hi}, ", x);
                    P.op("mov.b64 ", out, ", {%hi, %lo}");
                };
                if (kind == 1) {
                    for (int e = 0; e < D; ++e) {
                        mload(base + e);
                        for (uint32_t j = 0; j < (uint32_t)NA; ++j) {
                            if (pext(j, mask) != (uint32_t)e) continue;
                            swp("%a" + std::to_string(j), "%xs0");
                            P.op("fma.rn.f32x2 %y, %ml, %a", j, ", %zero");
                            P.op("fma.rn.f32x2 %a", j, ", %mh, %xs0, %y");
                            note_write(j);
                        }
                    }
                    continue;
                }
                const uint32_t rest = ((1u << M) - 1u) & ~mask;
                for (uint32_t gi = 0; gi < (uint32_t)NA / D; ++gi) {
                    const uint32_t b0 = pdep(gi, rest);
                    // a common input sign passes to the outputs; mixed signs are materialised
                    bool same = true;
                    for (int c = 1; c < D; ++c) same = same && sgn[b0 | pdep(c, mask)] == sgn[b0];
                    if (!same)
                        for (int c = 0; c < D; ++c) materialize(b0 | pdep(c, mask));
                    for (int c = 0; c < D; ++c) {
                        P.op("mov.b64 %x", c, ", %a", b0 | pdep(c, mask));
                        swp("%x" + std::to_string(c), "%xs" + std::to_string(c));
                    }
                    for (int rr = 0; rr < D; ++rr) {
                        const uint32_t dst = b0 | pdep(rr, mask);
                        note_write(dst);
                        for (int c = 0; c < D; ++c) {
                            mload(base + rr * D + c);
                            P.op("fma.rn.f32x2 %y, %ml, %x", c, ", ", c == 0 ? "%zero" : "%y");
                            P.op("fma.rn.f32x2 ", c == D - 1 ? "%a" + std::to_string(dst) : std::string("%y"), ", %mh, %xs", c,
                                 ", %y");
                        }
                    }
                }
            }
            if (last && cs.mode == 4)  // the pass scalar, explicitly
                for (int j = 0; j < NA; ++j) {
                    const bool ng = fold_out((uint32_t)j);
                    if (ng) sgn[j] ^= 1;
                    pmul("%a" + std::to_string(j), "%a" + std::to_string(j), cslot, ng);
                }
        };
        if (SVB_JIT_CZFOLD >= 2) {  // dry run: last writes and final signs
            const std::string saved = P.o.str();
            const int snr = P.nr, snrd = P.nrd, snp = P.np, srot = nrot;
            dry = true;
            wev = 0;
            std::fill(lastw.begin(), lastw.end(), -1);
            gates_body();
            need = sgn;
            P.o.str(saved);
            P.o.seekp(0, std::ios_base::end);
            P.nr = snr;
            P.nrd = snrd;
            P.np = snp;
            nrot = srot;
            dry = false;
            wev = 0;
            std::fill(sgn.begin(), sgn.end(), 0);
        }
        gates_body();
        for (int j = 0; j < NA; ++j) materialize((uint32_t)j);  // the phase's stores see true values
        if (last && direct) {
            P.op("add.s64 %gst, %gtile, %dg");
            if (lp.b0) {
                for (int j = 0; j < NA / 2; ++j)
                    P.op("st.global.cs.v2.b64 ", gaddr(P, "%gst", 8 * tm.dep(deposit(2u * j, lp.R))), ", {%a", 2 * j, ", %a",
                         2 * j + 1, "}");

            } else {
                for (int j = 0; j < NA; ++j)
                    P.op("st.global.cs.b64 ", gaddr(P, "%gst", 8 * tm.dep(deposit((uint32_t)j, lp.R))), ", %a", j);
            }
            if (bins)  // per bin slot: its registers, then the lanes holding bin bits
                for (uint32_t j0 = 0; j0 < (uint32_t)NA; ++j0) {
                    if (j0 & bin_regs) continue;
                    bool first = true;
                    for (uint32_t sub = 0; sub < (uint32_t)NA; ++sub)
                        if ((sub & ~bin_regs) == 0) {
                            wadd("%a" + std::to_string(j0 | sub), first);
                            first = false;
                        }
                    wstore(bin_lanes, gaddr_reg("%gst", 8 * tm.dep(deposit(j0, lp.R))));
                }
        } else {
            if (Ph.b0) {
                for (int j = 0; j < NA / 2; ++j) {
                    const std::string a = saddr(2u * j);
                    P.op("st.shared.v2.b64 [", a, "], {%a", 2 * j, ", %a", 2 * j + 1, "}");
                }
            } else {
                for (int j = 0; j < NA; ++j) {
                    const std::string a = saddr((uint32_t)j);
                    P.op("st.shared.b64 [", a, "], %a", j);
                }
            }
            P.op(gbar);
        }
    }
    if (!direct) {
        // write the tile back from shared memory: every unit into registers
        // first, so that the next tile's load can be issued before the stores
        // (the buffer is free once all threads have read it)
        for (int i = 0; i < UPT; ++i) {
            const std::string sa = P.r32();
            P.op("xor.b32 ", sa, ", %sthr, ", fold_swz(2u * nthr * i, T) << 3);
            P.op("add.s32 ", sa, ", ", sa, ", %cur");
            P.op("ld.shared.v2.b64 {%a", 2 * i, ", %a", 2 * i + 1, "}, [", sa, "]");
        }
        if (ring) {
            release();
        } else if (!zinit) {
            P.op("bar.sync 0");  // every thread is done with the tile buffer
            loadtile("%gnext", "@%p_next ", "%cur", pl ? 8u : 15u);
            P.op("cp.async.commit_group");
        }
        for (int i = 0; i < UPT; ++i)
            P.op("st.global.cs.v2.b64 ", gaddr(P, "%gcur", 8 * tm.dep(2ull * nthr * i)), ", {%a", 2 * i, ", %a", 2 * i + 1,
                 "}");
        if (bins)  // unit i: tile bit 0 = the pair, bits 1..3 = lane bits 0..2
            for (int i = 0; i < UPT; ++i) {
                wadd("%a" + std::to_string(2 * i), true);
                wadd("%a" + std::to_string(2 * i + 1), false);
                wstore(bin_lanes, gaddr_reg("%gcur", 8 * tm.dep(2ull * nthr * i)));
            }
    }
    if (ring) {
        // next tile of this group: k + 2 (buffer (bb + 2) mod 3)
        P.op("add.s64 %u, %u, %grid");
        P.op("add.s64 %u, %u, %grid");
        P.op("add.u32 %kk, %kk, 2");
        P.op("add.u32 %bb, %bb, 2");
        P.op("setp.ge.u32 %p_w, %bb, 3");
        P.op("@%p_w sub.u32 %bb, %bb, 3");
        P.op("setp.lt.u64 %p_w, %u, %ntiles");
        P.op("@%p_w bra $LOOP");
    } else if (db) {
        P.op("mov.u32 %r_c, %cur");
        P.op("mov.u32 %cur, %alt");
        P.op("mov.u32 %alt, %r_c");
        P.op("add.s64 %u, %u, %grid");
        P.op("setp.lt.u64 %p_w, %u, %ntiles");
        P.op("@%p_w bra $LOOP");
    } else {
        P.op("mov.b64 %gcur, %gnext");
        P.op("mov.b64 %gtile, %gtile_next");
        P.op("mov.b64 %u, %un");
        P.op("@%p_next bra $LOOP");
    }
    P.o << "$DONE:\n";
    if (ring) P.op("bar.sync 0");  // both groups: every load either group issued has been consumed
    P.op("ret");

    std::ostringstream k;
    k << "// pass-specialised register-blocked kernel (generated by rpass_jit.cpp)\n";
    k << "// T=" << T << " r=" << pd.r << " n=" << n_local << " S={";
    for (int q : pd.S) k << q << ",";
    k << "} gates " << g0 << ".." << g1 << " phases " << nph << (zinit ? " zinit" : "") << (pinit ? " product-start" : "")
      << (direct ? " direct" : "") << (bins ? " bins" : "") << (ring ? " ring" : "") << (pl ? " prelanded" : "") << "\n";
    k << ".version 8.8\n.target sm_100a\n.address_size 64\n";
    k << ".extern .shared .align 16 .b8 rsm[];\n";
    k << ".visible .entry rpj(.param .align 16 .b8 rpj_param_0[" << pbytes << "])\n";
    k << ".maxntid " << (ring ? 2 * nthr : nthr) << ", 1, 1\n.maxnreg " << (M >= 6 ? 255 : M == 5 ? 128 : 64) << "\n{\n";
    k << "\t.reg .pred %p<" << std::max(P.np, 1) << ">;\n\t.reg .pred %p_out, %p_next, %p_z, %p_bw, %p_w;\n";
    k << "\t.reg .b32 %rsm0, %grp, %bid, %mb0, %fb, %kk, %bb, %par, %alt, %spr, %qt, %pb<4>;\n\t.reg .b64 %rdk;\n";
    k << "\t.reg .f64 %dre, %dim, %dp;\n\t.reg .b64 %w, %wt, %bo, %bins;\n\t.reg .b32 %wl, %wh, %wl2, %wh2;\n";
    k << "\t.reg .b32 %r<" << std::max(P.nr, 1) << ">;\n\t.reg .b32 %t_id, %cur, %sthr, %tb, %zone, %r_c, %lo, %hi, %nhi, %h1;\n";
    k << "\t.reg .b64 %rd<" << std::max(P.nrd, 1) << ">;\n";
    k << "\t.reg .b64 %a<" << NA << ">;\n\t.reg .b64 %x<4>;\n\t.reg .b64 %xs<4>;\n";
    k << "\t.reg .f32 %rlo, %rhi, %rnl, %rnh;\n\t.reg .b64 %rt<8>, %po0, %po1, %pt, %py, %qsr, %qsi, %pone, %mneg1, %csg;\n";
    k << "\t.reg .b64 %y, %ml, %mh, %zero, %dthr, %dg, %psi, %ntiles, %u, %un, %grid, %tbo, %gtile, %gcur, %gtile_next, "
         "%gnext, %gst, %tf, %tabA, %tabB, %rdA, %rdB;\n";
    k << "\tmov.b64 %zero, 0;\n\tmov.b64 %pone, 4575657222473777152;\n\tmov.b64 %mneg1, -4647714812233515008;\n";  // (1, 1), (-1, -1)
    k << P.o.str();
    k << "}\n";
    return k.str();
}

// Assemble the PTX for this device through the driver's JIT (ptxas; the
// driver also caches the result across processes) and look the kernel up,
// which forces the module load under lazy loading.
// ---------------------------------------------------------------------------
// complex128 states (NEXT-1, Fig. 8): the same pass structure
// with 16 B amplitudes -- 16 per thread (M = 4; 64 fp64 registers), one
// LDS.128 / cp.async per amplitude, the wide fold swizzle (amplitude bits
// 0..2 ^= bits 3..5 ^ 6..8 ^ ...: 8 consecutive lanes hit 8 distinct 16 B
// bank groups), fp64 FMAs (4 per complex MAC).  Matrices travel as fp64.
uint32_t fold64(uint32_t t, int T) {
    uint32_t f = 0;
    for (int q = 3; q < T; ++q)
        if ((t >> q) & 1u) f ^= 1u << ((q - 3) % 3);
    return t ^ f;
}

std::string gen_chunk64(const PassDesc& pd, int n_local, size_t g0, size_t g1, bool zinit, size_t& nm,
                        std::vector<double>& mats, bool emit = true) {
    const int M = jit_m(pd), NA = 1 << M, UPT = NA;
    const int T = (int)pd.S.size();
    const int tbits = T - M;
    const uint32_t nthr = 1u << tbits;
    TileMap tm;
    tm.r = pd.r;
    for (int i = pd.r; i < T; ++i) tm.H.push_back(pd.S[i]);
    const auto phs = phases_cached(pd, g0, g1, M, true);
    const int nph = (int)phs.size();
    const RpPhaseHost& lp = phs.back();
    const bool direct = lp.lanes.size() >= 3 && lp.lanes[0] == 0 && lp.lanes[1] == 1 && lp.lanes[2] == 2;
    const bool early = direct && !zinit;
    mats.clear();
    // structured one-qubit gates (R11) as in gen_chunk: fp64 additions on
    // (re, im) register pairs, complex multipliers (s re, s im) per slot
    const ChunkSpec cs = chunk_spec(pd, g0, g1, zinit);
    auto put_s = [&](cd z) {
        mats.push_back(z.real());
        mats.push_back(z.imag());
    };
    std::vector<size_t> gbase(pd.gates.size(), 0);
    for (int ph = 0; ph < nph; ++ph)
        for (int g : phs[ph].gates) {
            const PassGate& pg = pd.gates[g];
            const int kind = gate_kind(pd, pg);
            const GSpec& x = cs.g[g];
            gbase[g] = mats.size() / 2;
            if (x.cls == 2) {
                put_s(x.mu);
                continue;
            }
            if (x.cls) {
                for (int r = 0; r < 2; ++r)
                    if (!x.unit[r]) put_s(x.s[r]);
                continue;
            }
            if (kind == 2) continue;
            const int D = 1 << pg.k;
            const double* mg = pd.mats64.data() + pg.moff;
            const cd f = cs.mode == 2 && g == cs.fold ? cs.C : cd(1.0);
            const int ne = kind == 1 ? D : D * D;
            for (int e = 0; e < ne; ++e) {
                const int src = kind == 1 ? e * D + e : e;
                put_s(cd(mg[2 * src], mg[2 * src + 1]) * f);
            }
        }
    size_t cslot = 0;
    if (cs.mode == 1 && pd.pinit_v.empty()) {  // the start amplitude
        cslot = mats.size() / 2;
        put_s(cs.C);
    } else if (cs.mode == 4) {
        cslot = mats.size() / 2;
        put_s(cs.C);
    }
    const bool pinit = zinit && !pd.pinit_v.empty();
    size_t reg0 = 0, lane0 = 0;
    if (pinit) {
        const RpPhaseHost& P0 = phs[0];
        reg0 = mats.size() / 2;
        for (uint32_t j = 0; j < NA; ++j) {
            std::complex<double> z = cs.mode == 1 ? cs.C : cd(1.0);
            for (int b = 0; b < M; ++b) z *= pd.pinit_v[2 * P0.R[b] + ((j >> b) & 1u)];
            mats.push_back(z.real());
            mats.push_back(z.imag());
        }
        lane0 = mats.size() / 2;
        for (int b = 0; b < tbits; ++b)
            for (int v = 0; v < 2; ++v) {
                mats.push_back(pd.pinit_v[2 * P0.lanes[b] + v].real());
                mats.push_back(pd.pinit_v[2 * P0.lanes[b] + v].imag());
            }
    }
    nm = mats.size() / 2;
    const size_t off_psi = std::max<size_t>(nm, 1) * 16, off_nt = off_psi + 8, off_zone = off_psi + 16,
                 off_h1 = off_psi + 20, off_ta = off_psi + 24, off_tb = off_psi + 32;
    const size_t pbytes = off_psi + 48;
    if (!emit) return std::string();

    Ptx P;
    P.op("mov.u32 %t_id, %tid.x");
    P.op("mov.u32 %cur, rsm");
    P.op("mov.b64 %dthr, 0");
    P.op("mov.b32 %sthr, 0");
    if (direct) P.op("mov.b64 %dg, 0");
    for (int b = 0; b < tbits; ++b) {
        const std::string t = P.r32(), q = P.pr();
        P.op("and.b32 ", t, ", %t_id, ", 1u << b);
        P.op("setp.ne.u32 ", q, ", ", t, ", 0");
        P.op("@", q, " add.s64 %dthr, %dthr, ", 16 * tm.dep(1ull << b));
        P.op("@", q, " xor.b32 %sthr, %sthr, ", fold64(1u << b, T) << 4);
        if (direct) P.op("@", q, " add.s64 %dg, %dg, ", 16 * tm.dep(1ull << lp.lanes[b]));
    }
    auto cmul = [&](const std::string& ar, const std::string& ai, const std::string& br, const std::string& bi,
                    const std::string& orr, const std::string& oi) {  // (or, oi) = a * b
        P.op("mul.rn.f64 %t0, ", ar, ", ", br);
        P.op("mul.rn.f64 %t1, ", ar, ", ", bi);
        P.op("neg.f64 %t2, ", ai);
        P.op("fma.rn.f64 ", orr, ", %t2, ", bi, ", %t0");
        P.op("fma.rn.f64 ", oi, ", ", ai, ", ", br, ", %t1");
    };
    // ---- structured gates (GSpec) on (re, im) pairs: i^k (x + i y) is a
    // choice of components and signs, so out = i^q (a0 + i^p a1) is two
    // DADDs; a multiplier s t is a complex multiply (2 DMUL + 2 DFMA)
    struct SV {  // signed component references of a complex value
        std::string r, i;
        bool nr, ni;
    };
    auto rotv = [](const std::string& xr, const std::string& xi, int k) -> SV {
        switch (k & 3) {
            case 0: return {xr, xi, false, false};
            case 1: return {xi, xr, true, false};   // i (x + i y) = -y + i x
            case 2: return {xr, xi, true, true};
            default: return {xi, xr, false, true};  // -i (x + i y) = y - i x
        }
    };
    auto sadd = [&](const std::string& d, const std::string& a, bool na, const std::string& b, bool nb) {
        if (!na && !nb) {
            P.op("add.rn.f64 ", d, ", ", a, ", ", b);
        } else if (!na) {
            P.op("sub.rn.f64 ", d, ", ", a, ", ", b);
        } else if (!nb) {
            P.op("sub.rn.f64 ", d, ", ", b, ", ", a);
        } else {
            P.op("neg.f64 %t2, ", a);
            P.op("sub.rn.f64 ", d, ", %t2, ", b);
        }
    };
    auto vadd = [&](const std::string& dr, const std::string& di, const SV& u, const SV& v) {
        sadd(dr, u.r, u.nr, v.r, v.nr);
        sadd(di, u.i, u.ni, v.i, v.ni);
    };
    auto smul = [&](const std::string& dr, const std::string& di, const std::string& tr, const std::string& ti,
                    size_t slot) {  // (dr, di) = s (tr, ti); d may alias t
        P.op("ld.param.v2.f64 {%mr, %mi}, [rpj_param_0+", 16 * slot, "]");
        cmul("%mr", "%mi", tr, ti, "%zr", "%zi");
        P.op("mov.f64 ", dr, ", %zr");
        P.op("mov.f64 ", di, ", %zi");
    };
    auto emit_spec64 = [&](const GSpec& x, uint32_t mask, size_t base) {
        size_t sl[2] = {base, base};
        if (!x.unit[0]) sl[1] = base + 1;
        auto AR = [](uint32_t j) { return "%ar" + std::to_string(j); };
        auto AI = [](uint32_t j) { return "%ai" + std::to_string(j); };
        if (x.cls == 3) {
            for (uint32_t j = 0; j < (uint32_t)NA; ++j) {
                const int r = (j & mask) ? 1 : 0;
                if (!x.unit[r]) {
                    smul(AR(j), AI(j), AR(j), AI(j), sl[r]);
                } else if (x.q[r] & 3) {
                    const SV v = rotv(AR(j), AI(j), x.q[r]);
                    P.op(v.nr ? "neg.f64 %zr, " : "mov.f64 %zr, ", v.r);
                    P.op(v.ni ? "neg.f64 %zi, " : "mov.f64 %zi, ", v.i);
                    P.op("mov.f64 ", AR(j), ", %zr");
                    P.op("mov.f64 ", AI(j), ", %zi");
                }
            }
            return;
        }
        for (uint32_t j0 = 0; j0 < (uint32_t)NA; ++j0) {
            if (j0 & mask) continue;
            const uint32_t j1 = j0 | mask;
            if (x.cls == 2) {  // out0 = a0 + mu a1, out1 = i^p0 a0 + i^p1 (mu a1)
                smul("%ptr", "%pti", AR(j1), AI(j1), sl[0]);
                vadd("%por0", "%poi0", rotv(AR(j0), AI(j0), 0), rotv("%ptr", "%pti", 0));
                vadd("%por1", "%poi1", rotv(AR(j0), AI(j0), x.p[0]), rotv("%ptr", "%pti", x.p[1]));
            } else {  // row form: out_r = s_r (a0 + i^p_r a1)
                for (int r = 0; r < 2; ++r) {
                    const std::string dr = "%por" + std::to_string(r), di = "%poi" + std::to_string(r);
                    if (x.unit[r]) {
                        vadd(dr, di, rotv(AR(j0), AI(j0), x.q[r]), rotv(AR(j1), AI(j1), x.p[r] + x.q[r]));
                    } else {
                        vadd("%ptr", "%pti", rotv(AR(j0), AI(j0), 0), rotv(AR(j1), AI(j1), x.p[r]));
                        smul(dr, di, "%ptr", "%pti", sl[r]);
                    }
                }
            }
            P.op("mov.f64 ", AR(j0), ", %por0");
            P.op("mov.f64 ", AI(j0), ", %poi0");
            P.op("mov.f64 ", AR(j1), ", %por1");
            P.op("mov.f64 ", AI(j1), ", %poi1");
        }
    };
    if (pinit) {
        P.op("mov.f64 %tfr, 0d3FF0000000000000");
        P.op("mov.f64 %tfi, 0d0000000000000000");
        for (int b = 0; b < tbits; ++b) {
            const std::string t = P.r32(), q = P.pr();
            P.op("and.b32 ", t, ", %t_id, ", 1u << b);
            P.op("setp.ne.u32 ", q, ", ", t, ", 0");
            P.op("ld.param.v2.f64 {%mr, %mi}, [rpj_param_0+", 16 * (lane0 + 2 * b), "]");
            P.op("ld.param.v2.f64 {%yr, %yi}, [rpj_param_0+", 16 * (lane0 + 2 * b + 1), "]");
            P.op("selp.f64 %mr, %yr, %mr, ", q);
            P.op("selp.f64 %mi, %yi, %mi, ", q);
            cmul("%tfr", "%tfi", "%mr", "%mi", "%tfr", "%tfi");
        }
        P.op("ld.param.u32 %h1, [rpj_param_0+", off_h1, "]");
        P.op("ld.param.u64 %tabA, [rpj_param_0+", off_ta, "]");
        P.op("ld.param.u64 %tabB, [rpj_param_0+", off_tb, "]");
    }
    P.op("ld.param.u64 %psi, [rpj_param_0+", off_psi, "]");
    P.op("ld.param.u64 %ntiles, [rpj_param_0+", off_nt, "]");
    P.op("ld.param.u32 %zone, [rpj_param_0+", off_zone, "]");
    P.op("mov.u32 %r_c, %ctaid.x");
    P.op("cvt.u64.u32 %u, %r_c");
    P.op("mov.u32 %r_c, %nctaid.x");
    P.op("cvt.u64.u32 %grid, %r_c");
    P.op("setp.ge.u64 %p_out, %u, %ntiles");
    P.op("@%p_out bra $DONE");
    // tile base (bytes) = 2 x the 8 B deposit
    emit_tbase(P, pd.S, n_local, "%u", "%tbo");
    P.op("shl.b64 %tbo, %tbo, 1");
    P.op("add.s64 %gtile, %psi, %tbo");
    P.op("add.s64 %gcur, %gtile, %dthr");
    auto loadtile = [&](const std::string& g, const std::string& pred) {
        for (int i = 0; i < UPT; ++i) {
            const std::string sa = P.r32();
            P.op("xor.b32 ", sa, ", %sthr, ", fold64(nthr * i, T) << 4);
            P.op("add.s32 ", sa, ", ", sa, ", %cur");
            const std::string ga = gaddr(P, g, 16 * tm.dep((uint64_t)nthr * i));
            P.op(pred, "cp.async.cg.shared.global [", sa, "], ", ga, ", 16");
        }
    };
    if (!zinit) loadtile("%gcur", "");
    P.op("cp.async.commit_group");
    P.o << "$LOOP:\n";
    P.op("add.s64 %un, %u, %grid");
    P.op("setp.lt.u64 %p_next, %un, %ntiles");
    emit_tbase(P, pd.S, n_local, "%un", "%tbo");
    P.op("shl.b64 %tbo, %tbo, 1");
    P.op("add.s64 %gtile_next, %psi, %tbo");
    P.op("add.s64 %gnext, %gtile_next, %dthr");
    P.op("cp.async.wait_group 0");
    P.op("bar.sync 0");
    auto ar = [](int j) { return "%ar" + std::to_string(j); };
    auto ai = [](int j) { return "%ai" + std::to_string(j); };
    for (int ph = 0; ph < nph; ++ph) {
        const RpPhaseHost& Ph = phs[ph];
        const bool last = ph == nph - 1;
        P.o << "\t// phase " << ph << ": R = {";
        for (int q : Ph.R) P.o << q << ",";
        P.o << "}, " << Ph.gates.size() << " gates\n";
        P.op("mov.b32 %tb, 0");
        for (int b = 0; b < tbits; ++b) {
            const std::string t = P.r32(), q = P.pr();
            P.op("and.b32 ", t, ", %t_id, ", 1u << b);
            P.op("setp.ne.u32 ", q, ", ", t, ", 0");
            P.op("@", q, " xor.b32 %tb, %tb, ", fold64(1u << Ph.lanes[b], T) << 4);
        }
        auto saddr = [&](uint32_t j) {
            const std::string t = P.r32();
            P.op("xor.b32 ", t, ", %tb, ", fold64(deposit(j, Ph.R), T) << 4);
            P.op("add.s32 ", t, ", ", t, ", %cur");
            return t;
        };
        if (ph == 0 && pinit) {
            // tile factor (two table entries) x thread factor, then x the register factor
            P.op("mov.b64 %rdB, 1");
            P.op("shl.b64 %rdB, %rdB, %h1");
            P.op("sub.s64 %rdB, %rdB, 1");
            P.op("and.b64 %rdB, %u, %rdB");
            P.op("shl.b64 %rdB, %rdB, 4");
            P.op("add.s64 %rdB, %tabA, %rdB");
            P.op("ld.global.nc.v2.f64 {%xr0, %xi0}, [%rdB]");
            P.op("shr.u64 %rdB, %u, %h1");
            P.op("shl.b64 %rdB, %rdB, 4");
            P.op("add.s64 %rdB, %tabB, %rdB");
            P.op("ld.global.nc.v2.f64 {%xr1, %xi1}, [%rdB]");
            cmul("%xr0", "%xi0", "%xr1", "%xi1", "%xr2", "%xi2");
            cmul("%xr2", "%xi2", "%tfr", "%tfi", "%xr3", "%xi3");
            for (int j = 0; j < NA; ++j) {
                P.op("ld.param.v2.f64 {%mr, %mi}, [rpj_param_0+", 16 * (reg0 + j), "]");
                cmul("%mr", "%mi", "%xr3", "%xi3", ar(j), ai(j));
            }
        } else if (ph == 0 && zinit) {
            for (int j = 0; j < NA; ++j) {
                P.op("mov.f64 ", ar(j), ", 0d0000000000000000");
                P.op("mov.f64 ", ai(j), ", 0d0000000000000000");
            }
            P.op("setp.ne.u32 %p_z, %zone, 0");
            P.op("setp.eq.and.u64 %p_z, %u, 0, %p_z");
            P.op("setp.eq.and.u32 %p_z, %t_id, 0, %p_z");
            if (cs.mode == 1 && !pinit)  // the pass scalar C as the start amplitude
                P.op("@%p_z ld.param.v2.f64 {%ar0, %ai0}, [rpj_param_0+", 16 * cslot, "]");
            else
                P.op("@%p_z mov.f64 %ar0, 0d3FF0000000000000");
        } else {
            for (int j = 0; j < NA; ++j) {
                const std::string a = saddr((uint32_t)j);
                P.op("ld.shared.v2.f64 {", ar(j), ", ", ai(j), "}, [", a, "]");
            }
        }
        if (last && early) {
            P.op("bar.sync 0");
            loadtile("%gnext", "@%p_next ");
            P.op("cp.async.commit_group");
        }
        for (int g : Ph.gates) {
            const PassGate& pg = pd.gates[g];
            const int kind = gate_kind(pd, pg);
            uint32_t mask = 0, tmask = 0;
            for (int b = 0; b < pg.k; ++b) {
                const auto it = std::find(Ph.R.begin(), Ph.R.end(), pg.pos[b]);
                if (it != Ph.R.end()) mask |= 1u << (int)(it - Ph.R.begin());
                else tmask |= 1u << (int)(std::find(Ph.lanes.begin(), Ph.lanes.end(), pg.pos[b]) - Ph.lanes.begin());
            }
            const int D = 1 << pg.k;
            P.o << "\t// gate " << g << ": k=" << pg.k << " kind=" << kind << " mask=" << mask << " tmask=" << tmask
                << " cls=" << cs.g[g].cls << "\n";
            if (cs.g[g].cls) {
                emit_spec64(cs.g[g], mask, gbase[g]);
                continue;
            }
            if (kind == 2) {
                std::string pred;
                if (popc(mask) != 2) {
                    const std::string t = P.r32();
                    pred = P.pr();
                    P.op("and.b32 ", t, ", %t_id, ", tmask);
                    P.op("setp.eq.u32 ", pred, ", ", t, ", ", tmask);
                    pred = "@" + pred + " ";
                }
                for (uint32_t j = 0; j < (uint32_t)NA; ++j)
                    if ((j & mask) == mask) {
                        P.op(pred, "neg.f64 ", ar(j), ", ", ar(j));
                        P.op(pred, "neg.f64 ", ai(j), ", ", ai(j));
                    }
                continue;
            }
            const size_t base = gbase[g];
            auto mload = [&](size_t e) {
                P.op("ld.param.v2.f64 {%mr, %mi}, [rpj_param_0+", 16 * e, "]");
                P.op("neg.f64 %nmi, %mi");
            };
            if (kind == 1) {
                for (int e = 0; e < D; ++e) {
                    mload(base + e);
                    for (uint32_t j = 0; j < (uint32_t)NA; ++j) {
                        if (pext(j, mask) != (uint32_t)e) continue;
                        P.op("mov.f64 %xr0, ", ar(j));
                        P.op("mul.rn.f64 ", ar(j), ", %mr, %xr0");
                        P.op("fma.rn.f64 ", ar(j), ", %nmi, ", ai(j), ", ", ar(j));
                        P.op("mul.rn.f64 %yi, %mr, ", ai(j));
                        P.op("fma.rn.f64 ", ai(j), ", %mi, %xr0, %yi");
                    }
                }
                continue;
            }
            const uint32_t rest = ((1u << M) - 1u) & ~mask;
            for (uint32_t gi = 0; gi < (uint32_t)NA / D; ++gi) {
                const uint32_t b0 = pdep(gi, rest);
                for (int c = 0; c < D; ++c) {
                    P.op("mov.f64 %xr", c, ", ", ar(b0 | pdep(c, mask)));
                    P.op("mov.f64 %xi", c, ", ", ai(b0 | pdep(c, mask)));
                }
                for (int rr = 0; rr < D; ++rr) {
                    const uint32_t dst = b0 | pdep(rr, mask);
                    for (int c = 0; c < D; ++c) {
                        mload(base + rr * D + c);
                        if (c == 0) {
                            P.op("mul.rn.f64 %yr, %mr, %xr0");
                            P.op("mul.rn.f64 %yi, %mr, %xi0");
                        } else {
                            P.op("fma.rn.f64 %yr, %mr, %xr", c, ", %yr");
                            P.op("fma.rn.f64 %yi, %mr, %xi", c, ", %yi");
                        }
                        P.op("fma.rn.f64 %yr, %nmi, %xi", c, ", %yr");
                        P.op("fma.rn.f64 %yi, %mi, %xr", c, ", %yi");
                    }
                    P.op("mov.f64 ", ar(dst), ", %yr");
                    P.op("mov.f64 ", ai(dst), ", %yi");
                }
            }
        }
        if (last && cs.mode == 4)  // the pass scalar, explicitly
            for (int j = 0; j < NA; ++j) smul(ar(j), ai(j), ar(j), ai(j), cslot);
        if (last && direct) {
            P.op("add.s64 %gst, %gtile, %dg");
            for (int j = 0; j < NA; ++j)
                P.op("st.global.cs.v2.f64 ", gaddr(P, "%gst", 16 * tm.dep(deposit((uint32_t)j, lp.R))), ", {", ar(j), ", ",
                     ai(j), "}");
        } else {
            for (int j = 0; j < NA; ++j) {
                const std::string a = saddr((uint32_t)j);
                P.op("st.shared.v2.f64 [", a, "], {", ar(j), ", ", ai(j), "}");
            }
            P.op("bar.sync 0");
        }
    }
    if (!direct) {
        for (int i = 0; i < UPT; ++i) {
            const std::string sa = P.r32();
            P.op("xor.b32 ", sa, ", %sthr, ", fold64(nthr * i, T) << 4);
            P.op("add.s32 ", sa, ", ", sa, ", %cur");
            P.op("ld.shared.v2.f64 {", ar(i), ", ", ai(i), "}, [", sa, "]");
        }
        if (!zinit) {
            P.op("bar.sync 0");
            loadtile("%gnext", "@%p_next ");
            P.op("cp.async.commit_group");
        }
        for (int i = 0; i < UPT; ++i)
            P.op("st.global.cs.v2.f64 ", gaddr(P, "%gcur", 16 * tm.dep((uint64_t)nthr * i)), ", {", ar(i), ", ", ai(i), "}");
    }
    P.op("mov.b64 %gcur, %gnext");
    P.op("mov.b64 %gtile, %gtile_next");
    P.op("mov.b64 %u, %un");
    P.op("@%p_next bra $LOOP");
    P.o << "$DONE:\n";
    P.op("ret");

    std::ostringstream k;
    k << "// pass-specialised register-blocked kernel, complex128 (generated by rpass_jit.cpp)\n";
    k << "// T=" << T << " r=" << pd.r << " n=" << n_local << " S={";
    for (int q : pd.S) k << q << ",";
    k << "} gates " << g0 << ".." << g1 << " phases " << nph << (zinit ? " zinit" : "") << (pinit ? " product-start" : "")
      << (direct ? " direct" : "") << "\n";
    k << ".version 8.8\n.target sm_100a\n.address_size 64\n";
    k << ".extern .shared .align 16 .b8 rsm[];\n";
    k << ".visible .entry rpj(.param .align 16 .b8 rpj_param_0[" << pbytes << "])\n";
    k << ".maxntid " << nthr << ", 1, 1\n.maxnreg " << (M >= 5 ? 255 : 128) << "\n{\n";
    k << "\t.reg .pred %p<" << std::max(P.np, 1) << ">;\n\t.reg .pred %p_out, %p_next, %p_z;\n";
    k << "\t.reg .b32 %r<" << std::max(P.nr, 1) << ">;\n\t.reg .b32 %t_id, %cur, %sthr, %tb, %zone, %r_c, %h1;\n";
    k << "\t.reg .b64 %rd<" << std::max(P.nrd, 1) << ">;\n";
    k << "\t.reg .f64 %ar<" << NA << ">, %ai<" << NA << ">, %xr<4>, %xi<4>, %yr, %yi, %mr, %mi, %nmi, %t0, %t1, %t2, %tfr, %tfi, %zr, %zi, "
         "%ptr, %pti, %por<2>, %poi<2>;\n";
    k << "\t.reg .b64 %dthr, %dg, %psi, %ntiles, %u, %un, %grid, %tbo, %gtile, %gcur, %gtile_next, %gnext, %gst, "
         "%tabA, %tabB, %rdB;\n";
    k << P.o.str();
    k << "}\n";
    return k.str();
}

int compile_one(RpJitKernel& K, int dev, std::string& log) {
    const auto t0 = std::chrono::steady_clock::now();
    cudaError_t e = cudaSetDevice(dev);  // worker threads start on device 0
    if (e != cudaSuccess) {
        log = cudaGetErrorString(e);
        return SV_ECUDA;
    }
    std::vector<char> elog(8192, 0);
    cudaJitOption opt[2] = {cudaJitErrorLogBuffer, cudaJitErrorLogBufferSizeBytes};
    void* val[2] = {elog.data(), (void*)(uintptr_t)elog.size()};
    e = cudaLibraryLoadData(&K.lib, K.src.c_str(), opt, val, 2, nullptr, nullptr, 0);
    if (e == cudaSuccess) e = cudaLibraryGetKernel(&K.kern, K.lib, "rpj");
    if (e == cudaSuccess) e = cudaKernelSetAttributeForDevice(K.kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)K.smem, dev);
    if (e != cudaSuccess) {
        log = std::string(cudaGetErrorString(e)) + ": " + elog.data();
        cudaGetLastError();
        return SV_ECUDA;
    }
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, (const void*)K.kern, K.nthr, K.smem) != cudaSuccess || nb < 1) {
        cudaGetLastError();
        nb = std::max(1, (int)((227u * 1024u) / (K.smem + 1024u)));
    }
    K.blocks_per_sm = nb;
    K.dev_mask |= 1ull << dev;
    g_compiled++;
    g_compile_ns += (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now() - t0).count();
    return SV_OK;
}

// find or create the cache entry of a chunk key; `fresh` = needs compiling
std::shared_ptr<RpJitKernel> lookup(const std::string& key, bool& fresh) {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    auto it = g_cache.find(key);
    if (it != g_cache.end()) {
        fresh = false;
        g_hits++;
        return it->second;
    }
    auto K = std::make_shared<RpJitKernel>();
    K->key = key;
    g_cache[key] = K;
    fresh = true;
    return K;
}

void drop(const std::string& key) {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    g_cache.erase(key);
}

}  // namespace

int rpass_jit_prepare(const PassDesc& pd, int n_local, bool zinit, bool compile, std::vector<RpJitLaunch>& out,
                      std::vector<std::string>* sources) {
    std::vector<const PassDesc*> one{&pd};
    if (!compile) {
        out.clear();
        const int T = (int)pd.S.size();
        bool first = true;
        for (const auto& ch : jit_chunks(pd)) {
            RpJitLaunch l;
            size_t nm = 0;
            const std::string src = pd.wide ? gen_chunk64(pd, n_local, ch.first, ch.second, zinit && first, nm, l.mats64)
                                            : gen_chunk(pd, n_local, ch.first, ch.second, zinit && first, nm, l.mats);
            if (sources) sources->push_back(src);
            l.c0 = ch.first;
            l.c1 = ch.second;
            l.zinit = zinit && first;
            (void)T;
            (void)n_local;
            out.push_back(std::move(l));
            first = false;
        }
        return SV_OK;
    }
    std::vector<std::vector<RpJitLaunch>> all;
    std::vector<char> z{(char)zinit};
    int rc = rpass_jit_prepare_many(one, n_local, z, all);
    if (rc) return rc;
    out = std::move(all[0]);
    if (sources)
        for (auto& l : out) sources->push_back(l.kern->src);
    return SV_OK;
}

int rpass_jit_prepare_many(const std::vector<const PassDesc*>& pds, int n_local, const std::vector<char>& zinit,
                           std::vector<std::vector<RpJitLaunch>>& out) {
    out.assign(pds.size(), {});
    std::vector<std::shared_ptr<RpJitKernel>> todo;
    for (size_t i = 0; i < pds.size(); ++i) {
        const PassDesc& pd = *pds[i];
        const int T = (int)pd.S.size();
        const int M = jit_m(pd);
        bool first = true;
        for (const auto& ch : jit_chunks(pd)) {
            RpJitLaunch l;
            size_t nm = 0;
            const bool z = zinit[i] && first;
            bool fresh = false;
            l.kern = lookup(chunk_key(pd, n_local, ch.first, ch.second, z), fresh);
            if (pd.wide) {
                gen_chunk64(pd, n_local, ch.first, ch.second, z, nm, l.mats64, false);
            } else {
                gen_chunk(pd, n_local, ch.first, ch.second, z, nm, l.mats, false);
                for (const auto& ms : pd.mats_shard) {
                    l.mats_shard.emplace_back();
                    gen_chunk(pd, n_local, ch.first, ch.second, z, nm, l.mats_shard.back(), false, &ms);
                }
            }
            if (fresh) {
                l.kern->src = pd.wide ? gen_chunk64(pd, n_local, ch.first, ch.second, z, nm, l.mats64)
                                      : gen_chunk(pd, n_local, ch.first, ch.second, z, nm, l.mats);
                const bool ring = SVB_JIT_RING && !pd.wide;
                l.kern->nthr = (1 << (T - M)) * (ring ? 2 : 1);
                const bool db = SVB_JIT_DB && !ring && !z && !pd.wide;  // as gen_chunk
                const bool pl = SVB_JIT_PL && !ring && !db && !z && !pd.wide && M >= 3;
                l.kern->smem = ((size_t)(pd.wide ? 16 : 8) << T) * (ring ? 3 : db ? 2 : 1) + (ring ? 64 : 0) +
                               (pl ? ((size_t)6 << T) : 0);  // 3/4 tile spare buffer
                l.kern->T = T;
                l.kern->nm = nm;
                l.kern->param_bytes = std::max<size_t>(nm, 1) * 16 + 48;  // as in gen_chunk
                todo.push_back(l.kern);
            }
            l.c0 = ch.first;
            l.c1 = ch.second;
            l.zinit = z;
            l.wide = pd.wide;
            out[i].push_back(std::move(l));
            first = false;
        }
    }
    if (todo.empty()) return SV_OK;
    // assemble the new kernels in parallel host threads
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) {
        cudaGetLastError();
        for (auto& K : todo) drop(K->key);
        return fail(SV_ECUDA, "no CUDA device for the pass kernels");
    }
    std::atomic<size_t> next{0};
    std::atomic<int> failed{0};
    std::string first_log;
    std::mutex log_mu;
    auto worker = [&]() {
        for (;;) {
            const size_t i = next++;
            if (i >= todo.size()) return;
            std::string log;
            if (compile_one(*todo[i], dev, log) != SV_OK) {
                failed++;
                std::lock_guard<std::mutex> lk(log_mu);
                if (first_log.empty()) first_log = log;
            }
        }
    };
    const unsigned hw = std::max(1u, std::thread::hardware_concurrency());
    const size_t nt = std::min<size_t>(todo.size(), std::min(hw, 16u));
    std::vector<std::thread> th;
    for (size_t t = 1; t < nt; ++t) th.emplace_back(worker);
    worker();
    for (auto& t : th) t.join();
    cudaSetDevice(dev);
    if (failed) {
        for (auto& K : todo) drop(K->key);
        return fail(SV_ECUDA, "PTX JIT of a pass kernel failed: " + first_log.substr(0, 2000));
    }
    return SV_OK;
}

cudaError_t launch_rpass_jit(void* psi, int n_local, const RpJitLaunch& l, bool one_here, cudaStream_t st, int slot,
                             uint64_t* bins) {
    RpJitKernel& K = *l.kern;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev >= 64) return cudaErrorInvalidDevice;
    if (!((K.dev_mask >> dev) & 1ull)) {  // first use on another device
        std::lock_guard<std::mutex> lk(K.mu);
        if (!((K.dev_mask >> dev) & 1ull)) {
            std::string log;
            if (!K.lib) {
                if (compile_one(K, dev, log) != SV_OK) return cudaErrorInvalidPtx;
            } else {
                e = cudaKernelSetAttributeForDevice(K.kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)K.smem, dev);
                if (e != cudaSuccess) return e;
                K.dev_mask |= 1ull << dev;
            }
        }
    }
    const int T = K.T;
    const uint64_t n_tiles = 1ull << (n_local - T);
    const uint64_t grid = std::min<uint64_t>(n_tiles, (uint64_t)pass_sms() * K.blocks_per_sm);
    std::vector<unsigned char> prm(K.param_bytes, 0);
    if (l.wide) {
        std::memcpy(prm.data(), l.mats64.data(), l.mats64.size() * sizeof(double));
    } else {
        const std::vector<float>& mats = l.mats_shard.empty() ? l.mats : l.mats_shard[slot];
        std::memcpy(prm.data(), mats.data(), mats.size() * sizeof(float));
    }
    const size_t off = std::max<size_t>(K.nm, 1) * 16;
    const void* cpsi = psi;
    std::memcpy(prm.data() + off, &cpsi, 8);
    std::memcpy(prm.data() + off + 8, &n_tiles, 8);
    const int zone = one_here ? 1 : 0;
    std::memcpy(prm.data() + off + 16, &zone, 4);
    std::memcpy(prm.data() + off + 20, &l.h1, 4);
    std::memcpy(prm.data() + off + 24, &l.tabA, 8);
    std::memcpy(prm.data() + off + 32, &l.tabB, 8);
    std::memcpy(prm.data() + off + 40, &bins, 8);
    void* args[] = {prm.data()};
    return cudaLaunchKernel((const void*)K.kern, dim3((unsigned)grid), dim3((unsigned)K.nthr), args, K.smem, st);
}

void rpass_jit_counters(uint64_t* compiled, uint64_t* cache_hits, double* compile_s) {
    if (compiled) *compiled = g_compiled;
    if (cache_hits) *cache_hits = g_hits;
    if (compile_s) *compile_s = (double)g_compile_ns * 1e-9;
}

uint64_t rpass_jit_ops_per_amp(const PassDesc& pd, bool zinit) {
    if (!pd.spec) return rpass_fma_per_amp(pd);
    uint64_t f = 0;
    bool first = true;
    for (const auto& ch : jit_chunks(pd)) {
        const ChunkSpec cs = chunk_spec(pd, ch.first, ch.second, zinit && first);
        for (size_t g = ch.first; g < ch.second; ++g) {
            const GSpec& x = cs.g[g];
            const int kind = gate_kind(pd, pd.gates[g]);
            const uint64_t nu = (x.unit[0] ? 0 : 2) + (x.unit[1] ? 0 : 2);
            uint64_t mono = 0;  // monomial: per 4 amplitudes 2 per rotation, 4 per multiply
            for (int r = 0; r < 4; ++r) mono += !x.munit[r] ? 4 : (x.mq[r] & 3) ? 2 : 0;
            switch (x.cls) {
                case 4: f += (mono + 3) / 4; break;
                case 1: f += 2 + nu; break;  // 2 FADDs per output, 4 ops per multiplier (per pair)
                case 2: f += 4; break;
                case 3: f += nu; break;
                default: f += kind == 0 ? 4ull << pd.gates[g].k : kind == 1 ? 4 : 0;
            }
        }
        if (cs.mode == 4) f += 4;
        first = false;
    }
    return f;
}

}  // namespace svb
