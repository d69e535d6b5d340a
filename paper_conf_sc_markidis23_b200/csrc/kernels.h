// kernels.h -- launch descriptors and launchers of the device kernels
// (internal to libsvb200; host code never sees a template).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <memory>
#include <string>
#include <utility>
#include <vector>

#include "sv_internal.h"

namespace svb {

// Qubit-class split (qsim splits at log2(32) = 5 for a
// 32-lane warp of 1 amplitude/lane).  On B200 a lane moves 16 B (2 amps) and
// 8 lanes fill a 128 B line, so a gate is "high" when none of its qubits is
// 1, 2 or 3 (qubit 0 lives inside a lane's float4).  Everything else is
// "low" and goes through a shared-memory tile.
constexpr uint64_t kLowMask = 0xEull;  // qubits {1,2,3}

struct ApplyDesc {
    int k = 0;
    int q[SV_MAX_FUSED] = {0};        // ascending physical qubits (within a shard)
    std::vector<cf> m;                // 2^k x 2^k row-major over ascending q, complex64
    std::vector<std::complex<double>> m64;  // the same in complex128 (int8 tensor-core packer)
    bool high = false;                // kernel class
    bool mono = false;                // one nonzero per row (exact permutation/diagonal path)
    int nc = 0;                       // control qubits (controlled gate, NEXT-4): only the
    int cq[SV_MAX_FUSED] = {0};       //   amplitudes with every control bit 1 are transformed
    int tc_mode = 3;                  // dense-gate path: 3 auto, 2 int8 k>=4, 0 SIMT (sv_set_option)
    bool tc = false;                  // tensor-core path
    bool tci = false;                 //   ... exact int8-slice variant (needs dev_wi8)
    const uint8_t* dev_wi8 = nullptr; // int8 W slices + column exponents (pack_wi8), device
    // low-kernel tile plan (host-computed once)
    int T = 0, r = 0;                 // tile bits, run bits
    // device copy of m for k == 6 (owned by the circuit / state scratch)
    const float2* dev_m = nullptr;
};

// Decide high/low and the tile plan for a gate on `n` local qubits.
void plan_apply(int n_local, ApplyDesc& d);

// Dense k = 4, 5 gates run on the tensor cores (tcgen05, TF32 x3) when the
// shard has at least 2^13 amplitudes.
bool tc_supported(int n_local, const ApplyDesc& d);
size_t wi8_bytes(int k);
void pack_wi8(const ApplyDesc& d, uint8_t* out);

// ---- complex128 states (apply64.cu, NEXT-1) --------------------------------
struct Apply64Desc {
    int k = 0;
    int q[SV_MAX_FUSED] = {0};          // ascending
    std::vector<cd> m;                  // 2^k x 2^k row-major over ascending q (fp64)
    const double* dev_planes = nullptr; // planes P, S, Q on the device (k = 6 and tiny states)
    const void* small_scratch = nullptr;  // device int[6] with q (tiny states)
};
void pack_planes64(const Apply64Desc& d, double* out);  // 3 * 4^k doubles
cudaError_t launch_apply64(double2* psi, int n, const Apply64Desc& d, cudaStream_t st);
cudaError_t launch_reset64(double2* psi, uint64_t n_amps, bool one, cudaStream_t st);
cudaError_t launch_gather64(const double2* psi, const uint64_t* phys, uint64_t count, double2* out, cudaStream_t st);
// exact in-place swap of local index bits a and b of a complex128 shard (2^l amplitudes)
cudaError_t launch_swap_bits64(double2* psi, int l, int a, int b, cudaStream_t st);

// Whole circuit in one CTA with the state in shared memory (n <= 13).
constexpr int kSmallCircuitMaxQubits = 13;
struct SmallGateDesc {
    int k;
    int q[SV_MAX_FUSED];  // ascending
    uint32_t mat_off;     // offset (complex elements) of the 2^k x 2^k matrix
};
size_t small_circuit_smem(int n);
cudaError_t launch_small_circuit(float2* psi, int n, int ngates, const SmallGateDesc* gates_dev,
                                 const float2* mats_dev, cudaStream_t st);

// Cache-blocked pass (blocked.cu): all gates of the pass act on qubits in S
// (|S| = tile bits, contains 0..r-1); one HBM read + write per pass.
constexpr int kPassMaxGates = 64;
constexpr int kPassPlaneFloats = 6144;
// 14-qubit tiles exist only as pass-specialised kernels, whose matrices are
// launch parameters (<= 32 KB) rather than a fixed parameter struct: a pass
// of such tiles may hold up to kJitPassMaxGates gates per launch
constexpr int kJitPassMaxGates = 256;
struct PassGate {
    int k;          // 1..4
    int pos[4];     // tile-local positions (rank of the qubit in sorted S), ascending
    uint32_t poff;  // offset (floats) of the gate's planes P, S, Q (3 x 4^k floats)
    uint32_t moff;  // offset (floats) of the gate's matrix in PassDesc::mats
    int kind = -1;  // gate_kind override (shard-dependent gates: the kind that fits every shard)
};
struct PassDesc {
    std::vector<int> S;  // qubits of the tile
    int r = 0;           // run bits (S[0..r) == 0..r-1)
    std::vector<PassGate> gates;
    std::vector<float> planes;
    std::vector<float> mats;  // per gate: 2^k x 2^k complex64, row-major (re, im pairs)
    // sharded runs with the diagonal exchange skip: mats of every local shard
    // slot (a gate block-diagonal in a global qubit has a block per shard);
    // empty when every shard runs `mats`
    std::vector<std::vector<float>> mats_shard;
    uint64_t fma_per_amp = 0;  // rpass FMAs per amplitude (stats), set at circuit creation
    std::vector<int> src;      // index of each gate in the planner's input run (sv_block_plan)
    // product-state start (first pass of a circuit run from |0...0>, pass-
    // specialised kernels only): the first gate of every qubit, when it is a
    // one-qubit gate, moved to time 0 (it commutes with every earlier gate),
    // so the pass starts from prod_q v_q[bit q] with v_q = that gate's first
    // column (identity: (1, 0)).  pinit_v: v of tile position p at [2p, 2p+1]
    std::vector<std::complex<double>> pinit_v;
    std::vector<double> mats64;  // complex128 states: the matrices in fp64 (same layout as mats)
    bool wide = false;           // complex128 state: pass-specialised fp64 kernel, 16 amplitudes per thread
    bool bins = false;           // last pass of an unsharded complex64 circuit: also write the sampler's bins
    // structured one-qubit gates (pass-specialised complex64 kernels, reading
    // R11): a one-qubit gate c * B with B's rows (or columns) of the form
    // (1, i^p) runs as additions; the scalars c of the pass are multiplied
    // out once per pass.  Only when every shard runs `mats` (no mats_shard).
    bool spec = false;
};
void plan_pass_tile(PassDesc& pd);
cudaError_t launch_pass(float2* psi, int n_local, const PassDesc& pd, cudaStream_t st);
// Register-blocked pass (k <= 2 gates, 10 <= T <= 13): each thread holds 32
// amplitudes of the tile in registers and applies every gate of a phase
// there; phases exchange through the shared-memory tile.
bool rpass_supported(const PassDesc& pd);
// fp32 FMAs per amplitude the rpass kernel executes for this pass (dense
// 2^k x 2^k: 4 * 2^k, diagonal: 4, CZ-like: 0)
uint64_t rpass_fma_per_amp(const PassDesc& pd);
// zero_init: the tiles are |0...0> (not loaded); one_here: this shard holds
// amplitude 0 (= 1)
cudaError_t launch_rpass(float2* psi, int n_local, const PassDesc& pd, cudaStream_t st, bool zero_init = false,
                         bool one_here = false, int slot = 0);
// Host model of the rpass phase plan (tests / tools): number of phases and
// the worst bank-conflict degree of their gathers.
void rpass_plan_stats(const PassDesc& pd, int* n_phases, int* worst_conflict);
// The rpass phase plan of a whole pass (host; sv_block_plan): per phase its
// register positions R (ascending tile positions) and its gates (pass-local
// indices, in application order).
void rpass_phase_plan(const PassDesc& pd, std::vector<std::vector<int>>& R, std::vector<std::vector<int>>& gates);

// ---- rpass host planning, shared by the generic kernel (blocked.cu) and the
// pass-specialised kernels compiled at circuit creation (rpass_jit.cpp)
struct RpPhaseHost {
    std::vector<int> gates;  // pass gate indices, in application order
    std::vector<int> R;      // M tile positions, ascending (register bit j <-> R[j])
    std::vector<int> lanes;  // T-M positions: thread-index bit i <-> lanes[i]
    bool b0;                 // tile position 0 is a register bit (16 B gathers)
};
constexpr int kRpMaxPhases = 48;  // per launch (parameter space of the generic kernel)
constexpr int kRpMaxGates = 64;
// fold swizzle of a tile index (16 B chunk bits 1..3 ^= tile bits 4..6 ^ 7..9 ^ 10..12)
uint32_t fold_swz(uint32_t t, int T);
uint32_t deposit(uint32_t v, const std::vector<int>& pos);
int rpass_m();
// 0 dense, 1 diagonal, 2 CZ-like (diag(1, 1, 1, -1)), exact in fp32
int gate_kind(const PassDesc& pd, const PassGate& pg);
// phases of pass gates [g0, g1) for M register bits
// wide: 16 B (complex128) amplitudes -- lanes for LDS.128 of single
// amplitudes under the wide fold swizzle (amplitude bits 0..2 ^= 3..5 ^ 6..8 ...)
std::vector<RpPhaseHost> plan_phases(const PassDesc& pd, size_t g0, size_t g1, int M, bool wide = false);
// The gates [g0, g1) of a pass as launch chunks: each chunk [c0, c1) fits one
// launch (<= kRpMaxGates gates, <= kRpMaxPhases phases).
std::vector<std::pair<size_t, size_t>> rpass_chunks(const PassDesc& pd, int M, bool wide = false);
int pass_sms();

// Pass-specialised register-blocked kernels (rpass_jit.cpp): the phase plan,
// gate kinds, register masks and every address offset of one launch chunk
// are compiled into a kernel (PTX -> sm_100a via nvJitLink) at circuit creation; only the
// matrices, the state pointer and the tile count are launch parameters.
// Kernels are cached per process by their PTX text.
struct RpJitKernel;
struct RpJitLaunch {
    std::shared_ptr<RpJitKernel> kern;
    std::vector<float> mats;  // float4 (mr, mr, -mi, mi) per matrix element, launch order
    std::vector<std::vector<float>> mats_shard;  // per local shard slot (PassDesc::mats_shard)
    std::vector<double> mats64;  // complex128 kernels: (mr, mi) per matrix element
    bool wide = false;
    size_t c0 = 0, c1 = 0;    // gate chunk
    bool zinit = false;
    // product-state start: tile factor = tabA[u & (2^h1 - 1)] * tabB[u >> h1]
    // (device tables owned by the circuit, complex64)
    const void* tabA = nullptr;  // complex64 (complex128 for wide kernels)
    const void* tabB = nullptr;
    int h1 = 0;
};
// Generate (and compile unless compile == false) the kernels of one pass;
// returns SV_OK or an error code with the message set (the compiler log).
int rpass_jit_prepare(const PassDesc& pd, int n_local, bool zinit, bool compile, std::vector<RpJitLaunch>& out,
                      std::vector<std::string>* sources = nullptr);
// Prepare many passes at once (compiles in parallel host threads).
int rpass_jit_prepare_many(const std::vector<const PassDesc*>& pds, int n_local, const std::vector<char>& zinit,
                           std::vector<std::vector<RpJitLaunch>>& out);
// bins: the sampler's bin array (kernels of a pass with PassDesc::bins write
// the 16-amplitude S5 bin weights of the final state there)
cudaError_t launch_rpass_jit(void* psi, int n_local, const RpJitLaunch& l, bool one_here, cudaStream_t st,
                             int slot = 0, uint64_t* bins = nullptr);
// fp32 pipe operations per amplitude of the pass-specialised kernels of this
// pass (zinit: the |0...0>-start variant): as rpass_fma_per_amp for generic
// gates, fewer for the structured gates of PassDesc::spec (one FADD, FMUL or
// FFMA = 1)
uint64_t rpass_jit_ops_per_amp(const PassDesc& pd, bool zinit);
// process-wide counters (sv_jit_stats)
void rpass_jit_counters(uint64_t* compiled, uint64_t* cache_hits, double* compile_s);

// Launch one fused-gate apply on a shard of 2^n_local amplitudes.
cudaError_t launch_apply(float2* psi, int n_local, const ApplyDesc& d, cudaStream_t st);

// |0...0> on a shard (one=true puts 1 at index 0).
cudaError_t launch_reset(float2* psi, uint64_t n_amps, bool one, cudaStream_t st);

// out[i] = psi_shard[ phys_index[i] ] for entries owned by this shard
// (owner[i] == shard), others untouched.
cudaError_t launch_gather(const float2* psi, const uint64_t* phys, const int32_t* owner, int shard,
                          uint64_t count, float2* out, cudaStream_t st);

// ---- sampling (S5) ----------------------------------------------------------
constexpr int kSampleBinBits = 4;  // 16 amplitudes per fine bin (= the 128 B runs of a blocked pass, whose
                                   // last pass can write the bin weights itself)
// bins[b] = sum over the 16 amplitudes of bin b of floor(p * 2^62)
cudaError_t launch_bin_weights(const void* psi, bool fp64, uint64_t n_amps, uint64_t* bins, cudaStream_t st);
// inclusive prefix sum in place over `count` uint64 (scratch: >= scan_scratch_elems(count))
size_t scan_scratch_elems(uint64_t count);
cudaError_t launch_inclusive_scan(uint64_t* data, uint64_t count, uint64_t* scratch, cudaStream_t st);
// Resolve samples s in [0, n_samples): t_s = (splitmix64#(s+1)(seed) * T) >> 64
// (T == 0 or T >= 3.99 * 2^62: every out[s] = UINT64_MAX, *status = 1 / 2)
// with T = *total_dev (+ global offset); samples whose t falls into this
// shard's range [range_lo, range_lo + local_total) are written as
// logical index = index_base + local index.  Others untouched.
cudaError_t launch_sample_resolve(const void* psi, bool fp64, uint64_t n_amps, const uint64_t* cum_bins,
                                  uint64_t n_bins, const uint64_t* range_lo_dev, const uint64_t* total_dev,
                                  uint64_t seed, uint64_t n_samples, uint64_t index_base, uint64_t* out,
                                  uint64_t* status, cudaStream_t st);

// offsets of shard totals in LOGICAL shard order: lo[d] = sum of totals of
// shards whose logical index sigma[d'] < sigma[d]; *total = sum of all.
// totals_src[d] points at shard d's total (last inclusive-prefix element).
cudaError_t launch_shard_offsets(const uint64_t* const* totals_src_dev, const int32_t* sigma_dev, int world,
                                 uint64_t* lo_dev, uint64_t* total_dev, cudaStream_t st);
// out[i] = min over r < world of src[r][i] (merge of per-rank partial results)
cudaError_t launch_merge_min(const uint64_t* const* src_dev, int world, uint64_t count, uint64_t* out, cudaStream_t st);
// device-side barrier over P2P-mapped flag words (multi-process sharded mode)
cudaError_t launch_barrier(uint64_t* const* flags_dev, int world, int me, uint64_t epoch, cudaStream_t st);

// ---- sharded exchange (S4 semantics) -----------------------------------------
struct ExchangeDesc {
    int l = 0;                       // local bits
    int s = 0;                       // number of pairs
    int P[8] = {0}, p[8] = {0};      // global positions (>= l) and local positions
};
// Swap chunks among shards: shards[d] points at shard d's amplitudes (local or
// peer-mapped).  Work is split so that rank `me` of `world` does its share of
// every pair (all pairs of all shards when me < 0: virtual mode).
cudaError_t launch_exchange(float2* const* shards_dev, int world, int me, const ExchangeDesc& x, cudaStream_t st);

}  // namespace svb
