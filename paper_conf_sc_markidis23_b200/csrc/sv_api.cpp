// sv_api.cpp -- the C ABI of include/sv.h: validation, error handling, the
// dispatcher that turns a circuit into kernel launches (SURVEY.md §8 rows
// a0-a9, b), and the sharded-mode plumbing.
//
// PAPER.md §3 (L128-135) describes the layering this replaces: an app reads
// a circuit and "maximum number of fused gates" (L128), a simulator class
// applies gates and launches the kernels (L129-130), a state-space class
// sets states, gets amplitudes and samples (L131-132).  Here all of it sits
// behind plain C calls; PyTorch is only a possible owner of the buffer and
// stream.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: ranges for nsys / ncu --nvtx

#include "kernels.h"
#include "sv_internal.h"

using namespace svb;

#ifndef SVB_PASS_COMMUTE
#define SVB_PASS_COMMUTE 1  // pass formation: a left-out diagonal gate blocks only non-diagonal gates on its qubits
#endif
#ifndef SVB_PASS_LOOKAHEAD
#define SVB_PASS_LOOKAHEAD 1  // pass qubit sets chosen by lookahead (0: first-come greedy)
#endif
#ifndef SVB_FUSED_BINS
#define SVB_FUSED_BINS 1  // the last register-blocked pass writes the sampler's bin weights
#endif
#ifndef SVB_PASS_BEAM
#define SVB_PASS_BEAM 5  // pass formation search width (reading R7): 1 = the greedy lookahead alone
#endif
#ifndef SVB_PASS_PIN
#define SVB_PASS_PIN 4  // qubits 0..PIN-1 in every blocked-pass tile (runs of 8 * 2^PIN bytes)
#endif

namespace svb {

static thread_local std::string g_err;

void set_error(const std::string& msg) { g_err = msg; }
int fail(int code, const std::string& msg) {
    g_err = msg;
    return code;
}

}  // namespace svb

namespace {

// NVTX range for the duration of a scope (host side: fuse, plan, pass
// kernels, upload, apply / exchange / sample launches)
struct Nvtx {
    explicit Nvtx(const char* name) { nvtxRangePushA(name); }
    ~Nvtx() { nvtxRangePop(); }
    Nvtx(const Nvtx&) = delete;
    Nvtx& operator=(const Nvtx&) = delete;
};

double now_s() {
    return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

struct Ctrl {               // per-rank control block (device memory, IPC-shared)
    uint64_t flags[64];     // barrier epochs written by each rank
    uint64_t total;         // this rank's sampling total
    uint64_t pad[63];
};

constexpr size_t kXferBytes = 64ull << 20;  // per-rank exchange area for samples / amplitudes

enum class LaunchClass { HIGH = 0, LOW = 1, EXCH = 2, OTHER = 3 };

}  // namespace

struct sv_state {
    int n = 0, g = 0, l = 0;
    int world = 1;            // P
    int rank = 0;
    bool virt = true;         // all shards on this GPU
    int device = 0;
    int vmin = 5;
    int block_bits = -1;      // cache-blocked passes: tile qubits (0 = off, -1 = auto, see sv_circuit_create)
    bool fp64 = false;        // complex128 amplitudes (NEXT-1)
    bool ext_buf = false;     // the state lives in a caller-owned buffer (sv_config.dev_buf)
    int tc_mode = 3;          // SV_OPT_APPLY_PATH
    int pass_jit = 1;         // SV_OPT_PASS_JIT
    int diag_skip = 1;        // SV_OPT_DIAG_SKIP
    int pass_pin = SVB_PASS_PIN;  // SV_OPT_PASS_PIN: qubits 0..pin-1 in every blocked-pass tile
    int pass_spec = 1;            // SV_OPT_PASS_SPEC: structured one-qubit gates as additions (reading R11)
    int pass_beam = SVB_PASS_BEAM;  // SV_OPT_PASS_SEARCH: pass-formation search width (reading R7)
    bool sample_pending = false;  // a sv_sample_device status word not yet checked
    // the sampler's bins hold the current state's S5 weights (written by the
    // last register-blocked pass of the last circuit); any state change clears it
    bool bins_valid = false;
    size_t elem = 8;          // bytes per amplitude
    // staging ring for per-call device inputs of sv_apply_fused /
    // sv_apply_controlled (k = 6 matrices, int8 W slices, fp64 planes): a
    // slot is reused only after the launch that read it has completed (its
    // event), so the calls stay asynchronous
    struct StageSlot {
        char* host = nullptr;  // pinned
        char* dev = nullptr;
        cudaEvent_t ev = nullptr;
        bool used = false;
    };
    std::vector<StageSlot> stage;
    size_t stage_next = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    std::vector<float2*> shard;        // shard pointers (local or peer-mapped)
    float2** shard_dev = nullptr;      // device copy of shard pointers
    void* alloc = nullptr;             // library-owned state allocation
    std::vector<int> pos;              // logical -> physical
    int sticky = SV_OK;
    // |0...0> requested by sv_reset but not yet written (complex64): the next
    // circuit whose first step is a register-blocked pass synthesises the
    // zero tiles instead of loading them; any other access writes it first
    bool zero_pending = false;
    // scratch
    uint64_t* bins = nullptr;          // world_local * n_bins
    uint64_t* scan_scratch = nullptr;
    uint64_t* misc = nullptr;          // [0..63] lo, [64] total, [65..] totals ptrs area
    uint64_t** totals_ptr_dev = nullptr;
    int32_t* sigma_dev = nullptr;
    // multi-process
    Ctrl* ctrl = nullptr;
    uint64_t* xfer = nullptr;          // kXferBytes
    std::vector<Ctrl*> peer_ctrl;
    std::vector<uint64_t*> peer_xfer;
    uint64_t** flags_dev = nullptr;
    uint64_t** xfer_dev = nullptr;
    uint64_t epoch = 0;
    bool attached = false;
    std::vector<void*> ipc_opened;
    // timing
    bool timing = false;
    struct Rec {
        LaunchClass cls;
        cudaEvent_t a, b;
    };
    std::vector<Rec> recs;
    std::vector<cudaEvent_t> ev_pool;
    std::vector<uint64_t> pass_bytes, pass_fma;  // per blocked pass of the last run (per shard)
    size_t ev_used = 0;
    sv_stats stats{};
    // reusable device buffers
    uint64_t* idx_dev = nullptr;
    size_t idx_cap = 0;
    float2* amp_dev = nullptr;
    size_t amp_cap = 0;
    uint64_t* samp_dev = nullptr;
    size_t samp_cap = 0;

    uint64_t local_amps() const { return 1ull << l; }
    int local_shards() const { return virt ? world : 1; }
};

struct sv_circuit {
    sv_state* owner = nullptr;
    std::vector<int> pos_in, pos_out;
    struct Step {
        Event::Type type;
        bool block = false;                   // APPLY of a cache-blocked pass (pass below)
        ApplyDesc apply;
        Apply64Desc a64;  // complex128 states
        PassDesc pass;
        std::vector<ApplyDesc> apply_shard;   // per local shard slot (diagonal exchange skip)
        std::vector<RpJitLaunch> jit, jitz;   // pass-specialised kernels (jitz: first pass from |0...0>)
        ExchangeDesc exch;
        std::vector<ApplyDesc> perm_applies;  // PERMUTE lowered to SWAP passes
        std::vector<int> perm;                // PERMUTE (complex128: exact bit swaps)
    };
    bool a64 = false;  // complex128, one apply64 launch per fused gate (not register-blocked)
    std::vector<Step> steps;
    // the same circuit for runs that start from a pending |0...0>: the first
    // gate of every qubit (a one-qubit gate) folded into a product-state
    // first pass (PassDesc::pinit_v); empty when not applicable
    std::vector<Step> steps_z;
    sv_stats stats_z{};
    bool zero_only = false;  // only steps_z was built (a one-shot run from the pending |0...0>)
    void* ptab = nullptr;  // its tile-factor tables (device, complex64 / complex128)
    float2* dev_mats = nullptr;
    double* planes64 = nullptr;  // complex128 states: planes of every gate
    uint8_t* wi8 = nullptr;      // int8 tensor-core W slices of every tensor-core gate
    int* q64 = nullptr;          // complex128 states: qubits of every gate (int[6] each)
    // small states (n <= 13, unsharded): whole circuit in one CTA (small.cu)
    bool small = false;
    int n_small = 0;
    SmallGateDesc* small_gates = nullptr;
    float2* small_mats = nullptr;
    sv_stats stats{};
};

namespace {

int cuda_fail(sv_state* s, cudaError_t e, const char* what) {
    if (s) s->sticky = SV_EBADSTATE;
    return fail(SV_ECUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

#define CK(s, expr)                                             \
    do {                                                        \
        cudaError_t e__ = (expr);                               \
        if (e__ != cudaSuccess) return cuda_fail((s), e__, #expr); \
    } while (0)

int check_state(sv_state* s) {
    if (!s) return fail(SV_EINVAL, "state handle is NULL");
    if (s->sticky != SV_OK) return fail(SV_EBADSTATE, "state poisoned by an earlier device failure");
    return SV_OK;
}

cudaEvent_t next_event(sv_state* s) {
    if (s->ev_used == s->ev_pool.size()) {
        cudaEvent_t e;
        cudaEventCreate(&e);
        s->ev_pool.push_back(e);
    }
    return s->ev_pool[s->ev_used++];
}

// Launch wrapper: records events around the launch when timing is on.
template <class F>
int launch(sv_state* s, LaunchClass cls, F&& f) {
    cudaEvent_t a = nullptr, b = nullptr;
    if (s->timing) {
        a = next_event(s);
        b = next_event(s);
        cudaEventRecord(a, s->stream);
    }
    cudaError_t e = f();
    if (e != cudaSuccess) return cuda_fail(s, e, "kernel launch");
    if (s->timing) {
        cudaEventRecord(b, s->stream);
        s->recs.push_back({cls, a, b});
    }
    switch (cls) {
        case LaunchClass::HIGH: s->stats.n_launch_high++; break;
        case LaunchClass::LOW: s->stats.n_launch_low++; break;
        default: s->stats.n_launch_other++; break;
    }
    return SV_OK;
}

void reset_stats(sv_state* s) {
    s->stats = sv_stats{};
    s->recs.clear();
    s->ev_used = 0;
}

// Sum recorded event intervals into stats (requires the stream to be done).
void collect_timing(sv_state* s) {
    for (auto& r : s->recs) {
        float ms = 0.f;
        if (cudaEventElapsedTime(&ms, r.a, r.b) != cudaSuccess) continue;
        const double sec = ms * 1e-3;
        switch (r.cls) {
            case LaunchClass::HIGH: s->stats.t_apply_high_dev_s += sec; break;
            case LaunchClass::LOW: s->stats.t_apply_low_dev_s += sec; break;
            case LaunchClass::EXCH: s->stats.t_exchange_dev_s += sec; break;
            default: s->stats.t_other_dev_s += sec; break;
        }
    }
    s->recs.clear();
    s->ev_used = 0;
}

int sync(sv_state* s) {
    CK(s, cudaStreamSynchronize(s->stream));
    if (s->timing) collect_timing(s);
    return SV_OK;
}

template <class T>
int ensure(sv_state* s, T*& p, size_t& cap, size_t need) {
    if (need <= cap) return SV_OK;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    cudaError_t e = cudaMalloc(&p, std::max<size_t>(need, 1) * sizeof(T));
    if (e != cudaSuccess) return fail(SV_ENOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
    cap = need;
    return SV_OK;
}

// ---- multi-process barrier ---------------------------------------------------
int barrier(sv_state* s) {
    if (s->virt || s->world == 1) return SV_OK;
    if (!s->attached) return fail(SV_ECOMM, "sharded multi-process state used before sv_attach_peers");
    ++s->epoch;
    return launch(s, LaunchClass::OTHER,
                  [&] { return launch_barrier(s->flags_dev, s->world, s->rank, s->epoch, s->stream); });
}

// ---- building launch descriptors -------------------------------------------
void make_apply(int l, int k, const int* phys_in_order, const cd* M /* bit b <-> phys_in_order[b] */, ApplyDesc& d,
                int tc_mode = 3) {
    d.tc_mode = tc_mode;
    std::vector<cd> Ms((size_t)1 << (2 * k));
    int sq[SV_MAX_FUSED];
    sort_matrix_qubits<cd>(k, phys_in_order, M, sq, Ms.data());
    d.k = k;
    for (int b = 0; b < k; ++b) d.q[b] = sq[b];
    d.m.resize(Ms.size());
    for (size_t i = 0; i < Ms.size(); ++i) d.m[i] = cf((float)Ms[i].real(), (float)Ms[i].imag());
    d.m64 = Ms;
    plan_apply(l, d);
}

// Block of a fused gate (matrix M over bits b <-> phys[b]) on the shard whose
// device bits are d: rows/columns whose global bits (phys[b] >= l) equal d's
// bits; locq receives the local positions.  A gate with no local position
// becomes a phase on local bit 0 (diag(c, c)).  Mirrors oracle/plan.py
// shard_block (reading R10).
std::vector<cd> shard_block(int k, const int* phys, const std::vector<cd>& M, int l, int d, std::vector<int>& locq) {
    std::vector<int> gb, lb;
    for (int b = 0; b < k; ++b) (phys[b] >= l ? gb : lb).push_back(b);
    int x = 0;
    for (int b : gb) x |= ((d >> (phys[b] - l)) & 1) << b;
    const int Dk = 1 << k, Dl = 1 << (int)lb.size();
    std::vector<int> idx(Dl);
    for (int t = 0; t < Dl; ++t) {
        int r = x;
        for (size_t j = 0; j < lb.size(); ++j) r |= ((t >> j) & 1) << lb[j];
        idx[t] = r;
    }
    locq.clear();
    for (int b : lb) locq.push_back(phys[b]);
    if (lb.empty()) {
        locq.push_back(0);
        const cd c = M[(size_t)x * Dk + x];
        return {c, cd(0), cd(0), c};
    }
    std::vector<cd> B((size_t)Dl * Dl);
    for (int r = 0; r < Dl; ++r)
        for (int c = 0; c < Dl; ++c) B[(size_t)r * Dl + c] = M[(size_t)idx[r] * Dk + idx[c]];
    return B;
}

// PERMUTE (data at local bit b moves to bit perm[b]) as passes of disjoint
// transpositions, <= 2 per pass (a 4-qubit permutation matrix carried in the
// kernel parameters; the FMA chain of a 0/1 matrix is exact).
// the bit swaps (in order) that move original bit b's data to bit perm[b]
std::vector<std::pair<int, int>> permute_swaps(int l, const std::vector<int>& perm) {
    std::vector<int> where(l);  // where[orig] = current position of orig's data
    for (int b = 0; b < l; ++b) where[b] = b;
    std::vector<std::pair<int, int>> swaps;
    for (int b = 0; b < l; ++b) {
        // want orig b's data at perm[b]
        int cur = where[b];
        int dst = perm[b];
        if (cur == dst) continue;
        // which orig currently sits at dst?
        int other = -1;
        for (int o = 0; o < l; ++o)
            if (where[o] == dst) other = o;
        swaps.push_back({cur, dst});
        where[b] = dst;
        where[other] = cur;
    }
    return swaps;
}

void lower_permute(int l, const std::vector<int>& perm, std::vector<ApplyDesc>& out) {
    const std::vector<std::pair<int, int>> swaps = permute_swaps(l, perm);
    size_t i = 0;
    while (i < swaps.size()) {
        std::vector<std::pair<int, int>> pass;
        uint64_t used = 0;
        while (i < swaps.size() && pass.size() < 2) {
            const auto sw = swaps[i];
            const uint64_t m = (1ull << sw.first) | (1ull << sw.second);
            if (used & m) break;  // keep order: a later swap touching these bits goes to the next pass
            used |= m;
            pass.push_back(sw);
            ++i;
        }
        const int k = 2 * (int)pass.size();
        int qs[SV_MAX_FUSED];
        for (size_t t = 0; t < pass.size(); ++t) {
            qs[2 * t] = pass[t].first;
            qs[2 * t + 1] = pass[t].second;
        }
        // matrix over qs (bit 2t <-> first, 2t+1 <-> second): swaps bit pairs
        const int D = 1 << k;
        std::vector<cd> M((size_t)D * D, cd(0));
        for (int c = 0; c < D; ++c) {
            int r = c;
            for (size_t t = 0; t < pass.size(); ++t) {
                const int b0 = (c >> (2 * t)) & 1, b1 = (c >> (2 * t + 1)) & 1;
                r &= ~(3 << (2 * t));
                r |= (b1 << (2 * t)) | (b0 << (2 * t + 1));
            }
            M[(size_t)r * D + c] = 1.0;
        }
        ApplyDesc d;
        make_apply(l, k, qs, M.data(), d);
        out.push_back(std::move(d));
    }
}

int run_apply(sv_state* s, const ApplyDesc& d) {
    for (int sh = 0; sh < s->local_shards(); ++sh) {
        float2* psi = s->virt ? s->shard[sh] : s->shard[s->rank];
        int rc = launch(s, d.high ? LaunchClass::HIGH : LaunchClass::LOW,
                        [&] { return launch_apply(psi, s->l, d, s->stream); });
        if (rc) return rc;
    }
    const int k = d.k;
    s->stats.bytes_apply += 16ull << s->l;
    (d.high ? s->stats.bytes_apply_high : s->stats.bytes_apply_low) += 16ull << s->l;
    s->stats.flops_apply += (uint64_t)((8 << k) - 2) << s->l;
    return SV_OK;
}

// per-shard blocks of one fused gate (diagonal exchange skip)
int run_apply_shards(sv_state* s, const std::vector<ApplyDesc>& ds) {
    for (int sh = 0; sh < s->local_shards(); ++sh) {
        float2* psi = s->virt ? s->shard[sh] : s->shard[s->rank];
        const ApplyDesc& d = ds[sh];
        int rc = launch(s, d.high ? LaunchClass::HIGH : LaunchClass::LOW,
                        [&] { return launch_apply(psi, s->l, d, s->stream); });
        if (rc) return rc;
    }
    const ApplyDesc& d = ds[0];
    s->stats.bytes_apply += 16ull << s->l;
    (d.high ? s->stats.bytes_apply_high : s->stats.bytes_apply_low) += 16ull << s->l;
    s->stats.flops_apply += (uint64_t)((8 << d.k) - 2) << s->l;
    return SV_OK;
}

int run_exchange(sv_state* s, const ExchangeDesc& x0) {
    Nvtx nv("sv.exchange");
    // complex128 shards: the same chunk swap over 8 B units (an amplitude is
    // units 2i, 2i + 1), i.e. every local and global position one higher
    ExchangeDesc x = x0;
    if (s->fp64) {
        x.l += 1;
        for (int j = 0; j < x.s; ++j) {
            x.P[j] += 1;
            x.p[j] += 1;
        }
    }
    int rc = barrier(s);
    if (rc) return rc;
    rc = launch(s, LaunchClass::EXCH,
                [&] { return launch_exchange(s->shard_dev, s->world, s->virt ? -1 : s->rank, x, s->stream); });
    if (rc) return rc;
    s->stats.bytes_exchange += (uint64_t)((1.0 - 1.0 / (1 << x.s)) * (double)s->elem * (double)(1ull << s->l));
    s->stats.n_exchanges++;
    return barrier(s);
}

void apply_event_pairs(sv_state* s, const std::vector<std::pair<int, int>>& pairs) {
    std::vector<int> inv(s->n);
    for (int q = 0; q < s->n; ++q) inv[s->pos[q]] = q;
    for (auto& pr : pairs) {
        const int a = inv[pr.first], b = inv[pr.second];
        s->pos[a] = pr.second;
        s->pos[b] = pr.first;
        inv[pr.first] = b;
        inv[pr.second] = a;
    }
}

ExchangeDesc make_exchange(int l, const std::vector<std::pair<int, int>>& pairs) {
    ExchangeDesc x;
    x.l = l;
    x.s = (int)pairs.size();
    for (int j = 0; j < x.s; ++j) {
        x.P[j] = pairs[j].first;
        x.p[j] = pairs[j].second;
    }
    return x;
}

// local qubit permutation of complex128 shards: exact bit swaps (moves only)
int run_permute64(sv_state* s, const std::vector<int>& perm) {
    for (const auto& sw : permute_swaps(s->l, perm))
        for (int i = 0; i < s->local_shards(); ++i) {
            const int d = s->virt ? i : s->rank;
            int rc = launch(s, LaunchClass::OTHER, [&] {
                return launch_swap_bits64(reinterpret_cast<double2*>(s->shard[d]), s->l, sw.first, sw.second, s->stream);
            });
            if (rc) return rc;
        }
    return SV_OK;
}

// Bring the state to a canonical map (local part identity) -- needed before
// sampling / whole-state reads in sharded mode.
int canonicalize(sv_state* s) {
    if (s->g == 0) return SV_OK;
    std::vector<Event> ev;
    std::vector<int> pos = s->pos;
    plan_canonicalize(s->n, s->g, pos, ev);
    for (auto& e : ev) {
        if (e.type == Event::EXCHANGE) {
            int rc = run_exchange(s, make_exchange(s->l, e.pairs));
            if (rc) return rc;
            apply_event_pairs(s, e.pairs);
        } else if (e.type == Event::PERMUTE && s->fp64) {
            int rc = run_permute64(s, e.perm);
            if (rc) return rc;
        } else if (e.type == Event::PERMUTE) {
            std::vector<ApplyDesc> passes;
            lower_permute(s->l, e.perm, passes);
            for (auto& d : passes) {
                int rc = run_apply(s, d);
                if (rc) return rc;
            }
            for (int p = 0; p < s->l; ++p) s->pos[e.perm[p]] = e.perm[p];
        }
    }
    return SV_OK;
}

// logical shard index of physical shard d
int sigma_of(const sv_state* s, int d) {
    int sg = 0;
    for (int q = s->l; q < s->n; ++q) sg |= ((d >> (s->pos[q] - s->l)) & 1) << (q - s->l);
    return sg;
}

uint64_t phys_of(const sv_state* s, uint64_t i) {
    uint64_t p = 0;
    for (int q = 0; q < s->n; ++q) p |= ((i >> q) & 1ull) << s->pos[q];
    return p;
}

int alloc_scratch(sv_state* s) {
    const uint64_t nb_local = (s->local_amps() + (1u << kSampleBinBits) - 1) >> kSampleBinBits;
    const uint64_t nb = nb_local * s->local_shards();
    cudaError_t e = cudaMalloc(&s->bins, nb * sizeof(uint64_t));
    if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(bins) failed");
    e = cudaMalloc(&s->scan_scratch, scan_scratch_elems(nb_local) * sizeof(uint64_t));
    if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(scan scratch) failed");
    e = cudaMalloc(&s->misc, 256 * sizeof(uint64_t));
    if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(misc) failed");
    e = cudaMalloc(&s->totals_ptr_dev, 64 * sizeof(uint64_t*));
    if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc failed");
    e = cudaMalloc(&s->sigma_dev, 64 * sizeof(int32_t));
    if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc failed");
    return SV_OK;
}

void destroy_state(sv_state* s) {
    if (!s) return;
    if (s->stream) cudaStreamSynchronize(s->stream);
    for (void* p : s->ipc_opened) cudaIpcCloseMemHandle(p);
    if (s->alloc) cudaFree(s->alloc);
    for (void* p : {(void*)s->shard_dev, (void*)s->bins, (void*)s->scan_scratch, (void*)s->misc,
                    (void*)s->totals_ptr_dev, (void*)s->sigma_dev, (void*)s->ctrl, (void*)s->xfer,
                    (void*)s->flags_dev, (void*)s->xfer_dev, (void*)s->idx_dev, (void*)s->amp_dev,
                    (void*)s->samp_dev})
        if (p) cudaFree(p);
    for (auto& sl : s->stage) {
        if (sl.host) cudaFreeHost(sl.host);
        if (sl.dev) cudaFree(sl.dev);
        if (sl.ev) cudaEventDestroy(sl.ev);
    }
    for (auto e : s->ev_pool) cudaEventDestroy(e);
    if (s->own_stream && s->stream) cudaStreamDestroy(s->stream);
    delete s;
}

int upload_shard_table(sv_state* s) {
    CK(s, cudaMemcpyAsync(s->shard_dev, s->shard.data(), sizeof(float2*) * s->world, cudaMemcpyHostToDevice,
                          s->stream));
    return SV_OK;
}

// staging slot layout: k = 6 matrix (32 KB) at 0, int8 W slices at 32 KB;
// complex128 states: planes (<= 24 KB, k <= 5) at 0, qubits at 128 KB
constexpr size_t kStageSlots = 8;
constexpr size_t kStageBytes = 136u << 10;
constexpr size_t kStageW = 32u << 10, kStageQ = 128u << 10;

int stage_acquire(sv_state* s, sv_state::StageSlot*& out) {
    if (s->stage.empty()) {
        s->stage.resize(kStageSlots);
        for (auto& sl : s->stage) {
            if (cudaMallocHost((void**)&sl.host, kStageBytes) != cudaSuccess ||
                cudaMalloc((void**)&sl.dev, kStageBytes) != cudaSuccess ||
                cudaEventCreateWithFlags(&sl.ev, cudaEventDisableTiming) != cudaSuccess)
                return fail(SV_ENOMEM, "staging ring allocation failed");
        }
    }
    sv_state::StageSlot& sl = s->stage[s->stage_next++ % kStageSlots];
    if (sl.used) CK(s, cudaEventSynchronize(sl.ev));  // waits only if the GPU is kStageSlots applies behind
    out = &sl;
    return SV_OK;
}
// copy `bytes` at slot offset `off` to the device (stream-ordered)
int stage_put(sv_state* s, sv_state::StageSlot& sl, size_t off, const void* src, size_t bytes) {
    std::memcpy(sl.host + off, src, bytes);
    CK(s, cudaMemcpyAsync(sl.dev + off, sl.host + off, bytes, cudaMemcpyHostToDevice, s->stream));
    return SV_OK;
}
int stage_release(sv_state* s, sv_state::StageSlot& sl) {
    CK(s, cudaEventRecord(sl.ev, s->stream));
    sl.used = true;
    return SV_OK;
}

}  // namespace

// =============================================================================
namespace {

// One fused gate for build_passes: ascending local (physical) qubits and its
// fp64 matrix over them.
struct PassIn {
    int k = 0;
    int q[SV_MAX_FUSED] = {0};
    std::vector<cd> M;
    // shard-dependent gate (diagonal exchange skip): its block on every local
    // shard slot over the same local qubits q (M = Mshard[0])
    std::vector<std::vector<cd>> Mshard;
};

// rpass gate kind of a 2^k x 2^k matrix rounded to complex64 (as gate_kind):
// 0 dense, 1 diagonal, 2 CZ-like diag(1, 1, 1, -1)
// fp32 operations per amplitude of a pass's kernels (stats, roofline)
uint64_t pass_ops(const PassDesc& pd, bool zinit) {
    return pd.spec ? rpass_jit_ops_per_amp(pd, zinit) : rpass_fma_per_amp(pd);
}

int kind_of(const std::vector<cd>& M, int k) {
    const int D = 1 << k;
    bool diag = true, cz = k == 2;
    for (int r = 0; r < D; ++r)
        for (int c = 0; c < D; ++c) {
            const float re = (float)M[(size_t)r * D + c].real(), im = (float)M[(size_t)r * D + c].imag();
            if (r != c && (re != 0.f || im != 0.f)) diag = cz = false;
            if (r == c && (im != 0.f || re != (r == D - 1 ? -1.f : 1.f))) cz = false;
        }
    return cz ? 2 : diag ? 1 : 0;
}

// Cache-blocked passes (reading R7).  Passes are formed like fused
// gates (the S3 greedy, one level up): a pass starts at the first unplaced
// gate and absorbs every later one whose qubits keep the pass within
// T - kPassPinned free tile qubits, provided it does not touch a qubit of a
// gate skipped before it (so it only moves past gates it commutes with).
// Qubits 0..kPassPinned-1 are in every tile (runs of >= 128 B); the pass's
// tile set S is the pinned qubits, the pass's qubits, then the lowest
// remaining qubits (longer runs).  The state never moves: a pass only
// chooses which amplitudes share a tile.
// Pass qubit sets chosen for a fused-gate structure (masks, diagonal flags,
// tile, pinning, search width): the formation depends on nothing else, so
// circuits of the same structure reuse it (process-wide cache)
std::mutex g_form_mu;
std::map<std::string, std::vector<uint64_t>> g_form_cache;

std::vector<PassDesc> build_passes(int T, const std::vector<PassIn>& in, int kPassPinned = SVB_PASS_PIN,
                                   int beam = SVB_PASS_BEAM) {
    const uint64_t pin = (1ull << kPassPinned) - 1ull;
    // gates per pass: one launch of the generic kernel's parameter struct, or
    // (14-qubit tiles: pass-specialised kernels only) a larger JIT launch
    const size_t kMaxGates = T >= 14 ? (size_t)kJitPassMaxGates : (size_t)kPassMaxGates;
    const size_t kMaxPlanes = T >= 14 ? (size_t)kJitPassMaxGates * 48 : (size_t)kPassPlaneFloats;
    const int Fp = T - kPassPinned;
    const size_t nf = in.size();
    std::vector<uint64_t> fm(nf, 0);
    for (size_t i = 0; i < nf; ++i)
        for (int b = 0; b < in[i].k; ++b) fm[i] |= 1ull << in[i].q[b];
    // diagonal gates commute with each other: a left-out diagonal gate only
    // blocks the non-diagonal gates on its qubits
    std::vector<char> dg(nf, 0);
    if (SVB_PASS_COMMUTE)
        for (size_t i = 0; i < nf; ++i) dg[i] = kind_of(in[i].M, in[i].k) >= 1;
    std::vector<char> placed(nf, 0);
    std::vector<PassDesc> passes;
    auto add_gate = [&](PassDesc& cur, size_t i) {
        const PassIn& f = in[i];
        const int D = 1 << f.k;
        PassGate pg{};
        pg.k = f.k;
        for (int b = 0; b < f.k; ++b) pg.pos[b] = (int)(std::find(cur.S.begin(), cur.S.end(), f.q[b]) - cur.S.begin());
        pg.poff = (uint32_t)cur.planes.size();
        pg.moff = (uint32_t)cur.mats.size();
        for (int e = 0; e < D * D; ++e) {
            cur.mats.push_back((float)f.M[e].real());
            cur.mats.push_back((float)f.M[e].imag());
            cur.mats64.push_back(f.M[e].real());
            cur.mats64.push_back(f.M[e].imag());
        }
        std::vector<float> Pp(D * D), Sp(D * D), Qp(D * D);
        for (int e = 0; e < D * D; ++e) {
            const float re = (float)f.M[e].real(), im = (float)f.M[e].imag();
            Pp[e] = re;
            Sp[e] = re + im;
            Qp[e] = im - re;
        }
        cur.planes.insert(cur.planes.end(), Pp.begin(), Pp.end());
        cur.planes.insert(cur.planes.end(), Sp.begin(), Sp.end());
        cur.planes.insert(cur.planes.end(), Qp.begin(), Qp.end());
        cur.gates.push_back(pg);
    };
    // ---- pass formation (reading R7): the qubit set Q of each pass.  A set
    // absorbs every later unplaced gate inside Q | pinned that touches no
    // qubit of an earlier gate left out (diagonal gates only block
    // non-diagonal ones, R12).  Greedy lookahead: grow Q from the first
    // unplaced gate's qubits by the qubit set of a left-out gate (among the
    // next 40 distinct ones) that absorbs the most gates, until none helps.
    // Search (beam > 1): keep the `beam` best additions at every growth step
    // (at most beam^2 partial sets), and take the final set whose greedy
    // completion of the rest of the circuit needs the fewest passes (ties:
    // the set absorbing more gates now).  30q D14: 6 -> 5 passes, 34q D20:
    // 10 -> 8 (profiles/r2_ab.md).
    auto absorb = [&](size_t i0, uint64_t Qc, const std::vector<char>& pl, std::vector<size_t>* out) {
        uint64_t Bl = 0, Bd = 0;  // qubits of left-out gates: non-diagonal / diagonal
        size_t cnt = 0, planes = 0;
        for (size_t j = i0; j < nf; ++j) {
            if (pl[j]) continue;
            const uint64_t Sj = fm[j];
            const size_t pj = 3ull << (2 * in[j].k);
            if (!(Sj & (dg[j] ? Bl : Bl | Bd)) && !(Sj & ~(Qc | pin)) && cnt < kMaxGates && planes + pj <= kMaxPlanes) {
                ++cnt;
                planes += pj;
                if (out) out->push_back(j);
            } else if (dg[j]) {
                Bd |= Sj;
            } else {
                Bl |= Sj;
            }
        }
        return cnt;
    };
    // ties between additions that absorb as many gates with as many qubits:
    // the earlier candidate (value_ties false) or the smaller qubit mask
    auto grow = [&](size_t i0, const std::vector<char>& pl, int B, std::vector<uint64_t>& finals,
                    bool value_ties = false) {
        std::vector<uint64_t> states{fm[i0] & ~pin};
        std::vector<char> in_cur(nf, 0);
        while (!states.empty()) {
            std::vector<uint64_t> nxt;
            for (uint64_t Qs : states) {
                std::vector<size_t> cur;
                const size_t have = absorb(i0, Qs, pl, &cur);
                for (size_t j : cur) in_cur[j] = 1;
                std::vector<uint64_t> cands;
                for (size_t j = i0; j < nf && cands.size() < 40; ++j) {
                    if (pl[j] || in_cur[j]) continue;
                    const uint64_t add = fm[j] & ~pin & ~Qs;
                    if (!add || __builtin_popcountll(Qs | add) > Fp) continue;
                    if (std::find(cands.begin(), cands.end(), add) == cands.end()) cands.push_back(add);
                }
                for (size_t j : cur) in_cur[j] = 0;
                struct Sc { size_t c; int bits; size_t ord; uint64_t add; };
                std::vector<Sc> sc;
                for (size_t o = 0; o < cands.size(); ++o) {
                    const size_t c = absorb(i0, Qs | cands[o], pl, nullptr);
                    if (c > have) sc.push_back({c, __builtin_popcountll(cands[o]), o, cands[o]});
                }
                std::sort(sc.begin(), sc.end(), [&](const Sc& a, const Sc& b) {
                    if (a.c != b.c) return a.c > b.c;
                    if (a.bits != b.bits) return a.bits < b.bits;
                    return value_ties ? a.add < b.add : a.ord < b.ord;
                });
                if (sc.empty()) {
                    if (std::find(finals.begin(), finals.end(), Qs) == finals.end()) finals.push_back(Qs);
                    continue;
                }
                for (size_t t = 0; t < sc.size() && t < (size_t)B; ++t) {
                    const uint64_t Qn = Qs | sc[t].add;
                    if (std::find(nxt.begin(), nxt.end(), Qn) == nxt.end()) nxt.push_back(Qn);
                }
            }
            if (nxt.size() > (size_t)(B * B)) nxt.resize((size_t)(B * B));
            states.swap(nxt);
        }
    };
    auto greedy_rest = [&](std::vector<char> pl, bool value_ties) {
        int n = 0;
        for (size_t i0 = 0; i0 < nf; ++i0) {
            if (pl[i0]) continue;
            std::vector<uint64_t> f;
            grow(i0, pl, 1, f, value_ties);
            std::vector<size_t> m;
            absorb(i0, f[0], pl, &m);
            for (size_t j : m) pl[j] = 1;
            ++n;
        }
        return n;
    };
    std::vector<uint64_t> forms;  // Q of every pass
    if (SVB_PASS_LOOKAHEAD) {
        std::string key;
        key.reserve(16 * nf + 32);
        key += std::to_string(T) + "," + std::to_string(kPassPinned) + "," + std::to_string(beam) + ",";
        for (size_t i = 0; i < nf; ++i) key += std::to_string(fm[i]) + (dg[i] ? "d" : "") + ",";
        bool hit = false;
        {
            std::lock_guard<std::mutex> lk(g_form_mu);
            auto it = g_form_cache.find(key);
            if (it != g_form_cache.end()) {
                forms = it->second;
                hit = true;
            }
        }
        if (!hit) {
            // one formation per tie policy (policy 2: both tie orders'
            // candidates, optimistic rollouts); the plan with the fewest passes
            // wins (ties: the earlier policy).  The search is sensitive to
            // ties: 30q D14 from |0...0> gives 6 passes with one order, 5 with
            // the other.
            auto formation = [&](int policy) {
                std::vector<uint64_t> fs;
                std::vector<char> pl(nf, 0);
                const bool vt = policy == 1;
                for (size_t i0 = 0; i0 < nf; ++i0) {
                    if (pl[i0]) continue;
                    std::vector<uint64_t> finals;
                    grow(i0, pl, std::max(1, beam), finals, vt);
                    if (beam > 1 && policy == 2) grow(i0, pl, beam, finals, true);
                    uint64_t Qb = finals[0];
                    if (finals.size() > 1) {
                        int best_n = 1 << 30;
                        size_t best_c = 0;
                        for (uint64_t Qf : finals) {
                            std::vector<char> p2 = pl;
                            std::vector<size_t> m;
                            const size_t c = absorb(i0, Qf, p2, &m);
                            for (size_t j : m) p2[j] = 1;
                            const int nrest = policy == 2 ? std::min(greedy_rest(p2, false), greedy_rest(p2, true))
                                                          : greedy_rest(p2, vt);
                            if (nrest < best_n || (nrest == best_n && c > best_c)) {
                                best_n = nrest;
                                best_c = c;
                                Qb = Qf;
                            }
                        }
                    }
                    std::vector<size_t> m;
                    absorb(i0, Qb, pl, &m);
                    for (size_t j : m) pl[j] = 1;
                    fs.push_back(Qb);
                }
                return fs;
            };
            forms = formation(0);
            if (beam > 1)
                for (int policy = 1; policy <= 2; ++policy) {
                    std::vector<uint64_t> f2 = formation(policy);
                    if (f2.size() < forms.size()) forms.swap(f2);
                }
            std::lock_guard<std::mutex> lk(g_form_mu);
            if (g_form_cache.size() > 256) g_form_cache.clear();
            g_form_cache[key] = forms;
        }
    }
    size_t npass = 0;
    for (size_t i = 0; i < nf; ++i) {
        if (placed[i]) continue;
        std::vector<size_t> mem{i};
        placed[i] = 1;
        uint64_t Q = fm[i], B = 0;
        if (SVB_PASS_LOOKAHEAD) {
            placed[i] = 0;
            Q = forms[npass++];
            mem.clear();
            absorb(i, Q, placed, &mem);
            for (size_t j : mem) placed[j] = 1;
            Q = 0;
            for (size_t j : mem) Q |= fm[j];
        } else {
            size_t planes = 3ull << (2 * in[i].k);
            for (size_t j = i + 1; j < nf && mem.size() < kMaxGates; ++j) {
                if (placed[j]) continue;
                const uint64_t Sj = fm[j];
                const size_t pj = 3ull << (2 * in[j].k);
                if (Sj & B) {
                    B |= Sj;
                } else if (__builtin_popcountll((Q | Sj) & ~pin) <= Fp && planes + pj <= kMaxPlanes) {
                    Q |= Sj;
                    planes += pj;
                    mem.push_back(j);
                    placed[j] = 1;
                } else {
                    B |= Sj;
                }
            }
        }
        uint64_t tile = Q | pin;
        for (int q = 0; q < 64 && __builtin_popcountll(tile) < T; ++q) tile |= 1ull << q;
        PassDesc cur;
        for (int q = 0; q < 64; ++q)
            if ((tile >> q) & 1ull) cur.S.push_back(q);
        plan_pass_tile(cur);
        for (size_t j : mem) {
            add_gate(cur, j);
            cur.src.push_back((int)j);
        }
        // shard-dependent gates: per-slot copies of the pass's matrices, and a
        // gate kind that fits every slot (dense < diagonal < CZ-like)
        size_t slots = 0;
        for (size_t j : mem) slots = std::max(slots, in[j].Mshard.size());
        if (slots) {
            cur.mats_shard.assign(slots, cur.mats);
            for (size_t t = 0; t < mem.size(); ++t) {
                const PassIn& f = in[mem[t]];
                if (f.Mshard.empty()) continue;
                PassGate& pg = cur.gates[t];
                int kind = 2;
                for (size_t sl = 0; sl < slots; ++sl) {
                    kind = std::min(kind, kind_of(f.Mshard[sl], f.k));
                    for (size_t e = 0; e < f.Mshard[sl].size(); ++e) {
                        cur.mats_shard[sl][pg.moff + 2 * e] = (float)f.Mshard[sl][e].real();
                        cur.mats_shard[sl][pg.moff + 2 * e + 1] = (float)f.Mshard[sl][e].imag();
                    }
                }
                pg.kind = kind;
            }
        }
        passes.push_back(std::move(cur));
    }
    return passes;
}

}  // namespace

extern "C" {

const char* sv_last_error(void) { return g_err.c_str(); }
const char* sv_version(void) { return "svb200 0.1 (sm_100a)"; }

int sv_create(int n_qubits, sv_state** out) {
    sv_config c{};
    c.n_qubits = n_qubits;
    c.world = 1;
    c.exchange_vmin = -1;
    c.device = -1;
    return sv_create_ex(&c, out);
}

int sv_create_ex(const sv_config* cfg, sv_state** out) {
    if (!cfg || !out) return fail(SV_EINVAL, "cfg/out is NULL");
    *out = nullptr;
    const int n = cfg->n_qubits;
    if (n < 1 || n > SV_MAX_QUBITS) return fail(SV_EINVAL, "n_qubits out of range [1, 40]");
    const int world = cfg->world <= 1 ? 1 : cfg->world;
    if (world & (world - 1)) return fail(SV_EUNSUPPORTED, "world must be a power of two");
    if (world > 64) return fail(SV_EUNSUPPORTED, "world > 64");
    int g = 0;
    while ((1 << g) < world) ++g;
    const int l = n - g;
    if (world > 1 && l < std::max(SV_MAX_FUSED, 2) + 2)
        return fail(SV_EUNSUPPORTED, "shard too small: need n - log2(world) >= 8");
    const bool virt = world == 1 || cfg->virtual_shards != 0;
    if (!virt && (cfg->rank < 0 || cfg->rank >= world)) return fail(SV_EINVAL, "rank out of range");
    if (cfg->precision != 0 && cfg->precision != 1) return fail(SV_EINVAL, "precision must be 0 (complex64) or 1 (complex128)");
    const bool fp64 = cfg->precision == 1;
    const size_t shard_bytes = (size_t)(fp64 ? 16 : 8) << l;
    const size_t need_bytes = shard_bytes * (virt ? world : 1);
    if (cfg->dev_buf && cfg->buf_bytes < need_bytes) return fail(SV_EINVAL, "buf_bytes too small for the state");
    if (cfg->dev_buf && !virt) return fail(SV_EUNSUPPORTED, "multi-process mode owns its buffers (dev_buf must be NULL)");

    std::unique_ptr<sv_state, void (*)(sv_state*)> s(new sv_state(), destroy_state);
    s->n = n;
    s->g = g;
    s->l = l;
    s->world = world;
    s->rank = virt ? 0 : cfg->rank;
    s->virt = virt;
    s->vmin = cfg->exchange_vmin < 0 ? 5 : cfg->exchange_vmin;
    s->fp64 = fp64;
    s->elem = fp64 ? 16 : 8;
    s->ext_buf = cfg->dev_buf != nullptr;
    if (cfg->device >= 0) CK(nullptr, cudaSetDevice(cfg->device));
    CK(nullptr, cudaGetDevice(&s->device));
    if (cfg->cuda_stream) {
        s->stream = (cudaStream_t)cfg->cuda_stream;
    } else {
        CK(nullptr, cudaStreamCreateWithFlags(&s->stream, cudaStreamNonBlocking));
        s->own_stream = true;
    }
    char* base = nullptr;
    if (cfg->dev_buf) {
        base = (char*)cfg->dev_buf;
    } else {
        size_t free_b = 0, total_b = 0;
        cudaMemGetInfo(&free_b, &total_b);
        const size_t bins_bytes = 8 * ((((size_t)1 << l) >> kSampleBinBits) + 1) * (virt ? world : 1);
        if (need_bytes + bins_bytes + (64ull << 20) > free_b)
            return fail(SV_ENOMEM, "state does not fit in free device memory");
        cudaError_t e = cudaMalloc(&s->alloc, need_bytes);
        if (e != cudaSuccess) return fail(SV_ENOMEM, std::string("cudaMalloc(state): ") + cudaGetErrorString(e));
        base = (char*)s->alloc;
    }
    s->shard.assign(world, nullptr);
    if (virt) {
        for (int d = 0; d < world; ++d) s->shard[d] = (float2*)(base + shard_bytes * d);
    } else {
        s->shard[s->rank] = (float2*)base;
        cudaError_t e = cudaMalloc(&s->ctrl, sizeof(Ctrl));
        if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(ctrl)");
        CK(nullptr, cudaMemset(s->ctrl, 0, sizeof(Ctrl)));
        e = cudaMalloc(&s->xfer, kXferBytes);
        if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(xfer)");
        CK(nullptr, cudaMalloc(&s->flags_dev, sizeof(uint64_t*) * world));
        CK(nullptr, cudaMalloc(&s->xfer_dev, sizeof(uint64_t*) * world));
    }
    CK(nullptr, cudaMalloc(&s->shard_dev, sizeof(float2*) * world));
    int rc = alloc_scratch(s.get());
    if (rc) return rc;
    rc = upload_shard_table(s.get());
    if (rc) return rc;
    s->pos.resize(n);
    for (int q = 0; q < n; ++q) s->pos[q] = q;
    rc = sv_reset(s.get());
    if (rc) return rc;
    CK(nullptr, cudaStreamSynchronize(s->stream));
    *out = s.release();
    return SV_OK;
}

int sv_destroy(sv_state* s) {
    if (!s) return fail(SV_EINVAL, "state handle is NULL");
    destroy_state(s);
    return SV_OK;
}

static int write_zero_state(sv_state* s);

int sv_reset(sv_state* s) {
    if (!s) return fail(SV_EINVAL, "state handle is NULL");
    if (s->sticky) return fail(SV_EBADSTATE, "state poisoned by an earlier device failure");
    for (int q = 0; q < s->n; ++q) s->pos[q] = q;
    s->bins_valid = false;
    if (!s->ext_buf) {
        s->zero_pending = true;  // written lazily (see sv_state::zero_pending)
        return SV_OK;
    }
    // caller-owned buffers (the caller may read or write the memory
    // directly) are written now
    s->zero_pending = false;
    return write_zero_state(s);
}

// materialise a pending |0...0> (every entry point that reads or writes the
// state calls this first, except sv_circuit_run_device's fused path)
static int materialize(sv_state* s) {
    if (!s->zero_pending) return SV_OK;
    s->zero_pending = false;
    return write_zero_state(s);
}

static int write_zero_state(sv_state* s) {
    s->bins_valid = false;
    for (int d = 0; d < s->local_shards(); ++d) {
        const int shard = s->virt ? d : s->rank;
        float2* psi = s->shard[shard];
        int rc = launch(s, LaunchClass::OTHER, [&] {
            return s->fp64 ? launch_reset64(reinterpret_cast<double2*>(psi), s->local_amps(), shard == 0, s->stream)
                           : launch_reset(psi, s->local_amps(), shard == 0, s->stream);
        });
        if (rc) return rc;
    }
    return SV_OK;
}

static int apply_matrix(sv_state* s, int k, const int32_t* qubits, const std::vector<cd>& M);

int sv_apply_fused(sv_state* s, int k, const int32_t* qubits, const sv_c64* matrix) {
    Nvtx nv("sv.apply_fused");
    int rc = check_state(s);
    if (rc) return rc;
    if (k < 1 || k > SV_MAX_FUSED) return fail(SV_EINVAL, "k must be in [1, 6]");
    if (!qubits || !matrix) return fail(SV_EINVAL, "qubits/matrix is NULL");
    const int D = 1 << k;
    std::vector<cd> M((size_t)D * D);
    for (int i = 0; i < D * D; ++i) M[i] = cd(matrix[i].re, matrix[i].im);
    return apply_matrix(s, k, qubits, M);
}

int sv_apply_fused_c128(sv_state* s, int k, const int32_t* qubits, const sv_c128* matrix) {
    int rc = check_state(s);
    if (rc) return rc;
    if (k < 1 || k > SV_MAX_FUSED) return fail(SV_EINVAL, "k must be in [1, 6]");
    if (!qubits || !matrix) return fail(SV_EINVAL, "qubits/matrix is NULL");
    const int D = 1 << k;
    std::vector<cd> M((size_t)D * D);
    for (int i = 0; i < D * D; ++i) M[i] = cd(matrix[i].re, matrix[i].im);
    return apply_matrix(s, k, qubits, M);
}

static int apply_matrix(sv_state* s, int k, const int32_t* qubits, const std::vector<cd>& Min) {
    // every argument is validated before any side effect (sv.h)
    int rc = SV_OK;
    uint64_t mask = 0;
    for (int b = 0; b < k; ++b) {
        if (qubits[b] < 0 || qubits[b] >= s->n) return fail(SV_EINVAL, "qubit out of range");
        if ((mask >> qubits[b]) & 1) return fail(SV_EINVAL, "duplicate qubit");
        mask |= 1ull << qubits[b];
    }
    if (s->g > 0 && k > s->l - 1) return fail(SV_EUNSUPPORTED, "gate wider than a shard allows");
    rc = materialize(s);
    if (rc) return rc;
    s->bins_valid = false;
    std::vector<cd> M = Min;
    std::vector<int> q(qubits, qubits + k);
    // sharded: bring global qubits local (one S4 step for this gate alone)
    if (s->g > 0) {
        std::vector<std::vector<int>> fq(1, q);
        std::vector<Event> ev;
        std::vector<int> pos = s->pos;
        plan_sharded(fq, s->n, s->g, s->vmin, ev, pos);
        for (auto& e : ev)
            if (e.type == Event::EXCHANGE) {
                rc = run_exchange(s, make_exchange(s->l, e.pairs));
                if (rc) return rc;
                apply_event_pairs(s, e.pairs);
            }
    }
    std::vector<int> phys(k);
    for (int b = 0; b < k; ++b) phys[b] = s->pos[q[b]];
    if (s->fp64) {
        Apply64Desc d;
        d.k = k;
        std::vector<cd> Ms(M.size());
        sort_matrix_qubits<cd>(k, phys.data(), M.data(), d.q, Ms.data());
        d.m = Ms;
        std::vector<double> planes(3 * M.size());
        pack_planes64(d, planes.data());
        sv_state::StageSlot* sl = nullptr;
        rc = stage_acquire(s, sl);
        if (rc) return rc;
        rc = stage_put(s, *sl, 0, planes.data(), planes.size() * sizeof(double));
        if (rc == SV_OK) rc = stage_put(s, *sl, kStageQ, d.q, sizeof(int) * SV_MAX_FUSED);
        if (rc) return rc;
        d.dev_planes = reinterpret_cast<const double*>(sl->dev);
        d.small_scratch = sl->dev + kStageQ;
        for (int i = 0; i < s->local_shards(); ++i) {
            const int sh = s->virt ? i : s->rank;
            rc = launch(s, LaunchClass::HIGH, [&] {
                return launch_apply64(reinterpret_cast<double2*>(s->shard[sh]), s->l, d, s->stream);
            });
            if (rc) return rc;
        }
        rc = stage_release(s, *sl);
        if (rc) return rc;
        s->stats.bytes_apply += 32ull << s->l;
        s->stats.bytes_apply_high += 32ull << s->l;
        s->stats.flops_apply += (uint64_t)((8 << k) - 2) << s->l;
        return SV_OK;
    }
    ApplyDesc d;
    make_apply(s->l, k, phys.data(), M.data(), d, s->tc_mode);
    sv_state::StageSlot* sl = nullptr;
    if (k == 6 || d.tci) {
        // device inputs staged through the ring (stream-ordered, no host sync)
        rc = stage_acquire(s, sl);
        if (rc) return rc;
        if (k == 6) {
            rc = stage_put(s, *sl, 0, d.m.data(), 64 * 64 * sizeof(float2));
            if (rc) return rc;
            d.dev_m = reinterpret_cast<const float2*>(sl->dev);
        }
        if (d.tci) {
            std::vector<uint8_t> w(wi8_bytes(k));
            pack_wi8(d, w.data());
            rc = stage_put(s, *sl, kStageW, w.data(), w.size());
            if (rc) return rc;
            d.dev_wi8 = reinterpret_cast<const uint8_t*>(sl->dev + kStageW);
        }
    }
    rc = run_apply(s, d);
    if (rc) return rc;
    return sl ? stage_release(s, *sl) : SV_OK;
}

int sv_apply_controlled(sv_state* s, int n_ctrl, const int32_t* controls, int k, const int32_t* targets,
                        const sv_c64* matrix) {
    int rc = check_state(s);
    if (rc) return rc;
    if (k < 1 || k > SV_MAX_FUSED) return fail(SV_EINVAL, "k must be in [1, 6]");
    if (n_ctrl < 0 || n_ctrl > SV_MAX_FUSED) return fail(SV_EINVAL, "n_ctrl must be in [0, 6]");
    if (!targets || !matrix || (n_ctrl > 0 && !controls)) return fail(SV_EINVAL, "NULL argument");
    uint64_t mask = 0;
    for (int b = 0; b < k + n_ctrl; ++b) {
        const int q = b < k ? targets[b] : controls[b - k];
        if (q < 0 || q >= s->n) return fail(SV_EINVAL, "qubit out of range");
        if ((mask >> q) & 1) return fail(SV_EINVAL, "duplicate qubit");
        mask |= 1ull << q;
    }
    if (n_ctrl == 0) return sv_apply_fused(s, k, targets, matrix);
    const int D = 1 << k;
    std::vector<cd> M((size_t)D * D);
    for (int i = 0; i < D * D; ++i) M[i] = cd(matrix[i].re, matrix[i].im);
    int minc = s->n;
    for (int c = 0; c < n_ctrl; ++c) minc = std::min(minc, (int)controls[c]);
    const bool subspace = !s->fp64 && s->g == 0 && minc >= 1;
    if (!subspace && k + n_ctrl > SV_MAX_FUSED)
        return fail(SV_EUNSUPPORTED, "controlled gate needs k + n_ctrl <= 6 here (control on qubit 0, sharded or fp64)");
    if (subspace) {
        rc = materialize(s);
        if (rc) return rc;
        s->bins_valid = false;
        // tile engine over the control-1 subspace only: 2^-n_ctrl of the state
        ApplyDesc d;
        make_apply(s->l, k, targets, M.data(), d);
        d.nc = n_ctrl;
        for (int c = 0; c < n_ctrl; ++c) d.cq[c] = controls[c];
        d.tc = false;
        plan_apply(s->l, d);
        d.tc = false;
        sv_state::StageSlot* sl = nullptr;
        if (k == 6) {
            rc = stage_acquire(s, sl);
            if (rc == SV_OK) rc = stage_put(s, *sl, 0, d.m.data(), 64 * 64 * sizeof(float2));
            if (rc) return rc;
            d.dev_m = reinterpret_cast<const float2*>(sl->dev);
        }
        rc = launch(s, d.high ? LaunchClass::HIGH : LaunchClass::LOW,
                    [&] { return launch_apply(s->shard[0], s->l, d, s->stream); });
        if (rc) return rc;
        if (sl) {
            rc = stage_release(s, *sl);
            if (rc) return rc;
        }
        s->stats.bytes_apply += 16ull << (s->l - n_ctrl);
        (d.high ? s->stats.bytes_apply_high : s->stats.bytes_apply_low) += 16ull << (s->l - n_ctrl);
        s->stats.flops_apply += (uint64_t)((8 << k) - 2) << (s->l - n_ctrl);
        return SV_OK;
    }
    // dense block expansion over targets ++ controls: U on the all-ones control block, identity elsewhere
    const int kk = k + n_ctrl, DD = 1 << kk;
    std::vector<int32_t> qs(targets, targets + k);
    for (int c = 0; c < n_ctrl; ++c) qs.push_back(controls[c]);
    std::vector<cd> F((size_t)DD * DD, cd(0));
    const int call = ((1 << n_ctrl) - 1) << k;
    for (int r = 0; r < DD; ++r) {
        if ((r & call) == call) {
            for (int c = 0; c < D; ++c) F[(size_t)r * DD + (call | c)] = M[(size_t)(r & (D - 1)) * D + c];
        } else {
            F[(size_t)r * DD + r] = 1.0;
        }
    }
    return apply_matrix(s, kk, qs.data(), F);
}

int sv_fusion_plan(const sv_gate* gates, size_t n_gates, int max_fused, int32_t* buf, size_t cap, size_t* need) {
    if (!need) return fail(SV_EINVAL, "need is NULL");
    if (max_fused < 0 || max_fused > SV_MAX_FUSED) return fail(SV_EINVAL, "max_fused must be in [0, 6]");
    int rc = validate_gates(gates, n_gates, -1);
    if (rc) return rc;
    std::vector<FusedGate> plan;
    fuse_plan(gates, n_gates, max_fused, plan);
    size_t len = 0;
    for (auto& f : plan) len += 2 + f.k + f.mem.size();
    *need = len;
    if (cap < len) return fail(SV_EINVAL, "cap too small");
    if (len && !buf) return fail(SV_EINVAL, "buf is NULL");
    size_t o = 0;
    for (auto& f : plan) {
        buf[o++] = f.k;
        for (int b = 0; b < f.k; ++b) buf[o++] = f.q[b];
        buf[o++] = (int32_t)f.mem.size();
        for (int32_t m : f.mem) buf[o++] = m;
    }
    return SV_OK;
}

int sv_block_plan(const sv_gate* gates, size_t n_gates, int max_fused, int tile_bits, int32_t* buf, size_t cap,
                  size_t* need) {
    if (!need) return fail(SV_EINVAL, "need is NULL");
    if (max_fused < 1 || max_fused > 4) return fail(SV_EINVAL, "max_fused must be in [1, 4] for blocked passes");
    if (tile_bits < 10 || tile_bits > 14) return fail(SV_EINVAL, "tile_bits must be in [10, 14]");
    int rc = validate_gates(gates, n_gates, -1);
    if (rc) return rc;
    std::vector<FusedGate> plan;
    fuse_plan(gates, n_gates, max_fused, plan);
    std::vector<PassIn> in;
    for (auto& f : plan) {
        build_fused_matrix(gates, f);
        PassIn pi;
        pi.k = f.k;
        for (int b = 0; b < f.k; ++b) pi.q[b] = f.q[b];
        pi.M = f.M;
        in.push_back(std::move(pi));
    }
    std::vector<int32_t> o;
    for (auto& pd : build_passes(tile_bits, in)) {
        o.push_back((int32_t)pd.S.size());
        for (int q : pd.S) o.push_back(q);
        o.push_back((int32_t)pd.src.size());
        for (int j : pd.src) o.push_back(j);
        std::vector<std::vector<int>> R, G;
        if (rpass_supported(pd)) rpass_phase_plan(pd, R, G);
        o.push_back((int32_t)R.size());
        for (size_t i = 0; i < R.size(); ++i) {
            o.push_back((int32_t)R[i].size());
            for (int r : R[i]) o.push_back(r);
            o.push_back((int32_t)G[i].size());
            for (int g : G[i]) o.push_back(g);
        }
    }
    *need = o.size();
    if (cap < o.size()) return fail(SV_EINVAL, "cap too small");
    if (!o.empty() && !buf) return fail(SV_EINVAL, "buf is NULL");
    std::copy(o.begin(), o.end(), buf);
    return SV_OK;
}

int sv_fused_matrix(const sv_gate* gates, size_t n_gates, int max_fused, size_t index, sv_c128* out, size_t cap) {
    if (max_fused < 0 || max_fused > SV_MAX_FUSED) return fail(SV_EINVAL, "max_fused must be in [0, 6]");
    int rc = validate_gates(gates, n_gates, -1);
    if (rc) return rc;
    std::vector<FusedGate> plan;
    fuse_plan(gates, n_gates, max_fused, plan);
    if (index >= plan.size()) return fail(SV_EINVAL, "index out of range");
    FusedGate& f = plan[index];
    build_fused_matrix(gates, f);
    if (!out || cap < f.M.size()) return fail(SV_EINVAL, "out too small");
    for (size_t i = 0; i < f.M.size(); ++i) out[i] = sv_c128{f.M[i].real(), f.M[i].imag()};
    return SV_OK;
}

static void write_events(const std::vector<Event>& ev, std::vector<int32_t>& o) {
    for (auto& e : ev) {
        if (e.type == Event::EXCHANGE) {
            o.push_back(-1);
            o.push_back((int32_t)e.pairs.size());
            for (auto& pr : e.pairs) {
                o.push_back(pr.first);
                o.push_back(pr.second);
            }
        } else if (e.type == Event::APPLY) {
            o.push_back(e.fused);
            o.push_back(e.k);
            for (int b = 0; b < e.k; ++b) o.push_back(e.phys[b]);
        } else {
            o.push_back(-2);
            o.push_back((int32_t)e.perm.size());
            for (int v : e.perm) o.push_back(v);
        }
    }
}

static int shard_plan_impl(const int32_t* fs, size_t len, const uint64_t* diag, int n, int g, int vmin, int32_t* buf,
                           size_t cap, size_t* need, int32_t* final_pos);

int sv_shard_plan(const int32_t* fs, size_t len, int n, int g, int vmin, int32_t* buf, size_t cap, size_t* need,
                  int32_t* final_pos) {
    return shard_plan_impl(fs, len, nullptr, n, g, vmin, buf, cap, need, final_pos);
}

int sv_shard_plan_diag(const int32_t* fs, size_t len, const uint64_t* diag, int n, int g, int vmin, int32_t* buf,
                       size_t cap, size_t* need, int32_t* final_pos) {
    if (!diag && len) return fail(SV_EINVAL, "diag is NULL");
    return shard_plan_impl(fs, len, diag, n, g, vmin, buf, cap, need, final_pos);
}

int sv_fusion_diag_masks(const sv_gate* gates, size_t n_gates, int max_fused, uint64_t* out, size_t cap, size_t* need) {
    if (!need) return fail(SV_EINVAL, "need is NULL");
    if (max_fused < 0 || max_fused > SV_MAX_FUSED) return fail(SV_EINVAL, "max_fused must be in [0, 6]");
    int rc = validate_gates(gates, n_gates, -1);
    if (rc) return rc;
    std::vector<FusedGate> plan;
    fuse_plan(gates, n_gates, max_fused, plan);
    *need = plan.size();
    if (cap < plan.size()) return fail(SV_EINVAL, "cap too small");
    if (!plan.empty() && !out) return fail(SV_EINVAL, "out is NULL");
    for (size_t i = 0; i < plan.size(); ++i) {
        build_fused_matrix(gates, plan[i]);
        out[i] = diag_mask(plan[i]);
    }
    return SV_OK;
}

static int shard_plan_impl(const int32_t* fs, size_t len, const uint64_t* diag, int n, int g, int vmin, int32_t* buf,
                           size_t cap, size_t* need, int32_t* final_pos) {
    if (!need) return fail(SV_EINVAL, "need is NULL");
    if (n < 1 || n > SV_MAX_QUBITS || g < 0 || g >= n) return fail(SV_EINVAL, "bad n / log2_world");
    if (len && !fs) return fail(SV_EINVAL, "fusion stream is NULL");
    std::vector<std::vector<int>> fq;
    size_t o = 0;
    while (o < len) {
        const int k = fs[o++];
        if (k < 1 || k > SV_MAX_FUSED || o + k + 1 > len) return fail(SV_EINVAL, "malformed fusion stream");
        std::vector<int> q(fs + o, fs + o + k);
        for (int x : q)
            if (x < 0 || x >= n) return fail(SV_EINVAL, "qubit out of range in fusion stream");
        if (k > n - g) return fail(SV_EUNSUPPORTED, "fused gate wider than a shard");
        o += k;
        const int nm = fs[o++];
        if (nm < 0 || o + nm > len) return fail(SV_EINVAL, "malformed fusion stream");
        o += nm;
        fq.push_back(q);
    }
    std::vector<Event> ev;
    std::vector<int> pos;
    std::vector<uint64_t> dm;
    if (diag) dm.assign(diag, diag + fq.size());
    plan_sharded(fq, n, g, vmin < 0 ? 5 : vmin, ev, pos, diag ? &dm : nullptr);
    std::vector<int32_t> outv;
    write_events(ev, outv);
    *need = outv.size();
    if (cap < outv.size()) return fail(SV_EINVAL, "cap too small");
    if (!outv.empty() && !buf) return fail(SV_EINVAL, "buf is NULL");
    std::copy(outv.begin(), outv.end(), buf);
    if (final_pos)
        for (int q = 0; q < n; ++q) final_pos[q] = pos[q];
    return SV_OK;
}

static int circuit_create_impl(sv_state* s, const sv_gate* gates, size_t n_gates, int max_fused, sv_circuit** out,
                               bool zero_only);

int sv_circuit_create(sv_state* s, const sv_gate* gates, size_t n_gates, int max_fused, sv_circuit** out) {
    return circuit_create_impl(s, gates, n_gates, max_fused, out, false);
}

static int circuit_create_impl(sv_state* s, const sv_gate* gates, size_t n_gates, int max_fused, sv_circuit** out,
                               bool zero_only) {
    int rc = check_state(s);
    if (rc) return rc;
    if (!out) return fail(SV_EINVAL, "out is NULL");
    if (max_fused < 0 || max_fused > SV_MAX_FUSED) return fail(SV_EINVAL, "max_fused must be in [0, 6]");
    rc = validate_gates(gates, n_gates, s->n);
    if (rc) return rc;
    if (s->g > 0 && std::max(max_fused, 2) > s->l - 1) return fail(SV_EUNSUPPORTED, "fused gates wider than a shard allows");
    Nvtx nv("sv.circuit_create");
    std::unique_ptr<sv_circuit> c(new sv_circuit());
    c->owner = s;
    const double t0 = now_s();
    std::vector<FusedGate> plan;
    {
        Nvtx nf("sv.fuse");
        fuse_plan(gates, n_gates, max_fused, plan);
        for (auto& f : plan) build_fused_matrix(gates, f);
    }
    const double t1 = now_s();
    Nvtx np_("sv.plan");
    c->stats.t_fuse_s = t1 - t0;
    c->stats.n_fused = (int)plan.size();
    for (auto& f : plan) c->stats.fused_hist[f.k]++;
    // Cache-blocked passes (complex64, large shards, k <= 4; sharded or not):
    // each maximal run of APPLY events between exchanges is cut into passes
    // by build_passes (reading R7); exchanges and permutations stay as they are.
    // complex128 states: pass-specialised fp64 kernels (16 amplitudes per
    // thread) for max_fused <= 2.
    // auto tile: 14 qubits for the complex64 pass kernels (512 threads, 128 KB;
    // 30q D14 F=1 24.7 ms vs 26.1 at 13, 32q D20 145 vs 166 ms: fewer passes
    // for the same runs), 13 for the generic kernel, 13 for complex128 (512
    // threads, 128 KB; with the structured gates 30q D14 F=1 57.6 ms, 7
    // passes, vs 61.6 ms, 9 passes, at 12)
    int T = s->block_bits >= 0 ? s->block_bits
                               : (max_fused <= 2 && s->l >= 20 ? (s->fp64 ? 13 : s->pass_jit ? 14 : 13) : 0);
    if (T == 14 && (s->fp64 || !s->pass_jit || max_fused > 2)) T = 13;  // 14-qubit tiles: complex64 pass kernels only
    const bool blocked = (!s->fp64 || (s->pass_jit && max_fused <= 2)) && T >= 10 && s->l >= T + 2 &&
                         s->n > kSmallCircuitMaxQubits && max_fused <= 4 && max_fused >= 1;
    // plan (sharded) or trivial apply list
    std::vector<Event> ev;
    c->pos_in = s->pos;
    std::vector<int> pos = s->pos;
    if (s->g > 0) {
        std::vector<std::vector<int>> fq;
        for (auto& f : plan) fq.emplace_back(f.q, f.q + f.k);
        // diagonal exchange skip (reading R10): per-shard blocks run on the
        // per-gate SIMT path or in register-blocked passes (k <= 2)
        const bool skip = s->diag_skip && !s->fp64 && (!blocked || max_fused <= 2);
        std::vector<uint64_t> dm;
        if (skip)
            for (auto& f : plan) dm.push_back(diag_mask(f));
        plan_sharded(fq, s->n, s->g, s->vmin, ev, pos, skip ? &dm : nullptr);
        plan_canonicalize(s->n, s->g, pos, ev);
    } else {
        for (size_t i = 0; i < plan.size(); ++i) {
            Event a;
            a.type = Event::APPLY;
            a.fused = (int)i;
            a.k = plan[i].k;
            for (int b = 0; b < a.k; ++b) a.phys[b] = plan[i].q[b];
            ev.push_back(a);
        }
    }
    c->pos_out = pos;
    const double t2 = now_s();
    c->stats.t_plan_s = t2 - t1;
    if (s->fp64 && !blocked) {
        // complex128: one apply64 launch per fused gate (per local shard, on
        // its physical positions) and the plan's exchanges; all planes and
        // qubit lists uploaded once (row a4)
        c->a64 = true;
        std::vector<double> planes;
        std::vector<int> qs;
        std::vector<size_t> poff;
        for (auto& e : ev) {
            sv_circuit::Step st;
            st.type = e.type;
            poff.push_back(planes.size());
            if (e.type == Event::EXCHANGE) {
                st.exch = make_exchange(s->l, e.pairs);
                c->stats.n_exchanges++;
            } else if (e.type == Event::PERMUTE) {
                st.perm = e.perm;
            } else {
                const FusedGate& f = plan[e.fused];
                st.a64.k = f.k;
                st.a64.m.resize(f.M.size());
                // fp64, ascending physical qubits: no rounding to complex64
                sort_matrix_qubits<cd>(f.k, e.phys, f.M.data(), st.a64.q, st.a64.m.data());
                planes.resize(planes.size() + 3 * f.M.size());
                pack_planes64(st.a64, planes.data() + poff.back());
            }
            for (int b = 0; b < SV_MAX_FUSED; ++b) qs.push_back(st.a64.q[b]);
            c->steps.push_back(std::move(st));
        }
        if (!planes.empty()) {
            cudaError_t e = cudaMalloc(&c->planes64, planes.size() * sizeof(double));
            if (e == cudaSuccess) e = cudaMalloc(&c->q64, qs.size() * sizeof(int));
            if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(fp64 circuit)");
            CK(s, cudaMemcpyAsync(c->planes64, planes.data(), planes.size() * sizeof(double), cudaMemcpyHostToDevice,
                                  s->stream));
            CK(s, cudaMemcpyAsync(c->q64, qs.data(), qs.size() * sizeof(int), cudaMemcpyHostToDevice, s->stream));
            CK(s, cudaStreamSynchronize(s->stream));
            for (size_t i = 0; i < c->steps.size(); ++i) {
                c->steps[i].a64.dev_planes = c->planes64 + poff[i];
                c->steps[i].a64.small_scratch = c->q64 + SV_MAX_FUSED * i;
            }
        }
        c->stats.t_upload_s = now_s() - t2;
        *out = c.release();
        return SV_OK;
    }
    // lower events to launch descriptors
    size_t n6 = 0;
    std::vector<PassIn> run, run_all;
    auto flush_passes = [&]() {
        if (run.empty()) return;
        for (auto& pd : build_passes(T, run, s->pass_pin, s->pass_beam)) {
            pd.wide = s->fp64;
            pd.spec = s->pass_spec && s->pass_jit && pd.mats_shard.empty();
            pd.fma_per_amp = rpass_supported(pd) ? pass_ops(pd, false) : 0;
            c->stats.fma_apply += pd.fma_per_amp << s->l;
            c->stats.n_passes++;
            sv_circuit::Step st;
            st.type = Event::APPLY;
            st.block = true;
            st.pass = std::move(pd);
            c->steps.push_back(std::move(st));
        }
        run.clear();
    };
    if (blocked) c->stats.block_bits = T;
    for (auto& e : ev) {
        // APPLY on global positions (diagonal skip): the block of every local
        // shard slot over the gate's local qubits
        std::vector<int> locq;
        std::vector<std::vector<cd>> blocks;
        if (e.type == Event::APPLY && s->g > 0) {
            bool gl = false;
            for (int b = 0; b < e.k; ++b) gl |= e.phys[b] >= s->l;
            if (gl) {
                for (int sl = 0; sl < s->local_shards(); ++sl)
                    blocks.push_back(shard_block(e.k, e.phys, plan[e.fused].M, s->l, s->virt ? sl : s->rank, locq));
            }
        }
        if (blocked && e.type == Event::APPLY) {
            PassIn pi;
            if (!blocks.empty()) {
                pi.k = (int)locq.size();
                for (auto& B : blocks) {
                    std::vector<cd> Ms(B.size());
                    sort_matrix_qubits<cd>(pi.k, locq.data(), B.data(), pi.q, Ms.data());
                    pi.Mshard.push_back(std::move(Ms));
                }
                pi.M = pi.Mshard[0];
            } else {
                pi.k = e.k;
                pi.M.resize((size_t)1 << (2 * e.k));
                sort_matrix_qubits<cd>(e.k, e.phys, plan[e.fused].M.data(), pi.q, pi.M.data());
            }
            if (s->g == 0) run_all.push_back(pi);
            run.push_back(std::move(pi));
            continue;
        }
        flush_passes();
        sv_circuit::Step st;
        st.type = e.type;
        if (e.type == Event::APPLY && !blocks.empty()) {
            for (auto& B : blocks) {  // SIMT: no per-shard int8 slices
                st.apply_shard.emplace_back();
                make_apply(s->l, (int)locq.size(), locq.data(), B.data(), st.apply_shard.back(), 0);
            }
            st.apply = st.apply_shard[0];
        } else if (e.type == Event::APPLY) {
            make_apply(s->l, e.k, e.phys, plan[e.fused].M.data(), st.apply, s->tc_mode);
            if (e.k == 6) ++n6;
        } else if (e.type == Event::EXCHANGE) {
            st.exch = make_exchange(s->l, e.pairs);
            c->stats.n_exchanges++;
        } else if (s->fp64) {
            st.perm = e.perm;
        } else {
            lower_permute(s->l, e.perm, st.perm_applies);
        }
        c->steps.push_back(std::move(st));
    }
    // product-state start (unsharded, pass-specialised kernels): the first
    // gate of each qubit, if it is a one-qubit gate, commutes with every gate
    // before it, so a run from |0...0> may apply all of them first -- i.e.
    // start from the product state prod_q v_q[bit q] (v_q = that gate's first
    // column) and skip them.  Built as a second step list (steps_z) used when
    // the state is a pending |0...0> at run time.
    std::vector<cd> pv;  // v_q, 2 per qubit
    if (blocked && s->pass_jit && s->g == 0 && !run_all.empty()) {
        pv.assign(2 * (size_t)s->n, cd(0));
        for (int q = 0; q < s->n; ++q) pv[2 * q] = 1.0;
        std::vector<char> seen(s->n, 0);
        std::vector<PassIn> rest;
        int nfold = 0;
        for (auto& g : run_all) {
            if (g.k == 1 && !seen[g.q[0]]) {
                pv[2 * g.q[0]] = g.M[0];      // column 0 of the 2 x 2 matrix
                pv[2 * g.q[0] + 1] = g.M[2];
                ++nfold;
            } else {
                rest.push_back(g);
            }
            for (int b = 0; b < g.k; ++b) seen[g.q[b]] = 1;
        }
        std::vector<PassDesc> pz = (nfold && !rest.empty()) ? build_passes(T, rest, s->pass_pin, s->pass_beam) : std::vector<PassDesc>{};
        if (!pz.empty() && rpass_supported(pz[0])) {
            for (int p = 0; p < (int)pz[0].S.size(); ++p) {
                pz[0].pinit_v.push_back(pv[2 * pz[0].S[p]]);
                pz[0].pinit_v.push_back(pv[2 * pz[0].S[p] + 1]);
            }
            c->stats_z = c->stats;
            c->stats_z.n_passes = 0;
            c->stats_z.fma_apply = 0;
            for (auto& pd : pz) {
                pd.wide = s->fp64;
                pd.spec = s->pass_spec && s->pass_jit && pd.mats_shard.empty();
                pd.fma_per_amp = rpass_supported(pd) ? pass_ops(pd, &pd == &pz[0]) : 0;
                c->stats_z.fma_apply += pd.fma_per_amp << s->l;
                c->stats_z.n_passes++;
                sv_circuit::Step st;
                st.type = Event::APPLY;
                st.block = true;
                st.pass = std::move(pd);
                c->steps_z.push_back(std::move(st));
            }
        }
    }
    // a circuit created for one run from the pending |0...0> (sv_run_circuit)
    // needs only the product-state steps: skip planning the others
    if (zero_only && !c->steps_z.empty()) {
        run.clear();
        c->zero_only = true;
        c->stats.n_passes = c->stats_z.n_passes;
        c->stats.fma_apply = c->stats_z.fma_apply;
    }
    flush_passes();
    // the last pass of an unsharded complex64 circuit also writes the
    // sampler's bin weights (sv_sample then skips its read of the state)
    if (SVB_FUSED_BINS && blocked && s->pass_jit && s->g == 0 && !s->fp64)
        for (auto* list : {&c->steps, &c->steps_z})
            if (!list->empty() && list->back().block && rpass_supported(list->back().pass) &&
                list->back().pass.r >= kSampleBinBits)  // bins = 16 consecutive amplitudes = tile bits 0..3
                list->back().pass.bins = true;
    // pass-specialised kernels of every register-blocked pass (compiled in
    // parallel, cached per process; the first pass also in its |0...0> form)
    if (blocked && s->pass_jit) {
        std::vector<const PassDesc*> pds;
        std::vector<char> zs;
        std::vector<std::vector<RpJitLaunch>*> dst;
        for (auto* list : {&c->steps, &c->steps_z}) {
            for (size_t i = 0; i < list->size(); ++i) {
                auto& st = (*list)[i];
                if (!st.block || !rpass_supported(st.pass)) continue;
                const bool z = list == &c->steps_z && i == 0;
                pds.push_back(&st.pass);
                zs.push_back(z ? 1 : 0);
                dst.push_back(z ? &st.jitz : &st.jit);
                if (list == &c->steps && i == 0 && c->steps_z.empty()) {  // lazy |0...0> without the fold
                    pds.push_back(&st.pass);
                    zs.push_back(1);
                    dst.push_back(&st.jitz);
                }
            }
        }
        if (!pds.empty()) {
            Nvtx nk("sv.pass_kernels");
            std::vector<std::vector<RpJitLaunch>> got;
            rc = rpass_jit_prepare_many(pds, s->l, zs, got);
            if (rc) return rc;
            for (size_t i = 0; i < got.size(); ++i) *dst[i] = std::move(got[i]);
        }
        if (!c->steps_z.empty()) {
            // tile-factor tables of the product-state pass: tile index bit i
            // <-> the i-th qubit outside its tile (ascending); A over the low
            // h1 bits, B over the rest; fp64 products rounded once
            const PassDesc& p0 = c->steps_z[0].pass;
            std::vector<int> out_q;
            for (int q = 0; q < s->l; ++q)
                if (std::find(p0.S.begin(), p0.S.end(), q) == p0.S.end()) out_q.push_back(q);
            const int h = (int)out_q.size(), h1 = h / 2, h2 = h - h1;
            const size_t nA = (size_t)1 << h1, nB = (size_t)1 << h2;
            std::vector<cd> tab(nA + nB);
            for (int part = 0; part < 2; ++part) {
                const int nb = part ? h2 : h1, b0 = part ? h1 : 0;
                cd* t = tab.data() + (part ? nA : 0);
                for (size_t x = 0; x < ((size_t)1 << nb); ++x) {
                    cd z = 1.0;
                    for (int i = 0; i < nb; ++i) z *= pv[2 * out_q[b0 + i] + ((x >> i) & 1)];
                    t[x] = z;
                }
            }
            // complex64 tables (rounded once) or complex128 ones (fp64 states)
            std::vector<float2> tab32;
            for (const cd& z : tab) tab32.push_back(make_float2((float)z.real(), (float)z.imag()));
            const size_t esz = s->fp64 ? sizeof(cd) : sizeof(float2);
            const void* host = s->fp64 ? (const void*)tab.data() : (const void*)tab32.data();
            cudaError_t e = cudaMalloc(&c->ptab, tab.size() * esz);
            if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(product-state tables)");
            CK(s, cudaMemcpyAsync(c->ptab, host, tab.size() * esz, cudaMemcpyHostToDevice, s->stream));
            CK(s, cudaStreamSynchronize(s->stream));
            for (auto& l : c->steps_z[0].jitz) {
                l.tabA = c->ptab;
                l.tabB = (const char*)c->ptab + nA * esz;
                l.h1 = h1;
            }
        }
    }
    // int8 tensor-core W slices of every tensor-core gate: one H2D upload
    {
        size_t total = 0;
        for (auto& st : c->steps)
            if (st.type == Event::APPLY && st.apply.tci) total += wi8_bytes(st.apply.k);
        if (total) {
            std::vector<uint8_t> host(total);
            std::vector<size_t> offs;
            size_t o = 0;
            for (auto& st : c->steps)
                if (st.type == Event::APPLY && st.apply.tci) {
                    pack_wi8(st.apply, host.data() + o);
                    offs.push_back(o);
                    o += wi8_bytes(st.apply.k);
                }
            cudaError_t e = cudaMalloc(&c->wi8, total);
            if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(int8 W slices)");
            CK(s, cudaMemcpyAsync(c->wi8, host.data(), total, cudaMemcpyHostToDevice, s->stream));
            CK(s, cudaStreamSynchronize(s->stream));
            size_t i = 0;
            for (auto& st : c->steps)
                if (st.type == Event::APPLY && st.apply.tci) st.apply.dev_wi8 = c->wi8 + offs[i++];
        }
    }
    // one H2D upload of all k = 6 matrices (smaller ones travel as kernel params)
    if (n6) {
        cudaError_t e = cudaMalloc(&c->dev_mats, n6 * 64 * 64 * sizeof(float2));
        if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(fused matrices)");
        std::vector<float2> host(n6 * 64 * 64);
        size_t i6 = 0;
        for (auto& st : c->steps)
            if (st.type == Event::APPLY && st.apply.k == 6) {
                std::memcpy(&host[i6 * 4096], st.apply.m.data(), 4096 * sizeof(float2));
                st.apply.dev_m = c->dev_mats + i6 * 4096;
                ++i6;
            }
        CK(s, cudaMemcpyAsync(c->dev_mats, host.data(), host.size() * sizeof(float2), cudaMemcpyHostToDevice,
                              s->stream));
        CK(s, cudaStreamSynchronize(s->stream));
    }
    if (s->g == 0 && s->n <= kSmallCircuitMaxQubits && !s->fp64) {
        std::vector<SmallGateDesc> gd;
        std::vector<float2> mats;
        for (auto& st : c->steps) {
            SmallGateDesc g{};
            g.k = st.apply.k;
            for (int b = 0; b < g.k; ++b) g.q[b] = st.apply.q[b];
            g.mat_off = (uint32_t)mats.size();
            for (const cf& m : st.apply.m) mats.push_back(make_float2(m.real(), m.imag()));
            gd.push_back(g);
        }
        c->n_small = (int)gd.size();
        if (c->n_small > 0) {
            cudaError_t e = cudaMalloc(&c->small_gates, gd.size() * sizeof(SmallGateDesc));
            if (e == cudaSuccess) e = cudaMalloc(&c->small_mats, mats.size() * sizeof(float2));
            if (e != cudaSuccess) return fail(SV_ENOMEM, "cudaMalloc(small circuit)");
            CK(s, cudaMemcpyAsync(c->small_gates, gd.data(), gd.size() * sizeof(SmallGateDesc), cudaMemcpyHostToDevice,
                                  s->stream));
            CK(s, cudaMemcpyAsync(c->small_mats, mats.data(), mats.size() * sizeof(float2), cudaMemcpyHostToDevice,
                                  s->stream));
            CK(s, cudaStreamSynchronize(s->stream));
        }
        c->small = true;
    }
    c->stats.t_upload_s = now_s() - t2;
    *out = c.release();
    return SV_OK;
}

int sv_circuit_run_device(sv_state* s, const sv_circuit* c) {
    int rc = check_state(s);
    if (rc) return rc;
    if (!c || c->owner != s) return fail(SV_EINVAL, "circuit is NULL or belongs to another state");
    if (s->pos != c->pos_in) return fail(SV_EINVAL, "state qubit map differs from the circuit's (sv_reset first)");
    if (c->zero_only && !s->zero_pending) return fail(SV_EINVAL, "circuit was built for a run from |0...0> only");
    Nvtx nv("sv.circuit_run");
    s->bins_valid = false;
    s->pass_bytes.clear();
    s->pass_fma.clear();
    const sv_stats keep = c->stats;
    reset_stats(s);
    s->stats.t_fuse_s = keep.t_fuse_s;
    s->stats.t_plan_s = keep.t_plan_s;
    s->stats.t_upload_s = keep.t_upload_s;
    s->stats.n_fused = keep.n_fused;
    for (int k = 0; k < 7; ++k) s->stats.fused_hist[k] = keep.fused_hist[k];
    // a pending |0...0> is synthesised inside the first pass when the circuit
    // starts with a register-blocked pass (no reset write, no first-pass read)
    bool zinit = false;
    // a run from a pending |0...0> takes the product-state step list when
    // the circuit has one (first gates folded into the first pass)
    const bool use_z = s->zero_pending && !c->steps_z.empty();
    const std::vector<sv_circuit::Step>& steps = use_z ? c->steps_z : c->steps;
    if (s->zero_pending) {
        zinit = !c->small && !steps.empty() && steps[0].block && rpass_supported(steps[0].pass) &&
                (!s->fp64 || !steps[0].jitz.empty());
        if (zinit) {
            s->zero_pending = false;
        } else {
            rc = materialize(s);
            if (rc) return rc;
        }
    }
    if (c->small) {
        if (c->n_small > 0) {
            rc = launch(s, LaunchClass::HIGH, [&] {
                return launch_small_circuit(s->shard[0], s->n, c->n_small, c->small_gates, c->small_mats, s->stream);
            });
            if (rc) return rc;
            for (auto& st : c->steps) {
                s->stats.bytes_apply += 16ull << s->l;
                s->stats.flops_apply += (uint64_t)((8 << st.apply.k) - 2) << s->l;
            }
        }
        s->pos = c->pos_out;
        return SV_OK;
    }
    if (c->a64) {
        for (auto& st : c->steps) {
            if (st.type == Event::EXCHANGE) {
                rc = run_exchange(s, st.exch);
            } else if (st.type == Event::PERMUTE) {
                rc = run_permute64(s, st.perm);
            } else {
                for (int i = 0; i < s->local_shards() && !rc; ++i) {
                    const int sh = s->virt ? i : s->rank;
                    rc = launch(s, LaunchClass::HIGH, [&] {
                        return launch_apply64(reinterpret_cast<double2*>(s->shard[sh]), s->l, st.a64, s->stream);
                    });
                }
                s->stats.bytes_apply += 32ull << s->l;
                s->stats.flops_apply += (uint64_t)((8 << st.a64.k) - 2) << s->l;
            }
            if (rc) return rc;
        }
        s->pos = c->pos_out;
        return SV_OK;
    }
    for (auto& st : steps) {
        if (st.block) {
            for (int sh = 0; sh < s->local_shards(); ++sh) {
                const int shard = s->virt ? sh : s->rank;
                float2* psi = s->shard[shard];
                const bool z = zinit && &st == &steps[0];
                const std::vector<RpJitLaunch>& jl = z ? st.jitz : st.jit;
                if (!jl.empty()) {
                    for (const auto& l : jl) {
                        rc = launch(s, LaunchClass::HIGH, [&] {
                            return launch_rpass_jit(psi, s->l, l, shard == 0, s->stream, sh,
                                                    st.pass.bins ? s->bins : nullptr);
                        });
                        if (rc) return rc;
                    }
                    continue;
                }
                rc = launch(s, LaunchClass::HIGH, [&] {
                    return rpass_supported(st.pass) ? launch_rpass(psi, s->l, st.pass, s->stream, z, shard == 0, sh)
                                                    : launch_pass(psi, s->l, st.pass, s->stream);
                });
                if (rc) return rc;
            }
            // algorithmic bytes: read + write, or write only when |0...0> is synthesised
            const uint64_t pass_bytes = ((zinit && &st == &steps[0]) ? 1ull : 2ull) * s->elem << s->l;
            s->stats.bytes_apply += pass_bytes;
            s->stats.bytes_apply_high += pass_bytes;
            if (!(zinit && &st == &steps[0] ? st.jitz : st.jit).empty()) s->stats.n_jit_passes += 1;
            for (auto& g : st.pass.gates) s->stats.flops_apply += (uint64_t)((8 << g.k) - 2) << s->l;
            s->stats.fma_apply += st.pass.fma_per_amp << s->l;
            s->pass_bytes.push_back(pass_bytes);
            s->pass_fma.push_back(st.pass.fma_per_amp << s->l);
            s->stats.n_passes += 1;
            s->stats.block_bits = (int)st.pass.S.size();
            continue;
        }
        if (st.type == Event::APPLY && !st.apply_shard.empty()) {
            rc = run_apply_shards(s, st.apply_shard);
        } else if (st.type == Event::APPLY) {
            rc = run_apply(s, st.apply);
        } else if (st.type == Event::EXCHANGE) {
            rc = run_exchange(s, st.exch);
        } else if (s->fp64) {
            rc = run_permute64(s, st.perm);
        } else {
            for (auto& d : st.perm_applies) {
                rc = run_apply(s, d);
                if (rc) break;
            }
        }
        if (rc) return rc;
    }
    s->pos = c->pos_out;
    // the last pass wrote the final state's sampling bins
    s->bins_valid = s->g == 0 && !s->fp64 && !steps.empty() && steps.back().block && steps.back().pass.bins &&
                    !(zinit && steps.size() == 1 ? steps.back().jitz : steps.back().jit).empty();
    return SV_OK;
}

int sv_circuit_stats(const sv_circuit* c, sv_stats* st) {
    if (!c || !st) return fail(SV_EINVAL, "NULL argument");
    *st = c->stats;
    return SV_OK;
}

int sv_circuit_destroy(sv_circuit* c) {
    if (!c) return fail(SV_EINVAL, "circuit is NULL");
    if (c->dev_mats || c->small_gates || c->small_mats || c->planes64 || c->q64 || c->wi8 || c->ptab) {
        if (c->owner && c->owner->stream) cudaStreamSynchronize(c->owner->stream);
        if (c->ptab) cudaFree(c->ptab);
        if (c->wi8) cudaFree(c->wi8);
        if (c->planes64) cudaFree(c->planes64);
        if (c->q64) cudaFree(c->q64);
        if (c->dev_mats) cudaFree(c->dev_mats);
        if (c->small_gates) cudaFree(c->small_gates);
        if (c->small_mats) cudaFree(c->small_mats);
    }
    delete c;
    return SV_OK;
}

int sv_run_circuit(sv_state* s, const sv_gate* gates, size_t n_gates, int max_fused, sv_stats* stats) {
    const double t0 = now_s();
    sv_circuit* c = nullptr;
    int rc = check_state(s);
    if (rc) return rc;
    rc = circuit_create_impl(s, gates, n_gates, max_fused, &c, s->zero_pending);
    if (rc) return rc;
    rc = sv_circuit_run_device(s, c);
    if (rc == SV_OK) rc = sync(s);
    sv_circuit_destroy(c);
    if (rc) return rc;
    s->stats.t_total_s = now_s() - t0;
    if (stats) *stats = s->stats;
    return SV_OK;
}

// ---- amplitudes ----------------------------------------------------------------
static int gather_units(sv_state* s, const std::vector<uint64_t>& loc, const std::vector<int32_t>& own, void* out_host);
// complex128 states (single shard): gather into double2, D2H
static int amplitudes64(sv_state* s, const uint64_t* idx, size_t count, sv_c128* out) {
    const uint64_t dim = 1ull << s->n;
    for (size_t i = 0; i < count; ++i)
        if (idx[i] >= dim) return fail(SV_EINVAL, "amplitude index out of range");
    int rc = materialize(s);
    if (rc) return rc;
    if (s->g > 0) {  // sharded: the two 8 B units of every amplitude
        std::vector<uint64_t> loc(2 * count);
        std::vector<int32_t> own(2 * count);
        for (size_t i = 0; i < count; ++i) {
            const uint64_t p = phys_of(s, idx[i]);
            loc[2 * i] = 2 * (p & (s->local_amps() - 1));
            loc[2 * i + 1] = loc[2 * i] + 1;
            own[2 * i] = own[2 * i + 1] = (int32_t)(p >> s->l);
        }
        return gather_units(s, loc, own, out);
    }
    rc = ensure(s, s->idx_dev, s->idx_cap, count);
    if (rc) return rc;
    rc = ensure(s, s->amp_dev, s->amp_cap, 2 * count);
    if (rc) return rc;
    CK(s, cudaMemcpyAsync(s->idx_dev, idx, count * 8, cudaMemcpyHostToDevice, s->stream));
    rc = launch(s, LaunchClass::OTHER, [&] {
        return launch_gather64(reinterpret_cast<const double2*>(s->shard[0]), s->idx_dev, count,
                               reinterpret_cast<double2*>(s->amp_dev), s->stream);
    });
    if (rc) return rc;
    CK(s, cudaMemcpyAsync(out, s->amp_dev, count * 16, cudaMemcpyDeviceToHost, s->stream));
    return sync(s);
}

int sv_amplitudes_c128(sv_state* s, const uint64_t* idx, size_t count, sv_c128* out) {
    int rc = check_state(s);
    if (rc) return rc;
    if (count == 0) return SV_OK;
    if (!idx || !out) return fail(SV_EINVAL, "idx/out is NULL");
    if (s->fp64) return amplitudes64(s, idx, count, out);
    std::vector<sv_c64> tmp(count);
    rc = sv_amplitudes(s, idx, count, tmp.data());
    if (rc) return rc;
    for (size_t i = 0; i < count; ++i) out[i] = sv_c128{tmp[i].re, tmp[i].im};
    return SV_OK;
}

int sv_amplitudes(sv_state* s, const uint64_t* idx, size_t count, sv_c64* out) {
    int rc = check_state(s);
    if (rc) return rc;
    if (count == 0) return SV_OK;
    if (!idx || !out) return fail(SV_EINVAL, "idx/out is NULL");
    if (s->fp64) {
        std::vector<sv_c128> tmp(count);
        rc = amplitudes64(s, idx, count, tmp.data());
        if (rc) return rc;
        for (size_t i = 0; i < count; ++i) out[i] = sv_c64{(float)tmp[i].re, (float)tmp[i].im};
        return SV_OK;
    }
    const uint64_t dim = 1ull << s->n;
    std::vector<uint64_t> loc(count);
    std::vector<int32_t> own(count);
    for (size_t i = 0; i < count; ++i) {
        if (idx[i] >= dim) return fail(SV_EINVAL, "amplitude index out of range");
        const uint64_t p = phys_of(s, idx[i]);
        loc[i] = p & (s->local_amps() - 1);
        own[i] = (int32_t)(p >> s->l);
    }
    rc = materialize(s);
    if (rc) return rc;
    return gather_units(s, loc, own, out);
}

// Gather 8 B units (unit loc[i] of shard own[i]) of a sharded state into
// host memory (virtual shards: every shard's kernel writes its own units;
// multi-process: through the xfer areas, min-merged over ~0 fills)
static int gather_units(sv_state* s, const std::vector<uint64_t>& loc, const std::vector<int32_t>& own, void* out_host) {
    int rc = SV_OK;
    const size_t count = loc.size();
    char* out = (char*)out_host;
    const size_t chunk = s->virt ? count : std::min<size_t>(count, kXferBytes / 8);
    for (size_t o = 0; o < count; o += chunk) {
        const size_t cnt = std::min(chunk, count - o);
        rc = ensure(s, s->idx_dev, s->idx_cap, 2 * cnt);
        if (rc) return rc;
        rc = ensure(s, s->amp_dev, s->amp_cap, cnt);
        if (rc) return rc;
        CK(s, cudaMemcpyAsync(s->idx_dev, loc.data() + o, cnt * 8, cudaMemcpyHostToDevice, s->stream));
        int32_t* own_dev = reinterpret_cast<int32_t*>(s->idx_dev + cnt);
        CK(s, cudaMemcpyAsync(own_dev, own.data() + o, cnt * 4, cudaMemcpyHostToDevice, s->stream));
        if (s->virt) {
            for (int d = 0; d < s->world; ++d) {
                rc = launch(s, LaunchClass::OTHER, [&] {
                    return launch_gather(s->shard[d], s->idx_dev, s->world > 1 ? own_dev : nullptr, d, cnt,
                                         s->amp_dev, s->stream);
                });
                if (rc) return rc;
            }
        } else {
            // owner writes into its xfer area; everyone merges (min over ~0-filled areas)
            CK(s, cudaMemsetAsync(s->xfer, 0xff, cnt * 8, s->stream));
            rc = launch(s, LaunchClass::OTHER, [&] {
                return launch_gather(s->shard[s->rank], s->idx_dev, own_dev, s->rank, cnt,
                                     reinterpret_cast<float2*>(s->xfer), s->stream);
            });
            if (rc) return rc;
            rc = barrier(s);
            if (rc) return rc;
            rc = launch(s, LaunchClass::OTHER, [&] {
                return launch_merge_min(s->xfer_dev, s->world, cnt, reinterpret_cast<uint64_t*>(s->amp_dev),
                                        s->stream);
            });
            if (rc) return rc;
            rc = barrier(s);
            if (rc) return rc;
        }
        CK(s, cudaMemcpyAsync(out + 8 * o, s->amp_dev, cnt * 8, cudaMemcpyDeviceToHost, s->stream));
        rc = sync(s);
        if (rc) return rc;
    }
    return SV_OK;
}

// ---- sampling --------------------------------------------------------------------
constexpr size_t kMiscStatus = 200;  // s->misc slot of the sampling status word

// Synchronise and report the status word of the last sampling call:
// SV_EINVAL if its total weight was zero or >= 3.99 * 2^62.
static int sample_status(sv_state* s) {
    uint64_t st = 0;
    if (s->sample_pending) CK(s, cudaMemcpyAsync(&st, s->misc + kMiscStatus, 8, cudaMemcpyDeviceToHost, s->stream));
    int rc = sync(s);
    if (rc) return rc;
    s->sample_pending = false;
    if (st == 1) return fail(SV_EINVAL, "state has zero total weight (no samples drawn)");
    if (st == 2) return fail(SV_EINVAL, "sum |c|^2 >= 3.99 (uint64 overflow risk; no samples drawn)");
    return SV_OK;
}
static int sample_impl(sv_state* s, uint64_t seed, size_t N, uint64_t* dev_out) {
    Nvtx nv("sv.sample");
    {
        const int rz = materialize(s);
        if (rz) return rz;
    }
    int rc = canonicalize(s);
    if (rc) return rc;
    const uint64_t La = s->local_amps();
    const uint64_t nb = (La + (1u << kSampleBinBits) - 1) >> kSampleBinBits;
    const int nloc = s->local_shards();
    // per local shard: bin weights + inclusive scan
    for (int i = 0; i < nloc; ++i) {
        const int d = s->virt ? i : s->rank;
        uint64_t* bins = s->bins + (size_t)i * nb;
        if (!s->bins_valid) {  // else the circuit's last pass wrote them
            rc = launch(s, LaunchClass::OTHER,
                        [&] { return launch_bin_weights(s->shard[d], s->fp64, La, bins, s->stream); });
            if (rc) return rc;
        }
        rc = launch(s, LaunchClass::OTHER, [&] { return launch_inclusive_scan(bins, nb, s->scan_scratch, s->stream); });
        if (rc) return rc;
    }
    s->bins_valid = false;  // the scan ran in place: the weights are consumed
    // totals pointers (shard d's total = last element of its prefix) and sigma
    std::vector<const uint64_t*> tp(s->world);
    std::vector<int32_t> sig(s->world);
    for (int d = 0; d < s->world; ++d) sig[d] = sigma_of(s, d);
    if (s->virt) {
        for (int d = 0; d < s->world; ++d) tp[d] = s->bins + (size_t)d * nb + (nb - 1);
    } else {
        CK(s, cudaMemcpyAsync(&s->ctrl->total, s->bins + (nb - 1), 8, cudaMemcpyDeviceToDevice, s->stream));
        rc = barrier(s);
        if (rc) return rc;
        for (int d = 0; d < s->world; ++d) tp[d] = &s->peer_ctrl[d]->total;
    }
    CK(s, cudaMemcpyAsync(s->totals_ptr_dev, tp.data(), sizeof(void*) * s->world, cudaMemcpyHostToDevice, s->stream));
    CK(s, cudaMemcpyAsync(s->sigma_dev, sig.data(), sizeof(int32_t) * s->world, cudaMemcpyHostToDevice, s->stream));
    uint64_t* lo = s->misc;
    uint64_t* total = s->misc + 64;
    rc = launch(s, LaunchClass::OTHER, [&] {
        return launch_shard_offsets(s->totals_ptr_dev, s->sigma_dev, s->world, lo, total, s->stream);
    });
    if (rc) return rc;
    // the total weight is checked on the device (sample_resolve_kernel): no
    // host round trip; an invalid total sets the status word
    uint64_t* status = s->misc + kMiscStatus;
    CK(s, cudaMemsetAsync(status, 0, 8, s->stream));
    s->sample_pending = true;
    if (s->virt) {
        for (int d = 0; d < s->world; ++d) {
            const uint64_t base = (uint64_t)sig[d] << s->l;
            rc = launch(s, LaunchClass::OTHER, [&] {
                return launch_sample_resolve(s->shard[d], s->fp64, La, s->bins + (size_t)d * nb, nb, lo + d, total, seed, N,
                                             base, dev_out, status, s->stream);
            });
            if (rc) return rc;
        }
    } else {
        const size_t chunk = kXferBytes / 8;
        for (size_t o = 0; o < N; o += chunk) {
            const size_t cnt = std::min(chunk, N - o);
            CK(s, cudaMemsetAsync(s->xfer, 0xff, cnt * 8, s->stream));
            const uint64_t base = (uint64_t)sig[s->rank] << s->l;
            // resolve samples o..o+cnt: shift the counter by o through the seed stream
            rc = launch(s, LaunchClass::OTHER, [&] {
                return launch_sample_resolve(s->shard[s->rank], s->fp64, La, s->bins, nb, lo + s->rank, total,
                                             seed + (uint64_t)o * 0x9E3779B97F4A7C15ull, cnt, base, s->xfer, status,
                                             s->stream);
            });
            if (rc) return rc;
            rc = barrier(s);
            if (rc) return rc;
            rc = launch(s, LaunchClass::OTHER,
                        [&] { return launch_merge_min(s->xfer_dev, s->world, cnt, dev_out + o, s->stream); });
            if (rc) return rc;
            rc = barrier(s);
            if (rc) return rc;
        }
    }
    return SV_OK;
}

int sv_sample_device(sv_state* s, uint64_t seed, size_t n_samples, uint64_t* dev_out) {
    int rc = check_state(s);
    if (rc) return rc;
    if (n_samples == 0) return SV_OK;
    if (!dev_out) return fail(SV_EINVAL, "dev_out is NULL");
    return sample_impl(s, seed, n_samples, dev_out);
}

int sv_sample(sv_state* s, uint64_t seed, size_t n_samples, uint64_t* out) {
    int rc = check_state(s);
    if (rc) return rc;
    if (n_samples == 0) return SV_OK;
    if (!out) return fail(SV_EINVAL, "out is NULL");
    rc = ensure(s, s->samp_dev, s->samp_cap, n_samples);
    if (rc) return rc;
    rc = sample_impl(s, seed, n_samples, s->samp_dev);
    if (rc) return rc;
    CK(s, cudaMemcpyAsync(out, s->samp_dev, n_samples * 8, cudaMemcpyDeviceToHost, s->stream));
    return sample_status(s);
}

// ---- whole state ------------------------------------------------------------------
static int set_state_bytes(sv_state* s, const void* host) {
    s->zero_pending = false;  // every amplitude is overwritten
    s->bins_valid = false;
    for (int q = 0; q < s->n; ++q) s->pos[q] = q;
    const size_t sb = s->elem << s->l;
    for (int i = 0; i < s->local_shards(); ++i) {
        const int d = s->virt ? i : s->rank;
        CK(s, cudaMemcpyAsync(s->shard[d], (const char*)host + sb * d, sb, cudaMemcpyHostToDevice, s->stream));
    }
    int rc = sync(s);
    if (rc) return rc;
    return barrier(s) ? fail(SV_ECOMM, "barrier failed") : sync(s);
}

int sv_set_state(sv_state* s, const sv_c64* host, size_t count) {
    int rc = check_state(s);
    if (rc) return rc;
    if (count != (1ull << s->n) || !host) return fail(SV_EINVAL, "count must be 2^n and host non-NULL");
    if (!s->fp64) return set_state_bytes(s, host);
    std::vector<sv_c128> up(count);
    for (size_t i = 0; i < count; ++i) up[i] = sv_c128{host[i].re, host[i].im};
    return set_state_bytes(s, up.data());
}

int sv_set_state_c128(sv_state* s, const sv_c128* host, size_t count) {
    int rc = check_state(s);
    if (rc) return rc;
    if (count != (1ull << s->n) || !host) return fail(SV_EINVAL, "count must be 2^n and host non-NULL");
    if (s->fp64) return set_state_bytes(s, host);
    std::vector<sv_c64> dn(count);
    for (size_t i = 0; i < count; ++i) dn[i] = sv_c64{(float)host[i].re, (float)host[i].im};
    return set_state_bytes(s, dn.data());
}

static int get_state_bytes(sv_state* s, void* host) {
    {
        const int rz = materialize(s);
        if (rz) return rz;
    }
    int rc = canonicalize(s);
    if (rc) return rc;
    rc = barrier(s);
    if (rc) return rc;
    rc = sync(s);
    if (rc) return rc;
    const size_t sb = s->elem << s->l;
    for (int d = 0; d < s->world; ++d) {
        const int sg = sigma_of(s, d);
        CK(s, cudaMemcpyAsync((char*)host + sb * sg, s->shard[d], sb, cudaMemcpyDeviceToHost, s->stream));
    }
    rc = sync(s);
    if (rc) return rc;
    rc = barrier(s);
    if (rc) return rc;
    return sync(s);
}

int sv_get_state(sv_state* s, sv_c64* host, size_t count) {
    int rc = check_state(s);
    if (rc) return rc;
    if (count != (1ull << s->n) || !host) return fail(SV_EINVAL, "count must be 2^n and host non-NULL");
    if (!s->fp64) return get_state_bytes(s, host);
    std::vector<sv_c128> full(count);
    rc = get_state_bytes(s, full.data());
    if (rc) return rc;
    for (size_t i = 0; i < count; ++i) host[i] = sv_c64{(float)full[i].re, (float)full[i].im};
    return SV_OK;
}

int sv_get_state_c128(sv_state* s, sv_c128* host, size_t count) {
    int rc = check_state(s);
    if (rc) return rc;
    if (count != (1ull << s->n) || !host) return fail(SV_EINVAL, "count must be 2^n and host non-NULL");
    if (s->fp64) return get_state_bytes(s, host);
    std::vector<sv_c64> low(count);
    rc = get_state_bytes(s, low.data());
    if (rc) return rc;
    for (size_t i = 0; i < count; ++i) host[i] = sv_c128{low[i].re, low[i].im};
    return SV_OK;
}

int sv_device_ptr(sv_state* s, int shard, void** out) {
    int rc = check_state(s);
    if (rc) return rc;
    if (!out) return fail(SV_EINVAL, "NULL argument");
    if (shard < 0 || shard >= s->world || !s->shard[shard]) return fail(SV_EINVAL, "shard not available here");
    if (!s->virt && shard != s->rank) return fail(SV_EINVAL, "multi-process mode: only this rank's shard");
    s->bins_valid = false;  // the caller may write the memory
    if (s->zero_pending) {  // the caller may read the memory: write |0...0> now
        int rc = materialize(s);
        if (rc == SV_OK) rc = sync(s);
        if (rc) return rc;
    }
    *out = s->shard[shard];
    return SV_OK;
}

int sv_qubit_map(const sv_state* s, int32_t* pos) {
    if (!s || !pos) return fail(SV_EINVAL, "NULL argument");
    for (int q = 0; q < s->n; ++q) pos[q] = s->pos[q];
    return SV_OK;
}

// ---- multi-process plumbing -------------------------------------------------------
struct IpcBlob {
    int32_t magic, rank, world, l;
    cudaIpcMemHandle_t state, ctrl, xfer;
};

int sv_ipc_handle(sv_state* s, void* out, size_t cap, size_t* need) {
    if (!s || !need) return fail(SV_EINVAL, "NULL argument");
    *need = sizeof(IpcBlob);
    if (s->virt) return fail(SV_EINVAL, "not a multi-process sharded state");
    if (cap < sizeof(IpcBlob) || !out) return fail(SV_EINVAL, "cap too small");
    IpcBlob b{};
    b.magic = 0x53564232;
    b.rank = s->rank;
    b.world = s->world;
    b.l = s->l;
    CK(s, cudaIpcGetMemHandle(&b.state, s->alloc));
    CK(s, cudaIpcGetMemHandle(&b.ctrl, s->ctrl));
    CK(s, cudaIpcGetMemHandle(&b.xfer, s->xfer));
    std::memcpy(out, &b, sizeof(b));
    return SV_OK;
}

int sv_attach_peers(sv_state* s, const void* handles, size_t each) {
    int rc = check_state(s);
    if (rc) return rc;
    if (s->virt) return fail(SV_EINVAL, "not a multi-process sharded state");
    if (!handles || each < sizeof(IpcBlob)) return fail(SV_EINVAL, "bad handle blobs");
    s->peer_ctrl.assign(s->world, nullptr);
    s->peer_xfer.assign(s->world, nullptr);
    for (int r = 0; r < s->world; ++r) {
        IpcBlob b;
        std::memcpy(&b, (const char*)handles + each * r, sizeof(b));
        if (b.magic != 0x53564232 || b.rank != r || b.world != s->world || b.l != s->l)
            return fail(SV_ECOMM, "peer handle blob mismatch");
        if (r == s->rank) {
            s->peer_ctrl[r] = s->ctrl;
            s->peer_xfer[r] = s->xfer;
            continue;
        }
        void* p = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, b.state, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) return fail(SV_ECOMM, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
        s->ipc_opened.push_back(p);
        s->shard[r] = (float2*)p;
        e = cudaIpcOpenMemHandle(&p, b.ctrl, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) return fail(SV_ECOMM, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
        s->ipc_opened.push_back(p);
        s->peer_ctrl[r] = (Ctrl*)p;
        e = cudaIpcOpenMemHandle(&p, b.xfer, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) return fail(SV_ECOMM, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
        s->ipc_opened.push_back(p);
        s->peer_xfer[r] = (uint64_t*)p;
    }
    std::vector<uint64_t*> fl(s->world);
    for (int r = 0; r < s->world; ++r) fl[r] = s->peer_ctrl[r]->flags;
    CK(s, cudaMemcpy(s->flags_dev, fl.data(), sizeof(void*) * s->world, cudaMemcpyHostToDevice));
    CK(s, cudaMemcpy(s->xfer_dev, s->peer_xfer.data(), sizeof(void*) * s->world, cudaMemcpyHostToDevice));
    rc = upload_shard_table(s);
    if (rc) return rc;
    s->attached = true;
    rc = barrier(s);
    if (rc) return rc;
    return sync(s);
}

int sv_set_blocking(sv_state* s, int tile_bits) {
    if (!s) return fail(SV_EINVAL, "state handle is NULL");
    if (tile_bits != 0 && tile_bits != -1 && (tile_bits < 10 || tile_bits > 14))
        return fail(SV_EINVAL, "tile_bits must be 0 (off), -1 (auto) or in [10, 14]");
    s->block_bits = tile_bits;
    return SV_OK;
}

int sv_set_option(sv_state* s, int option, int value) {
    if (!s) return fail(SV_EINVAL, "state handle is NULL");
    switch (option) {
        case SV_OPT_BLOCK_BITS: return sv_set_blocking(s, value);
        case SV_OPT_PASS_JIT:
            if (value != 0 && value != 1) return fail(SV_EINVAL, "SV_OPT_PASS_JIT takes 0 or 1");
            s->pass_jit = value;
            return SV_OK;
        case SV_OPT_APPLY_PATH:
            if (value != SV_PATH_AUTO && value != SV_PATH_SIMT && value != SV_PATH_INT8)
                return fail(SV_EINVAL, "SV_OPT_APPLY_PATH takes SV_PATH_AUTO, SV_PATH_SIMT or SV_PATH_INT8");
            s->tc_mode = value == SV_PATH_AUTO ? 3 : value == SV_PATH_INT8 ? 2 : 0;
            return SV_OK;
        case SV_OPT_TIMING: return sv_set_timing(s, value);
        case SV_OPT_PASS_PIN:
            if (value < 3 || value > 5) return fail(SV_EINVAL, "SV_OPT_PASS_PIN takes 3, 4 or 5");
            s->pass_pin = value;
            return SV_OK;
        case SV_OPT_DIAG_SKIP:
            if (value != 0 && value != 1) return fail(SV_EINVAL, "SV_OPT_DIAG_SKIP takes 0 or 1");
            s->diag_skip = value;
            return SV_OK;
        case SV_OPT_PASS_SEARCH:
            if (value < 1 || value > 8) return fail(SV_EINVAL, "SV_OPT_PASS_SEARCH takes 1..8");
            s->pass_beam = value;
            return SV_OK;
        case SV_OPT_PASS_SPEC:
            if (value != 0 && value != 1) return fail(SV_EINVAL, "SV_OPT_PASS_SPEC takes 0 or 1");
            s->pass_spec = value;
            return SV_OK;
        default: return fail(SV_EINVAL, "unknown option");
    }
}

int sv_pass_kernels(const sv_gate* gates, size_t n_gates, int max_fused, int tile_bits, int compile, char* buf,
                    size_t cap, size_t* need) {
    if (!need) return fail(SV_EINVAL, "need is NULL");
    if (max_fused < 1 || max_fused > 2) return fail(SV_EINVAL, "max_fused must be in [1, 2] for register-blocked passes");
    const bool wide = tile_bits < 0;  // complex128 kernels
    if (wide) tile_bits = -tile_bits;
    if (tile_bits < 10 || tile_bits > (wide ? 13 : 14))
        return fail(SV_EINVAL, "tile_bits must be in [10, 14] (complex128: -13..-10)");
    int rc = validate_gates(gates, n_gates, -1);
    if (rc) return rc;
    std::vector<FusedGate> plan;
    fuse_plan(gates, n_gates, max_fused, plan);
    int nq = 0;
    std::vector<PassIn> in;
    for (auto& f : plan) {
        build_fused_matrix(gates, f);
        PassIn pi;
        pi.k = f.k;
        for (int b = 0; b < f.k; ++b) {
            pi.q[b] = f.q[b];
            nq = std::max(nq, f.q[b] + 1);
        }
        pi.M = f.M;
        in.push_back(std::move(pi));
    }
    std::string all;
    bool first = true;
    auto passes = build_passes(tile_bits, in);
    if (!wide && !passes.empty() && rpass_supported(passes.back()) && passes.back().r >= kSampleBinBits)
        passes.back().bins = true;  // as sv_circuit_create
    for (auto& pd : passes) {
        pd.wide = wide;
        pd.spec = true;  // as sv_circuit_create with the default SV_OPT_PASS_SPEC
        if (!rpass_supported(pd)) continue;
        for (int z = 0; z < (first ? 2 : 1); ++z) {
            std::vector<RpJitLaunch> ls;
            std::vector<std::string> srcs;
            rc = rpass_jit_prepare(pd, std::max(nq, tile_bits + 2), z == 1, compile != 0, ls, &srcs);
            if (rc) return rc;
            for (auto& x : srcs) all += x + "\n//----\n";
        }
        first = false;
    }
    *need = all.size() + 1;
    if (cap == 0 && !buf) return SV_OK;
    if (cap < all.size() + 1 || !buf) return fail(SV_EINVAL, "cap too small");
    std::memcpy(buf, all.c_str(), all.size() + 1);
    return SV_OK;
}

int sv_jit_stats(uint64_t* compiled, uint64_t* cache_hits, double* compile_seconds) {
    rpass_jit_counters(compiled, cache_hits, compile_seconds);
    return SV_OK;
}

int sv_set_timing(sv_state* s, int enable) {
    if (!s) return fail(SV_EINVAL, "state handle is NULL");
    s->timing = enable != 0;
    return SV_OK;
}

int sv_last_pass_costs(const sv_state* s, uint64_t* bytes, uint64_t* fmas, size_t cap, size_t* need) {
    if (!s || !need) return fail(SV_EINVAL, "NULL argument");
    *need = s->pass_bytes.size();
    if (cap < *need) return fail(SV_EINVAL, "cap too small");
    if (*need && (!bytes || !fmas)) return fail(SV_EINVAL, "bytes/fmas is NULL");
    for (size_t i = 0; i < *need; ++i) {
        bytes[i] = s->pass_bytes[i];
        fmas[i] = s->pass_fma[i];
    }
    return SV_OK;
}

int sv_last_stats(const sv_state* s_, sv_stats* out) {
    sv_state* s = const_cast<sv_state*>(s_);
    if (!s || !out) return fail(SV_EINVAL, "NULL argument");
    if (s->timing && !s->recs.empty()) {
        int rc = sync(s);
        if (rc) return rc;
    }
    *out = s->stats;
    return SV_OK;
}

int sv_synchronize(sv_state* s) {
    if (!s) return fail(SV_EINVAL, "state handle is NULL");
    return sample_status(s);
}

}  // extern "C"
