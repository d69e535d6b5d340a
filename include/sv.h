/*
 * sv.h -- C ABI of the B200 state-vector hot path (libsvb200.so).
 *
 * What the library computes (citations: /root/reference/PAPER.md line Lnnn):
 *   - a state of n qubits is 2^n complex amplitudes; |c_i|^2 is the
 *     probability of |i> (L69, §2.2);
 *   - a gate G acts as psi' = G psi, applied matrix-free and in place
 *     (L71-93, §2.2, Figs. 3-4); the 2^n outputs split into 2^(n-k)
 *     independent groups of a 2^k x 2^k complex matvec (L93);
 *   - gates are fused in space (tensor product) and time (ordered matrix
 *     product) up to a "maximum of fused gates" (L98-104, Fig. 5);
 *   - gates on high qubits and on low qubits run in different kernels
 *     (L110-112, §2.3);
 *   - amplitudes can be read and measurement outcomes sampled (L131-132, §3);
 *   - several fused gates can share one pass over the state (cache blocking,
 *     related work [12], L221): the default for max_fused <= 2
 *     (sv_set_blocking, sv_block_plan).
 *
 * Conventions (SURVEY.md §8c readings Q1/Q3):
 *   - qubit q is bit q of the basis index (little-endian, qubit 0 = stride 1);
 *   - amplitudes are interleaved complex64 (sv_c64 == cuFloatComplex ==
 *     torch.complex64), fp32 arithmetic on the device;
 *   - a k-qubit matrix is row-major 2^k x 2^k; bit b of its row/column index
 *     belongs to qubits[b]; qubits[] may be in any order.
 *
 * Errors: every call returns int; SV_OK = 0, negative = error.  Nothing
 * throws or exits.  sv_last_error() returns a thread-local message for the
 * last failing call on this thread.  Arguments are validated before any side
 * effect.  After a failed asynchronous device operation a handle is sticky
 * SV_EBADSTATE until sv_destroy().
 *
 * Ownership: every input array is caller-owned and fully consumed (copied)
 * before the call returns; the library keeps no caller pointers except a
 * caller-provided device buffer (sv_config.dev_buf), which the caller must
 * keep alive until sv_destroy().  Output arrays are caller-allocated host
 * memory.
 *
 * Streams / sync: all device work of a handle runs on its stream (its own, or
 * sv_config.cuda_stream).  sv_apply_fused and sv_circuit_run_device are
 * asynchronous w.r.t. the host; sv_run_circuit, sv_amplitudes, sv_sample and
 * sv_get_state synchronise the stream before returning.
 *
 * Threading: a handle is not thread-safe; distinct handles are independent.
 *
 * Sharded mode (north star; PAPER.md L209/L229 name multi-GPU as future
 * work): the 2^n state is split into P = 2^g shards of 2^(n-g) amplitudes by
 * the top g PHYSICAL qubits.  Either all P shards live on this GPU
 * (virtual_shards = 1, used to test the exchange path on one device) or each
 * of P processes owns one shard and the processes exchange peer-memory
 * handles with sv_ipc_handle / sv_attach_peers (one GPU per process, NVLink
 * P2P).  In multi-process mode every rank makes the same calls with the same
 * arguments (collective semantics) and receives identical results.
 */
#ifndef SV_B200_H
#define SV_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SV_OK 0
#define SV_EINVAL (-1)        /* bad argument (range, NULL with count>0, dup qubit, ...) */
#define SV_ENOMEM (-2)        /* device or host allocation failed                          */
#define SV_ECUDA (-3)         /* CUDA runtime error (message in sv_last_error)            */
#define SV_ECOMM (-4)         /* peer attach / P2P error in sharded mode                   */
#define SV_EUNSUPPORTED (-5)  /* world not a power of two, shard too small, ...          */
#define SV_EBADSTATE (-6)     /* handle poisoned by an earlier asynchronous failure        */

#define SV_MAX_QUBITS 40      /* per handle (all shards) */
#define SV_MAX_FUSED 6        /* k <= 6: dense 64 x 64 fused matrices */

typedef struct sv_state sv_state;       /* opaque: device state + qubit map */
typedef struct sv_circuit sv_circuit;   /* opaque: fused, planned and uploaded circuit */

typedef struct { float re, im; } sv_c64;
typedef struct { double re, im; } sv_c128;

/* One input gate (1 or 2 qubits).  m is row-major 2^nq x 2^nq (a 1-qubit gate
 * uses m[0..3]); bit b of the matrix index <-> q[b].  fp64 so that fusion
 * (in fp64) rounds to complex64 once per fused gate. */
typedef struct {
    int32_t nq;
    int32_t q[2];
    int32_t pad_;
    sv_c128 m[16];
} sv_gate;

/* Statistics of the last sv_run_circuit / sv_circuit_run_device.  (SURVEY.md
 * §8b proposed a smaller struct; this one adds launch counts per kernel class,
 * device-side times, the blocked-pass and FMA counters and a byte split by
 * class -- every §8b field keeps its meaning.)  Host times
 * are wall-clock; t_apply_*_dev / t_exchange_dev / t_sample_dev are summed
 * CUDA-event durations around each launch and are filled only when timing is
 * enabled with sv_set_timing(s, 1).  Bytes are ALGORITHMIC: 16 B per
 * amplitude per apply pass, sent bytes per exchange. */
typedef struct {
    int32_t n_fused;            /* fused gates in the plan                       */
    int32_t n_exchanges;        /* exchange events (sharded)                     */
    int32_t fused_hist[7];      /* fused gates by size k = 0..6                  */
    int32_t n_launch_high;      /* high-qubit apply launches                     */
    int32_t n_launch_low;       /* low/mixed-qubit apply launches                */
    int32_t n_launch_other;     /* reset / permute / exchange / sample launches  */
    double t_fuse_s, t_plan_s, t_upload_s, t_total_s;
    double t_apply_high_dev_s, t_apply_low_dev_s, t_exchange_dev_s, t_other_dev_s;
    uint64_t bytes_apply;       /* per shard */
    uint64_t bytes_exchange;    /* sent per shard */
    uint64_t flops_apply;       /* (8*2^k - 2) per amplitude per fused gate, per shard */
    int32_t n_passes;           /* cache-blocked passes (0: one launch per fused gate) */
    int32_t block_bits;         /* tile qubits of the blocked passes (0: not blocked)  */
    uint64_t fma_apply;         /* fp32 FMAs the register-blocked passes execute (dense
                                   2^k x 2^k: 4*2^k per amplitude, diagonal: 4, CZ: 0),
                                   per shard; 0 for other kernels                       */
    uint64_t bytes_apply_high;  /* bytes_apply split by kernel class: high-qubit kernels  */
    uint64_t bytes_apply_low;   /*   (incl. all blocked passes) / low-qubit kernels       */
    int32_t n_jit_passes;       /* blocked passes run by pass-specialised kernels          */
    int32_t reserved2_;
} sv_stats;

typedef struct {
    int32_t n_qubits;        /* total qubits n, 1..SV_MAX_QUBITS                          */
    int32_t world;           /* P = number of shards (power of two); 0 or 1 = unsharded   */
    int32_t rank;            /* this process's shard in multi-process mode, else 0        */
    int32_t virtual_shards;  /* 1: all P shards on this GPU (single process)              */
    int32_t exchange_vmin;   /* planner victim floor (S4); < 0 = default 5                */
    int32_t device;          /* CUDA device ordinal; < 0 = current device                 */
    void* dev_buf;           /* optional caller-owned device buffer for the state, or NULL */
    size_t buf_bytes;        /* size of dev_buf: >= 8 * 2^n / (world if multi-process)    */
    void* cuda_stream;       /* optional cudaStream_t; NULL = library-owned stream        */
    int32_t precision;       /* 0: complex64 (fp32, default); 1: complex128 (fp64, NEXT-1;
                                PAPER.md L191 Fig. 8) -- sharded as complex64, fused k <= 6 */
    int32_t reserved_;
} sv_config;

/* ---- lifetime ------------------------------------------------------------- */
/* 1 GPU (current device), state = |0...0>.  n in [1, SV_MAX_QUBITS]. */
int sv_create(int n_qubits, sv_state** out);
/* General form (sharded / caller-owned buffer / caller stream). */
int sv_create_ex(const sv_config* cfg, sv_state** out);
int sv_destroy(sv_state* s);
/* |0...0> and the identity qubit map. Asynchronous.  On complex64 states in
 * library-owned memory the write is deferred: a circuit that starts with a
 * register-blocked pass builds the zero tiles itself (no extra pass over
 * HBM); every other call that reads or writes the state (or sv_device_ptr)
 * writes |0...0> first.  States in a caller-owned buffer (sv_config.dev_buf)
 * and complex128 states are written immediately (stream-ordered). */
int sv_reset(sv_state* s);

/* ---- the hot path ----------------------------------------------------------- */
/* Apply one dense k-qubit matrix (1 <= k <= 6) in place.  qubits distinct and
 * < n in any order; matrix row-major 2^k x 2^k complex64, bit b <-> qubits[b]
 * (logical qubits: in sharded mode an exchange is inserted when needed).
 * Asynchronous: matrices that do not travel as kernel parameters (k = 6,
 * int8 tensor-core slices, complex128 planes) are copied into a pinned
 * staging ring before return; the call blocks only when the GPU is more than
 * 8 such applies behind. */
int sv_apply_fused(sv_state* s, int k, const int32_t* qubits, const sv_c64* matrix);

/* Controlled gate (qsim ApplyControlledGate; SURVEY.md
 * NEXT-4): the k-qubit matrix acts on targets[] only where every one of the
 * n_ctrl control qubits is 1 (0 <= n_ctrl <= 6, all qubits distinct).  On
 * unsharded complex64 states with no control on qubit 0 only the
 * control-1 subspace (2^-n_ctrl of the state) is read and written; otherwise
 * the block matrix over targets ++ controls is applied (k + n_ctrl <= 6). */
int sv_apply_controlled(sv_state* s, int n_ctrl, const int32_t* controls, int k, const int32_t* targets,
                        const sv_c64* matrix);

/* Same with a complex128 matrix (no rounding on complex128 states; rounded to
 * complex64 on complex64 states). */
int sv_apply_fused_c128(sv_state* s, int k, const int32_t* qubits, const sv_c128* matrix);

/* Fuse (max_fused in [0,6]; 0 = no fusion), plan (sharded), upload and apply a
 * whole circuit of 1-2 qubit gates, synchronising before return.  stats may be
 * NULL. Equivalent to sv_circuit_create + sv_circuit_run + sv_circuit_destroy. */
int sv_run_circuit(sv_state* s, const sv_gate* gates, size_t n_gates, int max_fused, sv_stats* stats);

/* Prepared circuits: fusion, planning and the single H2D upload of all fused
 * matrices happen in sv_circuit_create; sv_circuit_run_device only launches
 * kernels (asynchronous; the timed "device" step of bench.py). */
int sv_circuit_create(sv_state* s, const sv_gate* gates, size_t n_gates, int max_fused, sv_circuit** out);
int sv_circuit_run_device(sv_state* s, const sv_circuit* c);
int sv_circuit_stats(const sv_circuit* c, sv_stats* stats);
int sv_circuit_destroy(sv_circuit* c);

/* Read `count` amplitudes at LOGICAL indices idx[] into out[] (host). */
int sv_amplitudes(sv_state* s, const uint64_t* idx, size_t count, sv_c64* out);

/* complex128 output (exact on complex128 states). */
int sv_amplitudes_c128(sv_state* s, const uint64_t* idx, size_t count, sv_c128* out);

/* Draw n_samples basis states (LOGICAL indices) with the integer fixed-point
 * sampler: bit-identical for a given complex64 state and
 * seed under any parallel decomposition.  SV_EINVAL if the total weight is 0
 * or sum |c|^2 >= 3.99.  out[] is host memory of n_samples uint64.  On
 * complex128 states p = fl(fl(re^2) + fl(im^2)) (reading R5). */
int sv_sample(sv_state* s, uint64_t seed, size_t n_samples, uint64_t* out);
/* Device form: writes n_samples uint64 into device memory dev_out
 * (asynchronous, no host round trip; the bench's device step).  The total
 * weight is checked on the device: if it is 0 or sum |c|^2 >= 3.99 every
 * output is UINT64_MAX (not a basis index) and the next sv_synchronize (or
 * sv_sample) on this handle returns SV_EINVAL once. */
int sv_sample_device(sv_state* s, uint64_t seed, size_t n_samples, uint64_t* dev_out);

/* ---- whole-state access (tests, debugging) ------------------------------ */
/* Copy 2^n amplitudes in LOGICAL order from host (set) / to host (get). In
 * multi-process mode each rank passes/receives the FULL vector. */
int sv_set_state(sv_state* s, const sv_c64* host, size_t count);
int sv_get_state(sv_state* s, sv_c64* host, size_t count);
/* complex128 forms (converting on complex64 states). */
int sv_set_state_c128(sv_state* s, const sv_c128* host, size_t count);
int sv_get_state_c128(sv_state* s, sv_c128* host, size_t count);
/* Device pointer of shard `shard` (virtual mode) / of this rank's shard
 * (multi-process mode: shard must equal the rank; peers' shards are not
 * handed out).  Materialises a pending |0...0> first. */
int sv_device_ptr(sv_state* s, int shard, void** out);

/* ---- pure host helpers (no GPU needed) ------------------------------------ */
/* Fusion plan as a flat int32 stream: per fused gate
 *   k, q_0..q_{k-1} (ascending), n_mem, mem_0..mem_{n_mem-1} (ascending).
 * *need gets the required length; if cap < *need returns SV_EINVAL and
 * writes nothing to buf.  (SURVEY.md §8b / §8c-S3.) */
int sv_fusion_plan(const sv_gate* gates, size_t n_gates, int max_fused, int32_t* buf, size_t cap, size_t* need);
/* Cache-blocked pass plan (pure host; reading R7, §7) of the fusion
 * plan for max_fused in [1,4] and tile_bits in [10,14], as a flat int32 stream:
 * per pass  T, S_0..S_{T-1} (tile qubits, ascending), n, f_0..f_{n-1} (fused-
 * gate indices of sv_fusion_plan, in pass order), n_phases, then per phase of
 * the register-blocked kernel (0 phases when the pass has a gate with k > 2)
 *   m, R_0..R_{m-1} (tile positions held in registers, ascending), g,
 *   j_0..j_{g-1} (indices into the pass's f list, in application order).
 * *need gets the length; cap < *need returns SV_EINVAL, writing nothing. */
int sv_block_plan(const sv_gate* gates, size_t n_gates, int max_fused, int tile_bits, int32_t* buf, size_t cap,
                  size_t* need);
/* Fused matrix of fused gate `index` of that plan, complex128 row-major over
 * the ascending qubit list (computed in fp64). out holds 4^k entries. */
int sv_fused_matrix(const sv_gate* gates, size_t n_gates, int max_fused, size_t index, sv_c128* out, size_t cap);
/* Sharded plan (S4) for fused qubit sets given as the sv_fusion_plan stream.
 * Output stream: per event  X: -1, s, P_0, p_0, ...;  A: i, k, phys_0..phys_{k-1}.
 * final_pos (n entries, may be NULL) receives logical -> physical positions. */
int sv_shard_plan(const int32_t* fusion_stream, size_t len, int n_qubits, int log2_world, int vmin,
                  int32_t* buf, size_t cap, size_t* need, int32_t* final_pos);
/* The same with the diagonal exchange skip (DESIGN.md
 * reading R10): diag[i] = mask of the logical qubits fused gate i is
 * block-diagonal in (sv_fusion_diag_masks); such a qubit, when global, does
 * not force an exchange, and APPLY events may then list global physical
 * positions (each shard runs the block its device bits select). */
int sv_shard_plan_diag(const int32_t* fusion_stream, size_t len, const uint64_t* diag, int n_qubits, int log2_world,
                       int vmin, int32_t* buf, size_t cap, size_t* need, int32_t* final_pos);
/* Pure host: per fused gate of sv_fusion_plan's plan, the mask of logical
 * qubits in which its fp64 fused matrix is block-diagonal (every entry
 * between a row and a column that differ in that qubit's bit has |entry| <=
 * 1e-10: fp64 rounding residue of exact zeros).
 * *need = number of fused gates; cap < *need -> SV_EINVAL. */
int sv_fusion_diag_masks(const sv_gate* gates, size_t n_gates, int max_fused, uint64_t* out, size_t cap, size_t* need);
/* Current logical -> physical qubit map (n entries). */
int sv_qubit_map(const sv_state* s, int32_t* pos);

/* ---- sharded multi-process plumbing --------------------------------------- */
/* Opaque bytes describing this rank's shard and control block for peers
 * (CUDA IPC handles). *need gets the size; cap < *need -> SV_EINVAL. */
int sv_ipc_handle(sv_state* s, void* out, size_t cap, size_t* need);
/* handles: world blobs of `each` bytes in rank order (from an all-gather). */
int sv_attach_peers(sv_state* s, const void* handles, size_t each);

/* ---- misc ------------------------------------------------------------------- */
/* Cache-blocked circuit execution (related work [12],
 * PAPER.md L221): sv_circuit_create on an unsharded complex64 state with
 * max_fused in [1,4] groups the fused gates into passes whose qubits all lie
 * in one set of tile_bits qubits (qubits 0..3 always included); each pass is
 * ONE HBM read + write of the state.  Passes of gates with k <= 2 run in the
 * register-blocked kernel (32 amplitudes per thread, gates applied in
 * registers); others in the shared-memory pass kernel.
 * tile_bits in [10,14]; 0 disables (one launch per fused gate); -1 (default)
 * = auto: when max_fused <= 2 and the shard has >= 20 qubits, 14 (complex64
 * with SV_OPT_PASS_JIT), 13 (generic kernel or complex128), else off.
 * 14-qubit tiles (512 threads, 128 KB of shared memory per pass CTA) exist
 * only as pass-specialised complex64 kernels: a circuit created with 14 and
 * SV_OPT_PASS_JIT 0, complex128 or max_fused > 2 uses 13.  Takes effect for
 * circuits created afterwards.  Errors: SV_EINVAL for other values. */
int sv_set_blocking(sv_state* s, int tile_bits);
/* 1: record CUDA events around every launch and fill the *_dev_s stats. */
int sv_set_timing(sv_state* s, int enable);
/* Per register-blocked pass of the most recent circuit run (per shard): the
 * algorithmic HBM bytes (16 B per amplitude; 8 B for a first pass that builds
 * its tiles) and the fp32 FMAs it executed -- the inputs of a per-pass
 * roofline floor max(bytes / HBM peak, FMAs / FMA peak).  *need = passes;
 * cap < *need -> SV_EINVAL. */
int sv_last_pass_costs(const sv_state* s, uint64_t* bytes, uint64_t* fmas, size_t cap, size_t* need);
/* Stats of the most recent run on this handle. */
int sv_last_stats(const sv_state* s, sv_stats* out);
/* Synchronise the handle's stream.  Returns SV_EINVAL (once) if an earlier
 * sv_sample_device found an invalid total weight (see there). */
int sv_synchronize(sv_state* s);

/* Per-handle execution options (replace process-wide environment switches):
 *   SV_OPT_BLOCK_BITS  = sv_set_blocking (tile qubits of the blocked passes);
 *   SV_OPT_PASS_JIT    1 (default): register-blocked passes run kernels
 *                      specialised to each pass (PTX for sm_100a, compiled in
 *                      sv_circuit_create and cached per process); 0: the
 *                      generic apply_rpass kernel.  Both give bit-identical
 *                      states when SV_OPT_PASS_SPEC is 0;
 *   SV_OPT_APPLY_PATH  dense fused gates of one launch each:
 *                      SV_PATH_AUTO (default: k = 5, 6 on the exact int8
 *                      tensor-core path, k <= 4 SIMT), SV_PATH_SIMT,
 *                      SV_PATH_INT8 (int8 tensor cores for k = 4..6);
 *   SV_OPT_TIMING      = sv_set_timing;
 *   SV_OPT_PASS_PIN    v in {3, 4, 5}: every blocked-pass tile holds qubits
 *                      0..v-1 (contiguous runs of 8 * 2^v bytes; default 4 =
 *                      128 B).  64 B runs leave one more tile slot per pass
 *                      (fewer passes) at some DRAM efficiency: which wins
 *                      depends on the circuit (30q D14: 3, 32q D20: 4);
 *   SV_OPT_DIAG_SKIP   1 (default): sharded circuits (sv_circuit_create) do
 *                      not exchange a global qubit for a fused gate that is
 *                      block-diagonal in it (sv_shard_plan_diag); 0: plain S4;
 *   SV_OPT_PASS_SPEC   1 (default): the pass-specialised kernels apply
 *                      structured one-qubit gates (rows or columns multiples
 *                      of (1, i^p), diagonals; H, sqrt(X), sqrt(Y), T and
 *                      their products) as fp32 additions with the gates'
 *                      scalar factors multiplied in once per pass (DESIGN.md
 *                      R11): same result up to fp32 rounding order, fewer
 *                      operations; 0: every gate as a dense complex matrix;
 *   SV_OPT_PASS_SEARCH v in [1, 8], default 5: width of the pass-formation
 *                      search (R7): 1 = the greedy lookahead alone;
 *                      v > 1 keeps the v best qubit-set additions per growth
 *                      step and takes the set whose greedy completion needs
 *                      the fewest passes (34q D20: 10 -> 8 passes); which
 *                      width runs faster depends on the circuit.
 * Takes effect for circuits created / gates applied afterwards.  SV_EINVAL
 * for unknown options or values. */
#define SV_OPT_BLOCK_BITS 1
#define SV_OPT_PASS_JIT 2
#define SV_OPT_APPLY_PATH 3
#define SV_OPT_TIMING 4
#define SV_OPT_DIAG_SKIP 5  /* 1 (default): sharded circuits plan with the diagonal exchange skip */
#define SV_OPT_PASS_PIN 6   /* qubits 0..v-1 in every blocked-pass tile (runs of 8*2^v bytes): 3, 4 (default), 5 */
#define SV_OPT_PASS_SPEC 7  /* 1 (default): structured one-qubit gates as additions in the pass kernels */
#define SV_OPT_PASS_SEARCH 8 /* pass-formation search width 1..8 (default 5) */
#define SV_PATH_AUTO 0
#define SV_PATH_SIMT 1
#define SV_PATH_INT8 2
int sv_set_option(sv_state* s, int option, int value);

/* PTX of the pass-specialised kernels of every register-blocked pass of a
 * circuit (max_fused in [1, 2], tile_bits in [10, 14]; the first pass also
 * in its |0...0> form), separated by "//----" lines.  Pure host unless
 * compile != 0, which also assembles them through the driver JIT on the
 * current device (SV_ECUDA with the JIT log on failure).  tile_bits < 0:
 * the complex128 (wide) kernels for tiles of |tile_bits| qubits.  *need gets the
 * length including the terminating NUL; cap < *need returns SV_EINVAL unless
 * buf is NULL and cap is 0 (size query). */
int sv_pass_kernels(const sv_gate* gates, size_t n_gates, int max_fused, int tile_bits, int compile, char* buf,
                    size_t cap, size_t* need);
/* Process-wide counters of the pass-kernel compiler: kernels compiled, cache
 * hits, seconds spent compiling.  Pointers may be NULL. */
int sv_jit_stats(uint64_t* compiled, uint64_t* cache_hits, double* compile_seconds);
const char* sv_last_error(void);
/* Library version string. */
const char* sv_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SV_B200_H */
