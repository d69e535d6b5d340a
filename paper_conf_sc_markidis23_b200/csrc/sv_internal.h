// sv_internal.h -- internal types of libsvb200 (not part of the C ABI).
#pragma once

#include <complex>
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/sv.h"

namespace svb {

using cd = std::complex<double>;
using cf = std::complex<float>;

// ---- errors ---------------------------------------------------------------
void set_error(const std::string& msg);
int fail(int code, const std::string& msg);

// ---- host fusion (S3) -------------------------------------------------------
struct FusedGate {
    int k = 0;                    // number of qubits
    int q[SV_MAX_FUSED] = {0};    // ascending logical qubits
    std::vector<int32_t> mem;     // member gate indices, ascending
    std::vector<cd> M;            // 2^k x 2^k row-major, bit b <-> q[b] (fp64)
};

// Validates gates; returns SV_OK or SV_EINVAL (message set).
int validate_gates(const sv_gate* g, size_t m, int n_qubits /* <0: skip range check */);
// Greedy qsim-style fusion plan.  Integer part only.
void fuse_plan(const sv_gate* g, size_t m, int max_fused, std::vector<FusedGate>& out);
// M = E_{mem[-1]} ... E_{mem[0]} in fp64 for one fused gate (fills fg.M).
void build_fused_matrix(const sv_gate* g, FusedGate& fg);

// Reorder a 2^k matrix whose index bit b <-> qubits[b] into ascending-qubit
// order.  sorted_q receives the ascending qubits.
template <typename T>
void sort_matrix_qubits(int k, const int* qubits, const T* in, int* sorted_q, T* out);

// ---- sharded planning (S4) --------------------------------------------------
struct Event {
    enum Type { APPLY = 0, EXCHANGE = 1, PERMUTE = 2 } type = APPLY;
    int fused = -1;                       // APPLY: fused gate index
    int k = 0;                            // APPLY: qubits
    int phys[SV_MAX_FUSED] = {0};         // APPLY: physical bits in sorted-logical order
    std::vector<std::pair<int, int>> pairs;  // EXCHANGE: (global P, local p)
    std::vector<int> perm;                // PERMUTE: new local position of local bit b (size l)
};
// S4 exactly; events + final pos (logical -> physical).
// diag (optional): per fused gate the mask of logical qubits it is
// block-diagonal in (the diagonal exchange skip, reading R10).
void plan_sharded(const std::vector<std::vector<int>>& fused_q, int n, int g, int vmin,
                  std::vector<Event>& ev, std::vector<int>& pos, const std::vector<uint64_t>* diag = nullptr);
// Logical qubits of a fused gate in which its fp64 matrix is block-diagonal
// (entries between rows and columns differing in that bit are exactly 0).
uint64_t diag_mask(const FusedGate& f);
// Canonicalisation events appended after a plan so that the final map is the
// identity up to a relabelling of the global bits (Readings R9).
void plan_canonicalize(int n, int g, std::vector<int>& pos, std::vector<Event>& ev);

}  // namespace svb
