// fuser.cpp -- host gate fusion.
//
// PAPER.md L98 (§2.2, Fig. 5): gates on disjoint qubits fuse "in space" by a
// tensor product, gates on the same qubits "in time" by an ordered matrix
// product; L104: fusion is "given as input the maximum of fused gates"
// (reading Q4: max qubits per fused gate; 0 = no fusion).  The greedy scan is
// the deterministic reading S3 of SURVEY.md §8c; it must reproduce the
// oracle's plan bit for bit (tests/test_host_lib.py).  Qubit sets are kept
// as 64-bit masks; the fused matrix is accumulated in fp64 by applying each
// member gate to the columns of the running product (E_j * M), and is rounded
// to complex64 only when a launch descriptor is built.
#include <algorithm>
#include <cstring>

#include "sv_internal.h"

namespace svb {

static inline int popc64(uint64_t x) { return __builtin_popcountll(x); }

int validate_gates(const sv_gate* g, size_t m, int n_qubits) {
    if (m > 0 && g == nullptr) return fail(SV_EINVAL, "gates is NULL with n_gates > 0");
    for (size_t i = 0; i < m; ++i) {
        const sv_gate& x = g[i];
        if (x.nq != 1 && x.nq != 2) return fail(SV_EINVAL, "gate " + std::to_string(i) + ": nq must be 1 or 2");
        for (int b = 0; b < x.nq; ++b) {
            if (x.q[b] < 0 || x.q[b] >= SV_MAX_QUBITS || (n_qubits >= 0 && x.q[b] >= n_qubits))
                return fail(SV_EINVAL, "gate " + std::to_string(i) + ": qubit out of range");
        }
        if (x.nq == 2 && x.q[0] == x.q[1]) return fail(SV_EINVAL, "gate " + std::to_string(i) + ": duplicate qubit");
    }
    return SV_OK;
}

static inline uint64_t gate_mask(const sv_gate& x) {
    uint64_t s = 0;
    for (int b = 0; b < x.nq; ++b) s |= 1ull << x.q[b];
    return s;
}

static void mask_to_fused(uint64_t Q, FusedGate& fg) {
    fg.k = 0;
    for (int q = 0; q < 64; ++q)
        if ((Q >> q) & 1) fg.q[fg.k++] = q;
}

void fuse_plan(const sv_gate* g, size_t m, int F, std::vector<FusedGate>& out) {
    out.clear();
    if (F == 0) {
        for (size_t i = 0; i < m; ++i) {
            FusedGate fg;
            mask_to_fused(gate_mask(g[i]), fg);
            fg.mem.push_back((int32_t)i);
            out.push_back(std::move(fg));
        }
        return;
    }
    std::vector<uint64_t> S(m);
    for (size_t i = 0; i < m; ++i) S[i] = gate_mask(g[i]);
    std::vector<char> done(m, 0);
    for (size_t i = 0; i < m; ++i) {
        if (done[i]) continue;
        done[i] = 1;
        uint64_t Q = S[i];
        FusedGate fg;
        fg.mem.push_back((int32_t)i);
        if (popc64(Q) > F) {
            mask_to_fused(Q, fg);
            out.push_back(std::move(fg));
            continue;
        }
        uint64_t B = 0;
        for (size_t j = i + 1; j < m; ++j) {
            if (done[j]) continue;
            const uint64_t s = S[j];
            if (s & B) {
                B |= s;
            } else if (popc64(Q | s) <= F) {
                Q |= s;
                fg.mem.push_back((int32_t)j);
                done[j] = 1;
            } else {
                B |= s;
            }
            if (popc64(Q) == F && (Q & ~B) == 0) break;
        }
        mask_to_fused(Q, fg);
        out.push_back(std::move(fg));
    }
}

// Apply a 1- or 2-qubit gate (local bit positions lp[b] <-> gate index bit b)
// to one column vector v of length 2^k, in place.
static void apply_local(int k, const sv_gate& x, const int* lp, cd* v) {
    const int nq = x.nq;
    const int d = 1 << nq;
    const int ngroups = 1 << (k - nq);
    int s[2] = {lp[0], nq == 2 ? lp[1] : 0};
    if (nq == 2 && s[0] > s[1]) std::swap(s[0], s[1]);
    cd a[4];
    for (int j = 0; j < ngroups; ++j) {
        unsigned base = (unsigned)j;
        for (int b = 0; b < nq; ++b) {
            unsigned lo = base & ((1u << s[b]) - 1);
            base = ((base >> s[b]) << (s[b] + 1)) | lo;
        }
        unsigned off[4];
        for (int c = 0; c < d; ++c) {
            unsigned o = 0;
            for (int b = 0; b < nq; ++b)
                if ((c >> b) & 1) o |= 1u << lp[b];
            off[c] = base | o;
            a[c] = v[off[c]];
        }
        for (int r = 0; r < d; ++r) {
            cd y = 0;
            for (int c = 0; c < d; ++c) y += cd(x.m[r * d + c].re, x.m[r * d + c].im) * a[c];
            v[off[r]] = y;
        }
    }
}

void build_fused_matrix(const sv_gate* g, FusedGate& fg) {
    const int k = fg.k;
    const int d = 1 << k;
    // column-major work array: col[c] is column c of M (a vector of length d)
    std::vector<cd> col((size_t)d * d, cd(0));
    for (int c = 0; c < d; ++c) col[(size_t)c * d + c] = 1.0;
    for (int32_t j : fg.mem) {
        const sv_gate& x = g[j];
        int lp[2] = {0, 0};
        for (int b = 0; b < x.nq; ++b) {
            int p = -1;
            for (int t = 0; t < k; ++t)
                if (fg.q[t] == x.q[b]) p = t;
            lp[b] = p;
        }
        for (int c = 0; c < d; ++c) apply_local(k, x, lp, &col[(size_t)c * d]);
    }
    fg.M.assign((size_t)d * d, cd(0));
    for (int r = 0; r < d; ++r)
        for (int c = 0; c < d; ++c) fg.M[(size_t)r * d + c] = col[(size_t)c * d + r];
}

template <typename T>
void sort_matrix_qubits(int k, const int* qubits, const T* in, int* sorted_q, T* out) {
    int order[SV_MAX_FUSED];  // order[j] = b such that sorted_q[j] = qubits[b]
    for (int b = 0; b < k; ++b) order[b] = b;
    std::sort(order, order + k, [&](int a, int b) { return qubits[a] < qubits[b]; });
    for (int j = 0; j < k; ++j) sorted_q[j] = qubits[order[j]];
    const int d = 1 << k;
    // new index bit j <-> old index bit order[j]
    std::vector<int> map(d);
    for (int nidx = 0; nidx < d; ++nidx) {
        int o = 0;
        for (int j = 0; j < k; ++j)
            if ((nidx >> j) & 1) o |= 1 << order[j];
        map[nidx] = o;
    }
    for (int r = 0; r < d; ++r)
        for (int c = 0; c < d; ++c) out[(size_t)r * d + c] = in[(size_t)map[r] * d + map[c]];
}

template void sort_matrix_qubits<cd>(int, const int*, const cd*, int*, cd*);
template void sort_matrix_qubits<cf>(int, const int*, const cf*, int*, cf*);

}  // namespace svb
