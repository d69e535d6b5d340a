// planner.cpp -- global/local qubit-map planning for the sharded mode
// (reading S4; north star "qubit-remapping exchange ...
// batched across consecutive gates"; PAPER.md L209/L229 name multi-GPU as
// the future work this realises).
//
// The 2^n state is split into P = 2^g shards by the top g PHYSICAL bits
// (positions l = n-g .. n-1).  Before a fused gate touching a logical qubit
// that sits at a global position, an EXCHANGE swaps physical bits (P_j, p_j)
// (global, local) for a batch of pairs chosen by Belady next-use order with
// a victim floor vmin.  Must match oracle/plan.py bit for bit.
//
// Diagonal skip (diag != nullptr; reading R10, SURVEY.md §8f
// NEXT-4): a fused gate forces an exchange only for its global qubits in
// which it is not block-diagonal (diag[i] = logical-qubit mask of the
// qubits it is block-diagonal in); next use counts non-diagonal uses only.
// Such an APPLY lists global physical positions; the dispatcher runs the
// block selected by each shard's device bits.
#include <algorithm>
#include <complex>
#include <limits>

#include "sv_internal.h"

namespace svb {

void plan_sharded(const std::vector<std::vector<int>>& fq, int n, int g, int vmin, std::vector<Event>& ev,
                  std::vector<int>& pos, const std::vector<uint64_t>* diag) {
    const int l = n - g;
    const int nf = (int)fq.size();
    const int INF = std::numeric_limits<int>::max();
    if ((int)pos.size() != n) {
        pos.resize(n);
        for (int q = 0; q < n; ++q) pos[q] = q;
    }
    std::vector<int> inv(n);
    for (int q = 0; q < n; ++q) inv[pos[q]] = q;
    // next_use[i][q] = min{ j >= i : q in Q_j } (INF if none), built backwards
    std::vector<std::vector<int>> next_use(nf + 1, std::vector<int>(n, INF));
    auto uses = [&](int i, int q) { return !diag || !(((*diag)[i] >> q) & 1ull); };
    for (int i = nf - 1; i >= 0; --i) {
        next_use[i] = next_use[i + 1];
        for (int q : fq[i])
            if (uses(i, q)) next_use[i][q] = i;
    }
    ev.clear();
    for (int i = 0; i < nf; ++i) {
        const std::vector<int>& Qi = fq[i];
        auto inQ = [&](int q) { return std::find(Qi.begin(), Qi.end(), q) != Qi.end(); };
        int need = 0;
        for (int q : Qi)
            if (pos[q] >= l && uses(i, q)) ++need;
        const std::vector<int>& nu = next_use[i];
        if (need) {
            std::vector<int> glob;
            for (int p = l; p < n; ++p) glob.push_back(inv[p]);
            std::stable_sort(glob.begin(), glob.end(), [&](int a, int b) {
                if (nu[a] != nu[b]) return nu[a] < nu[b];
                return a < b;
            });
            std::vector<int> cand;
            for (int p = std::max(vmin, 0); p < l; ++p)
                if (!inQ(inv[p])) cand.push_back(inv[p]);
            if ((int)cand.size() < need) {
                cand.clear();
                for (int p = 0; p < l; ++p)
                    if (!inQ(inv[p])) cand.push_back(inv[p]);
            }
            std::stable_sort(cand.begin(), cand.end(), [&](int a, int b) {
                if (nu[a] != nu[b]) return nu[a] > nu[b];
                return pos[a] > pos[b];
            });
            Event x;
            x.type = Event::EXCHANGE;
            for (size_t t = 0; t < glob.size() && t < cand.size(); ++t) {
                const int a = glob[t], b = cand[t];
                if (nu[a] < nu[b]) x.pairs.push_back({pos[a], pos[b]});
                else break;
            }
            for (auto& pr : x.pairs) {
                const int a = inv[pr.first], b = inv[pr.second];
                pos[a] = pr.second;
                pos[b] = pr.first;
                inv[pr.first] = b;
                inv[pr.second] = a;
            }
            ev.push_back(std::move(x));
        }
        Event a;
        a.type = Event::APPLY;
        a.fused = i;
        std::vector<int> sq = Qi;
        std::sort(sq.begin(), sq.end());
        a.k = (int)sq.size();
        for (int b = 0; b < a.k; ++b) a.phys[b] = pos[sq[b]];
        ev.push_back(std::move(a));
    }
}

void plan_canonicalize(int n, int g, std::vector<int>& pos, std::vector<Event>& ev) {
    const int l = n - g;
    std::vector<int> inv(n);
    for (int q = 0; q < n; ++q) inv[pos[q]] = q;
    std::vector<int> wg, wl;
    for (int P = l; P < n; ++P)
        if (inv[P] < l) wg.push_back(P);
    for (int p = 0; p < l; ++p)
        if (inv[p] >= l) wl.push_back(p);
    if (!wg.empty()) {
        Event x;
        x.type = Event::EXCHANGE;
        for (size_t t = 0; t < wg.size(); ++t) x.pairs.push_back({wg[t], wl[t]});
        for (auto& pr : x.pairs) {
            const int a = inv[pr.first], b = inv[pr.second];
            pos[a] = pr.second;
            pos[b] = pr.first;
            inv[pr.first] = b;
            inv[pr.second] = a;
        }
        ev.push_back(std::move(x));
    }
    bool ident = true;
    for (int p = 0; p < l; ++p)
        if (inv[p] != p) ident = false;
    if (!ident) {
        Event x;
        x.type = Event::PERMUTE;
        x.perm.resize(l);
        for (int p = 0; p < l; ++p) x.perm[p] = inv[p];  // data at bit p moves to bit inv[p]
        for (int p = 0; p < l; ++p) pos[inv[p]] = inv[p];
        ev.push_back(std::move(x));
    }
}

}  // namespace svb

namespace svb {

// block-diagonal in qubit b: every entry between a row and a column that
// differ in bit b has |entry| <= 1e-10 (fp64 rounding residue of exact zeros;
// the blocks drop them -- reading R10; oracle/plan.py DIAG_TOL)
uint64_t diag_mask(const FusedGate& f) {
    const int D = 1 << f.k;
    uint64_t m = 0;
    for (int b = 0; b < f.k; ++b) {
        bool block = true;
        for (int r = 0; r < D && block; ++r)
            for (int c = 0; c < D; ++c)
                if ((((r ^ c) >> b) & 1) && std::abs(f.M[(size_t)r * D + c]) > 1e-10) {
                    block = false;
                    break;
                }
        if (block) m |= 1ull << f.q[b];
    }
    return m;
}

}  // namespace svb
