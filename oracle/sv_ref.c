/*
 * sv_ref.c -- S0 oracle simulator in plain C + OpenMP.
 * TEST INFRASTRUCTURE ONLY: loaded by tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs.  Shares nothing with the
 * product library under paper_conf_sc_markidis23_b200/.
 *
 * What it computes (§2.2, Figs. 3-4): psi' = G psi for one
 * gate at a time, matrix-free and in place.  Each of the 2^(n-k) independent
 * groups (L93: "2^(n-1) (one matrix multiply per thread)", generalised to k
 * qubits) is: base = j with a zero bit inserted at every gate qubit (ascending),
 *   a[c] = psi[base | sum_b c_b 2^{q[b]}],
 *   psi[base | sum_b r_b 2^{q[b]}] = sum_c G[r][c] a[c].
 * Bit b of the matrix index <-> qubits[b], complex128,
 * interleaved (re, im).  No fusion, no tiling, no blocking.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define MAXK 6

int svref_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

void svref_zero_state(int n, double* psi) {
    uint64_t dim = (uint64_t)1 << n;
    int64_t i;
#pragma omp parallel for schedule(static)
    for (i = 0; i < (int64_t)dim; ++i) {
        psi[2 * i] = 0.0;
        psi[2 * i + 1] = 0.0;
    }
    psi[0] = 1.0;
}

/* Apply a k-qubit gate (k <= 6).  Returns 0, or -1 on bad arguments. */
int svref_apply(int n, int k, const int* qubits, const double* mat, double* psi) {
    int s[MAXK];
    int b, t, r, c;
    uint64_t off[1 << MAXK];
    int64_t j, ngroups;
    if (k < 1 || k > MAXK || k > n) return -1;
    for (b = 0; b < k; ++b) {
        if (qubits[b] < 0 || qubits[b] >= n) return -1;
        for (t = 0; t < b; ++t)
            if (qubits[t] == qubits[b]) return -1;
        s[b] = qubits[b];
    }
    /* sort the qubit positions ascending (insertion sort) */
    for (b = 1; b < k; ++b) {
        int v = s[b];
        t = b - 1;
        while (t >= 0 && s[t] > v) { s[t + 1] = s[t]; --t; }
        s[t + 1] = v;
    }
    /* offset of matrix index c: sum_b c_b 2^{qubits[b]} */
    for (c = 0; c < (1 << k); ++c) {
        uint64_t o = 0;
        for (b = 0; b < k; ++b)
            if ((c >> b) & 1) o |= (uint64_t)1 << qubits[b];
        off[c] = o;
    }
    ngroups = (int64_t)1 << (n - k);
#pragma omp parallel for schedule(static)
    for (j = 0; j < ngroups; ++j) {
        double a[2 << MAXK];
        uint64_t base = (uint64_t)j;
        int bb, cc, rr;
        for (bb = 0; bb < k; ++bb) {
            uint64_t lo = base & (((uint64_t)1 << s[bb]) - 1);
            base = ((base >> s[bb]) << (s[bb] + 1)) | lo;
        }
        for (cc = 0; cc < (1 << k); ++cc) {
            a[2 * cc] = psi[2 * (base | off[cc])];
            a[2 * cc + 1] = psi[2 * (base | off[cc]) + 1];
        }
        for (rr = 0; rr < (1 << k); ++rr) {
            double yr = 0.0, yi = 0.0;
            for (cc = 0; cc < (1 << k); ++cc) {
                double gr = mat[2 * (rr * (1 << k) + cc)];
                double gi = mat[2 * (rr * (1 << k) + cc) + 1];
                yr += gr * a[2 * cc] - gi * a[2 * cc + 1];
                yi += gr * a[2 * cc + 1] + gi * a[2 * cc];
            }
            psi[2 * (base | off[rr])] = yr;
            psi[2 * (base | off[rr]) + 1] = yi;
        }
    }
    (void)r;
    return 0;
}

/* Run m gates (1 or 2 qubits each) in order on psi.  Layout per gate i:
 * nq[i], q[2*i .. 2*i+1], mat[32*i ..] = 16 complex (2x2 uses the first 4). */
int svref_run(int n, int64_t m, const int* nq, const int* q, const double* mat, double* psi) {
    int64_t i;
    for (i = 0; i < m; ++i) {
        int rc = svref_apply(n, nq[i], q + 2 * i, mat + 32 * i, psi);
        if (rc) return rc;
    }
    return 0;
}
