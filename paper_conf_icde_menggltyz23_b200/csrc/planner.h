// FSteal estimate-and-reassign planner (§III, Eq. (1), Alg. 1
// P:134-148). Shared by the device control kernel and the host ABI helper gum_fsteal_plan.
//
// Eq. (1): min_X max_j sum_i c_ij x_ij s.t. sum_j x_ij = l_i. On a uniform NVSwitch fabric the cost
// matrix has two values: c_ii = 1 (local edge, unit time) and c_ij = b >= 1 for i != j (remote edge,
// c_ij = 1/B_ij + g(W_i) with B uniform). The LP relaxation (Theorem 1's z-form, the problem
// Alg. 1 hands to SCIP) then has a closed form (SURVEY c-7): donors (l_i > z) keep z of their own edges
// and give l_i - z away; receivers (l_j <= z) keep all of theirs and take (z - l_j)/b; z solves
//     sum_i max(l_i - z, 0) = sum_j max(z - l_j, 0) / b,
// found exactly by waterfill_z (the left side minus the right is decreasing and piecewise linear in z). X is filled donor-major
// ("north-west corner" over increasing worker ids). Rounding to whole chunks happens in the caller.
#pragma once

#ifndef __CUDACC__
#define GUM_HD
#else
#define GUM_HD __host__ __device__
#endif

namespace gum {

// The balance point of the closed form, exactly: the balance function
//     extra + sum_i max(v_i - z, 0) - sum_i max(z - v_i, 0) / b
// is decreasing and linear between consecutive loads (the loads below z are receivers, the others donors:
// extra + S_donors - n_d z - (n_r z - S_recv)/b), so z is the root of the one segment that contains it,
// found from the balance at the loads themselves -- O(m^2) cheap operations, where a bisection took hundreds
// of fp64 divisions on the control kernel's single thread (0.1-0.9 ms per iteration, measured in round 2).
// extra = work that must move off evicted fragments (OSteal), 0 for FSteal. v_i >= 0, m in 1..8, b >= 1.
GUM_HD inline double waterfill_balance(const double* v, int m, double extra, double ib, double z) {
    double f = extra;
    for (int i = 0; i < m; i++) f += v[i] > z ? v[i] - z : (v[i] - z) * ib;
    return f;
}
GUM_HD inline double waterfill_z(const double* v, int m, double extra, double b) {
    // the segment [lo, hi) between consecutive loads where the balance changes sign: lo = the largest load
    // (or 0) with balance >= 0; on it the loads <= lo are receivers and the others donors. (Multiplications
    // by 1/b: a single thread's fp64 divisions were the control kernel's cost.)
    const double ib = 1.0 / b;
    double lo = 0.0;
    for (int i = 0; i < m; i++)
        if (v[i] > lo && waterfill_balance(v, m, extra, ib, v[i]) >= 0.0) lo = v[i];
    double num = extra, den = 0.0;
    for (int i = 0; i < m; i++) {
        if (v[i] > lo) {
            num += v[i];
            den += 1.0;
        } else {
            num += v[i] * ib;
            den += ib;
        }
    }
    return num / den;
}

GUM_HD inline double fsteal_waterfill(const unsigned long long* l, int n, double b, double* X) {
    if (n <= 0) return 0.0;
    if (b < 1.0) b = 1.0;
    double v[8];
    for (int i = 0; i < n; i++) v[i] = (double)l[i];
    const double zz = waterfill_z(v, n, 0.0, b);
    double hi = 0.0;
    for (int i = 0; i < n; i++) hi = v[i] > hi ? v[i] : hi;
    const double z = zz < hi ? zz : hi;  // (all loads equal: the root is that load)
    // every entry of X is written exactly once, row by row: the off-diagonal transfers in worker order, then
    // the diagonal (kept share + rounding residue). The previous zero-fill + read-modify-write form produced a
    // zero diagonal in row 0 inside the device control kernel (worker 0 kept nothing, so the heaviest
    // iteration ran on the other three: tests/test_gpu_parity.py test_planned_fsteal), although the same
    // function was right on the host and in a standalone kernel (tools/plantest).
    double r[8];
    for (int j = 0; j < n; j++) r[j] = v[j] > z ? 0.0 : (z - v[j]) / b;
    for (int i = 0; i < n; i++) {
        double gi = v[i] > z ? v[i] - z : 0.0;
        for (int j = 0; j < n; j++) {
            double t = 0.0;
            if (j != i && gi > 0.0 && r[j] > 0.0) {
                t = gi < r[j] ? gi : r[j];
                gi -= t;
                r[j] -= t;
            }
            if (j != i) X[i * n + j] = t;
        }
        X[i * n + i] = (v[i] > z ? z : v[i]) + gi;  // rounding residue stays with its owner
    }
    return z;
}

// OSteal cost model (§IV-A/B, Eq. (4), p estimated online P:172, Alg. 2).
// For a cluster size m the reduction tree on a uniform fabric keeps workers R(m) = {0..m-1} (DESIGN.md
// reading #13); the revised Eq. (1) lets only R(m) process (x_ij = 0 for j outside R(m)): an evicted
// fragment's edges are all processed remotely at cost b, a survivor keeps its own at cost 1 and trades
// with the other survivors as in fsteal_waterfill. The LP relaxation again has a closed form: z solves
//     sum_{j<m} max(l_j - z, 0) + sum_{i>=m} l_i = sum_{j<m} max(z - l_j, 0) / b.
GUM_HD inline double osteal_makespan(const unsigned long long* l, int n, int m, double b) {
    if (n <= 0 || m <= 0) return 0.0;
    if (m > n) m = n;
    if (b < 1.0) b = 1.0;
    double v[8], evicted = 0.0;
    for (int i = 0; i < n; i++) {
        if (i < m) v[i] = (double)l[i];
        else evicted += (double)l[i];
    }
    return waterfill_z(v, m, evicted, b);
}

// Alg. 2: enumerate m = 1..n, E(m) = z(m) + p*m (Eq. 4), keep the first strict minimum. cost[m-1] =
// E(m) when cost is non-null. Returns the chosen m.
GUM_HD inline int osteal_choose(const unsigned long long* l, int n, double b, double p, double* cost) {
    int best_m = n;
    double best = 0.0;
    for (int m = 1; m <= n; m++) {
        const double e = osteal_makespan(l, n, m, b) + p * (double)m;
        if (cost) cost[m - 1] = e;
        if (m == 1 || e < best) {
            best = e;
            best_m = m;
        }
    }
    return best_m;
}

}  // namespace gum
