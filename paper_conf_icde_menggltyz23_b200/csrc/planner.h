// FSteal estimate-and-reassign planner (§III, Eq. (1), Alg. 1
// P:134-148). Shared by the device control kernel and the host ABI helper gum_fsteal_plan.
//
// Eq. (1): min_X max_j sum_i c_ij x_ij s.t. sum_j x_ij = l_i. On a uniform NVSwitch fabric the cost
// matrix has two values: c_ii = 1 (local edge, unit time) and c_ij = b >= 1 for i != j (remote edge,
// c_ij = 1/B_ij + g(W_i) with B uniform). The LP relaxation (Theorem 1's z-form, the problem
// Alg. 1 hands to SCIP) then has a closed form (SURVEY c-7): donors (l_i > z) keep z of their own edges
// and give l_i - z away; receivers (l_j <= z) keep all of theirs and take (z - l_j)/b; z solves
//     sum_i max(l_i - z, 0) = sum_j max(z - l_j, 0) / b,
// found by bisection (the left side minus the right is decreasing in z). X is filled donor-major
// ("north-west corner" over increasing worker ids). Rounding to whole chunks happens in the caller.
#pragma once

#ifndef __CUDACC__
#define GUM_HD
#else
#define GUM_HD __host__ __device__
#endif

namespace gum {

GUM_HD inline double fsteal_waterfill(const unsigned long long* l, int n, double b, double* X) {
    for (int i = 0; i < n * n; i++) X[i] = 0.0;
    if (n <= 0) return 0.0;
    if (b < 1.0) b = 1.0;
    double lo = 0.0, hi = 0.0;
    for (int i = 0; i < n; i++) hi = (double)l[i] > hi ? (double)l[i] : hi;
    for (int it = 0; it < 200; it++) {  // bisection on the balance function
        const double z = 0.5 * (lo + hi);
        double give = 0.0, take = 0.0;
        for (int i = 0; i < n; i++) {
            const double li = (double)l[i];
            if (li > z) give += li - z;
            else take += (z - li) / b;
        }
        if (give > take) lo = z;
        else hi = z;
    }
    const double z = hi;
    double g[8], r[8];
    for (int i = 0; i < n; i++) {
        const double li = (double)l[i];
        X[i * n + i] = li > z ? z : li;
        g[i] = li > z ? li - z : 0.0;
        r[i] = li > z ? 0.0 : (z - li) / b;
    }
    for (int i = 0; i < n; i++) {
        for (int j = 0; j < n && g[i] > 0.0; j++) {
            if (j == i || r[j] <= 0.0) continue;
            const double t = g[i] < r[j] ? g[i] : r[j];
            X[i * n + j] += t;
            g[i] -= t;
            r[j] -= t;
        }
        X[i * n + i] += g[i];  // bisection residue stays with its owner
    }
    return z;
}

}  // namespace gum
