// Device check of the FSteal planner (planner.h) against its host result on the loads where the control
#ifndef PLANNER_H
#define PLANNER_H "../../paper_conf_icde_menggltyz23_b200/csrc/planner.h"
#endif
// kernel produced a zero diagonal (tuning / debugging aid).
#include <cstdio>
#include PLANNER_H
__global__ void k(double* out, double b) {
    unsigned long long l[4] = {229893, 218340, 189113, 167913};
    double X[64];
    out[16] = gum::fsteal_waterfill(l, 4, b, X);
    for (int i = 0; i < 16; i++) out[i] = X[i];
}
__global__ void k_noinline_caller(double* out, double b, const unsigned long long* lg) {
    unsigned long long l[8];
    for (int i = 0; i < 4; i++) l[i] = lg[i];
    double X[64];
    out[16] = gum::fsteal_waterfill(l, 4, b, X);
    for (int i = 0; i < 16; i++) out[i] = X[i];
}
int main() {
    double *d, h[17], hh[17];
    unsigned long long hl[4] = {229893, 218340, 189113, 167913}, *dl;
    cudaMalloc(&d, 17 * 8);
    cudaMalloc(&dl, 32);
    cudaMemcpy(dl, hl, 32, cudaMemcpyHostToDevice);
    int bad = 0;
    for (int v = 0; v < 2; v++) {
        for (double b : {1.0, 2.0}) {
            if (v == 0) k<<<1, 1>>>(d, b); else k_noinline_caller<<<1, 1>>>(d, b, dl);
            cudaMemcpy(h, d, 17 * 8, cudaMemcpyDeviceToHost);
            hh[16] = gum::fsteal_waterfill(hl, 4, b, hh);
            printf("variant %d b=%g z dev %.3f host %.3f\n", v, b, h[16], hh[16]);
            for (int i = 0; i < 4; i++) {
                for (int j = 0; j < 4; j++) {
                    printf("%10.1f/%-10.1f ", h[i * 4 + j], hh[i * 4 + j]);
                    if (h[i * 4 + j] != hh[i * 4 + j]) bad++;
                }
                printf("\n");
            }
        }
    }
    printf("PLANTEST mismatches %d\n", bad);
    return bad != 0;
}
