// Host-side launchers of the sm_100a kernels (kernels.cu) and of the setup kernels (setup.cu).
#pragma once
#include <cuda_runtime.h>

#include "gum_internal.h"

namespace gum {

enum { ALG_BFS = GUM_BFS, ALG_SSSP = GUM_SSSP, ALG_WCC = GUM_WCC, ALG_PR = GUM_PR, ALG_DPR = GUM_DPR };
constexpr int kNumAlgs = 5;

// One launch unit = the workers [w0, w0+nw) that live on one device.
struct LaunchCfg {
    int w0, nw;
    int adv_grid;     // persistent advance grid (multiple of nw)
    int filter_grid;  // persistent filter CTAs per fragment
    int fin_grid;     // PR finalize CTAs per fragment
    int init_grid;
    int tail_grid;    // tail engine CTAs (cooperative; 0 = engine disabled)
    int adv_grid_pr;  // PR warp-task push (single fragment): occupancy-sized grid
    int pull_grid;    // PR pull: CTAs per fragment
};

enum { KER_FILTER = 0, KER_CONTROL = 1, KER_ADVANCE = 2, KER_FINALIZE = 3, KER_INIT = 4, KER_TAIL = 5, KER_APPLY = 6, KER_PULL = 7, KER_COUNT = 8 };
cudaError_t launch_kernel(int alg, int kind, const DevCtx& c, const LaunchCfg& L, cudaStream_t s,
                          cudaGraphConditionalHandle h, int use_h);
int phase_kernels(int alg, int phase, int* kinds);
cudaError_t launch_phase(int alg, int phase, const DevCtx& c, const LaunchCfg& L, cudaStream_t s,
                         cudaGraphConditionalHandle h, int use_h);
cudaError_t launch_init(int alg, const DevCtx& c, const LaunchCfg& L, cudaStream_t s, int f0, int nf, double D0,
                        int src_frag, unsigned src_local);
cudaError_t launch_gather(const DevCtx& c, int f, void* out, int is_pr, cudaStream_t s, int grid);
// multi-process barrier: every rank signals epoch into every peer's pad, then waits for all peers
cudaError_t launch_mp_barrier(const MpPads& p, int P, int me, unsigned long long epoch, cudaStream_t s);
// device-resident multi-unit loop: unit u's barrier (phase 0 = before the filter, with OSteal membership
// changes and parking; phase 1 = before control)
cudaError_t launch_unit_bar(const DevCtx& c, int u, int phase, cudaStream_t s);
cudaError_t advance_occupancy(int alg, int multi, int* blocks_per_sm);
cudaError_t tail_occupancy(int* blocks_per_sm);
cudaError_t filter_occupancy(int* blocks_per_sm);
cudaError_t pr_push_occupancy(int* blocks_per_sm);
cudaError_t pr_pull_occupancy(int* blocks_per_sm);
// PR single fragment: cut the destination-blocked queue's entries into pieces of <= piece edges
// (q2_off gets n2 + 1 entries; *n2 = pieces). tmp sized by setup_scan_tmp_bytes(n).
cudaError_t setup_pr_pieces_count(const unsigned long long* q_off, unsigned long long n, unsigned piece,
                                  unsigned long long* cnt, void* tmp, size_t tmp_bytes, cudaStream_t s);
cudaError_t setup_pr_pieces_emit(const unsigned* q_v, const unsigned long long* q_off, unsigned long long n,
                                 unsigned piece, const unsigned long long* pos, unsigned* q2_v,
                                 unsigned long long* q2_off, cudaStream_t s);
// PR pull: fragment in-CSR (rows = the fragment's vertices, cols = global source ids, rebased row_ptr) ->
// source-block-major layout with u32 offsets (pl_off[B*Vf+1]) and the per-pass merge-path tile table.
// h_tb receives the B+1 tile-table bases (host); pl_tx must hold h_tb[B] entries (call with pl_tx = null
// first to size it). tmp sized by setup_pr_tmp_bytes(Vf, B).
cudaError_t setup_pr_pull(const unsigned long long* in_rp, const unsigned* in_col, unsigned Vf, unsigned long long Ein,
                          unsigned S, int B, unsigned tile, unsigned* pl_off, unsigned* pl_col, unsigned* pl_tx,
                          unsigned long long* h_tb, void* tmp, size_t tmp_bytes, cudaStream_t s);
// BFS propagation blocking: static per-block capacities (in-degree histogram of the blocks) -> pb_off
cudaError_t setup_pb_offsets(const unsigned* col, unsigned long long E, unsigned shift, unsigned nb,
                             unsigned long long* pb_off, void* tmp, size_t tmp_bytes, cudaStream_t s);
size_t setup_pb_tmp_bytes(unsigned nb);

// ---- setup (setup.cu): validation, partitioning, relabelling, symmetrisation -------------------
cudaError_t setup_validate(const unsigned long long* row_ptr, const unsigned* col, unsigned V, unsigned long long E,
                           unsigned* d_err, cudaStream_t s);
cudaError_t setup_seg_bounds(const unsigned long long* row_ptr, unsigned V, unsigned long long E, int P,
                             unsigned* d_bounds, cudaStream_t s);
// RANDOM partitioner: keyed Feistel permutation pi on [0, V) (cycle walking), inverse table, and the
// relabelled CSR (row of new id pi(v) = row of v, destinations mapped through pi).
cudaError_t setup_relabel(const unsigned long long* row_ptr, const unsigned* col, const unsigned* w, unsigned V,
                          unsigned long long E, unsigned long long seed, unsigned* d_inv, unsigned long long* r_row_ptr,
                          unsigned* r_col, unsigned* r_w, void* tmp, size_t tmp_bytes, cudaStream_t s);
size_t setup_scan_tmp_bytes(unsigned V);
size_t setup_relabel_tmp_bytes(unsigned V);  // RANDOM relabel: scan temp + hub-row list
// symmetric (out + in) CSR for WCC: sym row v = out-neighbours of v followed by in-neighbours of v.
cudaError_t setup_symmetrize(const unsigned long long* row_ptr, const unsigned* col, unsigned V, unsigned long long E,
                             unsigned long long* s_row_ptr, unsigned* s_col, unsigned long long* cursor, void* tmp,
                             size_t tmp_bytes, cudaStream_t s);
// fragment extraction: rebased row_ptr slice; orig ids slice (or identity when inv == null)
cudaError_t setup_transpose(const unsigned long long* row_ptr, const unsigned* col, unsigned V, unsigned long long E,
                            unsigned long long* t_row_ptr, unsigned* t_col, unsigned long long* cursor, void* tmp,
                            size_t tmp_bytes, cudaStream_t s);
cudaError_t setup_rebase_rows(const unsigned long long* row_ptr, unsigned b0, unsigned b1, unsigned long long* out,
                              cudaStream_t s);
// PR destination-blocked static queue: pcol may be null when B == 1 (then the fragment col is used as is)
size_t setup_pr_tmp_bytes(unsigned Vf, int B);
cudaError_t setup_pr_blocked(const unsigned long long* rp, const unsigned* col, unsigned Vf, unsigned long long Ef,
                             unsigned S, int B, unsigned chunk, unsigned* pcol, unsigned* q_v, unsigned long long* q_off,
                             unsigned* tile, unsigned long long* h_Q, void* tmp, size_t tmp_bytes, cudaStream_t s);
cudaError_t setup_count_dangling(const unsigned long long* row_ptr, unsigned V, unsigned long long* d_count,
                                 cudaStream_t s);
unsigned host_feistel(unsigned v, unsigned V, unsigned long long seed);
// DEGREE relabel: d_perm[old] = new, d_inv[new] = old, ids ordered by decreasing in-degree (stable)
size_t setup_degree_tmp_bytes(unsigned V);
cudaError_t setup_relabel_degree(const unsigned long long* row_ptr, const unsigned* col, const unsigned* w,
                                 unsigned V, unsigned long long E, unsigned* d_perm, unsigned* d_inv,
                                 unsigned long long* r_row_ptr, unsigned* r_col, unsigned* r_w, void* tmp,
                                 size_t tmp_bytes, cudaStream_t s);
// NEXT-1 hub cache: off[0..n] = exclusive prefix of the cached (out-degree > t4) list lengths of global rows
// [b0, b0+n) (off[n] = total; tmp sized by setup_scan_tmp_bytes(n)); then fill copies the lists and sets
// off[v] = ~0 for rows that are not cached. hw / w may be null.
cudaError_t setup_hub_offsets(const unsigned long long* row_ptr, unsigned b0, unsigned n, unsigned t4,
                              unsigned long long* off, void* tmp, size_t tmp_bytes, cudaStream_t s);
cudaError_t setup_hub_fill(const unsigned long long* row_ptr, const unsigned* col, const unsigned* w, unsigned b0,
                           unsigned n, unsigned t4, unsigned long long* off, unsigned* hcol, unsigned* hw,
                           cudaStream_t s);

}  // namespace gum
