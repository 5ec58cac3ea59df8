// Internal layout shared by the host runtime (runtime.cu) and the sm_100a kernels (kernels.cu).
// Everything a kernel touches for fragment f lives in fragment f's device memory and is reachable
// from every worker through the pointers in DevCtx (local pointers for virtual peers, P2P/IPC
// pointers for real peers): the one-sided "remote memory access" design of P:398.
#pragma once
#include <stdint.h>

#include "gum.h"

namespace gum {

constexpr int kMaxW = GUM_MAX_WORKERS;
constexpr int kThreads = 256;          // CTA size of advance / filter
#ifndef GUM_ADV_THREADS
#define GUM_ADV_THREADS 256
#endif
constexpr int kAdvThreads = GUM_ADV_THREADS;  // CTA size of the advance (its barrier domain)
#ifndef GUM_EPT
#define GUM_EPT 8
#endif
constexpr int kEdgesPerThread = GUM_EPT;
constexpr int kTileMax = kAdvThreads * kEdgesPerThread;  // max edges per claimable chunk (smem sized for it)
constexpr int kDenseVertsPerThread = 8;                           // dense filter: consecutive vertices per thread
constexpr int kDenseWordsPerWarp = 32 * kDenseVertsPerThread / 32;   // 8 bitmap words per warp
constexpr int kDenseWordsPerPart = (kThreads / 32) * kDenseWordsPerWarp;  // 64 words = 2048 vertices
constexpr int kFilterAppPerThread = 8;                            // sparse filter: list entries per thread
constexpr int kFilterAppPerPart = kThreads * kFilterAppPerThread; // 2048
constexpr int kTraceMax = 1 << 16;
constexpr unsigned kTailSlack = 1u << 20;  // tail-engine lists (q_v, app): entries beyond V (no-dedupe duplicates)
constexpr int kPbMaxBins = 1024;       // propagation blocking: max destination blocks per fragment
constexpr unsigned kPrPiece = 64;      // PR warp-task path: max edges per queue entry
#ifndef GUM_PULL_IPT
#define GUM_PULL_IPT 8
#endif
constexpr int kPullIPT = GUM_PULL_IPT;              // PR pull: merge-path items (rows + edges) per thread
constexpr int kPullTile = kThreads * kPullIPT;       // PR pull: merge-path items per CTA tile

// Per-fragment control block (fragment memory, peer-visible). Counters that thieves touch
// (claim) and that the filter publishes (qlen, qedges, ntiles) live here.
struct alignas(128) FragCtl {
    unsigned long long claim;    // chunk claim counter of the current advance (steal queue head)
    unsigned long long ntiles;   // chunks in the current frontier queue
    unsigned long long qlen;     // |f_g| (vertices with out-degree > 0)
    unsigned long long qedges;   // l_g: out-edges of the current frontier (P:87 workload L_k)
    unsigned int app_cnt;        // activations appended during advance (next frontier, sparse list)
    unsigned int err;            // sticky error flag (1 = SSSP distance overflow)
    unsigned int dense;          // last filter used the bitmap (1) or the list (0)
    unsigned int pad0;
    double pr_dang[2];           // PR: partial dangling mass of this fragment's new x (by iteration parity)
    double pr_resid[2];          // PR: partial residual (by iteration parity)
    // run-total counters
    unsigned long long edges_done;     // edges of this fragment's chunks processed (own + stolen)
    unsigned long long edges_stolen;   // ... of which by a non-owner
    unsigned long long chunks_stolen;
    unsigned long long chunks_done;
    unsigned long long frontier_edges; // sum over iterations of qedges
    unsigned long long remote_updates; // updates issued by this fragment's owner to other fragments
    unsigned long long activations;
    unsigned long long frontier_vertices; // sum over iterations of qlen
    unsigned long long far_cnt;        // SSSP near-far: vertices currently parked in the far set
    unsigned int far_n[2];             // SSSP near-far: entries of the far lists (by sweep parity)
    unsigned int far_min[2];           // SSSP near-far: min distance of far vertices, by sweep parity
    unsigned int tcnt[3];              // tail engine: list counters (current / next / next-but-one)
    unsigned long long tedges[3];      // tail engine: out-edges of the listed vertices
    unsigned long long pclaim[kMaxW];  // FSteal planned mode: per-worker claim counters of this queue
    unsigned long long pull_checked;   // bottom-up BFS: in-edges inspected
    unsigned long long remote_filtered;  // NEXT-1 mirrors: cross-fragment updates absorbed locally
    unsigned long long hub_edges;        // NEXT-1 hub cache: non-local edges expanded from a local copy
    unsigned long long tail_edges, tail_vertices, tail_acts;  // work done inside the tail engine (stats)
    unsigned long long migrated_q;       // NEXT-3 copy-migration: queue entries generated in a foster queue
    unsigned int qown, pad_q;            // NEXT-3 copy-migration: the worker whose memory holds the current queue
                                         // (set by the filter that generated it; the advance may run after an
                                         // owner change, so it follows this, not the current owner)
    unsigned long long fpack;            // one-pass filter: (queue entries << kFpackShift) | out-edges reserved so far
    unsigned int fdone;                  // one-pass filter: CTAs finished (the last one publishes and resets)
    unsigned int tail_ovf;               // tail-engine hand-backs after a no-dedupe list overflow (stats)
};
// one-pass filter reservation counter: entries in the high 27 bits, edges in the low 37 (runtime checks V_g and
// E_g fit, else the two-pass filter runs)
constexpr unsigned kFpackShift = 37;
constexpr unsigned long long kFpackEdgeMask = (1ull << kFpackShift) - 1;

// Per launch unit (device) run-control replica: decisions are computed redundantly and
// identically by every unit from the same gathered counts (no policy broadcast).
struct alignas(128) RunCtl {
    unsigned int iter;        // BSP iteration k
    unsigned int done;
    unsigned int m;           // active owners (OSteal): workers {0..m-1}
    unsigned int steal_ok;    // FSteal gate for the current advance
    unsigned int tail;        // tail engine active for the current iteration (k_tail runs it)
    unsigned int tbar_cnt, tbar_gen;  // tail engine grid barrier
    unsigned int tsplit_cnt[2];       // tail engine: high-degree vertices deferred to the split phase
    unsigned int fbar_cnt, fbar_gen;  // filter grid barrier
    unsigned int tail_iters;  // iterations run by the tail engine (stats)
    unsigned int bodies;      // iteration bodies executed (control launches that did work)
    unsigned int pb;          // the current advance bins its discoveries (apply runs next body)
    unsigned int pull;        // the current BFS iteration runs bottom-up (k_bfs_pull instead of advance)
    unsigned int skip_filter; // the first iteration's queue is static (WCC blocked): no filter pass
    unsigned int blocked;     // WCC: the current advance runs on the static destination-blocked queue
                              // (1 = every vertex active, 2 = sources masked by the frontier bitmap)
    unsigned int blocked_iters;
    unsigned int plan_lo[kMaxW][kMaxW], plan_hi[kMaxW][kMaxW];  // FSteal plan: chunks [lo,hi) of queue f -> worker w
    double plan_z;            // planned makespan (edges) of the current iteration
    unsigned int nf_sweep;    // SSSP near-far: the next filter also scans the far set
    unsigned int nf_sweeps;   // number of threshold bumps so far (far_min slot parity)
    unsigned long long nf_T;  // SSSP near-far: current split distance (near iff dist < nf_T)
    unsigned int next_dense;  // the current advance only sets bitmap bits (next filter scans the bitmap)
                              // instead of appending to the activation list
    unsigned int owner[kMaxW];// fragment -> worker (P_OSteal vector O)
    unsigned int err;
    unsigned int osteal_iter;
    unsigned long long epoch; // filter look-back epoch (monotone across runs)
    double pr_D;              // PR: global dangling mass D_k of the current x
    double pr_resid;
    unsigned int ticket[kMaxW];   // filter partition tickets per fragment (reset by control)
    unsigned int filt_done[kMaxW];
    // device-resident multi-unit loop: barrier members {0..mb-1}; mb_next takes effect at the
    // next phase-A barrier (units >= mb_next leave it and park until woken); wakes[u] counts unit u's
    // wake-ups (computed identically by every member; the signal pad holds the same count); bar_ep is the
    // epoch of this unit's last device barrier (monotone across runs, equal on all members)
    unsigned int fctl_cnt;    // fused control: filter CTAs that arrived in this iteration
    unsigned int mb, mb_next;
    unsigned int wakes[kMaxW];
    unsigned long long bar_ep;
    // NEXT-3 online estimate of p (Eq. 4; "p ... can be estimated during previous iterations"): unit
    // 0's history by iteration & 3 (control start time, advance window, frontier edges, owners, tail flag);
    // every unit reads unit 0's history and updates its own estimate identically
    unsigned long long h_tctl[4], h_adv0[4], h_adv1[4], h_edges[4];
    unsigned int h_m[4], h_tail[4];
    double os_p;
    unsigned int os_p_n, pad_p;
};

// Decoupled look-back slot of the filter scan (one per partition per fragment, unit-local).
struct alignas(64) LBSlot {
    unsigned long long flag;      // epoch*4 + {1 = aggregate ready, 2 = inclusive ready}
    unsigned long long agg_cnt, agg_deg;
    unsigned long long inc_cnt, inc_deg;
};

// Tail engine split-list entry: a high-degree vertex expanded by all warps in segments.
struct TailSplit {
    unsigned f, v, sval, pad;
    unsigned long long s0, s1;
};

struct FragPtrs {
    const unsigned long long* row_ptr;  // [V_f + 1], rebased to 0
    const unsigned int* col;            // [E_f] global (relabelled) destination ids
    const unsigned int* w;              // [E_f] or null
    unsigned int* state;                // [V_f] depth / dist / label
    double* x;                          // PR [V_f]
    double* acc;                        // PR [V_f]
    double* cx;                         // PR [V_f] x[u]/outdeg(u): the value pushed along out-edges
    // BFS propagation blocking (dense iterations): destination ids binned per block of 2^pb_shift ids
    const unsigned long long* pb_off;   // [nb+1] static bin capacity prefix (in-degree per block)
    unsigned int* pb_fill;              // [nb] entries written this iteration
    unsigned int* pb_done;              // [nb] apply CTAs finished with the bin
    unsigned int* pb_buf;               // [E_in] binned destination ids (local)
    // bottom-up BFS (NEXT-4 direction optimisation): in-edges of the fragment's vertices
    const unsigned long long* in_row_ptr;  // [V_f + 1]
    const unsigned int* in_col;            // [E_in] global source ids
    const unsigned int* orig;           // [V_f] original ids (RANDOM relabel) or null (identity)
    unsigned int* bm;                   // [ceil(V_f/32)] activation bitmap (dedupe + dense frontier)
    unsigned int* vis;                  // [ceil(V_f/32)] BFS visited bitmap (check-before-update)
    unsigned int* bm2;                  // [ceil(V_f/32)] tail engine: dedupe bits of odd-iteration lists
    unsigned int* far;                  // [ceil(V_f/32)] SSSP near-far: parked (far) vertices
    unsigned int* farl;                 // [2][V_f] SSSP near-far: the far set as lists (bit set <=> listed)
    unsigned int* app;                  // [V_f] activation list (sparse next frontier)
    unsigned int* q_v;                  // [V_f] frontier queue (local ids, out-degree > 0)
    unsigned long long* q_off;          // [V_f + 1] exclusive prefix of out-degrees over the queue
    long long* q_base;                  // [V_f] col index of edge j of queue entry i = q_off[i] + j + q_base[i]
    unsigned int* tile;                 // [ntiles_max + 1] chunk table: first queue entry of chunk t
    FragCtl* ctl;
    unsigned int V;                     // |V_f|
    unsigned int base;                  // global id of local vertex 0
    unsigned long long E;
    unsigned long long pr_qlen, pr_qedges;  // PR's static destination-blocked queue (gum_prepare)
    // PR single fragment: the same queue with entries cut to <= kPrPiece edges, expanded by k_pr_push
    const unsigned int* pr2_q_v;
    const unsigned long long* pr2_q_off;  // [pr2_len + 1]; col index of edge j of entry i = q_off[i] + j
    unsigned long long pr2_len;
    // WCC: static destination-blocked queue of the symmetric graph for iteration 0 (all vertices active)
    const unsigned int* sq_col;
    const unsigned int* sq_q_v;
    const unsigned long long* sq_q_off;
    const unsigned int* sq_tile;
    unsigned long long sq_len, sq_edges;
    // PR pull (default PR advance): the fragment's in-edges regrouped source-block-major.
    // Pass b covers the sources [b*S, (b+1)*S) (an L2-sized block of x/outdeg); its rows are this fragment's
    // vertices: row i = pl_col[pl_off[b*V + i] .. pl_off[b*V + i + 1]) (global source ids, absolute u32
    // offsets). pl_tx[pl_tb[b] + t] = first row of merge-path tile t of pass b (pl_tb[b+1] - pl_tb[b] - 1
    // tiles; the last entry is V).
    const unsigned* pl_off;
    const unsigned* pl_col;
    const unsigned* pl_tx;
    const unsigned long long* pl_tb;
    // NEXT-1 outer-vertex mirror of worker f (this fragment's memory), indexed by GLOBAL id; only
    // vertices of other fragments are ever touched ("outer" vertices)
    double* macc;                       // PR: [V] aggregated pushes to other fragments' vertices
    unsigned int* msent;                // BFS: [ceil(V/32)] already-sent / known-visited bits
    unsigned int* mmin;                 // SSSP/WCC: [V] upper bound of the owner's value (min sent/seen)
};

// A fragment's frontier queue (the filter's output, the advance's input): in the fragment's own memory, or --
// NEXT-3 copy-migration (osteal_migrate) -- in a "foster" queue in the memory of the worker that owns the
// fragment after OSteal evicted its GPU ("the generated frontier queue will directly be on another GPU").
struct QPtrs {
    unsigned* q_v;
    unsigned long long* q_off;
    long long* q_base;
    unsigned* tile;
};

// NEXT-1 hub cache: worker w's local copy of fragment f's hub adjacency lists.
struct HubPtrs {
    const unsigned long long* off;  // [V_f] col index of local vertex u's list in the copy, ~0 = not cached
    const unsigned int* col;        // cached destination ids
    const unsigned int* w;          // cached weights (SSSP) or null
};

// Signal pads of the multi-unit barriers (a10), one per launch unit in its device memory (peer / IPC
// mapped): words [0, kMaxW) = host-loop barrier epochs by sender; kPadTimeout = a peer never arrived;
// kPadWake = wake count written by unit 0 (OSteal give-back / end of run); kPadArr / kPadLastIt = this
// unit's device-barrier arrivals in the current run and the iteration of the last one (stats);
// [kPadGraph, kPadGraph + kMaxW) = device-loop barrier epochs by sender.
constexpr int kPadWords = 32;
constexpr int kPadTimeout = kMaxW;
constexpr int kPadWake = kMaxW + 1;
constexpr int kPadArr = kMaxW + 2;
constexpr int kPadLastIt = kMaxW + 3;
constexpr int kPadGraph = 16;
struct MpPads {
    unsigned long long* pad[kMaxW];
};

struct DevCtx {
    FragPtrs f[kMaxW];
    RunCtl* rctl[kMaxW];        // per worker: the replica of the unit that worker belongs to
    LBSlot* lb[kMaxW];          // per fragment: look-back slots in the filtering unit's memory
    unsigned int lb_parts;      // slots per fragment
    gum_iter_trace* trace[kMaxW];  // per worker's unit (nullable)
    TailSplit* tsplit[kMaxW];      // per unit: tail engine split list (kTailSplitCap entries)
    unsigned int bounds[kMaxW + 1];
    int P;                      // fragments == workers
    unsigned int chunk;         // edges per chunk
    unsigned int num_vertices;  // |V|
    int fsteal, osteal;         // fsteal: 0 off, 1 steal queue, 2 planned (Eq. 1 / Alg. 1)
    double remote_cost;         // planned FSteal: cost of a remote edge relative to a local one
    double os_p;                // OSteal cost model (osteal = 2): p of Eq. (4) in edges (initial value when online)
    int os_p_online;            // estimate p online from unit 0's iteration history (osteal_sync_edges == 0)
    unsigned long long t1, t2, os_thresh, os_epw;
    unsigned int max_iter;
    int pr_iters;
    double pr_d;
    double dpr_eps;             // delta-PageRank residual threshold (absolute)
    unsigned int force_mode;    // 0 auto, 1 sparse, 2 dense
    unsigned int dense_div;     // dense filter iff app_cnt > V_f / dense_div
    unsigned int nf_delta;      // SSSP near-far split increment (0 = plain BSP frontier, the paper's)
    unsigned int tail_enter;    // tail engine: enter when the frontier has <= tail_enter vertices (0 = off)
    unsigned int tail_exit;     // tail engine: hand back when the next frontier exceeds tail_exit vertices
    unsigned int tail_slack;    // tail engine: list entries usable beyond V (<= kTailSlack; smaller only to test the overflow path)
    unsigned int tail_nodedupe; // tail engine: improvements by returning atomicMin, no dedupe bits (duplicates allowed)
    unsigned int tail_local;    // tail engine: local relaxation rounds per CTA before each grid barrier
    unsigned int pb_shift;      // BFS propagation blocking: log2(block size); 0 = off
    unsigned int pb_nb;         // bins of fragment 0 (single-fragment only)
    unsigned int bfs_pull;      // direction-optimising BFS enabled (in-CSR built)
    unsigned long long total_edges;  // sum of the fragments' out-edges
    int mirrors;                // NEXT-1 outer-vertex mirrors (P > 1 only)
    unsigned int filter_onepass;  // filter: one pass, queue ranges reserved per tile with one packed atomic
    unsigned int filter_swizzle;  // filter: spread each CTA's tile range over the id space (stride permutation)
    unsigned int bfs_filter_depth;  // BFS: the filter writes the depth of the vertices it takes from the
                                    // activations (the advance only sets visited / frontier bits)
    unsigned int wcc_blocked;     // WCC static destination-blocked queue exists: dense iterations may run on
                                  // it (the filter keeps the frontier bitmap in F.far)
    // PR pull: pl_B source-block passes per iteration; every launch unit keeps a replica of the global
    // x/outdeg vector, double-buffered by iteration parity ([2][num_vertices] doubles): the finalize of
    // fragment f writes its slice into every replica (cxrep[0..n_rep)), the pull of worker w reads cxw[w]
    // (its unit's replica). 0 passes = push (k_advance with red.add.f64).
    unsigned pl_B;
    int n_rep;
    double* cxrep[kMaxW];
    const double* cxw[kMaxW];
    // device-resident multi-unit loop: one CUDA graph per launch unit, device barriers over the member
    // units through these pads (unit u's pad in unit u's memory); 0 = single unit or host-driven loop
    int units_dev;
    int n_units;
    int alg;                    // the running algorithm (control_body)
    int fuse_ctl;               // single unit, graph mode: the filter's last CTA runs the control decision
    unsigned long long* pad[kMaxW];
    int migrate;                // NEXT-3 copy-migration: evicted fragments' queues live with their owner
    QPtrs fq[kMaxW][kMaxW];     // [owner][fragment] foster queues (fragment > owner), in the owner's memory
    int hub_on;                 // NEXT-1 hub cache built for this algorithm
    HubPtrs hub[kMaxW][kMaxW];  // [worker][fragment] (fragment != worker)
};

}  // namespace gum
