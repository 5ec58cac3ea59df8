/*
 * gum.h -- C ABI of the B200-native GUM hot path (Meng et al., ICDE'23, "Efficient Multi-GPU Graph
 * Processing with Remote Work Stealing"). PAPER.md lines are cited as P:<line>.
 *
 * The library runs the frontier-driven advance/filter iteration of GAS algorithms in BSP mode
 * (§II "Graph algorithms") for BFS, SSSP, WCC and PageRank (§VI-A) over an n-way
 * edge-cut partition of a CSR graph (§II "Graph partitions"), with the paper's two load
 * balancers: frontier stealing (FSteal, §III) and ownership stealing (OSteal, §IV,
 * P:152-211). Kernels are hand-written CUDA for sm_100a; see DESIGN.md.
 *
 * Conventions (all entry points):
 *   - plain C; no exceptions or C++/torch types cross the ABI;
 *   - every call returns gum_status (0 = GUM_OK, < 0 = error); gum_last_error() gives the text;
 *   - after any GUM_ECUDA the context is poisoned: later calls return GUM_ESTATE;
 *   - pointers are HOST pointers unless a flag or parameter says "device";
 *   - the caller owns every buffer it passes; the library copies what it keeps (gum_load_csr) and
 *     owns its device memory until gum_destroy().
 *   - vertex ids are uint32 in [0, V), V <= 2^32-2; GUM_INF (0xFFFFFFFF) marks "unreached".
 */
#ifndef GUM_H
#define GUM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct gum_ctx gum_ctx; /* opaque, owned by the library */

typedef enum {
    GUM_OK = 0,
    GUM_EINVAL = -1, /* null pointer, malformed CSR (row_ptr not monotone, row_ptr[V] != E, col >= V),
                        SSSP without weights, buffer too small, bad config value */
    GUM_ENOMEM = -2, /* device allocation failed (the paper assumes the graph fits) */
    GUM_ESTATE = -3, /* wrong call order (run before partition, result before run) or poisoned ctx */
    GUM_ERANGE = -4, /* source >= V, or an SSSP distance reaches 2^32-1 */
    GUM_ECUDA = -5,  /* CUDA runtime error (context is poisoned) */
    GUM_ENCCL = -6,  /* multi-process exchange failed, or a peer never reached a barrier */
    GUM_EUNSUP = -7  /* configuration not supported by this build */
} gum_status;

/* Algorithms. Outputs (reading #1): BFS hop depth, SSSP distance (uint32 weights,
 * uint64 arithmetic), WCC = minimum ORIGINAL vertex id of the weakly connected component,
 * PR = x_K of the fixed-K power iteration with uniform dangling redistribution (fp64). */
/* GUM_DPR (NEXT-4, "delta-PageRank"): residual-push PageRank in frontier-driven rounds (DESIGN.md
 * reading #27): x -> x* = (I - d P^T)^{-1} (1-d)/V (dangling mass not redistributed), every vertex whose
 * residual exceeds eps = dpr_tolerance * (1-d)/V is active; output x as double[V], with
 * 0 <= x* - x and sum(x* - x) <= dpr_tolerance. */
typedef enum { GUM_BFS = 0, GUM_SSSP = 1, GUM_WCC = 2, GUM_PR = 3, GUM_DPR = 4 } gum_alg;

/* Partitioners (P:315, P:382 Exp-6): SEG = contiguous id ranges with ~equal out-edges; RANDOM =
 * keyed Feistel relabel of ids, then SEG (reading #17). metis is out of scope.
 * DEGREE (a B200 layout option, not in the paper): relabel ids by decreasing in-degree (ties by id), then
 * SEG -- the few destinations most edges point to share a few KB of every per-vertex array, so their
 * visited-bit / state probes hit L1/L2 instead of missing. Results are in original ids. */
typedef enum { GUM_PART_SEG = 0, GUM_PART_RANDOM = 1, GUM_PART_DEGREE = 2 } gum_part;

#define GUM_INF 0xFFFFFFFFu
#define GUM_MAX_WORKERS 8

/* gum_config.flags */
#define GUM_CFG_TRACE 0x1u        /* record a per-iteration, per-worker trace (gum_trace) */
#define GUM_CFG_HOST_LOOP 0x2u    /* drive iterations from the host instead of a CUDA-graph WHILE node */
#define GUM_CFG_FORCE_SPARSE 0x4u /* filter always compacts the activation list (never the bitmap) */
#define GUM_CFG_FORCE_DENSE 0x8u  /* filter always scans the bitmap */
#define GUM_CFG_SPLIT_UNITS 0x20u /* one launch unit (stream, control replica, kernels) per worker even
                                     when workers share a device: runs the multi-device code path
                                     (per-unit decisions, cross-unit barriers) on one GPU */
#define GUM_CFG_PROFILE 0x10u     /* host loop, one iteration per poll, CUDA events around every kernel
                                     launch (read back with gum_profile); for measurement only */

typedef struct {
    /* Workers = GPUs of the paper (one worker per GPU, one fragment per worker).
     * num_gpus fragments are created. device_ids[i] is worker i's CUDA device; NULL => every worker
     * on device 0 ("virtual peers": workers are disjoint CTA groups of one GPU, peer pointers are
     * local pointers -- the T3 fake backend of SURVEY.md §4). */
    int num_gpus;
    const int* device_ids;
    /* FSteal (§III) and its gating thresholds t1, t2 (P:248 Example 5): stealing is enabled in an
     * iteration only if max_i l_i >= t1 and max_i l_i - min_i l_i >= t2 (l_i = active edges).
     * fsteal = 0: off; 1: steal queue (idle workers claim chunks of the most loaded peer queue, the
     * default); 2: planned (NEXT-2): each iteration solves Eq. (1) on the uniform fabric (closed form,
     * see gum_fsteal_plan) and carves every queue into consecutive chunk ranges per worker (Alg. 1);
     * used while all workers own their fragment (no OSteal shrink), else falls back to the queue. */
    int fsteal;
    uint64_t t1_min_max_edges;
    uint64_t t2_min_spread_edges;
    /* OSteal (§IV): re-decided every iteration from the global counts. While the number of active
     * vertices is below osteal_active_threshold the active owners are the survivors {0..m'-1}
     * (uniform NVSwitch reduction tree, reading #13), m' = clamp(ceil(active_edges /
     * osteal_edges_per_worker), 1, num_gpus) (0 => m' = 1); above it ownership is given back.
     * Fragment f is owned by worker f if f < m', else by f mod m'.
     * osteal = 0: off; 1: this active-vertex threshold trigger (the north_star's rule, the default);
     * 2: the paper's cost model (NEXT-3, Alg. 2 P:188-211 with Eq. (4)): every iteration,
     * for m = 1..num_gpus, E(m) = z(m) + p*m with z(m) the Eq. (1) makespan when only workers {0..m-1}
     * process (evicted fragments' edges at the remote cost, see gum_osteal_plan) and p =
     * osteal_sync_edges (or its online estimate); the first m with the lowest E(m) becomes the active
     * owner set (shrinking or giving ownership back). */
    int osteal;
    uint64_t osteal_active_threshold;
    uint64_t osteal_edges_per_worker;
    /* Edges per claimable chunk of the edge-balanced steal queue (multiple of 32, <= 2048;
     * 0 => 2048). */
    uint32_t chunk_edges;
    int pr_iterations;   /* 0 => 20 */
    double pr_damping;   /* 0 => 0.85 */
    uint32_t max_iterations; /* safety cap on BSP iterations, 0 => 2^31 */
    uint32_t flags;      /* GUM_CFG_* */
    /* SSSP frontier split (near-far, Davidson et al. = the paper's ref [46]): activated vertices
     * with dist >= T are parked in a far set; when the near frontier empties T moves to
     * min(far dist) + sssp_delta and the far set is swept. 0 = plain BSP frontier (the paper's GUM).
     * Results are identical either way (unique fixpoint); only the amount of re-relaxation changes. */
    uint32_t sssp_delta;
    /* Long-tail engine = OSteal's m'=1 mode (needs osteal=1 and a single launch unit):
     * when the global frontier has <= tail_vertices vertices, worker 0 takes ownership of every
     * fragment and one cooperative persistent kernel runs iterations back to back with one grid
     * barrier each, until the frontier exceeds 4*tail_vertices or converges; ownership is then given
     * back. 0 = off; gum_config_default sets 16384 (C3: 8192 -> 16384 took 487 -> 309 ms). */
    uint32_t tail_vertices;
    /* BFS propagation blocking for dense iterations (single fragment): 17 = bin destination ids by
     * blocks of 2^17 and set visited bits per block in shared memory; 0 = off (the default: every edge
     * probes the visited bitmap directly, measured faster on B200). */
    uint32_t pb_block_log2;
    /* Planned FSteal: cost of processing a remote edge relative to a local one (c_ij / c_ii of
     * P:101-108 with uniform B_ij; 0 => 1). */
    double fsteal_remote_cost;
    /* NEXT-4 direction-optimising BFS (Beamer et al.): 1 = build the in-CSR at gum_prepare(BFS) and run
     * large-frontier iterations bottom-up (every unvisited vertex looks for a parent at the current
     * depth among its in-edges). Same depths; 0 = push only (the paper's GUM, the default). */
    int bfs_direction_opt;
    /* OSteal cost model (osteal = 2): p of Eq. (4), the per-worker synchronisation cost of one
     * iteration expressed in edge-processing time units (edges). > 0: this constant. 0 (default):
     * estimated during the run from previous iterations: p = S / (m * tau) with S the measured
     * non-advance time of an iteration and tau the advance time per edge and worker, averaged over
     * iterations (reading #23); 500000 until the first measurement. */
    double osteal_sync_edges;
    /* Optional device allocator (e.g. the PyTorch caching allocator) and per-worker streams. */
    void* (*alloc)(uint64_t bytes, int device, void* user);
    void (*free_fn)(void* ptr, uint64_t bytes, int device, void* user);
    void* alloc_user;
    void* const* streams; /* cudaStream_t per worker (NULL => library-owned non-blocking streams) */
    /* NEXT-1 communication reducers (§V-B "Optimizations"; only change anything when num_gpus > 1).
     * mirrors = 1: outer-vertex mirrors with early message aggregation ("the destination of
     * cross-fragment edges are also kept as outer vertices for message-aggregation optimization").
     * Every worker w keeps, in its own memory, a mirror of every vertex it does not own:
     *   PR:        a double[V] accumulator -- pushes to other fragments' vertices add into w's mirror
     *              (local red.add) instead of the owner's acc; the owner's finalize pulls and clears its
     *              slice of every peer mirror (one bulk read per iteration instead of one remote atomic
     *              per edge: an aggregated reduce-scatter over peer memory);
     *   BFS:       a bit[V] "already sent" filter -- a cross-fragment update is issued only the first time
     *              w discovers v (a set bit also caches "v is visited" seen in the owner's bitmap);
     *   SSSP/WCC:  a uint32[V] "minimum sent" value -- a cross-fragment update is issued only when the
     *              candidate beats every value w has sent to v before (the owner's value is <= it).
     * Results are unchanged (monotone min-fixpoints; PR sums the same terms in another order).
     * hub_cache = 1: hub adjacency caching (P:274 Example 6). At gum_prepare every worker copies the
     * adjacency lists (col, and weights for SSSP) of every other fragment's vertices with out-degree >
     * hub_degree (t4; 0 caches every list) into its own memory; a stolen (or OSteal-inherited) frontier
     * vertex whose list is cached is expanded from the local copy instead of the owner's CSR over
     * NVLink. BFS/SSSP/WCC (PR's static queue is destination-blocked; PR uses mirrors instead). */
    int mirrors;
    int hub_cache;
    uint32_t hub_degree;
    /* PageRank advance (a8 for PR). 0 (default): pull -- every vertex sums x[u]/outdeg(u) over its in-edges,
     * one pass per L2-sized block of sources, rows and edges balanced by merge path; the sum is the same
     * set of terms as the push ("PR pull"). 1: push -- one red.add.f64 of x[u]/outdeg(u) per
     * out-edge into the destination's accumulator (the GAS scatter of P:53; also used whenever mirrors = 1,
     * whose aggregation is a push). Results agree within the PR tolerance either way. */
    int pr_push;
    /* delta-PageRank (GUM_DPR): target L1 tolerance; the residual threshold is dpr_tolerance * (1-d)/V
     * (0 => 1e-6). Damping is pr_damping. */
    double dpr_tolerance;
    /* NEXT-3 copy-migration of evicted fragments' frontiers (P:238 Ex. 4 step 2: "the generated frontier
     * queue will directly be on another GPU"; "migrating the residual frontiers from victims").
     * 0 (default): an evicted fragment's queue, CSR and state stay in its GPU's memory and the new owner reads
     * them remotely ("extended memory"). 1: the owner's filter generates the evicted fragment's queue in a
     * foster buffer in the owner's own memory and the owner's advance reads it locally (state, bitmaps and
     * CSR stay remote; the CSR can be replicated with hub_cache = 1, hub_degree = 0). BFS/SSSP/WCC/DPR. */
    int osteal_migrate;
} gum_config;

/* Fills *cfg with the defaults: 1 worker, fsteal=1, osteal=1, t1=t2=0, osteal threshold 0 (off until
 * set), chunk 2048, PR 20 iterations d=0.85. */
void gum_config_default(gum_config* cfg);

typedef struct {
    uint32_t iterations;      /* BSP iterations executed (advance steps) */
    double ms;                /* device time of the run (CUDA events around the iteration loop) */
    uint64_t edges_expanded;  /* edges processed by advance, summed over iterations (own + stolen) */
    uint64_t edges_frontier;  /* sum over iterations of the frontier's out-edges (filter's count);
                                 conservation: == edges_expanded */
    uint64_t edges_stolen;    /* of edges_expanded, processed by a worker that does not own the chunk */
    uint64_t chunks_stolen;
    uint64_t chunks_total;
    uint64_t remote_updates;  /* atomic updates whose target fragment is not the processing worker's */
    uint64_t activations;     /* vertices appended to next frontiers */
    uint64_t vertices_frontier; /* sum over iterations of |f_k| (queue entries expanded) */
    uint32_t final_owners;    /* active owners at the end (OSteal) */
    uint32_t osteal_iteration;/* iteration of the last owner-set change (0 = never) */
    uint32_t tail_iterations; /* of `iterations`, run inside the tail engine */
    uint32_t bodies;          /* iteration bodies (filter/control/advance/tail launches) executed */
    double pr_last_residual;  /* PR: sum_v |x_K - x_{K-1}| */
    uint64_t kernel_launches; /* this process's kernel launches in the run: exact in host-loop and
                                 multi-process mode (incl. barrier kernels); CUDA-graph mode counts every
                                 body kernel once per executed WHILE iteration (iterations + 1) */
    uint64_t remote_filtered; /* NEXT-1 mirrors: cross-fragment updates absorbed by the local mirror
                                 (BFS/SSSP/WCC: not sent; PR: aggregated, then flushed in bulk) */
    uint64_t hub_cached_edges;/* NEXT-1 hub cache: edges of non-local fragments expanded from a local copy */
    uint64_t mirror_flush_bytes; /* PR mirrors: bytes the finalize read from peer mirrors */
    uint32_t blocked_iterations; /* WCC: iterations run on the static destination-blocked queue */
    uint32_t tail_overflows;  /* tail-engine hand-backs whose next list (no-dedupe mode) outgrew its buffer and
                                 went back to the regular path as a bitmap (0 in practice) */
    /* of edges_expanded / vertices_frontier (list entries) / activations: the share done inside the tail
     * engine (k_tail), so per-kernel byte counts can be attributed (bench.py roofline) */
    uint64_t tail_edges;
    uint64_t tail_vertices;
    uint64_t tail_activations;
    /* multi-unit runs in the device-resident loop (one CUDA graph per device / process): per launch
     * unit, the number of device barriers it arrived at and the iteration of its last arrival. A unit
     * evicted by OSteal stops arriving: its last arrival is the barrier right after the eviction. */
    uint32_t unit_barriers[GUM_MAX_WORKERS];
    uint32_t unit_last_iter[GUM_MAX_WORKERS];
    /* host-side launches of this process in the run (kernels + graph launches): in the device-resident
     * loops this does not depend on the number of iterations */
    uint64_t host_launches;
    /* OSteal cost model (osteal = 2): p of Eq. (4) used at the end of the run (edges) and the number of
     * iterations it was estimated from (0 = the configured / initial value) */
    double osteal_p;
    uint32_t osteal_p_samples;
    uint32_t pad1;
    /* NEXT-3 copy-migration: frontier-queue entries generated in a foster queue on an evicted fragment's owner */
    uint64_t migrated_queue_entries;
} gum_run_stats;

/* Per-iteration trace record (GUM_CFG_TRACE). Times are %globaltimer ns of the advance phase:
 * worker w's busy window is [t_start[w], t_end[w]] (min start / max end over its CTAs). */
typedef struct {
    uint64_t t_start[GUM_MAX_WORKERS];
    uint64_t t_end[GUM_MAX_WORKERS];
    uint64_t edges_own[GUM_MAX_WORKERS];    /* edges of chunks the worker owns, processed by it */
    uint64_t edges_stolen[GUM_MAX_WORKERS]; /* edges the worker processed from others' queues */
    uint64_t frontier_vertices;
    uint64_t frontier_edges;
    uint32_t owners;      /* active owners m in this iteration */
    uint32_t steal_ok;    /* FSteal gate open in this iteration */
} gum_iter_trace;

/* ---- lifecycle ------------------------------------------------------------------------------ */
gum_status gum_create(const gum_config* cfg, gum_ctx** out);
void gum_destroy(gum_ctx* ctx);
const char* gum_last_error(const gum_ctx* ctx);

/* ---- a1 graph setup ---------------------------------------------------------------------------
 * Host helper: stable counting sort of a raw edge multiset (src[i] -> dst[i], w[i]) into CSR
 * (self-loops and parallel edges kept). row_ptr: uint64[V+1]; col, wout:
 * uint32[E] (wout/w may be NULL). Caller-allocated outputs. OpenMP-parallel. */
gum_status gum_build_csr(uint32_t num_vertices, uint64_t num_edges, const uint32_t* src, const uint32_t* dst,
                         const uint32_t* w, uint64_t* row_ptr, uint32_t* col, uint32_t* wout);

/* Loads graph G = (V, E). row_ptr: uint64[V+1], monotone, row_ptr[0] = 0, row_ptr[V] = E;
 * col: uint32[E] destinations < V; weights: uint32[E] or NULL (required for SSSP).
 * flags: GUM_LOAD_DEVICE => the three pointers are device pointers on worker 0's device.
 * Copies everything; validates on the device (EINVAL on malformed input). Invalidates any previous
 * partition. */
#define GUM_LOAD_DEVICE 0x1u
gum_status gum_load_csr(gum_ctx* ctx, uint32_t num_vertices, uint64_t num_edges, const uint64_t* row_ptr,
                        const uint32_t* col_idx, const uint32_t* weights, uint32_t flags);

/* ---- a2 partition -----------------------------------------------------------------------------
 * n-way edge-cut: fragment g owns the relabelled id range [b_g, b_{g+1}) with ~E/n
 * out-edges and keeps global destination ids; per-fragment device CSR, state, bitmap, queues and
 * peer-visible control blocks are allocated on worker g's device. seed keys the RANDOM relabel. */
gum_status gum_partition(gum_ctx* ctx, gum_part kind, uint64_t seed);
/* Fragment bounds in relabelled id space: bounds[0..num_gpus]. */
gum_status gum_partition_bounds(const gum_ctx* ctx, uint32_t* bounds, int n);

/* Optional: build per-algorithm auxiliary structures outside the timed run (WCC: symmetric
 * out+in fragments; PR: nothing extra). gum_run calls it implicitly. */
gum_status gum_prepare(gum_ctx* ctx, gum_alg alg);

/* ---- a3..a11 the run ---------------------------------------------------------------------------
 * Runs algorithm alg from `source` (BFS/SSSP; ignored by WCC/PR) to convergence (BFS/SSSP/WCC:
 * global frontier empty; PR: pr_iterations iterations). Stream-ordered on the workers' streams;
 * returns after completion. stats may be NULL. ERANGE if source >= V or an SSSP distance
 * overflows; EINVAL if SSSP and no weights were loaded. */
gum_status gum_run(gum_ctx* ctx, gum_alg alg, uint32_t source, gum_run_stats* stats);

/* ---- a12 result --------------------------------------------------------------------------------
 * Writes the last run's output in ORIGINAL vertex ids into out (host): uint32[V] for BFS/SSSP/WCC,
 * double[V] for PR. out_bytes must be >= V * element size (EINVAL otherwise). */
gum_status gum_result(gum_ctx* ctx, void* out, uint64_t out_bytes);
/* Same, into a device buffer on worker 0's device. */
gum_status gum_result_device(gum_ctx* ctx, void* out_device, uint64_t out_bytes);

/* Copies up to max_records per-iteration trace records of the last run (GUM_CFG_TRACE). */
gum_status gum_trace(const gum_ctx* ctx, gum_iter_trace* out, uint32_t max_records, uint32_t* n_records);

/* Per-kernel device time of the last run, from CUDA events recorded on the launching stream around
 * every launch (only with GUM_CFG_PROFILE; one launch unit per process: single device, or this rank's
 * unit in multi-process mode). */
typedef struct {
    double filter_ms, control_ms, advance_ms, finalize_ms, init_ms, tail_ms;
    uint32_t filter_launches, control_launches, advance_launches, finalize_launches, init_launches, tail_launches;
} gum_kernel_times;
gum_status gum_profile(const gum_ctx* ctx, gum_kernel_times* out);

/* Host helper of the planned FSteal (NEXT-2): the LP relaxation of Eq. (1) for loads l[0..n)
 * with local cost 1 and remote cost remote_cost (uniform fabric). Writes X[i*n+j] = edges resident on
 * worker i assigned to worker j (row sums = loads) and *z = the min-max makespan. The device control
 * kernel runs the same routine each iteration. */
gum_status gum_fsteal_plan(const uint64_t* loads, int n, double remote_cost, double* X, double* z);

/* ---- multi-process mode: one process per GPU (SURVEY.md §8(b) "optional multi-process adapter",
 * §8(e); the paper runs one worker per GPU) ---------------------------------------------
 * Each of `world` processes owns fragment `rank` on CUDA device `device`. Peers' fragment arrays are
 * mapped into every process with CUDA IPC (cudaIpcGetMemHandle / cudaIpcOpenMemHandle), so the
 * advance's remote updates (a9), frontier steals (a7) and OSteal's "extended memory" reads (a6)
 * are the same one-sided loads/atomics as in single-process mode. The per-phase barrier (a10) is a
 * device-side signal-pad barrier (fence.sys + st.release.sys of an epoch into every peer's pad, then
 * ld.acquire.sys spin on the local pad); no collective is on the data path.
 *
 * exchange: host all-gather supplied by the caller (e.g. a torch.distributed gloo group). Every rank
 * passes `bytes` bytes in `send`; on return `recv` holds world*bytes bytes, rank r's block at
 * r*bytes. Returns 0 on success, nonzero on failure (reported as GUM_ENCCL). The library calls it
 * from gum_create_mp, gum_partition, gum_prepare/gum_run (handle exchange, convergence agreement once
 * per launch batch -- the "global convergence flag" of the north_star) and gum_destroy. */
typedef int (*gum_exchange_fn)(const void* send, uint64_t bytes, void* recv, void* user);
typedef struct {
    int rank;                 /* this process's worker id in [0, world) */
    int world;                /* number of processes == cfg->num_gpus, 1..GUM_MAX_WORKERS */
    int device;               /* CUDA device of this process */
    gum_exchange_fn exchange; /* host all-gather (required) */
    void* user;               /* passed to exchange */
} gum_mp_config;

/* Host-only (no GPU needed): all-gathers {magic, library version, ABI struct sizes, rank, world, hash of
 * every semantic gum_config field} and checks that the ranks form a permutation of [0, world), that
 * cfg->num_gpus == world on every rank and that every rank runs the same library and configuration.
 * Returns GUM_OK on every rank or the same error on every rank (GUM_EINVAL on mismatch, GUM_ENCCL if
 * the exchange fails). gum_create_mp calls it first. */
gum_status gum_mp_handshake(const gum_config* cfg, const gum_mp_config* mp);

/* Collective: creates this rank's context (fragment `rank` on `mp->device`). cfg->num_gpus must equal
 * mp->world; cfg->device_ids and cfg->alloc must be NULL (IPC needs whole cudaMalloc allocations).
 * Afterwards every ABI call is collective and must be made by all ranks with the same arguments:
 * gum_load_csr (every rank loads the whole graph; validated against the peers at gum_partition),
 * gum_partition (each rank builds and keeps only its own fragment, then the fragments are
 * IPC-exchanged), gum_prepare, gum_run (each rank drives its own unit; stats->ms is this rank's device
 * time -- take the max over ranks), gum_result (every rank gathers the full result through the peer
 * mappings), gum_destroy. GUM_CFG_PROFILE runs the host-driven loop and times this rank's kernels. */
gum_status gum_create_mp(const gum_config* cfg, const gum_mp_config* mp, gum_ctx** out);

/* Host helper of the OSteal cost model (NEXT-3): Alg. 2 over m = 1..n for per-fragment loads l[0..n)
 * (active edges), remote cost b (local 1) and sync cost p (edges). cost[m-1] = E(m) = z(m) + p*m
 * (nullable); *m_out = the chosen cluster size. The device control kernel runs the same routine. */
gum_status gum_osteal_plan(const uint64_t* loads, int n, double remote_cost, double p, double* cost, int* m_out);

/* Library version (major*10000 + minor*100 + patch). */
int gum_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GUM_H */
