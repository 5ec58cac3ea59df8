// Host runtime behind the C ABI (include/gum.h): context, device fragments, partition, the
// iteration driver (CUDA-graph WHILE loop, or host loop with launch batches) and result/stat
// readback. PAPER.md lines as P:<line>; SURVEY.md §8(b) is the ABI contract.
#include <cuda_runtime.h>
#include <omp.h>

#include <algorithm>
#include <cstdarg>
#include <map>
#include <utility>
#include <cstdio>
#include <cstring>
#include <ctime>
#include <cstdlib>
#include <string>
#include <vector>

#include "gum.h"
#include "gum_internal.h"
#include "kernels.h"
#include "planner.h"

using namespace gum;
#ifdef GUM_FILTER_TIMING
namespace gum { void dump_filter_timing(); }
#endif

namespace {

struct Alloc {
    void* p;
    size_t bytes;
    int dev;
};

struct FragBufs {
    int dev = 0;
    unsigned V = 0, base = 0;
    unsigned long long E = 0, sE = 0;
    unsigned long long* row_ptr = nullptr;
    unsigned* col = nullptr;
    unsigned* w = nullptr;
    unsigned long long* s_row_ptr = nullptr;
    unsigned* s_col = nullptr;
    unsigned* orig = nullptr;
    unsigned* state = nullptr;
    double* x = nullptr;
    double* acc = nullptr;
    unsigned* bm = nullptr;
    unsigned* vis = nullptr;
    unsigned* bm2 = nullptr;
    unsigned* far = nullptr;
    unsigned* farl = nullptr;  // SSSP near-far: [2][V] far lists (gum_prepare(SSSP) with sssp_delta)
    unsigned* app = nullptr;
    unsigned* q_v = nullptr;
    unsigned long long* q_off = nullptr;
    long long* q_base = nullptr;
    unsigned* tile = nullptr;
    unsigned long long tile_cap = 0;
    FragCtl* ctl = nullptr;
    double* cx = nullptr;
    // PR static destination-blocked queue (gum_prepare(PR))
    unsigned* pr_col = nullptr;
    unsigned* pr_q_v = nullptr;
    unsigned long long* pr_q_off = nullptr;
    unsigned* pr_tile = nullptr;
    unsigned long long pr_qlen = 0, pr_qedges = 0;
    unsigned* pr2_q_v = nullptr;             // PR single fragment: pieces of <= kPrPiece edges (k_pr_push)
    unsigned long long* pr2_q_off = nullptr;
    unsigned long long pr2_len = 0;
    // WCC iteration-0 static destination-blocked queue over the symmetric graph
    unsigned* sq_col = nullptr;
    unsigned* sq_q_v = nullptr;
    unsigned long long* sq_q_off = nullptr;
    unsigned* sq_tile = nullptr;
    unsigned long long sq_len = 0, sq_edges = 0;
    // BFS propagation blocking
    unsigned long long* in_row_ptr = nullptr;  // bottom-up BFS in-CSR
    unsigned* in_col = nullptr;
    unsigned long long* pb_off = nullptr;
    unsigned* pb_fill = nullptr;
    unsigned* pb_done = nullptr;
    unsigned* pb_buf = nullptr;
    // NEXT-1 outer-vertex mirror of this worker (V entries of 8 B; PR acc / BFS bits / SSSP-WCC min alias it)
    void* mbuf = nullptr;
    // PR pull (gum_prepare(PR) without pr_push): source-block-major in-edges + merge-path tile table
    unsigned* pl_off = nullptr;
    unsigned* pl_col = nullptr;
    unsigned* pl_tx = nullptr;
    unsigned long long* pl_tb = nullptr;
};

// NEXT-1 hub cache: worker w's copy of fragment f's hub lists
struct HubBufs {
    unsigned long long* off = nullptr;
    unsigned* col = nullptr;
    unsigned* w = nullptr;
};

}  // namespace

struct gum_ctx {
    gum_config cfg{};
    int P = 1;
    int dev[kMaxW] = {0};
    bool single_device = true;
    bool split = false;  // one launch unit per worker (multi-device, or GUM_CFG_SPLIT_UNITS on one device)
    int n_units = 1;
    cudaStream_t stream[kMaxW] = {nullptr};
    bool own_stream[kMaxW] = {false};
    int nsm = 148;
    int tail_occ = 1;
    int filter_occ = 2;
    int adv_occ[kNumAlgs][2] = {{4, 4}, {4, 4}, {4, 4}, {4, 4}, {4, 4}};  // advance CTAs per SM by [alg][multi]
    int pr_push_occ = 8;
    int pull_occ = 4;
    std::string err;
    bool poisoned = false;
    std::vector<Alloc> load_allocs, part_allocs, misc_allocs;
    // loaded graph (worker 0's device)
    bool loaded = false;
    unsigned V = 0;
    unsigned long long E = 0;
    bool has_w = false;
    unsigned long long* g_row_ptr = nullptr;
    unsigned* g_col = nullptr;
    unsigned* g_w = nullptr;
    // partition
    bool partitioned = false;
    int part_kind = GUM_PART_SEG;
    unsigned long long seed = 0;
    unsigned bounds[kMaxW + 1] = {0};
    unsigned* inv = nullptr;  // relabelled id -> original id (RANDOM, DEGREE)
    unsigned* perm = nullptr; // original id -> relabelled id (DEGREE; RANDOM computes it with the Feistel map)
    unsigned long long* p_row_ptr = nullptr;  // the partitioned global CSR (relabelled or original)
    unsigned* p_col = nullptr;
    unsigned* p_w = nullptr;
    bool sym_ready = false;
    bool pr_ready = false;
    bool pb_ready = false;
    bool in_ready = false;
    bool pl_ready = false;  // PR pull structures built (else PR pushes)
    unsigned pl_B = 0;      // PR pull: source-block passes per iteration
    double* cxg[kMaxW] = {nullptr};  // PR pull: per unit, replica of x/outdeg [2][V] (global ids)
    unsigned pb_shift = 0, pb_nb = 0;
    int pr_blocks = 1;
    FragBufs fr[kMaxW];
    unsigned long long* s_rp_g = nullptr;  // global symmetric CSR (WCC), kept for the hub cache
    unsigned* s_col_g = nullptr;
    int hub_kind = 0;                      // hub cache built from: 0 none, 1 out-CSR (BFS/SSSP), 2 symmetric (WCC)
    HubBufs hub[kMaxW][kMaxW];             // [worker][fragment]
    QPtrs fq[kMaxW][kMaxW] = {};           // NEXT-3 copy-migration: foster queues [owner][fragment > owner]
    unsigned long long fq_tile_cap[kMaxW][kMaxW] = {};
    unsigned long long fq_key = 0;         // edge counts the foster queues are sized for (same on every rank)
    std::vector<Alloc> hub_allocs;
    unsigned long long hub_entries = 0;    // cached list entries per worker copy set (stats / tests)
    unsigned long long n_dangling = 0;
    RunCtl* rctl[kMaxW] = {nullptr};
    LBSlot* lb[kMaxW] = {nullptr};
    unsigned lb_parts = 0;
    gum_iter_trace* trace[kMaxW] = {nullptr};
    TailSplit* tsplit[kMaxW] = {nullptr};
    RunCtl* h_rctl = nullptr;  // pinned
    void* d_res = nullptr;
    cudaGraphExec_t gexec[kNumAlgs] = {};
    cudaGraphExec_t gexec_u[kNumAlgs][kMaxW] = {};  // device-resident multi-unit loop: one graph per unit
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    std::vector<cudaEvent_t> bar_ev;
    std::vector<cudaEvent_t> prof_ev;  // pairs (start, end)
    std::vector<int> prof_kind;
    gum_kernel_times prof{};
    int last_alg = -1;
    bool has_result = false;
    unsigned last_iters = 0;
    // multi-process mode (gum_create_mp): this process is worker/unit `rank`; every other fragment's
    // arrays are CUDA-IPC mappings of the peer process's allocations.
    bool mp = false;
    int rank = 0;
    gum_exchange_fn xch = nullptr;
    void* xuser = nullptr;
    unsigned long long* pad[kMaxW] = {nullptr};  // per unit: signal pad (epochs by unit + timeout flag)
    unsigned long long mp_epoch = 0;
    unsigned long long launches = 0;  // kernel launches of the current run (gum_run_stats.kernel_launches)
    unsigned long long hlaunch = 0;   // host-side launches (kernels + graphs) of the current run
    std::map<std::pair<int, unsigned long long>, void*> ipc_map;  // (peer, peer pointer) -> mapped pointer
};

namespace {

gum_status fail(gum_ctx* c, gum_status st, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    if (c) {
        c->err = buf;
        if (st == GUM_ECUDA) c->poisoned = true;
    }
    return st;
}

#define CK(call)                                                                                  \
    do {                                                                                          \
        cudaError_t e_ = (call);                                                                  \
        if (e_ != cudaSuccess) return fail(c, GUM_ECUDA, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), \
                                           __FILE__, __LINE__);                                   \
    } while (0)

void* dalloc(gum_ctx* c, int dev, size_t bytes, std::vector<Alloc>& list) {
    bytes = std::max<size_t>(bytes, 256);
    bytes = (bytes + 255) & ~size_t(255);
    void* p = nullptr;
    if (c->cfg.alloc) {
        p = c->cfg.alloc(bytes, dev, c->cfg.alloc_user);
    } else {
        cudaSetDevice(dev);
        if (cudaMalloc(&p, bytes) != cudaSuccess) {
            cudaGetLastError();
            p = nullptr;
        }
    }
    if (p) list.push_back({p, bytes, dev});
    return p;
}

void free_list(gum_ctx* c, std::vector<Alloc>& list) {
    for (auto& a : list) {
        if (c->cfg.free_fn) {
            c->cfg.free_fn(a.p, a.bytes, a.dev, c->cfg.alloc_user);
        } else {
            cudaSetDevice(a.dev);
            cudaFree(a.p);
        }
    }
    list.clear();
}

// ---- multi-process mode helpers ------------------------------------------------------------------
gum_status mp_exchange(gum_ctx* c, const void* send, size_t bytes, void* recv) {
    if (c->xch(send, bytes, recv, c->xuser) != 0) return fail(c, GUM_ENCCL, "multi-process exchange failed");
    return GUM_OK;
}

// host barrier of all ranks (an all-gather of one word)
gum_status mp_host_barrier(gum_ctx* c) {
    unsigned long long me = 1, all[kMaxW];
    return mp_exchange(c, &me, sizeof(me), all);
}

void mp_close_maps(gum_ctx* c) {
    for (auto& kv : c->ipc_map) cudaIpcCloseMemHandle(kv.second);
    c->ipc_map.clear();
    cudaGetLastError();
}

void drop_graphs(gum_ctx* c) {
    for (auto& g : c->gexec) {
        if (g) cudaGraphExecDestroy(g);
        g = nullptr;
    }
    for (auto& row : c->gexec_u)
        for (auto& g : row) {
            if (g) cudaGraphExecDestroy(g);
            g = nullptr;
        }
}

void drop_partition(gum_ctx* c) {
    drop_graphs(c);
    for (int d = 0; d < c->P; d++) {
        cudaSetDevice(c->dev[d]);
        cudaStreamSynchronize(c->stream[d]);
    }
    if (c->mp && c->partitioned) {
        // peers may still read or update this rank's fragment until they are done with it: collective
        mp_host_barrier(c);
        mp_close_maps(c);
        mp_host_barrier(c);
    }
    c->mp_epoch = 0;
    for (auto& p : c->pad) p = nullptr;
    free_list(c, c->hub_allocs);
    c->hub_kind = 0;
    c->hub_entries = 0;
    for (auto& row : c->hub)
        for (auto& h : row) h = HubBufs{};
    for (int i = 0; i < kMaxW; i++)
        for (int j = 0; j < kMaxW; j++) {
            c->fq[i][j] = QPtrs{};
            c->fq_tile_cap[i][j] = 0;
        }
    c->fq_key = 0;
    c->s_rp_g = nullptr;
    c->s_col_g = nullptr;
    free_list(c, c->part_allocs);
    c->partitioned = false;
    c->sym_ready = false;
    c->pr_ready = false;
    c->pb_ready = false;
    c->in_ready = false;
    c->pl_ready = false;
    c->pl_B = 0;
    for (auto& p : c->cxg) p = nullptr;
    c->pb_shift = c->pb_nb = 0;
    c->has_result = false;
    c->inv = nullptr;
    c->perm = nullptr;
    c->p_row_ptr = nullptr;
    c->p_col = nullptr;
    c->p_w = nullptr;
    for (auto& f : c->fr) f = FragBufs{};
    for (int i = 0; i < kMaxW; i++) {
        c->rctl[i] = nullptr;
        c->lb[i] = nullptr;
        c->trace[i] = nullptr;
        c->tsplit[i] = nullptr;
    }
    c->d_res = nullptr;
}

// unit u covers workers [unit_w0(u), unit_w0(u)+unit_nw(u))
int unit_w0(const gum_ctx* c, int u) { return c->split ? u : 0; }
int unit_nw(const gum_ctx* c, int u) { return c->split ? 1 : c->P; }
int unit_dev(const gum_ctx* c, int u) { return c->dev[unit_w0(c, u)]; }
// multi-process mode: only this process's unit and fragment are built and launched here
bool unit_local(const gum_ctx* c, int u) { return !c->mp || u == c->rank; }
bool frag_local(const gum_ctx* c, int f) { return !c->mp || f == c->rank; }
int home_unit(const gum_ctx* c) { return c->mp ? c->rank : 0; }

LaunchCfg make_launch(const gum_ctx* c, int u, int alg) {
    LaunchCfg L;
    L.w0 = unit_w0(c, u);
    L.nw = unit_nw(c, u);
    int grid = c->nsm * c->adv_occ[alg][c->P > 1 ? 1 : 0];
    grid = (grid / L.nw) * L.nw;
    if (grid < L.nw) grid = L.nw;
    L.adv_grid = grid;
    // clamped to 8: lb_parts (one look-back slot per filter CTA) is sized for nsm * 8 CTAs
    static const int filter_per_sm = getenv("GUM_FILTER_CTAS_PER_SM") ? std::min(8, std::max(1, atoi(getenv("GUM_FILTER_CTAS_PER_SM")))) : 0;
    L.filter_grid = std::max(1, (c->nsm * (filter_per_sm ? filter_per_sm : c->filter_occ)) /
                                    (c->single_device ? std::min(c->P, 4) : 1));
    if (c->split && c->single_device) L.adv_grid = std::max(1, L.adv_grid / c->P);
    L.fin_grid = std::max(1, (c->nsm * 4) / L.nw);
    L.init_grid = std::max(1, (c->nsm * 4) / L.nw);
    // the tail engine (OSteal's m'=1 mode) runs on unit 0 over every fragment; with several units on one
    // device one CTA slot per SM is left for the parked units' barrier kernels (co-residency of the
    // cooperative grid)
    // (the host-driven multi-unit loop has no run-control hand-over between units, so it keeps the tail engine
    // off: the other units' iteration counters would not follow the engine's iterations)
    const bool tail_ok = c->n_units == 1 || !(c->cfg.flags & (GUM_CFG_HOST_LOOP | GUM_CFG_PROFILE));
    L.tail_grid = (u == 0 && tail_ok && c->cfg.tail_vertices && alg != GUM_PR && alg != GUM_DPR)
                      ? c->nsm * ((c->split && c->single_device && c->tail_occ > 1) ? c->tail_occ - 1 : c->tail_occ)
                      : 0;
    L.adv_grid_pr = c->nsm * c->pr_push_occ;
    L.pull_grid = std::max(1, (c->nsm * c->pull_occ) / L.nw);
    return L;
}

DevCtx make_devctx(const gum_ctx* c, int alg) {
    DevCtx d;
    memset(&d, 0, sizeof(d));
    for (int f = 0; f < c->P; f++) {
        const FragBufs& F = c->fr[f];
        FragPtrs& p = d.f[f];
        if (alg == GUM_WCC) {
            p.row_ptr = F.s_row_ptr;
            p.col = F.s_col;
            p.E = F.sE;
        } else {
            p.row_ptr = F.row_ptr;
            p.col = F.col;
            p.E = F.E;
        }
        p.w = F.w;
        p.state = F.state;
        p.x = F.x;
        p.acc = F.acc;
        p.cx = F.cx;
        p.pb_off = F.pb_off;
        p.pb_fill = F.pb_fill;
        p.pb_done = F.pb_done;
        p.pb_buf = F.pb_buf;
        p.in_row_ptr = F.in_row_ptr;
        p.in_col = F.in_col;
        if (alg == GUM_WCC && F.sq_col) {
            p.sq_col = F.sq_col;
            p.sq_q_v = F.sq_q_v;
            p.sq_q_off = F.sq_q_off;
            p.sq_tile = F.sq_tile;
            p.sq_len = F.sq_len;
            p.sq_edges = F.sq_edges;
        }
        p.orig = F.orig;
        p.bm = F.bm;
        p.vis = F.vis;
        p.bm2 = F.bm2;
        p.far = F.far;
        p.farl = (alg == GUM_SSSP) ? F.farl : nullptr;
        p.app = F.app;
        p.q_v = F.q_v;
        p.q_off = F.q_off;
        p.q_base = F.q_base;
        p.tile = F.tile;
        if (alg == GUM_PR) {
            p.col = F.pr_col;
            p.q_v = F.pr_q_v;
            p.q_off = F.pr_q_off;
            p.q_base = nullptr;
            p.tile = F.pr_tile;
            p.pr_qlen = F.pr_qlen;
            p.pr_qedges = F.pr_qedges;
            p.pr2_q_v = F.pr2_q_v;
            p.pr2_q_off = F.pr2_q_off;
            p.pr2_len = F.pr2_len;
        }
        p.ctl = F.ctl;
        p.V = F.V;
        p.base = F.base;
        if (alg == GUM_PR && c->pl_ready) {
            p.pl_off = F.pl_off;
            p.pl_col = F.pl_col;
            p.pl_tx = F.pl_tx;
            p.pl_tb = F.pl_tb;
        }
        p.macc = (double*)F.mbuf;
        p.msent = (unsigned*)F.mbuf;
        p.mmin = (unsigned*)F.mbuf;
        d.lb[f] = c->lb[f];
    }
    d.mirrors = (c->cfg.mirrors && c->P > 1 && c->fr[0].mbuf && alg != GUM_DPR) ? 1 : 0;
    d.migrate = (c->cfg.osteal_migrate && c->P > 1 && alg != GUM_PR) ? 1 : 0;
    for (int o = 0; o < c->P && d.migrate; o++)
        for (int f = o + 1; f < c->P; f++) d.fq[o][f] = c->fq[o][f];
    if (alg == GUM_PR && c->pl_ready) {
        // one replica of x/outdeg per launch unit; worker w pulls from its unit's
        d.pl_B = c->pl_B;
        d.n_rep = c->n_units;
        for (int u = 0; u < c->n_units; u++) d.cxrep[u] = c->cxg[unit_w0(c, u)];
        for (int w = 0; w < c->P; w++) d.cxw[w] = c->cxg[unit_w0(c, c->split ? w : 0)];
    }
    const int hk = alg == GUM_WCC ? 2 : ((alg == GUM_PR || alg == GUM_DPR) ? -1 : 1);
    d.hub_on = (c->hub_kind == hk) ? 1 : 0;
    for (int w = 0; w < c->P && d.hub_on; w++)
        for (int f = 0; f < c->P; f++) {
            d.hub[w][f].off = c->hub[w][f].off;
            d.hub[w][f].col = c->hub[w][f].col;
            d.hub[w][f].w = c->hub[w][f].w;
        }
    for (int w = 0; w < c->P; w++) {
        int u = c->split ? w : 0;
        d.rctl[w] = c->rctl[unit_w0(c, u)];
        d.trace[w] = c->trace[unit_w0(c, u)];
        d.tsplit[w] = c->tsplit[unit_w0(c, u)];
    }
    d.lb_parts = c->lb_parts;
    d.n_units = c->n_units;
    for (int u = 0; u < c->n_units; u++) d.pad[u] = c->pad[unit_w0(c, u)];
    d.units_dev = (c->n_units > 1 && !(c->cfg.flags & (GUM_CFG_HOST_LOOP | GUM_CFG_PROFILE))) ? 1 : 0;
    d.alg = alg;
    // control fused into the filter's last CTA: measured no faster on C2 (1.589 vs 1.570 ms per run), opt-in
    static const int env_fc = getenv("GUM_FUSE_CONTROL") ? atoi(getenv("GUM_FUSE_CONTROL")) : 0;
    d.fuse_ctl = (env_fc && c->n_units == 1 && alg != GUM_PR && !(c->cfg.flags & (GUM_CFG_HOST_LOOP | GUM_CFG_PROFILE))) ? 1 : 0;
    for (int i = 0; i <= c->P; i++) d.bounds[i] = c->bounds[i];
    d.P = c->P;
    d.chunk = c->cfg.chunk_edges;
    d.num_vertices = c->V;
    d.fsteal = c->cfg.fsteal;
    d.remote_cost = c->cfg.fsteal_remote_cost > 0.0 ? c->cfg.fsteal_remote_cost : 1.0;
    d.osteal = c->cfg.osteal;
    d.os_p = c->cfg.osteal_sync_edges > 0.0 ? c->cfg.osteal_sync_edges : 500000.0;
    d.os_p_online = c->cfg.osteal_sync_edges > 0.0 ? 0 : 1;  // 0 => estimated online (initial 500K)
    d.t1 = c->cfg.t1_min_max_edges;
    d.t2 = c->cfg.t2_min_spread_edges;
    d.os_thresh = c->cfg.osteal_active_threshold;
    d.os_epw = c->cfg.osteal_edges_per_worker;
    d.max_iter = c->cfg.max_iterations ? c->cfg.max_iterations : 0x7FFFFFFFu;
    d.pr_iters = c->cfg.pr_iterations;
    d.pr_d = c->cfg.pr_damping;
    d.dpr_eps = (c->cfg.dpr_tolerance > 0.0 ? c->cfg.dpr_tolerance : 1e-6) * (1.0 - c->cfg.pr_damping) / (double)c->V;
    d.force_mode = (c->cfg.flags & GUM_CFG_FORCE_DENSE) ? 2u : ((c->cfg.flags & GUM_CFG_FORCE_SPARSE) ? 1u : 0u);
    d.dense_div = 32;
    d.nf_delta = alg == GUM_SSSP ? c->cfg.sssp_delta : 0u;
    d.tail_enter = (alg != GUM_PR && alg != GUM_DPR && (c->n_units == 1 || !(c->cfg.flags & (GUM_CFG_HOST_LOOP | GUM_CFG_PROFILE))))
                       ? c->cfg.tail_vertices
                       : 0u;
    d.tail_exit = 4u * c->cfg.tail_vertices;
    // local relaxation rounds per CTA before each grid barrier of the tail engine (SSSP/WCC, one fragment):
    // C3 8192^2 grid 252 -> 241 ms at 6 rounds; the tail is bound by the per-hop chain of dependent loads,
    // not by the barriers (4096^2: 10186 -> 1281 engine iterations at 8 rounds, 103 -> 91 ms)
    // (32 rounds with the no-dedupe engine: C3 157.2 -> 153.6 ms at threshold 32768; ab_c3_tail_sweep.txt)
    static const int env_tl = getenv("GUM_TAIL_LOCAL") ? atoi(getenv("GUM_TAIL_LOCAL")) : 32;
    d.tail_local = (unsigned)std::max(0, env_tl);
    // tail engine without next-list dedupe bits (improvement = returning atomicMin): C3 208.9 -> 158.3 ms
    static const int env_nd = getenv("GUM_TAIL_NODEDUPE") ? atoi(getenv("GUM_TAIL_NODEDUPE")) : 1;
    d.tail_nodedupe = env_nd ? 1u : 0u;
    static const long long env_sl = getenv("GUM_TAIL_SLACK") ? atoll(getenv("GUM_TAIL_SLACK")) : (long long)kTailSlack;
    d.tail_slack = (unsigned)std::min<long long>(std::max(0ll, env_sl), (long long)kTailSlack);
    d.pb_shift = (alg == GUM_BFS && c->pb_ready) ? c->pb_shift : 0u;
    d.pb_nb = c->pb_nb;
    d.bfs_pull = (alg == GUM_BFS && c->in_ready) ? 1u : 0u;
    static const int env_sw = getenv("GUM_FILTER_SWIZZLE") ? atoi(getenv("GUM_FILTER_SWIZZLE")) : 1;
    d.filter_swizzle = env_sw ? 1u : 0u;
    // one-pass filter (queue ranges reserved per tile with one packed atomic): needs every fragment's queue
    // length < 2^27 and out-edges (symmetric for WCC) < 2^37, the packed counter's two fields
    static const int env_op = getenv("GUM_FILTER_ONEPASS") ? atoi(getenv("GUM_FILTER_ONEPASS")) : 1;
    bool op_fits = true;
    for (int f = 0; f < c->P; f++)
        op_fits = op_fits && c->fr[f].V < (1ull << (64 - kFpackShift)) &&
                  std::max(c->fr[f].E, c->fr[f].sE) <= kFpackEdgeMask;
    d.filter_onepass = (env_op && op_fits) ? 1u : 0u;
    d.bfs_filter_depth = alg == GUM_BFS ? 1u : 0u;  // (the advance no longer writes BFS depths)
    static const int env_wb = getenv("GUM_WCC_BLOCKED") ? atoi(getenv("GUM_WCC_BLOCKED")) : 1;
    d.wcc_blocked = (alg == GUM_WCC && c->fr[0].sq_col && c->cfg.fsteal != 2 && env_wb) ? 1u : 0u;
    for (int f = 0; f < c->P; f++) d.total_edges += c->fr[f].E;
    return d;
}

gum_status sync_all(gum_ctx* c) {
    for (int u = 0; u < c->n_units; u++) {
        if (!unit_local(c, u)) continue;
        CK(cudaSetDevice(unit_dev(c, u)));
        CK(cudaStreamSynchronize(c->stream[unit_w0(c, u)]));
    }
    return GUM_OK;
}

// cross-unit barrier (multi-device, single process): every unit's stream waits for every other's.
// multi-process: a device-side signal-pad barrier on this rank's stream (a10; kernels.cu k_mp_barrier)
gum_status unit_barrier(gum_ctx* c) {
    if (c->n_units == 1) return GUM_OK;
    if (c->mp) {
        MpPads p;
        memset(&p, 0, sizeof(p));
        for (int i = 0; i < c->P; i++) p.pad[i] = c->pad[i];
        CK(cudaSetDevice(c->dev[c->rank]));
        CK(launch_mp_barrier(p, c->P, c->rank, ++c->mp_epoch, c->stream[c->rank]));
        c->launches++;
        return GUM_OK;
    }
    for (int u = 0; u < c->n_units; u++) {
        CK(cudaSetDevice(unit_dev(c, u)));
        CK(cudaEventRecord(c->bar_ev[u], c->stream[unit_w0(c, u)]));
    }
    for (int u = 0; u < c->n_units; u++) {
        CK(cudaSetDevice(unit_dev(c, u)));
        for (int v = 0; v < c->n_units; v++)
            if (v != u) CK(cudaStreamWaitEvent(c->stream[unit_w0(c, u)], c->bar_ev[v], 0));
    }
    return GUM_OK;
}

// Multi-process: the device buffers of fragment f that peers map (everything a kernel may touch after
// OSteal hands the fragment to another worker), plus the unit's run control, trace and signal pad.
constexpr int kMpFields = 88;
int mp_fields(gum_ctx* c, int f, void** out[kMpFields]) {
    FragBufs& F = c->fr[f];
    int n = 0;
#define GUM_FLD(x) out[n++] = (void**)&(x)
    GUM_FLD(F.row_ptr); GUM_FLD(F.col); GUM_FLD(F.w); GUM_FLD(F.s_row_ptr); GUM_FLD(F.s_col); GUM_FLD(F.orig);
    GUM_FLD(F.state); GUM_FLD(F.x); GUM_FLD(F.acc); GUM_FLD(F.cx); GUM_FLD(F.bm); GUM_FLD(F.vis); GUM_FLD(F.bm2);
    GUM_FLD(F.far); GUM_FLD(F.app); GUM_FLD(F.q_v); GUM_FLD(F.q_off); GUM_FLD(F.q_base); GUM_FLD(F.tile);
    GUM_FLD(F.ctl); GUM_FLD(F.pr_col); GUM_FLD(F.pr_q_v); GUM_FLD(F.pr_q_off); GUM_FLD(F.pr_tile);
    GUM_FLD(F.sq_col); GUM_FLD(F.sq_q_v); GUM_FLD(F.sq_q_off); GUM_FLD(F.sq_tile); GUM_FLD(F.in_row_ptr);
    GUM_FLD(F.in_col); GUM_FLD(c->lb[f]); GUM_FLD(c->rctl[f]); GUM_FLD(c->trace[f]); GUM_FLD(c->pad[f]);
    GUM_FLD(F.mbuf); GUM_FLD(F.farl); GUM_FLD(F.pl_off); GUM_FLD(F.pl_col); GUM_FLD(F.pl_tx); GUM_FLD(F.pl_tb); GUM_FLD(c->cxg[f]);
    for (int g = 0; g < kMaxW; g++) {  // worker f's foster queues (NEXT-3 copy-migration)
        GUM_FLD(c->fq[f][g].q_v); GUM_FLD(c->fq[f][g].q_off); GUM_FLD(c->fq[f][g].q_base); GUM_FLD(c->fq[f][g].tile);
    }
#undef GUM_FLD
    return n;
}

struct MpBlob {
    unsigned magic, status, rank, nfields;
    unsigned long long V, E, bounds_hash, pr_qlen, sq_len, sE, tile_cap, pad0;
    unsigned long long ptr[kMpFields];
    cudaIpcMemHandle_t h[kMpFields];
};
constexpr unsigned kMpMagic = 0x47554d31u;  // "GUM1"

unsigned long long hash_words(const void* p, size_t n, unsigned long long h = 1469598103934665603ull) {
    const unsigned char* b = (const unsigned char*)p;
    for (size_t i = 0; i < n; i++) h = (h ^ b[i]) * 1099511628211ull;
    return h;
}

// Collective: publishes this rank's fragment buffers (IPC handles) and scalars, maps every peer's.
// local_st = this rank's status of the step just done; if any rank failed, every rank returns an error.
gum_status mp_publish(gum_ctx* c, gum_status local_st) {
    if (!c->mp) return local_st;
    cudaSetDevice(c->dev[c->rank]);
    if (cudaDeviceSynchronize() != cudaSuccess && local_st == GUM_OK)  // pads/ctl zeroed before peers map them
        local_st = fail(c, GUM_ECUDA, "device synchronize before the fragment exchange failed");
    std::vector<MpBlob> all(c->P);
    MpBlob me;
    memset(&me, 0, sizeof(me));
    me.magic = kMpMagic;
    me.rank = (unsigned)c->rank;
    void** fl[kMpFields];
    const int nf = mp_fields(c, c->rank, fl);
    me.nfields = (unsigned)nf;
    if (local_st == GUM_OK) {
        cudaSetDevice(c->dev[c->rank]);
        for (int i = 0; i < nf; i++) {
            void* p = *fl[i];
            me.ptr[i] = (unsigned long long)(uintptr_t)p;
            if (p && cudaIpcGetMemHandle(&me.h[i], p) != cudaSuccess) {
                cudaGetLastError();
                local_st = fail(c, GUM_ECUDA, "cudaIpcGetMemHandle failed (field %d)", i);
                break;
            }
        }
        const FragBufs& F = c->fr[c->rank];
        me.V = c->V;
        me.E = c->E;
        me.bounds_hash = hash_words(c->bounds, sizeof(unsigned) * (c->P + 1));
        me.pr_qlen = F.pr_qlen;
        me.sq_len = F.sq_len;
        me.sE = F.sE;
        me.tile_cap = F.tile_cap;
    }
    me.status = (unsigned)(-(int)local_st);
    gum_status st = mp_exchange(c, &me, sizeof(me), all.data());
    if (st != GUM_OK) return st;
    if (local_st != GUM_OK) return local_st;
    for (int r = 0; r < c->P; r++) {
        const MpBlob& b = all[r];
        if (b.magic != kMpMagic || b.rank != (unsigned)r || b.nfields != (unsigned)nf)
            return fail(c, GUM_EINVAL, "multi-process exchange: rank %d sent a malformed blob", r);
        if (b.status) return fail(c, GUM_ESTATE, "peer rank %d failed (status -%u)", r, b.status);
        if (b.V != me.V || b.E != me.E || b.bounds_hash != me.bounds_hash)
            return fail(c, GUM_EINVAL, "rank %d has a different graph or partition (V=%llu E=%llu)", r, b.V, b.E);
    }
    for (int r = 0; r < c->P; r++) {
        if (r == c->rank) continue;
        const MpBlob& b = all[r];
        void** pf[kMpFields];
        mp_fields(c, r, pf);
        for (int i = 0; i < nf; i++) {
            if (!b.ptr[i]) {
                *pf[i] = nullptr;
                continue;
            }
            auto key = std::make_pair(r, b.ptr[i]);
            auto it = c->ipc_map.find(key);
            if (it == c->ipc_map.end()) {
                void* q = nullptr;
                cudaError_t e = cudaIpcOpenMemHandle(&q, b.h[i], cudaIpcMemLazyEnablePeerAccess);
                if (e != cudaSuccess) {
                    cudaGetLastError();
                    return fail(c, GUM_ECUDA, "cudaIpcOpenMemHandle(rank %d, field %d): %s", r, i, cudaGetErrorString(e));
                }
                it = c->ipc_map.emplace(key, q).first;
            }
            *pf[i] = it->second;
        }
        FragBufs& F = c->fr[r];
        F.pr_qlen = b.pr_qlen;
        F.pr_qedges = F.E;
        F.sq_len = b.sq_len;
        F.sq_edges = b.sE;
        F.sE = b.sE;
        F.tile_cap = b.tile_cap;
    }
    return GUM_OK;
}

gum_status ensure_fragment_state(gum_ctx* c, int f, unsigned long long max_edges) {
    FragBufs& F = c->fr[f];
    const unsigned long long need = max_edges / c->cfg.chunk_edges + 2;
    if (F.tile && F.tile_cap >= need) return GUM_OK;
    F.tile = (unsigned*)dalloc(c, F.dev, need * sizeof(unsigned), c->part_allocs);
    if (!F.tile) return fail(c, GUM_ENOMEM, "tile table alloc failed (fragment %d)", f);
    F.tile_cap = need;
    return GUM_OK;
}

gum_status build_sym(gum_ctx* c) {
    if (c->sym_ready) return GUM_OK;
    const int d0 = c->dev[0];
    CK(cudaSetDevice(d0));
    cudaStream_t s = c->stream[0];
    const unsigned long long sE = 2ull * c->E;
    std::vector<Alloc> tmp;
    unsigned long long* srp = (unsigned long long*)dalloc(c, d0, (c->V + 1ull) * 8, c->part_allocs);
    unsigned* scol = (unsigned*)dalloc(c, d0, std::max<unsigned long long>(sE, 1) * 4, c->part_allocs);
    unsigned long long* cursor = (unsigned long long*)dalloc(c, d0, (c->V + 1ull) * 8, tmp);
    size_t tb = setup_scan_tmp_bytes(c->V);
    void* t = dalloc(c, d0, tb, tmp);
    if (!srp || !scol || !cursor || !t) {
        free_list(c, tmp);
        return fail(c, GUM_ENOMEM, "symmetric CSR alloc failed (%llu entries)", sE);
    }
    cudaError_t e = setup_symmetrize(c->p_row_ptr, c->p_col, c->V, c->E, srp, scol, cursor, t, tb, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    free_list(c, tmp);
    if (e != cudaSuccess) return fail(c, GUM_ECUDA, "symmetrize: %s", cudaGetErrorString(e));
    std::vector<unsigned long long> hb(c->P + 1);
    for (int f = 0; f <= c->P; f++) CK(cudaMemcpy(&hb[f], srp + c->bounds[f], 8, cudaMemcpyDeviceToHost));
    for (int f = 0; f < c->P; f++) {
        FragBufs& F = c->fr[f];
        F.sE = hb[f + 1] - hb[f];
        if (F.sE >= (1ull << 32)) return fail(c, GUM_EUNSUP, "symmetric fragment %d has >= 2^32 entries", f);
        if (!frag_local(c, f)) continue;
        if (c->P == 1 && c->single_device) {
            F.s_row_ptr = srp;
            F.s_col = scol;
        } else {
            F.s_row_ptr = (unsigned long long*)dalloc(c, F.dev, (F.V + 1ull) * 8, c->part_allocs);
            F.s_col = (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(F.sE, 1) * 4, c->part_allocs);
            if (!F.s_row_ptr || !F.s_col) return fail(c, GUM_ENOMEM, "sym fragment alloc failed");
            unsigned long long* tmp_rp = F.s_row_ptr;
            std::vector<Alloc> t2;
            if (F.dev != d0) tmp_rp = (unsigned long long*)dalloc(c, d0, (F.V + 1ull) * 8, t2);
            CK(setup_rebase_rows(srp, c->bounds[f], c->bounds[f + 1], tmp_rp, s));
            if (F.dev != d0) CK(cudaMemcpyPeerAsync(F.s_row_ptr, F.dev, tmp_rp, d0, (F.V + 1ull) * 8, s));
            if (F.sE) CK(cudaMemcpyPeerAsync(F.s_col, F.dev, scol + hb[f], d0, F.sE * 4, s));
            CK(cudaStreamSynchronize(s));
            free_list(c, t2);
        }
        gum_status st = ensure_fragment_state(c, f, std::max(F.E, F.sE));
        if (st != GUM_OK) return st;
    }
    // Iteration 0 of WCC has every vertex active: when the label array does not fit L2, regroup the
    // symmetric graph block-major by destination block (as for PR) so its atomics stay L2-resident.
    const unsigned long long block_bytes = getenv("GUM_WCC_BLOCK_BYTES") ? strtoull(getenv("GUM_WCC_BLOCK_BYTES"), 0, 10)
                                                                        : (48ull << 20);
    if ((unsigned long long)c->V * 4 > block_bytes + (block_bytes >> 1)) {
        unsigned long long S = std::max<unsigned long long>(256, block_bytes / 4);
        int B = (int)((c->V + S - 1) / S);
        if (B > 64) {
            B = 64;
            S = (c->V + 63) / 64;
        }
        for (int f = 0; f < c->P; f++) {
            if (!frag_local(c, f)) continue;
            FragBufs& F = c->fr[f];
            CK(cudaSetDevice(F.dev));
            cudaStream_t s2 = c->stream[c->split ? f : 0];
            const unsigned long long cap = std::min<unsigned long long>((unsigned long long)B * F.V, F.sE) + 1;
            F.sq_col = (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(F.sE, 1) * 4, c->part_allocs);
            F.sq_q_v = (unsigned*)dalloc(c, F.dev, cap * 4, c->part_allocs);
            F.sq_q_off = (unsigned long long*)dalloc(c, F.dev, (cap + 1) * 8, c->part_allocs);
            F.sq_tile = (unsigned*)dalloc(c, F.dev, (F.sE / c->cfg.chunk_edges + 2) * 4, c->part_allocs);
            std::vector<Alloc> tmp2;
            const size_t tb2 = setup_pr_tmp_bytes(F.V, B);
            void* t2 = dalloc(c, F.dev, tb2, tmp2);
            if (!F.sq_col || !F.sq_q_v || !F.sq_q_off || !F.sq_tile || !t2) {
                free_list(c, tmp2);
                return fail(c, GUM_ENOMEM, "WCC blocked queue alloc failed (fragment %d)", f);
            }
            unsigned long long Q = 0;
            cudaError_t e2 = setup_pr_blocked(F.s_row_ptr, F.s_col, F.V, F.sE, (unsigned)S, B, c->cfg.chunk_edges,
                                              F.sq_col, F.sq_q_v, F.sq_q_off, F.sq_tile, &Q, t2, tb2, s2);
            if (e2 == cudaSuccess) e2 = cudaStreamSynchronize(s2);
            free_list(c, tmp2);
            if (e2 != cudaSuccess) return fail(c, GUM_ECUDA, "WCC blocked queue: %s", cudaGetErrorString(e2));
            F.sq_len = Q;
            F.sq_edges = F.sE;
        }
        CK(cudaSetDevice(c->dev[0]));
    }
    c->s_rp_g = srp;
    c->s_col_g = scol;
    c->sym_ready = true;
    drop_graphs(c);
    return GUM_OK;
}

// NEXT-1 hub cache: every worker gets a local copy of the adjacency lists of every other fragment's
// vertices with out-degree > t4, built from the global (partitioned) CSR of the algorithm: the out-CSR for
// BFS/SSSP, the symmetric CSR for WCC. On one device the workers share one copy per fragment (their memory
// is the same); across devices each worker's copy lives on its own device; in multi-process mode each rank
// builds the copies it needs from its own full graph.
gum_status build_hub(gum_ctx* c, int alg) {
    if (!c->cfg.hub_cache || c->P == 1 || alg == GUM_PR) return GUM_OK;
    const int kind = alg == GUM_WCC ? 2 : 1;
    if (c->hub_kind == kind) return GUM_OK;
    free_list(c, c->hub_allocs);
    for (auto& row : c->hub)
        for (auto& h : row) h = HubBufs{};
    c->hub_kind = 0;
    c->hub_entries = 0;
    const unsigned long long* rp = kind == 2 ? c->s_rp_g : c->p_row_ptr;
    const unsigned* col = kind == 2 ? c->s_col_g : c->p_col;
    const unsigned* wt = kind == 2 ? nullptr : c->p_w;
    if (!rp || !col) return fail(c, GUM_ESTATE, "hub cache: global CSR not available");
    const int d0 = c->dev[0];
    CK(cudaSetDevice(d0));
    cudaStream_t s = c->stream[0];
    const unsigned t4 = c->cfg.hub_degree;
    for (int f = 0; f < c->P; f++) {
        const unsigned b0 = c->bounds[f], n = c->bounds[f + 1] - c->bounds[f];
        // the workers that need a copy of fragment f (built here), and where the copy lives
        bool need = false;
        for (int w = 0; w < c->P; w++) need = need || (w != f && (!c->mp || w == c->rank));
        if (!need) continue;
        unsigned long long* off = (unsigned long long*)dalloc(c, d0, (n + 1ull) * 8, c->hub_allocs);
        std::vector<Alloc> tmp;
        const size_t tb = setup_scan_tmp_bytes(n);
        void* t = dalloc(c, d0, tb, tmp);
        if (!off || !t) {
            free_list(c, tmp);
            return fail(c, GUM_ENOMEM, "hub cache offsets alloc failed");
        }
        CK(setup_hub_offsets(rp, b0, n, t4, off, t, tb, s));
        unsigned long long tot = 0;
        CK(cudaMemcpyAsync(&tot, off + n, 8, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        free_list(c, tmp);
        if (tot >= (1ull << 32)) return fail(c, GUM_EUNSUP, "hub cache of fragment %d has >= 2^32 entries", f);
        unsigned* hcol = (unsigned*)dalloc(c, d0, std::max<unsigned long long>(tot, 1) * 4, c->hub_allocs);
        unsigned* hw = wt ? (unsigned*)dalloc(c, d0, std::max<unsigned long long>(tot, 1) * 4, c->hub_allocs) : nullptr;
        if (!hcol || (wt && !hw)) return fail(c, GUM_ENOMEM, "hub cache alloc failed (%llu entries)", tot);
        CK(setup_hub_fill(rp, col, wt, b0, n, t4, off, hcol, hw, s));
        CK(cudaStreamSynchronize(s));
        c->hub_entries += tot;
        for (int w = 0; w < c->P; w++) {
            if (w == f || (c->mp && w != c->rank)) continue;
            HubBufs& H = c->hub[w][f];
            if (c->dev[w] == d0) {
                H.off = off;
                H.col = hcol;
                H.w = hw;
                continue;
            }
            const int dw = c->dev[w];
            H.off = (unsigned long long*)dalloc(c, dw, (n + 1ull) * 8, c->hub_allocs);
            H.col = (unsigned*)dalloc(c, dw, std::max<unsigned long long>(tot, 1) * 4, c->hub_allocs);
            H.w = hw ? (unsigned*)dalloc(c, dw, std::max<unsigned long long>(tot, 1) * 4, c->hub_allocs) : nullptr;
            if (!H.off || !H.col || (hw && !H.w)) return fail(c, GUM_ENOMEM, "hub cache copy alloc failed");
            CK(cudaMemcpyPeerAsync(H.off, dw, off, d0, (n + 1ull) * 8, s));
            if (tot) CK(cudaMemcpyPeerAsync(H.col, dw, hcol, d0, tot * 4, s));
            if (tot && hw) CK(cudaMemcpyPeerAsync(H.w, dw, hw, d0, tot * 4, s));
            CK(cudaStreamSynchronize(s));
        }
    }
    c->hub_kind = kind;
    drop_graphs(c);
    return GUM_OK;
}

// NEXT-3 copy-migration (osteal_migrate): worker o keeps a foster queue for every fragment f > o (the only
// fragments the survivors {0..m'-1} can inherit, owner(f) = f mod m'), in o's memory, so an evicted fragment's
// frontier queue is generated directly on its new owner and its advance reads it locally. Sized like
// the fragment's own queue (vertices, and chunks of the larger of the out / symmetric edge counts).
gum_status build_foster(gum_ctx* c, bool* built) {
    *built = false;
    if (!c->cfg.osteal_migrate || c->P == 1) return GUM_OK;
    // decided from global sizes only, so every rank of a multi-process run agrees (and publishes) together
    unsigned long long key = 1;
    for (int f = 0; f < c->P; f++) key = key * 1000003ull + std::max(c->fr[f].E, c->fr[f].sE);
    if (key == c->fq_key) return GUM_OK;
    c->fq_key = key;
    *built = true;
    for (int o = 0; o < c->P; o++) {
        if (!frag_local(c, o)) continue;  // (multi-process: every rank builds its own, peers map them)
        for (int f = o + 1; f < c->P; f++) {
            const FragBufs& F = c->fr[f];
            const unsigned long long need_t = std::max(F.E, F.sE) / c->cfg.chunk_edges + 2;
            QPtrs& Q = c->fq[o][f];
            const int dev = c->dev[o];
            const size_t Vn = std::max<size_t>(F.V, 1);
            if (!Q.q_v) {
                Q.q_v = (unsigned*)dalloc(c, dev, Vn * 4, c->part_allocs);
                Q.q_off = (unsigned long long*)dalloc(c, dev, (Vn + 1) * 8, c->part_allocs);
                Q.q_base = (long long*)dalloc(c, dev, Vn * 8, c->part_allocs);
                if (!Q.q_v || !Q.q_off || !Q.q_base) return fail(c, GUM_ENOMEM, "foster queue alloc failed (%d, %d)", o, f);
            }
            if (c->fq_tile_cap[o][f] < need_t) {
                Q.tile = (unsigned*)dalloc(c, dev, need_t * 4, c->part_allocs);
                if (!Q.tile) return fail(c, GUM_ENOMEM, "foster chunk table alloc failed (%d, %d)", o, f);
                c->fq_tile_cap[o][f] = need_t;
            }
        }
    }
    drop_graphs(c);
    return GUM_OK;
}

// kernels launch_phase issues for (alg, phase) under d/L (the skips of kernels.cu launch_phase)
int count_phase(int alg, int phase, const DevCtx& d, const LaunchCfg& L) {
    int kinds[4];
    const int n = phase_kernels(alg, phase, kinds);
    int k = 0;
    for (int i = 0; i < n; i++) {
        if (kinds[i] == KER_TAIL && L.tail_grid <= 0) continue;
        if (kinds[i] == KER_PULL && !d.bfs_pull) continue;
        if (kinds[i] == KER_APPLY && !d.pb_shift) continue;
        if (kinds[i] == KER_CONTROL && d.fuse_ctl && alg != GUM_PR) continue;
        k++;
    }
    return k;
}

// Launch one phase; in profile mode bracket every kernel with a pair of CUDA events.
gum_status run_phase(gum_ctx* c, int alg, int phase, const DevCtx& d, const LaunchCfg& L, cudaStream_t s) {
    c->launches += count_phase(alg, phase, d, L);
    if (!(c->cfg.flags & GUM_CFG_PROFILE)) {
        CK(launch_phase(alg, phase, d, L, s, 0, 0));
        return GUM_OK;
    }
    int kinds[4];
    const int n = phase_kernels(alg, phase, kinds);
    for (int i = 0; i < n; i++) {
        if (kinds[i] == KER_TAIL && L.tail_grid <= 0) continue;
        if (kinds[i] == KER_PULL && !d.bfs_pull) continue;
        cudaEvent_t a, b;
        CK(cudaEventCreate(&a));
        CK(cudaEventCreate(&b));
        CK(cudaEventRecord(a, s));
        CK(launch_kernel(alg, kinds[i], d, L, s, 0, 0));
        CK(cudaEventRecord(b, s));
        c->prof_ev.push_back(a);
        c->prof_ev.push_back(b);
        c->prof_kind.push_back(kinds[i]);
    }
    return GUM_OK;
}

// PR's frontier is every vertex with out-degree > 0 in every iteration: build it once, regrouped by
// destination block so that consecutive chunks push into one L2-resident slice of acc.
// PR pull (default): every fragment's in-edges regrouped by source block (an x/outdeg slice
// sized to stay L2-resident while a pass gathers from it), plus one replica of x/outdeg per launch unit.
gum_status build_pr_pull(gum_ctx* c) {
    const unsigned long long block_bytes = getenv("GUM_PR_PULL_BLOCK_BYTES")
                                               ? strtoull(getenv("GUM_PR_PULL_BLOCK_BYTES"), 0, 10)
                                               : (48ull << 20);
    unsigned long long S = std::max<unsigned long long>(1024, block_bytes / 8);
    int B = (int)((c->V + S - 1) / S);
    if (B > 64) {
        B = 64;
        S = (c->V + 63) / 64;
    }
    if (B < 1) B = 1;
    const int d0 = c->dev[0];
    CK(cudaSetDevice(d0));
    cudaStream_t s = c->stream[0];
    std::vector<Alloc> tmp;
    unsigned long long* trp = (unsigned long long*)dalloc(c, d0, (c->V + 1ull) * 8, tmp);
    unsigned* tcol = (unsigned*)dalloc(c, d0, std::max<unsigned long long>(c->E, 1) * 4, tmp);
    unsigned long long* cursor = (unsigned long long*)dalloc(c, d0, (c->V + 1ull) * 8, tmp);
    const size_t tb = setup_scan_tmp_bytes(c->V);
    void* t = dalloc(c, d0, tb, tmp);
    if (!trp || !tcol || !cursor || !t) {
        free_list(c, tmp);
        return fail(c, GUM_ENOMEM, "PR pull: transpose alloc failed");
    }
    cudaError_t e = setup_transpose(c->p_row_ptr, c->p_col, c->V, c->E, trp, tcol, cursor, t, tb, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) {
        free_list(c, tmp);
        return fail(c, GUM_ECUDA, "PR pull transpose: %s", cudaGetErrorString(e));
    }
    std::vector<unsigned long long> hb(c->P + 1);
    for (int f = 0; f <= c->P; f++) CK(cudaMemcpy(&hb[f], trp + c->bounds[f], 8, cudaMemcpyDeviceToHost));
    for (int f = 0; f < c->P; f++) {
        FragBufs& F = c->fr[f];
        F.pr_qlen = F.V;  // every vertex pulls (stats / byte model: one queue entry per vertex)
        F.pr_qedges = F.E;
        if (!frag_local(c, f)) continue;
        const unsigned long long Ein = hb[f + 1] - hb[f];
        if (Ein >= (1ull << 32)) {
            free_list(c, tmp);
            return fail(c, GUM_EUNSUP, "PR pull: fragment %d has >= 2^32 in-edges: use more workers", f);
        }
        std::vector<Alloc> t2;
        unsigned long long* irp = (unsigned long long*)dalloc(c, d0, (F.V + 1ull) * 8, t2);
        const size_t tb2 = setup_pr_tmp_bytes(F.V, B);
        void* tt = dalloc(c, d0, tb2, t2);
        if (!irp || !tt) {
            free_list(c, t2);
            free_list(c, tmp);
            return fail(c, GUM_ENOMEM, "PR pull: fragment %d temp alloc failed", f);
        }
        CK(setup_rebase_rows(trp, c->bounds[f], c->bounds[f + 1], irp, s));
        std::vector<unsigned long long> htb(B + 1);
        CK(setup_pr_pull(irp, tcol + hb[f], F.V, Ein, (unsigned)S, B, kPullTile, nullptr, nullptr, nullptr, htb.data(),
                         tt, tb2, s));
        const unsigned long long n_off = (unsigned long long)B * F.V + 1;
        // built on worker 0's device; copied to the fragment's device when it differs
        const bool here = F.dev == d0;
        std::vector<Alloc>& dst_list = here ? c->part_allocs : t2;
        unsigned* off = (unsigned*)dalloc(c, d0, n_off * 4, dst_list);
        unsigned* pcol = (unsigned*)dalloc(c, d0, std::max<unsigned long long>(Ein, 1) * 4, dst_list);
        unsigned* tx = (unsigned*)dalloc(c, d0, htb[B] * 4, dst_list);
        unsigned long long* tbd = (unsigned long long*)dalloc(c, d0, (B + 1) * 8, dst_list);
        if (!off || !pcol || !tx || !tbd) {
            free_list(c, t2);
            free_list(c, tmp);
            return fail(c, GUM_ENOMEM, "PR pull: fragment %d alloc failed (%llu in-edges)", f, Ein);
        }
        CK(setup_pr_pull(irp, tcol + hb[f], F.V, Ein, (unsigned)S, B, kPullTile, off, pcol, tx, htb.data(), tt, tb2,
                         s));
        CK(cudaMemcpyAsync(tbd, htb.data(), (B + 1) * 8, cudaMemcpyHostToDevice, s));
        CK(cudaStreamSynchronize(s));
        if (here) {
            F.pl_off = off;
            F.pl_col = pcol;
            F.pl_tx = tx;
            F.pl_tb = tbd;
        } else {
            F.pl_off = (unsigned*)dalloc(c, F.dev, n_off * 4, c->part_allocs);
            F.pl_col = (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(Ein, 1) * 4, c->part_allocs);
            F.pl_tx = (unsigned*)dalloc(c, F.dev, htb[B] * 4, c->part_allocs);
            F.pl_tb = (unsigned long long*)dalloc(c, F.dev, (B + 1) * 8, c->part_allocs);
            if (!F.pl_off || !F.pl_col || !F.pl_tx || !F.pl_tb) {
                free_list(c, t2);
                free_list(c, tmp);
                return fail(c, GUM_ENOMEM, "PR pull: fragment %d device copy alloc failed", f);
            }
            CK(cudaMemcpyPeerAsync(F.pl_off, F.dev, off, d0, n_off * 4, s));
            if (Ein) CK(cudaMemcpyPeerAsync(F.pl_col, F.dev, pcol, d0, Ein * 4, s));
            CK(cudaMemcpyPeerAsync(F.pl_tx, F.dev, tx, d0, htb[B] * 4, s));
            CK(cudaMemcpyPeerAsync(F.pl_tb, F.dev, tbd, d0, (B + 1) * 8, s));
            CK(cudaStreamSynchronize(s));
        }
        free_list(c, t2);
    }
    free_list(c, tmp);
    for (int u = 0; u < c->n_units; u++) {
        if (!unit_local(c, u)) continue;
        const int w0 = unit_w0(c, u);
        c->cxg[w0] = (double*)dalloc(c, unit_dev(c, u), 2ull * c->V * 8, c->part_allocs);
        if (!c->cxg[w0]) return fail(c, GUM_ENOMEM, "PR pull: x/outdeg replica alloc failed");
    }
    CK(cudaSetDevice(d0));
    c->pl_B = (unsigned)B;
    c->pl_ready = true;
    c->pr_ready = true;
    drop_graphs(c);
    return GUM_OK;
}

gum_status build_pr(gum_ctx* c) {
    if (c->pr_ready) return GUM_OK;
    // pull unless the caller asked for the push, or NEXT-1 mirrors (which aggregate pushes) are on
    if (!c->cfg.pr_push && !(c->cfg.mirrors && c->P > 1)) return build_pr_pull(c);
    const unsigned long long block_bytes = getenv("GUM_PR_BLOCK_BYTES") ? strtoull(getenv("GUM_PR_BLOCK_BYTES"), 0, 10)
                                                                       : (48ull << 20);
    unsigned long long S = std::max<unsigned long long>(1024, block_bytes / 8);
    int B = 1;
    if ((unsigned long long)c->V * 8 > block_bytes + (block_bytes >> 1)) B = (int)((c->V + S - 1) / S);
    if (B > 64) {
        B = 64;
        S = (c->V + 63) / 64;
    }
    if (B == 1) S = (unsigned long long)c->V + 1;
    c->pr_blocks = B;
    for (int f = 0; f < c->P; f++) {
        FragBufs& F = c->fr[f];
        F.pr_qedges = F.E;
        if (!frag_local(c, f)) continue;
        CK(cudaSetDevice(F.dev));
        cudaStream_t s = c->stream[c->split ? f : 0];
        const unsigned long long cap = std::min<unsigned long long>((unsigned long long)B * F.V, F.E) + 1;
        F.pr_col = B > 1 ? (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(F.E, 1) * 4, c->part_allocs) : F.col;
        F.pr_q_v = (unsigned*)dalloc(c, F.dev, cap * 4, c->part_allocs);
        F.pr_q_off = (unsigned long long*)dalloc(c, F.dev, (cap + 1) * 8, c->part_allocs);
        F.pr_tile = (unsigned*)dalloc(c, F.dev, (F.E / c->cfg.chunk_edges + 2) * 4, c->part_allocs);
        std::vector<Alloc> tmp;
        const size_t tb = setup_pr_tmp_bytes(F.V, B);
        void* t = dalloc(c, F.dev, tb, tmp);
        if (!F.pr_col || !F.pr_q_v || !F.pr_q_off || !F.pr_tile || !t) {
            free_list(c, tmp);
            return fail(c, GUM_ENOMEM, "PR blocked queue alloc failed (fragment %d, %d blocks)", f, B);
        }
        unsigned long long Q = 0;
        cudaError_t e = setup_pr_blocked(F.row_ptr, F.col, F.V, F.E, (unsigned)S, B, c->cfg.chunk_edges,
                                         B > 1 ? F.pr_col : nullptr, F.pr_q_v, F.pr_q_off, F.pr_tile, &Q, t, tb, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        free_list(c, tmp);
        if (e != cudaSuccess) return fail(c, GUM_ECUDA, "PR blocked queue: %s", cudaGetErrorString(e));
        F.pr_qlen = Q;
        F.pr_qedges = F.E;
        // opt-in (measured slower on C5: 12.0 vs 10.8 ms per iteration, the shuffle search is MIO-bound)
        static const int env_pp = getenv("GUM_PR_PUSH") ? atoi(getenv("GUM_PR_PUSH")) : 0;
        if (c->P == 1 && env_pp) {
            // single fragment: the warp-task push (k_pr_push) runs on the same queue cut into pieces
            std::vector<Alloc> t3;
            unsigned long long* pos = (unsigned long long*)dalloc(c, F.dev, (Q + 1) * 8, t3);
            const size_t tb3 = setup_scan_tmp_bytes((unsigned)std::min<unsigned long long>(Q, 0xFFFFFFF0ull));
            void* tt = dalloc(c, F.dev, tb3 + (Q > 0xFFFFFFF0ull ? 0 : 0), t3);
            if (!pos || !tt) {
                free_list(c, t3);
                return fail(c, GUM_ENOMEM, "PR pieces alloc failed");
            }
            unsigned long long n2 = 0;
            cudaError_t e3 = setup_pr_pieces_count(F.pr_q_off, Q, kPrPiece, pos, tt, tb3, s);
            if (e3 == cudaSuccess) e3 = cudaMemcpyAsync(&n2, pos + Q, 8, cudaMemcpyDeviceToHost, s);
            if (e3 == cudaSuccess) e3 = cudaStreamSynchronize(s);
            if (e3 == cudaSuccess) {
                F.pr2_q_v = (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(n2, 1) * 4, c->part_allocs);
                F.pr2_q_off = (unsigned long long*)dalloc(c, F.dev, (n2 + 1) * 8, c->part_allocs);
                if (!F.pr2_q_v || !F.pr2_q_off) {
                    free_list(c, t3);
                    return fail(c, GUM_ENOMEM, "PR pieces alloc failed (%llu pieces)", n2);
                }
                e3 = setup_pr_pieces_emit(F.pr_q_v, F.pr_q_off, Q, kPrPiece, pos, F.pr2_q_v, F.pr2_q_off, s);
                if (e3 == cudaSuccess) e3 = cudaStreamSynchronize(s);
            }
            free_list(c, t3);
            if (e3 != cudaSuccess) return fail(c, GUM_ECUDA, "PR pieces: %s", cudaGetErrorString(e3));
            F.pr2_len = n2;
        }
    }
    CK(cudaSetDevice(c->dev[0]));
    c->pr_ready = true;
    drop_graphs(c);
    return GUM_OK;
}

// BFS propagation blocking (single fragment): per destination block of 2^17 ids, a region of the binned
// buffer sized by the block's in-degree (an upper bound for any iteration: each edge is expanded once).
gum_status build_pb(gum_ctx* c) {
    if (c->pb_ready || c->P != 1 || c->cfg.pb_block_log2 == 0) return GUM_OK;
    const unsigned shift = c->cfg.pb_block_log2;
    if (shift != 17) return fail(c, GUM_EINVAL, "pb_block_log2 must be 0 or 17");
    const unsigned long long nb = ((unsigned long long)c->V + (1ull << shift) - 1) >> shift;
    if (nb > (unsigned long long)kPbMaxBins) return GUM_OK;  // too many blocks: keep the plain advance
    FragBufs& F = c->fr[0];
    CK(cudaSetDevice(F.dev));
    cudaStream_t s = c->stream[0];
    F.pb_off = (unsigned long long*)dalloc(c, F.dev, (nb + 1) * 8, c->part_allocs);
    F.pb_fill = (unsigned*)dalloc(c, F.dev, nb * 4, c->part_allocs);
    F.pb_done = (unsigned*)dalloc(c, F.dev, nb * 4, c->part_allocs);
    F.pb_buf = (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(F.E, 1) * 4, c->part_allocs);
    std::vector<Alloc> tmp;
    const size_t tb = setup_pb_tmp_bytes((unsigned)nb);
    void* t = dalloc(c, F.dev, tb, tmp);
    if (!F.pb_off || !F.pb_fill || !F.pb_done || !F.pb_buf || !t) {
        free_list(c, tmp);
        return fail(c, GUM_ENOMEM, "propagation-blocking buffers alloc failed");
    }
    CK(cudaMemsetAsync(F.pb_fill, 0, nb * 4, s));
    CK(cudaMemsetAsync(F.pb_done, 0, nb * 4, s));
    cudaError_t e = setup_pb_offsets(F.col, F.E, shift, (unsigned)nb, F.pb_off, t, tb, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    free_list(c, tmp);
    if (e != cudaSuccess) return fail(c, GUM_ECUDA, "pb offsets: %s", cudaGetErrorString(e));
    c->pb_shift = shift;
    c->pb_nb = (unsigned)nb;
    c->pb_ready = true;
    drop_graphs(c);
    return GUM_OK;
}

// In-CSR (transpose) of the partitioned graph, sliced per fragment, for bottom-up BFS iterations.
gum_status build_in(gum_ctx* c) {
    if (c->in_ready || !c->cfg.bfs_direction_opt) return GUM_OK;
    const int d0 = c->dev[0];
    CK(cudaSetDevice(d0));
    cudaStream_t s = c->stream[0];
    std::vector<Alloc> tmp;
    unsigned long long* trp = (unsigned long long*)dalloc(c, d0, (c->V + 1ull) * 8, c->part_allocs);
    unsigned* tcol = (unsigned*)dalloc(c, d0, std::max<unsigned long long>(c->E, 1) * 4, c->part_allocs);
    unsigned long long* cursor = (unsigned long long*)dalloc(c, d0, (c->V + 1ull) * 8, tmp);
    const size_t tb = setup_scan_tmp_bytes(c->V);
    void* t = dalloc(c, d0, tb, tmp);
    if (!trp || !tcol || !cursor || !t) {
        free_list(c, tmp);
        return fail(c, GUM_ENOMEM, "in-CSR alloc failed");
    }
    cudaError_t e = setup_transpose(c->p_row_ptr, c->p_col, c->V, c->E, trp, tcol, cursor, t, tb, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    free_list(c, tmp);
    if (e != cudaSuccess) return fail(c, GUM_ECUDA, "transpose: %s", cudaGetErrorString(e));
    std::vector<unsigned long long> hb(c->P + 1);
    for (int f = 0; f <= c->P; f++) CK(cudaMemcpy(&hb[f], trp + c->bounds[f], 8, cudaMemcpyDeviceToHost));
    for (int f = 0; f < c->P; f++) {
        FragBufs& F = c->fr[f];
        const unsigned long long iE = hb[f + 1] - hb[f];
        if (!frag_local(c, f)) continue;
        if (c->P == 1 && c->single_device) {
            F.in_row_ptr = trp;
            F.in_col = tcol;
            continue;
        }
        F.in_row_ptr = (unsigned long long*)dalloc(c, F.dev, (F.V + 1ull) * 8, c->part_allocs);
        F.in_col = (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(iE, 1) * 4, c->part_allocs);
        if (!F.in_row_ptr || !F.in_col) return fail(c, GUM_ENOMEM, "in-CSR fragment alloc failed");
        std::vector<Alloc> t2;
        unsigned long long* tmp_rp = F.in_row_ptr;
        if (F.dev != d0) tmp_rp = (unsigned long long*)dalloc(c, d0, (F.V + 1ull) * 8, t2);
        CK(setup_rebase_rows(trp, c->bounds[f], c->bounds[f + 1], tmp_rp, s));
        if (F.dev != d0) CK(cudaMemcpyPeerAsync(F.in_row_ptr, F.dev, tmp_rp, d0, (F.V + 1ull) * 8, s));
        if (iE) CK(cudaMemcpyPeerAsync(F.in_col, F.dev, tcol + hb[f], d0, iE * 4, s));
        CK(cudaStreamSynchronize(s));
        free_list(c, t2);
    }
    c->in_ready = true;
    drop_graphs(c);
    return GUM_OK;
}

gum_status capture_graph(gum_ctx* c, int alg, const DevCtx& d, const LaunchCfg& L) {
    if (c->gexec[alg]) return GUM_OK;
    cudaStream_t s = c->stream[0];
    cudaGraph_t g;
    CK(cudaGraphCreate(&g, 0));
    cudaGraphConditionalHandle h;
    CK(cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault));
    alignas(cudaGraphNodeParams) unsigned char pbuf[sizeof(cudaGraphNodeParams)];
    memset(pbuf, 0, sizeof(pbuf));
    cudaGraphNodeParams& p = *reinterpret_cast<cudaGraphNodeParams*>(pbuf);
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = cudaGraphCondTypeWhile;
    p.conditional.size = 1;
    cudaGraphNode_t node;
    CK(cudaGraphAddNode(&node, g, nullptr, 0, &p));
    cudaGraph_t body = p.conditional.phGraph_out[0];
    CK(cudaStreamBeginCaptureToGraph(s, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
    cudaError_t e = launch_phase(alg, 0, d, L, s, h, 1);
    if (e == cudaSuccess) e = launch_phase(alg, 1, d, L, s, h, 1);
    cudaGraph_t captured;
    cudaError_t e2 = cudaStreamEndCapture(s, &captured);
    if (e != cudaSuccess || e2 != cudaSuccess) {
        cudaGraphDestroy(g);
        return fail(c, GUM_ECUDA, "graph capture: %s / %s", cudaGetErrorString(e), cudaGetErrorString(e2));
    }
    cudaGraphExec_t ex;
    CK(cudaGraphInstantiate(&ex, g, 0));
    cudaGraphDestroy(g);
    c->gexec[alg] = ex;
    return GUM_OK;
}

// Device-resident multi-unit loop: unit u's graph = a conditional WHILE node whose body is
// unit barrier (phase A: OSteal membership, parking) -> phase-0 kernels -> unit barrier -> phase-1 kernels.
// Every unit decides convergence and OSteal redundantly in its control kernel and sets its own condition;
// a parked unit sits in its phase-A barrier until woken. No host round trip per iteration.
gum_status capture_unit_graph(gum_ctx* c, int alg, int u, const DevCtx& d, const LaunchCfg& L) {
    if (c->gexec_u[alg][u]) return GUM_OK;
    CK(cudaSetDevice(unit_dev(c, u)));
    cudaStream_t s = c->stream[L.w0];
    cudaGraph_t g;
    CK(cudaGraphCreate(&g, 0));
    cudaGraphConditionalHandle h;
    CK(cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault));
    alignas(cudaGraphNodeParams) unsigned char pbuf[sizeof(cudaGraphNodeParams)];
    memset(pbuf, 0, sizeof(pbuf));
    cudaGraphNodeParams& p = *reinterpret_cast<cudaGraphNodeParams*>(pbuf);
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = cudaGraphCondTypeWhile;
    p.conditional.size = 1;
    cudaGraphNode_t node;
    CK(cudaGraphAddNode(&node, g, nullptr, 0, &p));
    cudaGraph_t body = p.conditional.phGraph_out[0];
    CK(cudaStreamBeginCaptureToGraph(s, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
    cudaError_t e = launch_unit_bar(d, u, 0, s);
    if (e == cudaSuccess) e = launch_phase(alg, 0, d, L, s, h, 1);
    if (e == cudaSuccess) e = launch_unit_bar(d, u, 1, s);
    if (e == cudaSuccess) e = launch_phase(alg, 1, d, L, s, h, 1);
    cudaGraph_t captured;
    cudaError_t e2 = cudaStreamEndCapture(s, &captured);
    if (e != cudaSuccess || e2 != cudaSuccess) {
        cudaGraphDestroy(g);
        return fail(c, GUM_ECUDA, "unit %d graph capture: %s / %s", u, cudaGetErrorString(e), cudaGetErrorString(e2));
    }
    cudaGraphExec_t ex;
    CK(cudaGraphInstantiate(&ex, g, 0));
    cudaGraphDestroy(g);
    c->gexec_u[alg][u] = ex;
    return GUM_OK;
}

}  // namespace

// ================================================================================ C ABI
extern "C" {

int gum_version(void) { return 100; }

void gum_config_default(gum_config* cfg) {
    if (!cfg) return;
    memset(cfg, 0, sizeof(*cfg));
    cfg->num_gpus = 1;
    cfg->fsteal = 1;
    cfg->osteal = 1;
    cfg->chunk_edges = 2048;
    cfg->pr_iterations = 20;
    cfg->pr_damping = 0.85;
    cfg->tail_vertices = 16384;
    cfg->pb_block_log2 = 0;  // propagation blocking is opt-in (slower than the probe path)
}

const char* gum_last_error(const gum_ctx* ctx) { return ctx ? ctx->err.c_str() : "null context"; }

gum_status gum_create(const gum_config* cfg, gum_ctx** out) {
    if (!cfg || !out) return GUM_EINVAL;
    *out = nullptr;
    if (cfg->num_gpus < 1 || cfg->num_gpus > kMaxW) return GUM_EINVAL;
    gum_ctx* c = new gum_ctx();
    c->cfg = *cfg;
    if (const char* e = getenv("GUM_CHUNK")) c->cfg.chunk_edges = (uint32_t)atoi(e);  // tuning override
    if (c->cfg.chunk_edges == 0 || c->cfg.chunk_edges > (unsigned)kTileMax) c->cfg.chunk_edges = kTileMax;
    if (c->cfg.chunk_edges % 32 != 0) {
        delete c;
        return GUM_EINVAL;
    }
    if (c->cfg.pr_iterations <= 0) c->cfg.pr_iterations = 20;
    if (c->cfg.pr_damping <= 0.0) c->cfg.pr_damping = 0.85;
    c->P = cfg->num_gpus;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        delete c;
        return GUM_ECUDA;
    }
    for (int i = 0; i < c->P; i++) {
        c->dev[i] = cfg->device_ids ? cfg->device_ids[i] : 0;
        if (c->dev[i] < 0 || c->dev[i] >= ndev) {
            delete c;
            return GUM_EINVAL;
        }
    }
    c->single_device = true;
    for (int i = 1; i < c->P; i++)
        if (c->dev[i] != c->dev[0]) c->single_device = false;
    if (!c->single_device) {
        for (int i = 0; i < c->P; i++)
            for (int j = 0; j < c->P; j++)
                if (i != j && c->dev[i] == c->dev[j]) {
                    delete c;
                    return GUM_EUNSUP;  // mixed: some workers share a device, others do not
                }
    }
    c->split = !c->single_device || ((cfg->flags & GUM_CFG_SPLIT_UNITS) && c->P > 1);
    c->n_units = c->split ? c->P : 1;
    for (int u = 0; u < c->n_units; u++) {
        int d = unit_dev(c, u);
        int w0 = unit_w0(c, u);
        cudaSetDevice(d);
        if (cfg->streams && cfg->streams[w0]) {
            c->stream[w0] = (cudaStream_t)cfg->streams[w0];
        } else {
            if (cudaStreamCreateWithFlags(&c->stream[w0], cudaStreamNonBlocking) != cudaSuccess) {
                cudaGetLastError();
                delete c;
                return GUM_ECUDA;
            }
            c->own_stream[w0] = true;
        }
        if (!c->single_device) {
            for (int v = 0; v < c->P; v++) {
                if (v == u) continue;
                int can = 0;
                cudaDeviceCanAccessPeer(&can, d, c->dev[v]);
                if (!can) {
                    delete c;
                    return GUM_EUNSUP;
                }
                cudaError_t e = cudaDeviceEnablePeerAccess(c->dev[v], 0);
                if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
                    cudaGetLastError();
                    delete c;
                    return GUM_ECUDA;
                }
                cudaGetLastError();
            }
        }
        cudaEvent_t ev;
        cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
        c->bar_ev.push_back(ev);
    }
    cudaSetDevice(c->dev[0]);
    cudaDeviceGetAttribute(&c->nsm, cudaDevAttrMultiProcessorCount, c->dev[0]);
    for (int a = 0; a < kNumAlgs; a++)
        for (int m = 0; m < 2; m++) {
            int occ = 0;
            if (advance_occupancy(a, m, &occ) == cudaSuccess && occ > 0) c->adv_occ[a][m] = occ;
            if (const char* e = getenv("GUM_ADV_CTAS_PER_SM")) c->adv_occ[a][m] = std::max(1, atoi(e));
        }
    cudaGetLastError();
    {
        int occ = 0;
        if (tail_occupancy(&occ) == cudaSuccess && occ > 0) c->tail_occ = std::min(occ, 3);  // C3: 2 -> 3 per SM 253 -> 243 ms
        if (const char* e = getenv("GUM_TAIL_CTAS_PER_SM")) c->tail_occ = std::max(1, std::min(occ, atoi(e)));
        cudaGetLastError();
        occ = 0;
        if (filter_occupancy(&occ) == cudaSuccess && occ > 0) c->filter_occ = std::min(occ, 4);
        occ = 0;
        if (pr_push_occupancy(&occ) == cudaSuccess && occ > 0) c->pr_push_occ = occ;
        occ = 0;
        if (pr_pull_occupancy(&occ) == cudaSuccess && occ > 0) c->pull_occ = occ;
        if (const char* e = getenv("GUM_PULL_CTAS_PER_SM")) c->pull_occ = std::max(1, atoi(e));
        if (const char* e = getenv("GUM_PR_PUSH_CTAS_PER_SM")) c->pr_push_occ = std::max(1, atoi(e));
        cudaGetLastError();
    }
    cudaEventCreate(&c->ev0);
    cudaEventCreate(&c->ev1);
    if (cudaMallocHost(&c->h_rctl, sizeof(RunCtl)) != cudaSuccess) {
        cudaGetLastError();
        delete c;
        return GUM_ENOMEM;
    }
    *out = c;
    return GUM_OK;
}

static unsigned long long config_hash(const gum_config* cfg) {
    unsigned long long h = 1469598103934665603ull;
#define GUM_HC(x) h = hash_words(&cfg->x, sizeof(cfg->x), h)
    GUM_HC(num_gpus); GUM_HC(fsteal); GUM_HC(t1_min_max_edges); GUM_HC(t2_min_spread_edges); GUM_HC(osteal);
    GUM_HC(osteal_active_threshold); GUM_HC(osteal_edges_per_worker); GUM_HC(chunk_edges); GUM_HC(pr_iterations);
    GUM_HC(pr_damping); GUM_HC(max_iterations); GUM_HC(flags); GUM_HC(sssp_delta); GUM_HC(tail_vertices);
    GUM_HC(pb_block_log2); GUM_HC(fsteal_remote_cost); GUM_HC(bfs_direction_opt); GUM_HC(osteal_sync_edges);
    GUM_HC(mirrors); GUM_HC(hub_cache); GUM_HC(hub_degree); GUM_HC(pr_push); GUM_HC(dpr_tolerance);
    GUM_HC(osteal_migrate);
#undef GUM_HC
    return h;
}

gum_status gum_mp_handshake(const gum_config* cfg, const gum_mp_config* mp) {
    if (!cfg || !mp || !mp->exchange) return GUM_EINVAL;
    if (mp->world < 1 || mp->world > kMaxW) return GUM_EINVAL;
    struct Hello {
        unsigned magic, version, sz_cfg, sz_stats;
        int rank, world, num_gpus, pad;
        unsigned long long cfg_hash;
    } me, all[kMaxW];
    memset(&me, 0, sizeof(me));
    memset(all, 0, sizeof(all));
    me.magic = kMpMagic;
    me.version = (unsigned)gum_version();
    me.sz_cfg = sizeof(gum_config);
    me.sz_stats = sizeof(gum_run_stats);
    me.rank = mp->rank;
    me.world = mp->world;
    me.num_gpus = cfg->num_gpus;
    me.cfg_hash = config_hash(cfg);
    if (mp->exchange(&me, sizeof(me), all, mp->user) != 0) return GUM_ENCCL;
    // every rank evaluates the same gathered table, so every rank returns the same status
    for (int r = 0; r < mp->world; r++) {
        const Hello& h = all[r];
        if (h.magic != kMpMagic || h.version != me.version || h.sz_cfg != me.sz_cfg || h.sz_stats != me.sz_stats)
            return GUM_EINVAL;
        if (h.rank != r || h.world != all[0].world || h.num_gpus != h.world || h.cfg_hash != all[0].cfg_hash)
            return GUM_EINVAL;
    }
    return GUM_OK;
}

gum_status gum_create_mp(const gum_config* cfg, const gum_mp_config* mp, gum_ctx** out) {
    if (!cfg || !mp || !out || !mp->exchange) return GUM_EINVAL;
    *out = nullptr;
    if (mp->rank < 0 || mp->rank >= mp->world) return GUM_EINVAL;
    gum_status st = gum_mp_handshake(cfg, mp);
    if (st != GUM_OK) return st;
    gum_status local = GUM_OK;
    if (cfg->device_ids || cfg->alloc) local = GUM_EUNSUP;  // IPC maps whole cudaMalloc allocations
    gum_ctx* c = nullptr;
    if (local == GUM_OK) {
        gum_config c1 = *cfg;
        int devs[kMaxW];
        for (int i = 0; i < kMaxW; i++) devs[i] = mp->device;
        c1.device_ids = devs;
        c1.flags &= ~GUM_CFG_SPLIT_UNITS;
        local = gum_create(&c1, &c);
    }
    // agree: every rank creates its context or none keeps one
    long long mine = local, all[kMaxW];
    if (mp->exchange(&mine, sizeof(mine), all, mp->user) != 0) {
        gum_destroy(c);
        return GUM_ENCCL;
    }
    for (int r = 0; r < mp->world; r++)
        if (all[r] != GUM_OK) {
            gum_destroy(c);
            return local != GUM_OK ? local : GUM_ESTATE;
        }
    if (mp->world > 1) {
        c->mp = true;
        c->rank = mp->rank;
        c->xch = mp->exchange;
        c->xuser = mp->user;
        c->single_device = false;
        c->split = true;
        c->n_units = c->P;
        for (int i = 1; i < c->P; i++) c->stream[i] = c->stream[0];  // own_stream[0] stays the only owner
    }
    *out = c;
    return GUM_OK;
}

void gum_destroy(gum_ctx* c) {
    if (!c) return;
    drop_partition(c);
    free_list(c, c->load_allocs);
    free_list(c, c->misc_allocs);
    for (int i = 0; i < kMaxW; i++) {
        if (c->own_stream[i]) {
            cudaSetDevice(c->dev[i]);
            cudaStreamDestroy(c->stream[i]);
        }
    }
    for (auto e : c->bar_ev) cudaEventDestroy(e);
    if (c->ev0) cudaEventDestroy(c->ev0);
    if (c->ev1) cudaEventDestroy(c->ev1);
    if (c->h_rctl) cudaFreeHost(c->h_rctl);
    delete c;
}

gum_status gum_build_csr(uint32_t V, uint64_t E, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                         uint64_t* row_ptr, uint32_t* col, uint32_t* wout) {
    if ((!src || !dst || !col) && E) return GUM_EINVAL;
    if (!row_ptr) return GUM_EINVAL;
    if (w && !wout && E) return GUM_EINVAL;
    const int T = omp_get_max_threads();
    // per-thread histograms over contiguous edge ranges -> stable counting sort
    std::vector<std::vector<uint64_t>> hist(T);
    int bad = 0;
#pragma omp parallel num_threads(T) reduction(| : bad)
    {
        int t = omp_get_thread_num();
        auto& h = hist[t];
        h.assign((size_t)V + 1, 0);
        uint64_t lo = E * t / T, hi = E * (t + 1) / T;
        for (uint64_t i = lo; i < hi; i++) {
            if (src[i] >= V || dst[i] >= V) {
                bad = 1;
                continue;
            }
            h[src[i]]++;
        }
    }
    if (bad) return GUM_EINVAL;
    // row_ptr and per-thread write cursors (thread t's edges of row v follow threads < t)
    row_ptr[0] = 0;
    {
        // column-wise prefix over (v, t)
        std::vector<uint64_t> rowsum((size_t)V, 0);
#pragma omp parallel for num_threads(T) schedule(static)
        for (int64_t v = 0; v < (int64_t)V; v++) {
            uint64_t s = 0;
            for (int t = 0; t < T; t++) {
                uint64_t x = hist[t][v];
                hist[t][v] = s;
                s += x;
            }
            rowsum[v] = s;
        }
        for (uint64_t v = 0; v < V; v++) row_ptr[v + 1] = row_ptr[v] + rowsum[v];
    }
#pragma omp parallel num_threads(T)
    {
        int t = omp_get_thread_num();
        auto& h = hist[t];
        uint64_t lo = E * t / T, hi = E * (t + 1) / T;
        for (uint64_t i = lo; i < hi; i++) {
            uint32_t u = src[i];
            uint64_t pos = row_ptr[u] + h[u]++;
            col[pos] = dst[i];
            if (w) wout[pos] = w[i];
        }
    }
    return GUM_OK;
}

gum_status gum_load_csr(gum_ctx* c, uint32_t V, uint64_t E, const uint64_t* row_ptr, const uint32_t* col_idx,
                        const uint32_t* weights, uint32_t flags) {
    if (!c) return GUM_EINVAL;
    if (c->poisoned) return fail(c, GUM_ESTATE, "context poisoned by an earlier CUDA error");
    if (!row_ptr || (!col_idx && E)) return fail(c, GUM_EINVAL, "null row_ptr/col_idx");
    if (V == 0 || V > 0xFFFFFFFEu) return fail(c, GUM_EINVAL, "V must be in [1, 2^32-2]");
    drop_partition(c);
    free_list(c, c->load_allocs);
    c->loaded = false;
    const int d0 = c->dev[0];
    CK(cudaSetDevice(d0));
    cudaStream_t s = c->stream[0];
    c->g_row_ptr = (unsigned long long*)dalloc(c, d0, (V + 1ull) * 8, c->load_allocs);
    c->g_col = (unsigned*)dalloc(c, d0, std::max<uint64_t>(E, 1) * 4, c->load_allocs);
    c->g_w = weights ? (unsigned*)dalloc(c, d0, std::max<uint64_t>(E, 1) * 4, c->load_allocs) : nullptr;
    unsigned* d_err = (unsigned*)dalloc(c, d0, 256, c->load_allocs);
    if (!c->g_row_ptr || !c->g_col || (weights && !c->g_w) || !d_err) {
        free_list(c, c->load_allocs);
        return fail(c, GUM_ENOMEM, "graph alloc failed (V=%u E=%llu)", V, (unsigned long long)E);
    }
    const cudaMemcpyKind kind = (flags & GUM_LOAD_DEVICE) ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    CK(cudaMemcpyAsync(c->g_row_ptr, row_ptr, (V + 1ull) * 8, kind, s));
    if (E) CK(cudaMemcpyAsync(c->g_col, col_idx, E * 4, kind, s));
    if (weights && E) CK(cudaMemcpyAsync(c->g_w, weights, E * 4, kind, s));
    CK(cudaMemsetAsync(d_err, 0, 4, s));
    CK(setup_validate(c->g_row_ptr, c->g_col, V, E, d_err, s));
    unsigned herr = 0;
    CK(cudaMemcpyAsync(&herr, d_err, 4, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (herr) {
        free_list(c, c->load_allocs);
        return fail(c, GUM_EINVAL, "malformed CSR (code %u: 1=row_ptr[0]!=0 2=row_ptr[V]!=E 4=not monotone 8=col>=V)",
                    herr);
    }
    c->V = V;
    c->E = E;
    c->has_w = weights != nullptr;
    c->loaded = true;
    return GUM_OK;
}

static gum_status partition_body(gum_ctx* c, gum_part kind, uint64_t seed);

gum_status gum_partition(gum_ctx* c, gum_part kind, uint64_t seed) {
    if (!c) return GUM_EINVAL;
    if (c->poisoned) return fail(c, GUM_ESTATE, "context poisoned");
    if (!c->loaded) return fail(c, GUM_ESTATE, "gum_partition before gum_load_csr");
    if (kind != GUM_PART_SEG && kind != GUM_PART_RANDOM && kind != GUM_PART_DEGREE)
        return fail(c, GUM_EINVAL, "bad partition kind");
    drop_partition(c);
    gum_status st = partition_body(c, kind, seed);
    if (c->mp) {
        st = mp_publish(c, st);
        c->partitioned = st == GUM_OK;
    }
    return st;
}

static gum_status partition_body(gum_ctx* c, gum_part kind, uint64_t seed) {
    const int d0 = c->dev[0];
    CK(cudaSetDevice(d0));
    cudaStream_t s = c->stream[0];
    const unsigned V = c->V;
    const unsigned long long E = c->E;
    c->part_kind = kind;
    c->seed = seed;
    // ---- a2: relabel (RANDOM) then edge-balanced contiguous ranges (SEG)
    if (kind == GUM_PART_RANDOM || kind == GUM_PART_DEGREE) {
        c->inv = (unsigned*)dalloc(c, d0, (size_t)V * 4, c->part_allocs);
        c->perm = kind == GUM_PART_DEGREE ? (unsigned*)dalloc(c, d0, (size_t)V * 4, c->part_allocs) : nullptr;
        c->p_row_ptr = (unsigned long long*)dalloc(c, d0, (V + 1ull) * 8, c->part_allocs);
        c->p_col = (unsigned*)dalloc(c, d0, std::max<unsigned long long>(E, 1) * 4, c->part_allocs);
        c->p_w = c->has_w ? (unsigned*)dalloc(c, d0, std::max<unsigned long long>(E, 1) * 4, c->part_allocs) : nullptr;
        std::vector<Alloc> tmp;
        size_t tb = kind == GUM_PART_DEGREE ? setup_degree_tmp_bytes(V) : setup_relabel_tmp_bytes(V);
        void* t = dalloc(c, d0, tb, tmp);
        if (!c->inv || !c->p_row_ptr || !c->p_col || (c->has_w && !c->p_w) || !t ||
            (kind == GUM_PART_DEGREE && !c->perm)) {
            free_list(c, tmp);
            return fail(c, GUM_ENOMEM, "relabel alloc failed");
        }
        cudaError_t e = kind == GUM_PART_DEGREE
                            ? setup_relabel_degree(c->g_row_ptr, c->g_col, c->g_w, V, E, c->perm, c->inv, c->p_row_ptr,
                                                   c->p_col, c->p_w, t, tb, s)
                            : setup_relabel(c->g_row_ptr, c->g_col, c->g_w, V, E, seed, c->inv, c->p_row_ptr,
                                            c->p_col, c->p_w, t, tb, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        free_list(c, tmp);
        if (e != cudaSuccess) return fail(c, GUM_ECUDA, "relabel: %s", cudaGetErrorString(e));
    } else {
        c->inv = nullptr;
        c->p_row_ptr = c->g_row_ptr;
        c->p_col = c->g_col;
        c->p_w = c->g_w;
    }
    {
        std::vector<Alloc> tmp;
        unsigned* db = (unsigned*)dalloc(c, d0, 64, tmp);
        CK(setup_seg_bounds(c->p_row_ptr, V, E, c->P, db, s));
        CK(cudaMemcpyAsync(c->bounds, db, (c->P + 1) * 4, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        free_list(c, tmp);
    }
    std::vector<unsigned long long> eb(c->P + 1);
    for (int f = 0; f <= c->P; f++) CK(cudaMemcpy(&eb[f], c->p_row_ptr + c->bounds[f], 8, cudaMemcpyDeviceToHost));
    // ---- per-fragment device CSR + state + frontier + control
    for (int f = 0; f < c->P; f++) {
        FragBufs& F = c->fr[f];
        F.dev = c->dev[f];
        F.base = c->bounds[f];
        F.V = c->bounds[f + 1] - c->bounds[f];
        F.E = eb[f + 1] - eb[f];
        if (F.E >= (1ull << 32)) return fail(c, GUM_EUNSUP, "fragment %d has >= 2^32 edges: use more workers", f);
        if (!frag_local(c, f)) continue;  // multi-process: the peer's buffers are mapped by mp_publish
        const size_t Vn = std::max<size_t>(F.V, 1);
        if (c->P == 1 && c->single_device) {
            F.row_ptr = c->p_row_ptr;
            F.col = c->p_col;
            F.w = c->p_w;
            F.orig = c->inv;
        } else {
            F.row_ptr = (unsigned long long*)dalloc(c, F.dev, (F.V + 1ull) * 8, c->part_allocs);
            F.col = (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(F.E, 1) * 4, c->part_allocs);
            F.w = c->has_w ? (unsigned*)dalloc(c, F.dev, std::max<unsigned long long>(F.E, 1) * 4, c->part_allocs)
                           : nullptr;
            F.orig = c->inv ? (unsigned*)dalloc(c, F.dev, Vn * 4, c->part_allocs) : nullptr;
            if (!F.row_ptr || !F.col || (c->has_w && !F.w) || (c->inv && !F.orig))
                return fail(c, GUM_ENOMEM, "fragment %d CSR alloc failed", f);
            std::vector<Alloc> t2;
            unsigned long long* tmp_rp = F.row_ptr;
            if (F.dev != d0) tmp_rp = (unsigned long long*)dalloc(c, d0, (F.V + 1ull) * 8, t2);
            CK(setup_rebase_rows(c->p_row_ptr, c->bounds[f], c->bounds[f + 1], tmp_rp, s));
            if (F.dev != d0) CK(cudaMemcpyPeerAsync(F.row_ptr, F.dev, tmp_rp, d0, (F.V + 1ull) * 8, s));
            if (F.E) CK(cudaMemcpyPeerAsync(F.col, F.dev, c->p_col + eb[f], d0, F.E * 4, s));
            if (F.E && F.w) CK(cudaMemcpyPeerAsync(F.w, F.dev, c->p_w + eb[f], d0, F.E * 4, s));
            if (F.orig && F.V) CK(cudaMemcpyPeerAsync(F.orig, F.dev, c->inv + F.base, d0, (size_t)F.V * 4, s));
            CK(cudaStreamSynchronize(s));
            free_list(c, t2);
        }
        F.state = (unsigned*)dalloc(c, F.dev, Vn * 4, c->part_allocs);
        F.x = (double*)dalloc(c, F.dev, Vn * 8, c->part_allocs);
        F.acc = (double*)dalloc(c, F.dev, Vn * 8, c->part_allocs);
        F.cx = (double*)dalloc(c, F.dev, Vn * 8, c->part_allocs);
        F.bm = (unsigned*)dalloc(c, F.dev, ((F.V + 31) / 32 + 4) * 4, c->part_allocs);
        F.vis = (unsigned*)dalloc(c, F.dev, ((F.V + 31) / 32 + 4) * 4, c->part_allocs);
        F.bm2 = (unsigned*)dalloc(c, F.dev, ((F.V + 31) / 32 + 4) * 4, c->part_allocs);
        F.far = (unsigned*)dalloc(c, F.dev, ((F.V + 31) / 32 + 4) * 4, c->part_allocs);
        // (+ kTailSlack: the tail engine's no-dedupe mode may list a vertex more than once)
        F.app = (unsigned*)dalloc(c, F.dev, (Vn + kTailSlack) * 4, c->part_allocs);
        F.q_v = (unsigned*)dalloc(c, F.dev, (Vn + kTailSlack) * 4, c->part_allocs);
        F.q_off = (unsigned long long*)dalloc(c, F.dev, (Vn + 1) * 8, c->part_allocs);
        F.q_base = (long long*)dalloc(c, F.dev, Vn * 8, c->part_allocs);
        F.ctl = (FragCtl*)dalloc(c, F.dev, sizeof(FragCtl), c->part_allocs);
        if (!F.state || !F.x || !F.acc || !F.cx || !F.bm || !F.vis || !F.bm2 || !F.far || !F.app || !F.q_v || !F.q_off || !F.q_base || !F.ctl)
            return fail(c, GUM_ENOMEM, "fragment %d state alloc failed", f);
        if (c->cfg.mirrors && c->P > 1) {
            // NEXT-1: worker f's outer-vertex mirror (global id space, 8 B per vertex)
            F.mbuf = dalloc(c, F.dev, (size_t)V * 8, c->part_allocs);
            if (!F.mbuf) return fail(c, GUM_ENOMEM, "worker %d mirror alloc failed", f);
        }
        CK(cudaSetDevice(F.dev));
        CK(cudaMemset(F.ctl, 0, sizeof(FragCtl)));
        CK(cudaSetDevice(d0));
        gum_status st = ensure_fragment_state(c, f, F.E);
        if (st != GUM_OK) return st;
    }
    // look-back slots (per fragment, in the fragment's memory) and per-unit run control
    unsigned parts = 1;
    for (int f = 0; f < c->P; f++) {
        unsigned nwords = (c->fr[f].V + 31) / 32;
        unsigned a = (nwords + kDenseWordsPerPart - 1) / kDenseWordsPerPart;
        unsigned b = (c->fr[f].V + kFilterAppPerPart - 1) / kFilterAppPerPart;
        parts = std::max(parts, std::max(a, b) + 1);
    }
    parts = std::max<unsigned>(parts, (unsigned)c->nsm * 8);  // one aggregate slot per filter CTA
    c->lb_parts = parts;
    for (int f = 0; f < c->P; f++) {
        if (!frag_local(c, f)) continue;
        c->lb[f] = (LBSlot*)dalloc(c, c->fr[f].dev, (size_t)parts * sizeof(LBSlot), c->part_allocs);
        if (!c->lb[f]) return fail(c, GUM_ENOMEM, "look-back alloc failed");
        CK(cudaSetDevice(c->fr[f].dev));
        CK(cudaMemset(c->lb[f], 0, (size_t)parts * sizeof(LBSlot)));
    }
    for (int u = 0; u < c->n_units; u++) {
        if (!unit_local(c, u)) continue;
        int w0 = unit_w0(c, u), d = unit_dev(c, u);
        if (c->n_units > 1) {
            c->pad[w0] = (unsigned long long*)dalloc(c, d, kPadWords * 8, c->part_allocs);
            if (!c->pad[w0]) return fail(c, GUM_ENOMEM, "signal pad alloc failed");
            CK(cudaSetDevice(d));
            CK(cudaMemset(c->pad[w0], 0, kPadWords * 8));
        }
        c->rctl[w0] = (RunCtl*)dalloc(c, d, sizeof(RunCtl), c->part_allocs);
        c->tsplit[w0] = (TailSplit*)dalloc(c, d, 8192 * sizeof(TailSplit), c->part_allocs);
        if (!c->rctl[w0] || !c->tsplit[w0]) return fail(c, GUM_ENOMEM, "run control alloc failed");
        CK(cudaSetDevice(d));
        CK(cudaMemset(c->rctl[w0], 0, sizeof(RunCtl)));
        if (c->cfg.flags & GUM_CFG_TRACE) {
            c->trace[w0] = (gum_iter_trace*)dalloc(c, d, (size_t)kTraceMax * sizeof(gum_iter_trace), c->part_allocs);
            if (!c->trace[w0]) return fail(c, GUM_ENOMEM, "trace alloc failed");
        }
    }
    CK(cudaSetDevice(d0));
    {
        std::vector<Alloc> tmp;
        unsigned long long* dc = (unsigned long long*)dalloc(c, d0, 64, tmp);
        CK(cudaMemsetAsync(dc, 0, 8, s));
        CK(setup_count_dangling(c->p_row_ptr, V, dc, s));
        CK(cudaMemcpyAsync(&c->n_dangling, dc, 8, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        free_list(c, tmp);
    }
    c->d_res = dalloc(c, d0, (size_t)V * 8, c->part_allocs);
    if (!c->d_res) return fail(c, GUM_ENOMEM, "result buffer alloc failed");
    c->partitioned = true;
    return GUM_OK;
}

gum_status gum_partition_bounds(const gum_ctx* c, uint32_t* bounds, int n) {
    if (!c || !bounds) return GUM_EINVAL;
    if (!c->partitioned) return GUM_ESTATE;
    for (int i = 0; i <= c->P && i < n; i++) bounds[i] = c->bounds[i];
    return GUM_OK;
}

gum_status gum_prepare(gum_ctx* c, gum_alg alg) {
    if (!c) return GUM_EINVAL;
    if (c->poisoned) return fail(c, GUM_ESTATE, "context poisoned");
    if (!c->partitioned) return fail(c, GUM_ESTATE, "gum_prepare before gum_partition");
    if (alg < 0 || alg > GUM_DPR) return fail(c, GUM_EINVAL, "bad algorithm %d", (int)alg);
    gum_status st = GUM_OK;
    bool built = false;  // multi-process: new buffers must be published (all ranks agree: same state)
    if (alg == GUM_WCC) {
        built = !c->sym_ready;
        st = build_sym(c);
    } else if (alg == GUM_PR) {
        built = !c->pr_ready;
        st = build_pr(c);
    } else if (alg == GUM_BFS) {
        built = (!c->pb_ready && c->P == 1 && c->cfg.pb_block_log2) || (!c->in_ready && c->cfg.bfs_direction_opt);
        st = build_pb(c);
        if (st == GUM_OK) st = build_in(c);
    }
    if (st == GUM_OK) st = build_hub(c, alg);  // worker-local copies: nothing to publish
    if (st == GUM_OK && alg == GUM_SSSP && c->cfg.sssp_delta) {
        // near-far: the far set also kept as two lists, so a sweep reads the parked vertices instead of
        // scanning the whole far bitmap (one sweep per distance bucket)
        static const int env_fl = getenv("GUM_FAR_LIST") ? atoi(getenv("GUM_FAR_LIST")) : 1;
        bool any = false;
        for (int f = 0; f < c->P && env_fl; f++) {
            FragBufs& F = c->fr[f];
            if (!frag_local(c, f) || F.farl) continue;
            F.farl = (unsigned*)dalloc(c, F.dev, 2ull * std::max<size_t>(F.V, 1) * 4, c->part_allocs);
            if (!F.farl) st = fail(c, GUM_ENOMEM, "far list alloc failed (fragment %d)", f);
            any = true;
        }
        if (any) {
            drop_graphs(c);
            built = true;
        }
    }
    if (st == GUM_OK && alg != GUM_PR) {
        bool fb = false;
        st = build_foster(c, &fb);
        built = built || fb;
    }
    if (c->mp && built) st = mp_publish(c, st);
    return st;
}

gum_status gum_run(gum_ctx* c, gum_alg alg, uint32_t source, gum_run_stats* stats) {
    if (!c) return GUM_EINVAL;
    if (c->poisoned) return fail(c, GUM_ESTATE, "context poisoned");
    if (!c->partitioned) return fail(c, GUM_ESTATE, "gum_run before gum_partition");
    if (alg < GUM_BFS || alg > GUM_DPR) return fail(c, GUM_EINVAL, "bad algorithm %d", (int)alg);
    if (alg == GUM_SSSP && !c->has_w) return fail(c, GUM_EINVAL, "SSSP needs edge weights");
    if ((alg == GUM_BFS || alg == GUM_SSSP) && source >= c->V) return fail(c, GUM_ERANGE, "source %u >= V", source);
    gum_status st = gum_prepare(c, alg);
    if (st != GUM_OK) return st;
    c->has_result = false;
    const DevCtx d = make_devctx(c, alg);
    int src_frag = -1;
    unsigned src_local = 0;
    if (alg == GUM_BFS || alg == GUM_SSSP) {
        unsigned sp = source;
        if (c->perm) {
            CK(cudaSetDevice(c->dev[0]));
            CK(cudaMemcpy(&sp, c->perm + source, 4, cudaMemcpyDeviceToHost));
        } else if (c->inv) {
            sp = host_feistel(source, c->V, c->seed);
        }
        for (int f = 0; f < c->P; f++)
            if (sp >= c->bounds[f] && sp < c->bounds[f + 1]) src_frag = f;
        src_local = sp - c->bounds[src_frag];
    }
    const double D0 = (double)c->n_dangling / (double)c->V;
    const bool profile = (c->cfg.flags & GUM_CFG_PROFILE) != 0;
    // (one process per GPU: each rank profiles its own unit's launches)
    if (profile && c->n_units > 1 && !c->mp) return fail(c, GUM_EUNSUP, "GUM_CFG_PROFILE needs a single launch unit per process");
    const bool graph_mode = !(c->cfg.flags & (GUM_CFG_HOST_LOOP | GUM_CFG_PROFILE));
    for (auto e : c->prof_ev) cudaEventDestroy(e);
    c->prof_ev.clear();
    c->prof_kind.clear();
    memset(&c->prof, 0, sizeof(c->prof));
    cudaEvent_t init_a = nullptr, init_b = nullptr;
    if (graph_mode && c->n_units == 1) {
        CK(cudaSetDevice(c->dev[0]));
        st = capture_graph(c, alg, d, make_launch(c, 0, alg));
        if (st != GUM_OK) return st;
    } else if (graph_mode) {
        for (int u = 0; u < c->n_units; u++) {
            if (!unit_local(c, u)) continue;
            st = capture_unit_graph(c, alg, u, d, make_launch(c, u, alg));
            if (st != GUM_OK) return st;
        }
    }
    CK(cudaSetDevice(c->dev[0]));
    CK(cudaEventRecord(c->ev0, c->stream[0]));
    c->launches = 0;
    c->hlaunch = 0;
    if (c->n_units > 1) {
        st = unit_barrier(c);
        if (st != GUM_OK) return st;
    }
    if (profile) {
        CK(cudaEventCreate(&init_a));
        CK(cudaEventCreate(&init_b));
        CK(cudaEventRecord(init_a, c->stream[0]));
    }
    for (int u = 0; u < c->n_units; u++) {
        if (!unit_local(c, u)) continue;
        const LaunchCfg L = make_launch(c, u, alg);
        CK(cudaSetDevice(unit_dev(c, u)));
        CK(launch_init(alg, d, L, c->stream[L.w0], L.w0, L.nw, D0, src_frag, src_local));
        c->launches += 2 + ((src_frag >= L.w0 && src_frag < L.w0 + L.nw) ? 1 : 0);
    }
    if (profile) CK(cudaEventRecord(init_b, c->stream[0]));
    if (graph_mode && c->n_units > 1) {
        for (int u = 0; u < c->n_units; u++) {
            if (!unit_local(c, u)) continue;
            CK(cudaSetDevice(unit_dev(c, u)));
            CK(cudaGraphLaunch(c->gexec_u[alg][u], c->stream[unit_w0(c, u)]));
            c->hlaunch++;
        }
        if (c->mp) {  // peers read this rank's fragment until they finish: leave together (device barrier)
            st = unit_barrier(c);
            if (st != GUM_OK) return st;
        }
    } else if (graph_mode) {
        CK(cudaGraphLaunch(c->gexec[alg], c->stream[0]));
        c->hlaunch++;
        if (getenv("GUM_DEBUG")) {  // watchdog: sample the run control block from a side stream
            cudaStream_t side;
            cudaStreamCreateWithFlags(&side, cudaStreamNonBlocking);
            for (int i = 0; i < 50 && cudaStreamQuery(c->stream[0]) == cudaErrorNotReady; i++) {
                RunCtl r;
                cudaMemcpyAsync(&r, c->rctl[0], sizeof(RunCtl), cudaMemcpyDeviceToHost, side);
                cudaStreamSynchronize(side);
                fprintf(stderr, "[gum] graph running: iter=%u done=%u tail=%u err=%u bodies=%u tail_iters=%u tbar=%u/%u\n",
                        r.iter, r.done, r.tail, r.err, r.bodies, r.tail_iters, r.tbar_cnt, r.tbar_gen);
                struct timespec ts = {0, 100000000};
                nanosleep(&ts, nullptr);
            }
            cudaStreamDestroy(side);
        }
    } else {
        // host-driven loop: launch batches of iterations, then poll the device-side done flag
        const int B = profile ? 1 : 8;
        for (;;) {
            for (int b = 0; b < B; b++) {
                for (int phase = 0; phase < 2; phase++) {
                    st = unit_barrier(c);
                    if (st != GUM_OK) return st;
                    for (int u = 0; u < c->n_units; u++) {
                        if (!unit_local(c, u)) continue;
                        const LaunchCfg L = make_launch(c, u, alg);
                        CK(cudaSetDevice(unit_dev(c, u)));
                        st = run_phase(c, alg, phase, d, L, c->stream[L.w0]);
                        if (st != GUM_OK) return st;
                    }
                }
            }
            const int hu = home_unit(c);
            CK(cudaSetDevice(c->dev[hu]));
            CK(cudaMemcpyAsync(c->h_rctl, c->rctl[hu], sizeof(RunCtl), cudaMemcpyDeviceToHost, c->stream[hu]));
            CK(cudaStreamSynchronize(c->stream[hu]));
            if (getenv("GUM_DEBUG"))
                fprintf(stderr, "[gum] host loop: iter=%u done=%u tail=%u err=%u bodies=%u tail_iters=%u nf_sweeps=%u\n",
                        c->h_rctl->iter, c->h_rctl->done, c->h_rctl->tail, c->h_rctl->err, c->h_rctl->bodies,
                        c->h_rctl->tail_iters, c->h_rctl->nf_sweeps);
            if (c->mp) {
                // the global convergence flag: every unit decided it redundantly from the same counts;
                // the ranks leave the loop together (matching barrier sequences) once all agree
                unsigned long long mine = c->h_rctl->done ? 1ull : 0ull, flags[kMaxW];
                unsigned long long pad_err = 0;
                CK(cudaMemcpy(&pad_err, c->pad[c->rank] + kMaxW, 8, cudaMemcpyDeviceToHost));
                if (pad_err) mine = 2;
                st = mp_exchange(c, &mine, sizeof(mine), flags);
                if (st != GUM_OK) return st;
                bool all = true;
                for (int r = 0; r < c->P; r++) {
                    if (flags[r] == 2) return fail(c, GUM_ENCCL, "barrier timeout: rank %d never arrived", r);
                    all = all && flags[r] == 1;
                }
                if (all) break;
            } else if (c->h_rctl->done) {
                break;
            }
        }
        st = unit_barrier(c);
        if (st != GUM_OK) return st;
    }
    CK(cudaSetDevice(c->dev[0]));
    CK(cudaEventRecord(c->ev1, c->stream[0]));
    st = sync_all(c);
    if (st != GUM_OK) return st;
    CK(cudaMemcpy(c->h_rctl, c->rctl[home_unit(c)], sizeof(RunCtl), cudaMemcpyDeviceToHost));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, c->ev0, c->ev1));
    const RunCtl R = *c->h_rctl;
    if (profile) {
        float t = 0.f;
        CK(cudaEventElapsedTime(&t, init_a, init_b));
        c->prof.init_ms = t;
        c->prof.init_launches = (alg == GUM_BFS || alg == GUM_SSSP) ? 3 : (alg == GUM_PR ? 3 : 2);
        cudaEventDestroy(init_a);
        cudaEventDestroy(init_b);
        for (size_t i = 0; i < c->prof_kind.size(); i++) {
            CK(cudaEventElapsedTime(&t, c->prof_ev[2 * i], c->prof_ev[2 * i + 1]));
            switch (c->prof_kind[i]) {
                case KER_FILTER: c->prof.filter_ms += t; c->prof.filter_launches++; break;
                case KER_CONTROL: c->prof.control_ms += t; c->prof.control_launches++; break;
                case KER_ADVANCE: c->prof.advance_ms += t; c->prof.advance_launches++; break;
                case KER_TAIL: c->prof.tail_ms += t; c->prof.tail_launches++; break;
                default: c->prof.finalize_ms += t; c->prof.finalize_launches++; break;
            }
        }
    }
#ifdef GUM_FILTER_TIMING
    dump_filter_timing();
#endif
    c->last_alg = alg;
    c->last_iters = R.iter;
    if (R.err == 2) return fail(c, GUM_ENCCL, "device barrier timeout: a unit never arrived");
    if (R.err) return fail(c, GUM_ERANGE, "SSSP distance reached 2^32-1");
    if (stats) {
        memset(stats, 0, sizeof(*stats));
        stats->iterations = R.iter;
        stats->ms = ms;
        stats->final_owners = R.m;
        stats->osteal_iteration = R.osteal_iter;
        stats->pr_last_residual = R.pr_resid;
        stats->osteal_p = R.os_p_n ? R.os_p : d.os_p;
        stats->osteal_p_samples = R.os_p_n;
        stats->tail_iterations = R.tail_iters;
        stats->blocked_iterations = R.blocked_iters;
        stats->bodies = R.bodies;
        stats->kernel_launches = c->launches;
        stats->host_launches = c->launches + c->hlaunch;
        if (graph_mode && c->n_units == 1) {
            const LaunchCfg L0 = make_launch(c, 0, alg);
            stats->kernel_launches += (unsigned long long)(R.iter + 1) * (count_phase(alg, 0, d, L0) + count_phase(alg, 1, d, L0));
        } else if (graph_mode) {
            // per local unit: its executed bodies (control launches that did work, + the exiting one)
            for (int u = 0; u < c->n_units; u++) {
                if (!unit_local(c, u)) continue;
                RunCtl ru;
                CK(cudaSetDevice(unit_dev(c, u)));
                CK(cudaMemcpy(&ru, c->rctl[unit_w0(c, u)], sizeof(RunCtl), cudaMemcpyDeviceToHost));
                const LaunchCfg Lu = make_launch(c, u, alg);
                stats->kernel_launches += (unsigned long long)(ru.bodies + 1) * (count_phase(alg, 0, d, Lu) + count_phase(alg, 1, d, Lu) + 2);
            }
        }
        // device barrier arrivals per unit (multi-unit runs): an evicted unit stops arriving
        for (int u = 0; u < c->n_units && c->n_units > 1; u++) {
            unsigned long long pw[2] = {0, 0};
            const unsigned long long* pu = c->pad[unit_w0(c, u)];
            if (!pu) continue;
            CK(cudaSetDevice(unit_dev(c, u)));
            CK(cudaMemcpy(pw, pu + kPadArr, 16, cudaMemcpyDeviceToHost));
            stats->unit_barriers[u] = (uint32_t)pw[0];
            stats->unit_last_iter[u] = (uint32_t)pw[1];
        }
        unsigned long long qedges_total = 0;
        for (int f = 0; f < c->P; f++) {
            FragCtl fc;
            CK(cudaSetDevice(c->fr[f].dev));
            CK(cudaMemcpy(&fc, c->fr[f].ctl, sizeof(FragCtl), cudaMemcpyDeviceToHost));
            stats->edges_expanded += fc.edges_done;
            stats->edges_stolen += fc.edges_stolen;
            stats->chunks_stolen += fc.chunks_stolen;
            stats->chunks_total += fc.chunks_done;
            stats->edges_frontier += fc.frontier_edges;
            stats->remote_updates += fc.remote_updates;
            stats->activations += fc.activations;
            stats->vertices_frontier += fc.frontier_vertices;
            stats->remote_filtered += fc.remote_filtered;
            stats->hub_cached_edges += fc.hub_edges;
            stats->tail_edges += fc.tail_edges;
            stats->tail_vertices += fc.tail_vertices;
            stats->tail_activations += fc.tail_acts;
            stats->tail_overflows += fc.tail_ovf;
            stats->migrated_queue_entries += fc.migrated_q;
            if (getenv("GUM_DEBUG"))
                fprintf(stderr, "[gum] frag %d: V=%u E=%llu qlen=%llu edges_done=%llu frontier_edges=%llu frontier_vertices=%llu app_cnt=%u tcnt=%u,%u,%u\n",
                        f, c->fr[f].V, (unsigned long long)(alg == GUM_WCC ? c->fr[f].sE : c->fr[f].E), fc.qlen,
                        fc.edges_done, fc.frontier_edges, fc.frontier_vertices, fc.app_cnt, fc.tcnt[0], fc.tcnt[1], fc.tcnt[2]);
            qedges_total += fc.qedges;
        }
        if (alg == GUM_PR) {
            stats->edges_frontier = qedges_total * R.iter;
            stats->vertices_frontier = 0;
            for (int f = 0; f < c->P; f++) stats->vertices_frontier += c->fr[f].pr_qlen * R.iter;
            if (d.mirrors) stats->mirror_flush_bytes = (unsigned long long)R.iter * (c->P - 1) * c->V * 8ull;
        }
        CK(cudaSetDevice(c->dev[0]));
    }
    c->has_result = true;
    return GUM_OK;
}

static gum_status gather_result(gum_ctx* c, void* dst_dev) {
    const bool pr = c->last_alg == GUM_PR || c->last_alg == GUM_DPR;  // double results
    const DevCtx d = make_devctx(c, c->last_alg);
    for (int f = 0; f < c->P; f++) {
        CK(cudaSetDevice(c->fr[f].dev));
        CK(launch_gather(d, f, dst_dev, pr, c->stream[c->split ? f : 0], c->nsm * 4));
    }
    return sync_all(c);
}

gum_status gum_result(gum_ctx* c, void* out, uint64_t out_bytes) {
    if (!c) return GUM_EINVAL;
    if (c->poisoned) return fail(c, GUM_ESTATE, "context poisoned");
    if (!c->has_result) return fail(c, GUM_ESTATE, "gum_result before a successful gum_run");
    if (!out) return fail(c, GUM_EINVAL, "null output buffer");
    const size_t es = (c->last_alg == GUM_PR || c->last_alg == GUM_DPR) ? 8 : 4;
    if (out_bytes < (uint64_t)c->V * es) return fail(c, GUM_EINVAL, "output buffer too small");
    gum_status st = gather_result(c, c->d_res);
    if (st != GUM_OK) return st;
    CK(cudaSetDevice(c->dev[0]));
    CK(cudaMemcpyAsync(out, c->d_res, (size_t)c->V * es, cudaMemcpyDeviceToHost, c->stream[0]));
    CK(cudaStreamSynchronize(c->stream[0]));
    return GUM_OK;
}

gum_status gum_result_device(gum_ctx* c, void* out, uint64_t out_bytes) {
    if (!c) return GUM_EINVAL;
    if (c->poisoned) return fail(c, GUM_ESTATE, "context poisoned");
    if (!c->has_result) return fail(c, GUM_ESTATE, "gum_result_device before a successful gum_run");
    if (!out) return fail(c, GUM_EINVAL, "null output buffer");
    const size_t es = (c->last_alg == GUM_PR || c->last_alg == GUM_DPR) ? 8 : 4;
    if (out_bytes < (uint64_t)c->V * es) return fail(c, GUM_EINVAL, "output buffer too small");
    return gather_result(c, out);
}

gum_status gum_fsteal_plan(const uint64_t* loads, int n, double remote_cost, double* X, double* z) {
    if (!loads || !X || n < 1 || n > kMaxW) return GUM_EINVAL;
    unsigned long long l[kMaxW];
    for (int i = 0; i < n; i++) l[i] = loads[i];
    const double zz = fsteal_waterfill(l, n, remote_cost > 0.0 ? remote_cost : 1.0, X);
    if (z) *z = zz;
    return GUM_OK;
}

gum_status gum_osteal_plan(const uint64_t* loads, int n, double remote_cost, double p, double* cost, int* m_out) {
    if (!loads || !m_out || n < 1 || n > kMaxW || p < 0.0) return GUM_EINVAL;
    unsigned long long l[kMaxW];
    for (int i = 0; i < n; i++) l[i] = loads[i];
    *m_out = osteal_choose(l, n, remote_cost > 0.0 ? remote_cost : 1.0, p, cost);
    return GUM_OK;
}

gum_status gum_profile(const gum_ctx* c, gum_kernel_times* out) {
    if (!c || !out) return GUM_EINVAL;
    if (!(c->cfg.flags & GUM_CFG_PROFILE)) return GUM_ESTATE;
    *out = c->prof;
    return GUM_OK;
}

gum_status gum_trace(const gum_ctx* cc, gum_iter_trace* out, uint32_t max_records, uint32_t* n_records) {
    gum_ctx* c = const_cast<gum_ctx*>(cc);
    if (!c || !n_records) return GUM_EINVAL;
    *n_records = 0;
    if (!c->has_result) return fail(c, GUM_ESTATE, "no run to trace");
    if (!c->trace[0]) return fail(c, GUM_ESTATE, "tracing disabled (GUM_CFG_TRACE)");
    uint32_t n = std::min<uint32_t>(std::min<uint32_t>(c->last_iters, kTraceMax), max_records);
    if (n && out) {
        CK(cudaSetDevice(c->dev[0]));
        CK(cudaMemcpy(out, c->trace[0], n * sizeof(gum_iter_trace), cudaMemcpyDeviceToHost));
        // multi-device: worker w's busy window and edge counts live in its own unit's buffer
        if (c->split) {
            std::vector<gum_iter_trace> tmp(n);
            for (int w = 1; w < c->P; w++) {
                CK(cudaSetDevice(c->dev[w]));
                CK(cudaMemcpy(tmp.data(), c->trace[w], n * sizeof(gum_iter_trace), cudaMemcpyDeviceToHost));
                for (uint32_t i = 0; i < n; i++) {
                    out[i].t_start[w] = tmp[i].t_start[w];
                    out[i].t_end[w] = tmp[i].t_end[w];
                    out[i].edges_own[w] = tmp[i].edges_own[w];
                    out[i].edges_stolen[w] = tmp[i].edges_stolen[w];
                }
            }
        }
    }
    *n_records = n;
    return GUM_OK;
}

}  // extern "C"
