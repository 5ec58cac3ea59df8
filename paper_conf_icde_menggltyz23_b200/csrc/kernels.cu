// sm_100a kernels of the GUM hot path. PAPER.md lines as P:<line>.
//
// One BSP iteration (GAS on BSP; Example 4 P:234-242) is, per launch unit (a GPU):
//   k_filter   a4  "Step 1: generate frontiers": the owner compacts its activation bitmap
//                  (dense) or activation list (sparse) into a degree-filtered queue, with the
//                  exclusive prefix of out-degrees and the edge-balanced chunk table
//                  (Alg. 1 l.9-18 PrefixSum + SortedSearch) in ONE decoupled-look-back pass.
//   k_control  a5/a6/a7-gate  workload sync + convergence, OSteal owner-set shrink (§IV,
//                  P:158-160, reduction tree P:162), FSteal gating t1/t2.
//   k_advance  a7/a8/a9  persistent CTAs claim edge-balanced chunks of their own fragments' queues
//                  (atomic claim counter = steal-queue head); when drained they steal chunks of the
//                  most-loaded peer queue and read the victim's CSR in place. Per edge:
//                  GAS Apply as atomicMin / red.add into the OWNER fragment's state (local or peer),
//                  activation = atomicOr on the owner's bitmap + warp-aggregated append.
//   k_pr_finalize a11  x' = (1-d)/V + d(acc + D/V), dangling mass and residual (PR, fp64).
#include <cuda_runtime.h>
#include <cstdio>
#include <stdint.h>
#include <stdlib.h>

#include "gum_internal.h"
#include "kernels.h"
#include "planner.h"

namespace gum {

// ------------------------------------------------------------------------------------------ utils
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
template <typename T>
__device__ __forceinline__ T vload(const T* p) {
    return *(const volatile T*)p;
}
__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

__host__ __device__ __forceinline__ unsigned gcd_u32(unsigned a, unsigned b) {
    while (b) {
        const unsigned t = a % b;
        a = b;
        b = t;
    }
    return a;
}

// The frontier queue of fragment f when worker o owns it: a foster queue in o's memory under NEXT-3
// copy-migration, else the fragment's own.
__device__ __forceinline__ QPtrs queue_of(const DevCtx& c, int f, unsigned o) {
    if (c.migrate && o != (unsigned)f && c.fq[o][f].q_v) return c.fq[o][f];
    const FragPtrs& F = c.f[f];
    return QPtrs{F.q_v, F.q_off, F.q_base, F.tile};
}

// owner fragment of a global (relabelled) vertex id: <= 7 compares ("global to local id").
__device__ __forceinline__ int frag_of(const DevCtx& c, unsigned v) {
    int f = 0;
#pragma unroll
    for (int i = 1; i < kMaxW; i++) f += (i < c.P && v >= c.bounds[i]) ? 1 : 0;
    return f;
}

// ------------------------------------------------------------------------------------------ init
template <int ALG>
__global__ void k_init(const __grid_constant__ DevCtx c, int f0) {
    const int f = f0 + blockIdx.y;
    const FragPtrs& F = c.f[f];
    const unsigned nwords = (F.V + 31) / 32;
    const unsigned n = F.V > nwords ? F.V : nwords;
    for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        if (i < F.V) {
            if (ALG == ALG_BFS || ALG == ALG_SSSP) F.state[i] = GUM_INF;
            if (ALG == ALG_WCC) F.state[i] = F.orig ? F.orig[i] : F.base + i;
            if (ALG == ALG_WCC || ALG == ALG_PR || ALG == ALG_DPR) F.app[i] = i;  // all-active frontier as a list too
            if (ALG == ALG_DPR) {  // delta-PR: x = 0, residual (in acc) = (1-d)/V, every vertex active
                F.x[i] = 0.0;
                F.acc[i] = (1.0 - c.pr_d) / (double)c.num_vertices;
                F.cx[i] = 0.0;
            }
            if (ALG == ALG_PR) {
                const double x0 = 1.0 / (double)c.num_vertices;
                const unsigned long long od = F.row_ptr[i + 1] - F.row_ptr[i];
                F.x[i] = x0;
                F.acc[i] = 0.0;
                F.cx[i] = od ? x0 / (double)od : 0.0;  // the contribution x/outdeg pushed along out-edges
                for (int r = 0; r < c.n_rep; r++) c.cxrep[r][F.base + i] = F.cx[i];  // pull replicas, buffer 0
            }
        }
        if (i < nwords) {
            unsigned wv = 0;
            if (ALG == ALG_PR || ALG == ALG_DPR || (ALG == ALG_WCC && !F.sq_col)) {
                unsigned rem = F.V - i * 32;
                wv = rem >= 32 ? 0xFFFFFFFFu : ((1u << rem) - 1u);
            }
            F.bm[i] = wv;
            if (ALG == ALG_BFS) F.vis[i] = 0u;
            F.bm2[i] = 0u;
            if (ALG == ALG_SSSP) F.far[i] = 0u;
        }
    }
    // NEXT-1: worker f's outer-vertex mirror starts empty (global id space; own slice never touched)
    if (c.mirrors) {
        const unsigned NV = c.num_vertices;
        const unsigned nm = ALG == ALG_BFS ? (NV + 31) / 32 : NV;
        for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < nm; i += gridDim.x * blockDim.x) {
            if (ALG == ALG_PR) F.macc[i] = 0.0;
            if (ALG == ALG_BFS) F.msent[i] = 0u;
            if (ALG == ALG_SSSP || ALG == ALG_WCC) F.mmin[i] = GUM_INF;
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        FragCtl* ct = F.ctl;
        ct->claim = 0;
        // PR: the frontier is the static destination-blocked queue built by gum_prepare(PR)
        // WCC with a blocked symmetric graph: iteration 0 runs on that static queue (no filter pass)
        const bool sq = ALG == ALG_WCC && F.sq_col;
        ct->ntiles = (ALG == ALG_PR) ? (F.pr_qedges + c.chunk - 1) / c.chunk : (sq ? (F.sq_edges + c.chunk - 1) / c.chunk : 0);
        ct->qlen = (ALG == ALG_PR) ? F.pr_qlen : (sq ? F.sq_len : 0);
        ct->qedges = (ALG == ALG_PR) ? F.pr_qedges : (sq ? F.sq_edges : 0);
        ct->app_cnt = ((ALG == ALG_WCC && !sq) || ALG == ALG_DPR) ? F.V : 0;
        ct->err = 0;
        ct->dense = 0;
        ct->pr_dang[0] = ct->pr_dang[1] = 0.0;
        ct->pr_resid[0] = ct->pr_resid[1] = 0.0;
        ct->edges_done = ct->edges_stolen = ct->chunks_stolen = ct->chunks_done = 0;
        ct->frontier_edges = ct->remote_updates = ct->activations = 0;
        ct->frontier_vertices = 0;
        ct->far_cnt = 0;
        ct->far_min[0] = ct->far_min[1] = GUM_INF;
        ct->far_n[0] = ct->far_n[1] = 0;
        ct->pull_checked = 0;
        ct->remote_filtered = 0;
        ct->hub_edges = 0;
        ct->tail_edges = ct->tail_vertices = ct->tail_acts = 0;
        ct->tail_ovf = 0;
        ct->fpack = 0;  // one-pass filter reservation (a run that stopped mid-filter leaves no residue)
        ct->fdone = 0;
        ct->qown = (unsigned)f;
        ct->migrated_q = 0;
        if (sq) {
            ct->frontier_edges = F.sq_edges;
            ct->frontier_vertices = F.sq_len;
        }
    }
}

// source activation (BFS/SSSP): runs after k_init on the source's owner unit.
__global__ void k_init_source(const __grid_constant__ DevCtx c, int f, unsigned ls) {
    const FragPtrs& F = c.f[f];
    F.state[ls] = 0;
    if (F.vis) F.vis[ls >> 5] |= 1u << (ls & 31);
    F.bm[ls >> 5] |= 1u << (ls & 31);
    F.app[0] = ls;
    F.ctl->app_cnt = 1;
}

__global__ void k_init_run(const __grid_constant__ DevCtx c, int w0, double D0, unsigned next_dense0,
                           unsigned skip_filter0) {
    RunCtl* rc = c.rctl[w0];
    rc->next_dense = next_dense0;
    rc->skip_filter = skip_filter0;
    rc->blocked = skip_filter0 ? 1u : 0u;
    rc->blocked_iters = 0;
    rc->iter = 0;
    rc->done = 0;
    rc->m = c.P;
    rc->steal_ok = 0;
    for (int i = 0; i < kMaxW; i++) {
        rc->owner[i] = i;
        rc->ticket[i] = 0;
        rc->filt_done[i] = 0;
    }
    rc->err = 0;
    rc->osteal_iter = 0;
    rc->epoch = rc->epoch + 1;
    rc->pr_D = D0;
    rc->pr_resid = 0.0;
    rc->nf_sweep = 0;
    rc->nf_sweeps = 0;
    rc->tail = 0;
    rc->tbar_cnt = 0;
    rc->tail_iters = 0;
    rc->bodies = 0;
    rc->tsplit_cnt[0] = rc->tsplit_cnt[1] = 0;
    rc->fbar_cnt = 0;
    rc->fctl_cnt = 0;
    rc->pb = 0;
    rc->pull = 0;
    rc->nf_T = c.nf_delta ? (unsigned long long)c.nf_delta : 0xFFFFFFFFull;
    // device-resident multi-unit loop: every unit is a member at the start (bar_ep and wakes[] stay
    // monotone across runs: the pads keep their last values)
    rc->mb = rc->mb_next = (unsigned)c.n_units;
    rc->os_p = 0.0;
    rc->os_p_n = 0;
    for (int i = 0; i < 4; i++) {
        rc->h_tctl[i] = rc->h_adv1[i] = rc->h_edges[i] = 0;
        rc->h_adv0[i] = ~0ull;
        rc->h_m[i] = 1;
        rc->h_tail[i] = 1;  // no measurement from iterations that did not run
    }
    if (c.pad[w0]) {
        c.pad[w0][kPadArr] = 0;
        c.pad[w0][kPadLastIt] = 0;
    }
}

// ------------------------------------------------------------------------------------------ filter
// Block-wide exclusive scan of (count, degree-sum) pairs; returns the block totals.
struct Pair {
    unsigned long long cnt, deg;
};
__device__ __forceinline__ Pair block_excl_scan(Pair v, Pair* s_warp, Pair& total) {
    const unsigned lane = lane_id(), wid = threadIdx.x >> 5;
    Pair inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned long long c = __shfl_up_sync(0xffffffffu, inc.cnt, o);
        unsigned long long d = __shfl_up_sync(0xffffffffu, inc.deg, o);
        if (lane >= (unsigned)o) {
            inc.cnt += c;
            inc.deg += d;
        }
    }
    if (lane == 31) s_warp[wid] = inc;
    __syncthreads();
    Pair wexcl{0, 0};
    total = Pair{0, 0};
    for (int i = 0; i < kThreads / 32; i++) {
        if ((unsigned)i < wid) {
            wexcl.cnt += s_warp[i].cnt;
            wexcl.deg += s_warp[i].deg;
        }
        total.cnt += s_warp[i].cnt;
        total.deg += s_warp[i].deg;
    }
    __syncthreads();
    return Pair{wexcl.cnt + inc.cnt - v.cnt, wexcl.deg + inc.deg - v.deg};
}

// Block scan of one filter tile's (count, degree) pairs packed into one u64: a tile holds <= 2048
// accepted vertices (12 bits) and a degree sum < 2^52 edges, so each step is one 64-bit shuffle instead
// of two (C2 filter 0.396 -> 0.383 ms per run). Same contract as block_excl_scan.
static_assert(kThreads * kDenseVertsPerThread < 4096 && kThreads * kFilterAppPerThread < 4096,
              "block_excl_scan_tile keeps a tile's count in 12 bits");
__device__ __forceinline__ Pair block_excl_scan_tile(Pair v, Pair* s_warp, Pair& total) {
    constexpr unsigned kCntShift = 52;
    constexpr unsigned long long kDegMask = (1ull << kCntShift) - 1;
    const unsigned lane = lane_id(), wid = threadIdx.x >> 5;
    const unsigned long long key = (v.cnt << kCntShift) | v.deg;
    unsigned long long inc = key;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= (unsigned)o) inc += y;
    }
    unsigned long long* s_w = reinterpret_cast<unsigned long long*>(s_warp);
    if (lane == 31) s_w[wid] = inc;
    __syncthreads();
    unsigned long long wexcl = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < kThreads / 32; i++) {
        const unsigned long long x = s_w[i];
        if ((unsigned)i < wid) wexcl += x;
        tot += x;
    }
    __syncthreads();
    const unsigned long long ex = wexcl + inc - key;
    total = Pair{tot >> kCntShift, tot & kDegMask};
    return Pair{ex >> kCntShift, ex & kDegMask};
}

// Chunk-table runs of long adjacency lists (> kLongInline chunk starts) are deferred to a per-CTA list and
// written by whole warps after the tile (filter_flush_long): with a degree-ordered layout the hubs sit in
// the first tiles, and one thread writing hundreds of entries serialised the whole filter.
constexpr int kLongCap = 512;
constexpr unsigned kLongInline = 2;
__shared__ unsigned s_long_n;
__shared__ unsigned s_long_pos[kLongCap], s_long_t0[kLongCap], s_long_t1[kLongCap];
__shared__ QPtrs s_qo;  // the filter CTA's output queue (queue_of the fragment under its current owner)
__shared__ const unsigned* s_src;  // the filter CTA's sparse input: the activation list, or a far list (sweep)

__device__ __forceinline__ void emit_vertex(const FragPtrs& F, unsigned chunk, unsigned v, unsigned long long rp,
                                            unsigned long long deg, unsigned long long pos, unsigned long long off) {
    (void)F;
    s_qo.q_v[pos] = v;
    s_qo.q_off[pos] = off;
    s_qo.q_base[pos] = (long long)rp - (long long)off;
    // chunk table: every chunk whose first edge lies in [off, off+deg) starts at queue entry pos
    unsigned long long t = (off + chunk - 1) / chunk;
    const unsigned long long t1 = (off + deg + chunk - 1) / chunk;
    if (t1 - t > kLongInline) {
        const unsigned i = atomicAdd(&s_long_n, 1u);
        if (i < (unsigned)kLongCap) {
            s_long_pos[i] = (unsigned)pos;
            s_long_t0[i] = (unsigned)t;
            s_long_t1[i] = (unsigned)t1;
            return;
        }
    }
    for (; t < t1; t++) s_qo.tile[t] = (unsigned)pos;
}

// all threads of the CTA: write the deferred chunk-table runs (a warp per run, lanes over its chunks)
__device__ __forceinline__ void filter_flush_long(const FragPtrs& F) {
    __syncthreads();
    const unsigned n = s_long_n < (unsigned)kLongCap ? s_long_n : (unsigned)kLongCap;
    if (n == 0) return;  // CTA-uniform (read after the barrier; the next append follows another barrier)
    for (unsigned e = threadIdx.x >> 5; e < n; e += kThreads / 32) {
        const unsigned pos = s_long_pos[e], t1 = s_long_t1[e];
        for (unsigned t = s_long_t0[e] + (threadIdx.x & 31); t < t1; t += 32) s_qo.tile[t] = pos;
    }
    __syncthreads();
    if (threadIdx.x == 0) s_long_n = 0;
}

// Dense partitions: 8 warps x 32 bitmap words (8192 vertices); a warp walks its words i-major,
// lane-minor (vertex = word*32 + lane), so row_ptr reads are coalesced and the queue is sorted.

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long x) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    return x;
}
__device__ __forceinline__ unsigned long long warp_excl_scan_u64(unsigned long long x, unsigned long long& total) {
    unsigned long long inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned long long y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane_id() >= (unsigned)o) inc += y;
    }
    total = __shfl_sync(0xffffffffu, inc, 31);
    return inc - x;
}


#ifndef GUM_FILTER_MINB
#define GUM_FILTER_MINB 4
#endif

// One filter tile (2048 items: 64 bitmap words in dense mode, 2048 activation-list entries in sparse
// mode). Thread t owns 8 consecutive items; returns its (count, degree) of accepted vertices (out-degree
// > 0 and, with the SSSP near-far split, dist < T) in vertex order.
//   FT_CLASSIFY (pass 1): near-far parking happens here, once (far bit, far count, far minimum);
//   FT_COUNT    (pass 2a): pure re-count with the same acceptance (dist < T);
//   FT_EMIT     (pass 2b): writes the queue entries from pos/off on, clears the consumed bitmap words and
//                          the far bits of accepted vertices.
enum { FT_CLASSIFY = 0, FT_COUNT = 1, FT_EMIT = 2 };
// per-thread near-far bookkeeping, reduced per warp before touching the fragment's counters (they are
// single addresses: per-vertex atomics there serialise in the L2 atomic unit)
struct NfAcc {
    unsigned long long parked = 0, unparked = 0;
    unsigned min_dist = 0xFFFFFFFFu;
    unsigned fslot = 0;       // far list receiving new / still-parked vertices (nf_sweeps & 1)
    bool sweep_list = false;  // this filter sweeps the previous far list (its entries are all parked)
};
// Acceptance of a thread's 8 candidates (bit q of cand: vertex vs[q] has out-degree > 0) under the
// near-far split, batched so that the 8 state loads and then the 8 far-bit atomics are each in flight
// together (one dependent round trip per step instead of one per vertex). Returns the accepted mask.
template <int MODE>
__device__ __forceinline__ unsigned filter_accept8(const FragPtrs& F, const unsigned* vs, unsigned cand, bool nf,
                                                   unsigned nfT, NfAcc& acc) {
    if (!nf || !cand) return cand;
    unsigned st[8];
#pragma unroll
    for (int q = 0; q < 8; q++) st[q] = ((cand >> q) & 1u) ? F.state[vs[q]] : 0u;
    unsigned ok = 0, park = 0;
#pragma unroll
    for (int q = 0; q < 8; q++) {
        if (!((cand >> q) & 1u)) continue;
        if (st[q] < nfT) ok |= 1u << q;
        else park |= 1u << q;
    }
    if (MODE == FT_CLASSIFY && park) {
        unsigned ob[8];
#pragma unroll
        for (int q = 0; q < 8; q++)
            ob[q] = ((park >> q) & 1u) ? atomicOr(F.far + (vs[q] >> 5), 1u << (vs[q] & 31)) : 0xFFFFFFFFu;
        // the far set is also a list: a newly parked vertex is appended, and a sweep re-appends the entries
        // of the previous list that stay parked (a far bit is set <=> the vertex is in the current list)
        unsigned lst = 0;
#pragma unroll
        for (int q = 0; q < 8; q++) {
            if (!((park >> q) & 1u)) continue;
            const bool fresh = !(ob[q] & (1u << (vs[q] & 31)));
            if (fresh) acc.parked++;
            if (fresh || acc.sweep_list) lst |= 1u << q;
            acc.min_dist = st[q] < acc.min_dist ? st[q] : acc.min_dist;
        }
        if (lst && F.farl) {
            unsigned pos = atomicAdd(&F.ctl->far_n[acc.fslot], (unsigned)__popc(lst));
            unsigned* fl = F.farl + (size_t)acc.fslot * F.V;
#pragma unroll
            for (int q = 0; q < 8; q++)
                if ((lst >> q) & 1u) fl[pos++] = vs[q];
        }
    }
    // with far lists a vertex leaves the far set only when a sweep takes it: an entry accepted in a normal
    // iteration keeps its bit and is looked at again by the next sweep (one extra look, no duplicate entry)
    if (MODE == FT_EMIT && ok && (acc.sweep_list || !F.farl)) {
        // accepted vertices leave the far set (their bit may be left from an earlier parking)
        unsigned fw[8], ob[8];
#pragma unroll
        for (int q = 0; q < 8; q++) fw[q] = ((ok >> q) & 1u) ? F.far[vs[q] >> 5] : 0u;
#pragma unroll
        for (int q = 0; q < 8; q++)
            ob[q] = (((ok >> q) & 1u) && (fw[q] & (1u << (vs[q] & 31)))) ? atomicAnd(F.far + (vs[q] >> 5), ~(1u << (vs[q] & 31))) : 0u;
#pragma unroll
        for (int q = 0; q < 8; q++)
            if (ob[q] & (1u << (vs[q] & 31))) acc.unparked++;
    }
    return ok;
}

// warp-reduce the near-far counters and apply them to the fragment (lane 0 of each warp)
__device__ __forceinline__ void nf_flush(FragCtl* ct, unsigned fslot, const NfAcc& a) {
    const unsigned long long p = warp_sum_u64(a.parked), u = warp_sum_u64(a.unparked);
    const unsigned m = __reduce_min_sync(0xffffffffu, a.min_dist);
    if (lane_id() == 0) {
        if (p != u) atomicAdd(&ct->far_cnt, p - u);  // two's complement: a net decrement wraps correctly
        if (m != 0xFFFFFFFFu) atomicMin(&ct->far_min[fslot], m);
    }
}

// delta-PR (reading #27): an activated vertex hands its residual over when the filter takes it into the next
// frontier: x += r, push value cx = d*r/outdeg (0 for a dangling vertex), r = 0 (BSP: no advance runs now)
__device__ __forceinline__ void dpr_take(const FragPtrs& F, unsigned v, unsigned long long od, double dd) {
    const double dl = F.acc[v];
    F.x[v] += dl;
    F.acc[v] = 0.0;
    F.cx[v] = od ? dd * dl / (double)od : 0.0;
}

template <int MODE, bool DPR = false>
__device__ __forceinline__ Pair filter_tile(const FragPtrs& F, NfAcc& acc, bool keep_fbm, unsigned depth, unsigned tile, bool dense, bool sweep,
                                            bool nf, unsigned nfT, unsigned nwords, unsigned app_cnt, unsigned ipt,
                                            unsigned chunk, unsigned long long pos, unsigned long long off, double dd = 0.0) {
    const unsigned lane = lane_id();
    Pair mine{0, 0};
    if (dense) {
        const unsigned wbase = tile * kDenseWordsPerPart + (threadIdx.x >> 5) * kDenseWordsPerWarp;
        const unsigned vb = wbase * 32u + lane * kDenseVertsPerThread;
        const unsigned wi = wbase + (lane >> 2);
        unsigned word = 0;
        if (wi < nwords) {
            word = F.bm[wi];
            if (sweep) word |= F.far[wi];  // (sweep without a far list: the bitmap)
        }
        if (MODE == FT_EMIT) {
            __syncwarp();
            if ((lane & 3u) == 0 && wi < nwords) {
                if (keep_fbm) F.far[wi] = word;  // WCC: the frontier as a bitmap for a masked blocked pass
                if (F.bm[wi]) F.bm[wi] = 0u;
            }
        }
        const unsigned bits = (word >> ((lane & 3u) * 8u)) & 0xFFu;
        if (MODE == FT_EMIT && depth != GUM_INF && bits) {
            // BFS: the depth of every vertex activated by the previous advance is written here, in vertex
            // order, instead of by every discovering edge in the advance (a random 4-byte store each):
            // the thread's 8 consecutive states as two 16-byte read-modify-writes
            if (vb + kDenseVertsPerThread <= F.V) {
                uint4* sp = reinterpret_cast<uint4*>(F.state + vb);  // 32-byte aligned (vb % 8 == 0)
                uint4 a = bits == 0xFFu ? make_uint4(0, 0, 0, 0) : __ldcg(sp);
                uint4 b = bits == 0xFFu ? make_uint4(0, 0, 0, 0) : __ldcg(sp + 1);
                if (bits & 1u) a.x = depth;
                if (bits & 2u) a.y = depth;
                if (bits & 4u) a.z = depth;
                if (bits & 8u) a.w = depth;
                if (bits & 16u) b.x = depth;
                if (bits & 32u) b.y = depth;
                if (bits & 64u) b.z = depth;
                if (bits & 128u) b.w = depth;
                if (bits & 0x0Fu) sp[0] = a;
                if (bits & 0xF0u) sp[1] = b;
            } else {
#pragma unroll
                for (int q = 0; q < kDenseVertsPerThread; q++)
                    if ((bits >> q) & 1u) F.state[vb + q] = depth;
            }
        }
        if (bits) {
            unsigned long long rpv[kDenseVertsPerThread + 1];
            const unsigned long long* rp = F.row_ptr + vb;  // 64-byte aligned (vb % 8 == 0)
            if (vb + kDenseVertsPerThread <= F.V) {
#pragma unroll
                for (int q = 0; q < kDenseVertsPerThread / 2; q++) {
                    const ulonglong2 t2 = __ldg(reinterpret_cast<const ulonglong2*>(rp) + q);
                    rpv[2 * q] = t2.x;
                    rpv[2 * q + 1] = t2.y;
                }
                rpv[kDenseVertsPerThread] = __ldg(rp + kDenseVertsPerThread);
            } else {
#pragma unroll
                for (int q = 0; q <= kDenseVertsPerThread; q++) rpv[q] = (vb + q <= F.V) ? __ldg(rp + q) : 0ull;
            }
            if (DPR && MODE == FT_EMIT) {
#pragma unroll
                for (int q = 0; q < kDenseVertsPerThread; q++)
                    if ((bits >> q) & 1u) dpr_take(F, vb + q, rpv[q + 1] - rpv[q], dd);
            }
            static_assert(kDenseVertsPerThread == 8, "filter_accept8 takes 8 candidates");
            unsigned vs[8], cand = 0;
#pragma unroll
            for (int q = 0; q < kDenseVertsPerThread; q++) {
                vs[q] = vb + q;
                if (((bits >> q) & 1u) && rpv[q + 1] != rpv[q]) cand |= 1u << q;
            }
            const unsigned ok = filter_accept8<MODE>(F, vs, cand, nf, nfT, acc);
#pragma unroll
            for (int q = 0; q < kDenseVertsPerThread; q++) {
                if ((ok >> q) & 1u) {
                    const unsigned long long d = rpv[q + 1] - rpv[q];
                    if (MODE == FT_EMIT) emit_vertex(F, chunk, vb + q, rpv[q], d, pos + mine.cnt, off + mine.deg);
                    mine.cnt += 1;
                    mine.deg += d;
                }
            }
        }
    } else {
        // ipt (1..8) items per thread: short lists use small tiles so they spread over every SM
        const unsigned long long ibase = (unsigned long long)tile * (kThreads * ipt) + threadIdx.x * ipt;
        unsigned items[kFilterAppPerThread];
        unsigned long long rp0[kFilterAppPerThread], d[kFilterAppPerThread];
#pragma unroll
        for (int j = 0; j < kFilterAppPerThread; j++) {
            items[j] = 0xFFFFFFFFu;
            if ((unsigned)j < ipt && ibase + j < app_cnt) items[j] = s_src[ibase + j];
        }
#pragma unroll
        for (int j = 0; j < kFilterAppPerThread; j++) {
            d[j] = 0;
            rp0[j] = 0;
            if (items[j] != 0xFFFFFFFFu) {
                const unsigned v = items[j];
                // every set bit belongs to a listed vertex: clearing whole words is exact
                if (MODE == FT_EMIT) F.bm[v >> 5] = 0u;
                if (MODE == FT_EMIT && depth != GUM_INF) F.state[v] = depth;  // BFS (see the dense path)
                rp0[j] = __ldg(F.row_ptr + v);
                d[j] = __ldg(F.row_ptr + v + 1) - rp0[j];
                if (DPR && MODE == FT_EMIT) dpr_take(F, v, d[j], dd);
            }
        }
        static_assert(kFilterAppPerThread == 8, "filter_accept8 takes 8 candidates");
        unsigned cand = 0;
#pragma unroll
        for (int j = 0; j < kFilterAppPerThread; j++)
            if (d[j]) cand |= 1u << j;
        const unsigned ok = filter_accept8<MODE>(F, items, cand, nf, nfT, acc);
#pragma unroll
        for (int j = 0; j < kFilterAppPerThread; j++) {
            if ((ok >> j) & 1u) {
                if (MODE == FT_EMIT) emit_vertex(F, chunk, items[j], rp0[j], d[j], pos + mine.cnt, off + mine.deg);
                mine.cnt += 1;
                mine.deg += d[j];
            }
        }
    }
    return mine;
}

// Pass 2 of one dense tile without the near-far split (acceptance = out-degree > 0): the count, the
// block scan for the per-thread offsets and the emit in one walk of the tile (FT_COUNT + FT_EMIT read the
// bitmap word and the row_ptr run twice). Only the 8-bit accepted mask stays live across the scan; the
// row_ptr run is re-read after it from L1 (the same thread's lines). Returns the tile's totals.
// one-pass filter: thread 0 reserves the tile's queue range [cnt, cnt + tot.cnt) and edge range with ONE
// atomic on the packed counter (both ranges in the same order, so q_off stays the prefix of the degrees in
// queue order) and broadcasts the base; every thread returns the base in (pos, off)
__device__ __forceinline__ void filter_reserve(unsigned long long* fpack, const Pair& tot, unsigned long long& pos,
                                               unsigned long long& off) {
    __shared__ unsigned long long s_fbase;
    if (threadIdx.x == 0)
        s_fbase = tot.cnt ? atomicAdd(fpack, (tot.cnt << kFpackShift) | tot.deg) : 0ull;
    __syncthreads();
    pos = s_fbase >> kFpackShift;
    off = s_fbase & kFpackEdgeMask;
}

template <bool DPR = false>
__device__ __forceinline__ Pair filter_tile_dense_fused(const FragPtrs& F, bool keep_fbm, unsigned depth, unsigned tile,
                                                        unsigned nwords, unsigned chunk, unsigned long long pos,
                                                        unsigned long long off, Pair* s_warp, double dd = 0.0,
                                                        unsigned long long* fpack = nullptr) {
    const unsigned lane = lane_id();
    const unsigned wbase = tile * kDenseWordsPerPart + (threadIdx.x >> 5) * kDenseWordsPerWarp;
    const unsigned vb = wbase * 32u + lane * kDenseVertsPerThread;
    const unsigned wi = wbase + (lane >> 2);
    const bool full = vb + kDenseVertsPerThread <= F.V;
    const unsigned word = wi < nwords ? F.bm[wi] : 0u;
    __syncwarp();
    if ((lane & 3u) == 0 && wi < nwords) {
        if (keep_fbm) F.far[wi] = word;
        if (word) F.bm[wi] = 0u;
    }
    const unsigned bits = (word >> ((lane & 3u) * 8u)) & 0xFFu;
    if (depth != GUM_INF && bits) {
        if (full) {
            uint4* sp = reinterpret_cast<uint4*>(F.state + vb);
            uint4 a = bits == 0xFFu ? make_uint4(0, 0, 0, 0) : __ldcg(sp);
            uint4 b = bits == 0xFFu ? make_uint4(0, 0, 0, 0) : __ldcg(sp + 1);
            if (bits & 1u) a.x = depth;
            if (bits & 2u) a.y = depth;
            if (bits & 4u) a.z = depth;
            if (bits & 8u) a.w = depth;
            if (bits & 16u) b.x = depth;
            if (bits & 32u) b.y = depth;
            if (bits & 64u) b.z = depth;
            if (bits & 128u) b.w = depth;
            if (bits & 0x0Fu) sp[0] = a;
            if (bits & 0xF0u) sp[1] = b;
        } else {
#pragma unroll
            for (int q = 0; q < kDenseVertsPerThread; q++)
                if ((bits >> q) & 1u) F.state[vb + q] = depth;
        }
    }
    const unsigned long long* rp = F.row_ptr + vb;
    Pair mine{0, 0};
    unsigned ok = 0;
    if (bits) {
        unsigned long long rpv[kDenseVertsPerThread + 1];
        if (full) {
#pragma unroll
            for (int q = 0; q < kDenseVertsPerThread / 2; q++) {
                const ulonglong2 t2 = __ldg(reinterpret_cast<const ulonglong2*>(rp) + q);
                rpv[2 * q] = t2.x;
                rpv[2 * q + 1] = t2.y;
            }
            rpv[kDenseVertsPerThread] = __ldg(rp + kDenseVertsPerThread);
        } else {
#pragma unroll
            for (int q = 0; q <= kDenseVertsPerThread; q++) rpv[q] = (vb + q <= F.V) ? __ldg(rp + q) : 0ull;
        }
        if (DPR) {
#pragma unroll
            for (int q = 0; q < kDenseVertsPerThread; q++)
                if ((bits >> q) & 1u) dpr_take(F, vb + q, rpv[q + 1] - rpv[q], dd);
        }
#pragma unroll
        for (int q = 0; q < kDenseVertsPerThread; q++) {
            if (((bits >> q) & 1u) && rpv[q + 1] != rpv[q]) {
                ok |= 1u << q;
                mine.cnt += 1;
                mine.deg += rpv[q + 1] - rpv[q];
            }
        }
    }
    Pair tot;
    const Pair tex = block_excl_scan_tile(mine, s_warp, tot);
    if (fpack) filter_reserve(fpack, tot, pos, off);  // one-pass filter (CTA-uniform)
    if (ok) {
        unsigned long long p = pos + tex.cnt, o = off + tex.deg;
#pragma unroll
        for (int q = 0; q < kDenseVertsPerThread; q++) {
            if ((ok >> q) & 1u) {
                const unsigned long long r0 = __ldg(rp + q), r1 = __ldg(rp + q + 1);
                emit_vertex(F, chunk, vb + q, r0, r1 - r0, p, o);
                p += 1;
                o += r1 - r0;
            }
        }
    }
    return tot;
}

// a4 filter / frontier generation (Example 4 Step 1; Alg. 1's degree prefix sum): the
// fragment's activations (bitmap words when dense, the activation list when sparse) -> queue of
// vertices with out-degree > 0 (q_v), exclusive out-degree prefix (q_off), col base (q_base) and the
// edge-balanced chunk table. Reduce-then-scan over a static split of the tiles: CTA b (ticket order)
// counts its contiguous tile range, publishes the aggregate, sums its predecessors' aggregates (one
// parallel read, no serial look-back chain) and re-walks its range emitting entries in vertex order.
#ifdef GUM_FILTER_TIMING
__device__ unsigned long long g_ftime[1024][8];
__device__ unsigned g_fcall;
#define FT_MARK(i) do { if (threadIdx.x == 0 && g_fcall == GUM_FILTER_TIMING) g_ftime[blockIdx.x][i] = globaltimer(); } while (0)
#else
#define FT_MARK(i) do {} while (0)
#endif
// NF: SSSP near-far parking compiled in (its batched state loads and far-bit atomics cost registers the
// other algorithms' filters do not need)
__device__ __noinline__ void control_body(const DevCtx& c, const int alg, int w0, int nw, cudaGraphConditionalHandle h,
                                          int use_h);

// fuse_ctl (single launch unit, graph mode): every CTA of the filter grid arrives on a counter once it is done;
// the last one runs the iteration's control decision (control_body) -- one kernel launch less per iteration.
__device__ __forceinline__ void filter_arrive(const DevCtx& c, int w0, int nw, cudaGraphConditionalHandle h, int use_h) {
    __threadfence();  // every thread's queue / counter writes before the CTA's arrival
    __syncthreads();
    if (threadIdx.x == 0) {
        RunCtl* rc = c.rctl[w0];
        const unsigned total = gridDim.x * gridDim.y;
        if (atomicAdd(&rc->fctl_cnt, 1u) == total - 1) {
            __threadfence();
            rc->fctl_cnt = 0;
            control_body(c, c.alg, w0, nw, h, use_h);
        }
    }
}

template <bool NF, bool DPR = false>
__global__ void __launch_bounds__(kThreads, GUM_FILTER_MINB) k_filter(const __grid_constant__ DevCtx c, int w0, int nw,
                                                                      int fuse_ctl, cudaGraphConditionalHandle h, int use_h) {
    FT_MARK(0);
    // Prologue by thread 0 only, broadcast through shared memory: the run-control fields are a handful of
    // L2 lines that every CTA of every kernel reads, and per-warp loads of one address serialise in its
    // L2 slice (with ~600 CTAs x 8 warps that alone cost tens of microseconds per launch).
    struct Pro {
        unsigned go, sweep, dense, nfT, fslot, app_cnt, b, depth;
        unsigned long long epoch;
    };
    __shared__ Pro s_pro;
    __shared__ Pair s_warp[kThreads / 32];
    RunCtl* rc = c.rctl[w0];
    const int f = blockIdx.y;
    const FragPtrs& F = c.f[f];
    FragCtl* ct = F.ctl;
    const bool nf = NF && c.nf_delta != 0;
    if (threadIdx.x == 0) {
        Pro p{};
        const unsigned o = vload(&rc->owner[f]);
        p.go = !vload(&rc->done) && !vload(&rc->skip_filter) && (int)o >= w0 && (int)o < w0 + nw;
        if (p.go) {
            // SSSP near-far: only vertices with dist < T enter the queue; the rest are parked in F.far
            p.sweep = nf && vload(&rc->nf_sweep) != 0;
            const unsigned long long T = vload(&rc->nf_T);
            p.nfT = nf ? (unsigned)(T < 0xFFFFFFFFull ? T : 0xFFFFFFFFull) : GUM_INF;
            p.fslot = vload(&rc->nf_sweeps) & 1u;
            // the advance that produced these activations either appended them (sparse) or only set bits;
            // a near-far sweep (the near frontier is empty) reads the previous far list, or scans the far
            // bitmap when the list is not kept
            const bool swl = p.sweep && F.farl;
            p.dense = (p.sweep && !swl) || (!p.sweep && vload(&rc->next_dense) != 0);
            p.app_cnt = swl ? vload(&ct->far_n[p.fslot ^ 1u]) : (p.dense ? 0u : vload(&ct->app_cnt));
            s_src = swl ? F.farl + (size_t)(p.fslot ^ 1u) * F.V : F.app;
            p.epoch = vload(&rc->epoch);
            // BFS: activations of advance k-1 have depth k = the iteration counter before control runs
            p.depth = c.bfs_filter_depth ? vload(&rc->iter) : GUM_INF;
            p.b = atomicAdd(&rc->ticket[f], 1u);  // ticket order: predecessors are running
            s_qo = queue_of(c, f, o);
        }
        s_pro = p;
        s_long_n = 0;
    }
    __syncthreads();
    FT_MARK(1);
    if (!s_pro.go) {
        if (fuse_ctl) filter_arrive(c, w0, nw, h, use_h);
        return;
    }
    const bool sweep = s_pro.sweep != 0;
    const unsigned nfT = s_pro.nfT;
    const unsigned fslot = s_pro.fslot;
    const bool dense = s_pro.dense != 0;
    const unsigned app_cnt = s_pro.app_cnt;
    const bool keep_fbm = c.wcc_blocked != 0 && !nf;
    const unsigned depth = s_pro.depth;
    const double dd = DPR ? c.pr_d : 0.0;
    const unsigned nwords = (F.V + 31) / 32;
    const unsigned long long n_items = dense ? nwords : app_cnt;
    // sparse lists: items per thread so that the tiles cover the grid (1..8)
    unsigned ipt = kFilterAppPerThread;
    if (!dense) {
        const unsigned long long per_cta = (n_items + gridDim.x - 1) / gridDim.x;
        ipt = per_cta <= kThreads ? 1u : per_cta <= 2u * kThreads ? 2u : per_cta <= 4u * kThreads ? 4u : 8u;
    }
    const unsigned per = dense ? kDenseWordsPerPart : kThreads * ipt;
    const unsigned n_tiles = (unsigned)((n_items + per - 1) / per);
    const unsigned long long epoch = s_pro.epoch;
    const unsigned chunk = c.chunk;
    LBSlot* slots = c.lb[f];
    // small lists: only as many CTAs as tiles take part (the others leave before the prefix exchange)
    const unsigned G = n_tiles < gridDim.x ? (n_tiles ? n_tiles : 1u) : gridDim.x;
    const unsigned b = s_pro.b;
    if (b >= G) {
        if (fuse_ctl) filter_arrive(c, w0, nw, h, use_h);
        return;
    }
    const unsigned t_lo = (unsigned)(((unsigned long long)n_tiles * b) / G);
    const unsigned t_hi = (unsigned)(((unsigned long long)n_tiles * (b + 1)) / G);
    // logical tile t (queue order) -> physical tile (t * stride) mod n_tiles, stride coprime to n_tiles:
    // a CTA's contiguous logical range is spread over the id space, so activations clustered in one id
    // range (the DEGREE layout activates vertices of similar in-degree together) do not all land on a
    // few CTAs. The queue order is then a permutation of vertex order (nothing depends on it being sorted).
    unsigned stride = 1;
    if (c.filter_swizzle && n_tiles > 2u * G) {
        stride = 2053u;  // start at a prime; step until gcd(stride, n_tiles) == 1 (a bijection on the tiles)
        while (stride < n_tiles && gcd_u32(stride, n_tiles) != 1u) stride++;
        if (stride >= n_tiles) stride = 1;
    }

    if (!NF && c.filter_onepass) {
        // ---- one pass: per tile count -> block scan -> one packed atomic reserves the tile's queue and edge
        // ranges -> emit. No look-back and no second walk; the queue is in reservation order (nothing depends
        // on it being sorted: q_off is the prefix of the degrees in queue order, the chunk table follows it)
        unsigned long long* fpack = &ct->fpack;
        NfAcc nfo;
        for (unsigned t = t_lo; t < t_hi; t++) {
            const unsigned pt = (unsigned)((unsigned long long)t * stride % n_tiles);
            if (dense) {
                filter_tile_dense_fused<DPR>(F, keep_fbm, depth, pt, nwords, chunk, 0, 0, s_warp, dd, fpack);
            } else {
                const Pair q = filter_tile<FT_COUNT, DPR>(F, nfo, keep_fbm, depth, pt, dense, sweep, false, nfT, nwords,
                                                          app_cnt, ipt, chunk, 0, 0, dd);
                Pair tot;
                const Pair tex = block_excl_scan_tile(q, s_warp, tot);
                unsigned long long bp, bo;
                filter_reserve(fpack, tot, bp, bo);
                // (always: the emit walk also clears the consumed bitmap words and writes BFS depths)
                filter_tile<FT_EMIT, DPR>(F, nfo, keep_fbm, depth, pt, dense, sweep, false, nfT, nwords, app_cnt, ipt,
                                          chunk, bp + tex.cnt, bo + tex.deg, dd);
            }
            filter_flush_long(F);
        }
        // the last of the G participating CTAs publishes the queue and re-arms the counters
        __threadfence();
        __syncthreads();
        if (threadIdx.x == 0 && atomicAdd(&ct->fdone, 1u) == G - 1) {
            __threadfence();
            const unsigned long long pk = atomicExch(fpack, 0ull);
            ct->fdone = 0;
            const unsigned long long tc = pk >> kFpackShift, td = pk & kFpackEdgeMask;
            s_qo.q_off[tc] = td;
            ct->qlen = tc;
            ct->qown = vload(&rc->owner[f]);
            if (c.migrate && s_qo.q_v != F.q_v) ct->migrated_q += tc;
            ct->qedges = td;
            ct->ntiles = (td + chunk - 1) / chunk;
            ct->claim = 0;
            for (int q = 0; q < kMaxW; q++) ct->pclaim[q] = 0;
            ct->app_cnt = 0;
            ct->dense = dense ? 1u : 0u;
            ct->frontier_edges += td;
            ct->frontier_vertices += tc;
        }
        if (fuse_ctl) filter_arrive(c, w0, nw, h, use_h);
        return;
    }
    // ---- pass 1: aggregate of this CTA's tile range
    Pair mine{0, 0};
    NfAcc nfa;
    nfa.fslot = fslot;
    nfa.sweep_list = sweep && !dense;
    for (unsigned t = t_lo; t < t_hi; t++) {
        const Pair q = filter_tile<FT_CLASSIFY, DPR>(F, nfa, keep_fbm, depth, (unsigned)((unsigned long long)t * stride % n_tiles), dense, sweep, nf, nfT, nwords, app_cnt, ipt, chunk, 0, 0, dd);
        mine.cnt += q.cnt;
        mine.deg += q.deg;
    }
    FT_MARK(2);
    Pair agg;
    const Pair tex1 = block_excl_scan(mine, s_warp, agg);  // per-thread offsets when the CTA has one tile
    if (threadIdx.x == 0) {
        slots[b].agg_cnt = agg.cnt;
        slots[b].agg_deg = agg.deg;
        st_release_u64(&slots[b].flag, epoch * 4 + 1);
    }
    // ---- exclusive prefix: the aggregates of CTAs 0..b-1 (relaxed spin, then one acquire fence)
    Pair pre{0, 0};
    for (unsigned j = threadIdx.x; j < b; j += kThreads)
        while (vload(&slots[j].flag) < epoch * 4 + 1) __nanosleep(32);
    __threadfence();
    for (unsigned j = threadIdx.x; j < b; j += kThreads) {
        pre.cnt += __ldcg(&slots[j].agg_cnt);
        pre.deg += __ldcg(&slots[j].agg_deg);
    }
    FT_MARK(3);
    Pair excl;
    block_excl_scan(pre, s_warp, excl);  // excl = sum over all predecessors
    if (b == G - 1 && threadIdx.x == 0) {
        const unsigned long long tc = excl.cnt + agg.cnt, td = excl.deg + agg.deg;
        s_qo.q_off[tc] = td;
        ct->qlen = tc;
        ct->qown = vload(&rc->owner[f]);
        if (c.migrate && s_qo.q_v != F.q_v) ct->migrated_q += tc;
        ct->qedges = td;
        ct->ntiles = (td + chunk - 1) / chunk;
        ct->claim = 0;
        for (int q = 0; q < kMaxW; q++) ct->pclaim[q] = 0;
        ct->app_cnt = 0;
        ct->dense = dense ? 1u : 0u;
        ct->frontier_edges += td;
        ct->frontier_vertices += tc;
    }
    // ---- pass 2: per tile, re-count (L1/L2-resident re-read) for the per-thread offsets, then emit
    unsigned long long run_cnt = excl.cnt, run_deg = excl.deg;
    if (t_hi - t_lo == 1) {
        // one tile: pass 1's per-thread counts are this tile's (same acceptance), no re-count
        filter_tile<FT_EMIT, DPR>(F, nfa, keep_fbm, depth, (unsigned)((unsigned long long)t_lo * stride % n_tiles), dense, sweep, nf, nfT, nwords, app_cnt, ipt, chunk, run_cnt + tex1.cnt,
                                  run_deg + tex1.deg, dd);
        filter_flush_long(F);
    } else {
        for (unsigned t = t_lo; t < t_hi; t++) {
            const unsigned pt = (unsigned)((unsigned long long)t * stride % n_tiles);
            if (dense && !nf) {
                const Pair tot = filter_tile_dense_fused<DPR>(F, keep_fbm, depth, pt, nwords, chunk, run_cnt, run_deg, s_warp, dd);
                filter_flush_long(F);
                run_cnt += tot.cnt;
                run_deg += tot.deg;
                continue;
            }
            const Pair q = filter_tile<FT_COUNT, DPR>(F, nfa, keep_fbm, depth, pt, dense, sweep, nf, nfT, nwords, app_cnt, ipt, chunk, 0, 0, dd);
            Pair tot;
#ifdef GUM_PACK2
            const Pair tex = block_excl_scan_tile(q, s_warp, tot);  // A/B variant "pack2" (filter 0.390 ms/run on C2)
#else
            const Pair tex = block_excl_scan(q, s_warp, tot);  // "pack": packed scan in the fused dense tile only (0.384)
#endif
            filter_tile<FT_EMIT, DPR>(F, nfa, keep_fbm, depth, pt, dense, sweep, nf, nfT, nwords, app_cnt, ipt, chunk, run_cnt + tex.cnt,
                                      run_deg + tex.deg, dd);
            filter_flush_long(F);
            run_cnt += tot.cnt;
            run_deg += tot.deg;
        }
    }
    if (nf) nf_flush(ct, fslot, nfa);
    FT_MARK(4);
    if (fuse_ctl) filter_arrive(c, w0, nw, h, use_h);
#ifdef GUM_FILTER_TIMING
    if (threadIdx.x == 0 && g_fcall == GUM_FILTER_TIMING) { g_ftime[blockIdx.x][5] = b; g_ftime[blockIdx.x][6] = G; g_ftime[blockIdx.x][7] = app_cnt; }
#endif
}

// ------------------------------------------------------------------------------------------ control
// a5/a6/a7-gate: the control decision of one BSP iteration (1 thread). Runs as its own kernel (k_control),
// or -- single launch unit in graph mode -- inside the filter's last CTA (k_filter, fuse_ctl): one launch
// less per iteration. Not inlined: its planner arrays must not raise the filter's register count.
__device__ __noinline__ void control_body(const DevCtx& c, const int alg, int w0, int nw, cudaGraphConditionalHandle h,
                                          int use_h) {
    RunCtl* rc = c.rctl[w0];
#ifdef GUM_FILTER_TIMING
    g_fcall++;
#endif
    if (rc->done) {
        if (use_h) cudaGraphSetConditional(h, 0);
        return;
    }
    const unsigned long long t_ctl = globaltimer();
    const unsigned k = rc->iter;
    unsigned long long active = 0, total_edges = 0, l[kMaxW];
    unsigned err = 0;
    for (int i = 0; i < kMaxW; i++) l[i] = 0;
    double D = 0.0, R = 0.0;
    for (int f = 0; f < c.P; f++) {
        FragCtl* ct = c.f[f].ctl;
        unsigned long long q = vload(&ct->qlen), e = vload(&ct->qedges);
        err |= vload(&ct->err);
        active += q;
        total_edges += e;
        l[rc->owner[f]] += e;
        if (alg == ALG_PR && k > 0) {
            D += vload(&ct->pr_dang[(k - 1) & 1]);
            R += vload(&ct->pr_resid[(k - 1) & 1]);
        }
    }
    // SSSP near-far: when the near frontier is empty but vertices are parked, move the split to the
    // smallest parked distance + delta and sweep the far set in the next filter (this iteration's
    // advance has an empty queue).
    bool nf_bump = false;
    if (alg == ALG_SSSP && c.nf_delta) {
        unsigned long long far_total = 0;
        unsigned fmin = GUM_INF;
        const unsigned slot = rc->nf_sweeps & 1u;
        for (int f = 0; f < c.P; f++) {
            far_total += vload(&c.f[f].ctl->far_cnt);
            const unsigned fm = vload(&c.f[f].ctl->far_min[slot]);
            fmin = fm < fmin ? fm : fmin;
        }
        rc->nf_sweep = 0;
        if (active == 0 && far_total > 0 && err == 0) {
            nf_bump = true;
            unsigned long long T = rc->nf_T + c.nf_delta;
            const unsigned long long T2 = (unsigned long long)fmin + c.nf_delta;
            rc->nf_T = T2 > T ? T2 : T;
            rc->nf_sweep = 1;
            rc->nf_sweeps = rc->nf_sweeps + 1;
            // the next epoch's minimum slot starts empty (only the owner resets; others read `slot`)
            for (int f = 0; f < c.P; f++)
                if ((int)rc->owner[f] >= w0 && (int)rc->owner[f] < w0 + nw) {
                    c.f[f].ctl->far_min[slot ^ 1u] = GUM_INF;
                    c.f[f].ctl->far_n[slot ^ 1u] = 0;  // consumed by the previous sweep; receives this one's
                }
        }
    }
    bool done;
    if (alg == ALG_PR) {
        if (k > 0) {
            rc->pr_D = D;
            rc->pr_resid = R;
        }
        // the finalize of iteration k accumulates into parity slot k&1: clear it for owned fragments
        // (other units only ever read the opposite slot in this phase)
        for (int f = 0; f < c.P; f++) {
            if ((int)rc->owner[f] >= w0 && (int)rc->owner[f] < w0 + nw) {
                c.f[f].ctl->pr_dang[k & 1] = 0.0;
                c.f[f].ctl->pr_resid[k & 1] = 0.0;
            }
        }
        done = (int)k >= c.pr_iters;
    } else {
        done = err != 0 || (active == 0 && !nf_bump) || k >= c.max_iter;
    }
    unsigned m = rc->m;
    unsigned grow_to = 0;  // device-resident multi-unit loop: members to wake for the next iteration
    if (!done) {
        // a6 OSteal: the active owner set is re-decided every iteration from the global
        // counts. Below the active-vertex threshold the survivors are {0..m'-1} (uniform-fabric
        // reduction tree) with m' = clamp(ceil(active edges / edges-per-worker), 1, P); above it
        // ownership is given back. Fragment f is owned by f when f < m', else by f mod m'.
        if (c.osteal && c.P > 1) {
            unsigned mp = (unsigned)c.P;
            if (c.osteal == 2) {
                // NEXT-3: Alg. 2 with Eq. (4) on this iteration's per-fragment active edges
                unsigned long long lf[kMaxW];
                for (int f = 0; f < c.P; f++) lf[f] = vload(&c.f[f].ctl->qedges);
                double p = c.os_p;
                if (c.os_p_online) {
                    // p from unit 0's iteration k-2 (complete, and on one clock): its period (control to next
                    // control) minus its advance window is the per-iteration synchronisation time S; the
                    // advance processed e edges over m workers in A, i.e. tau = A*m/e per edge; Eq. 4's
                    // T_hat = p*m gives p = S/(m*tau) edges. Halved-weight running average; iterations
                    // touching the tail engine are skipped (their period holds many engine iterations).
                    const RunCtl* r0 = c.rctl[0];
                    if (k >= 2) {
                        const unsigned a = (k - 2) & 3u, b2 = (k - 1) & 3u;
                        const unsigned long long ta = vload(&r0->h_tctl[a]), tb = vload(&r0->h_tctl[b2]);
                        const unsigned long long a0 = vload(&r0->h_adv0[a]), a1 = vload(&r0->h_adv1[a]);
                        const unsigned long long e = vload(&r0->h_edges[a]);
                        const unsigned m2 = vload(&r0->h_m[a]);
                        const bool clean = !vload(&r0->h_tail[a]) && !vload(&r0->h_tail[b2]);
                        if (clean && a1 > a0 && a1 - a0 > 2000ull && tb > ta && tb - ta > a1 - a0 && m2 >= 1 &&
                            e >= 64ull * m2) {
                            const double A = (double)(a1 - a0), S = (double)(tb - ta) - A;
                            const double pk = S * (double)e / (A * (double)m2 * (double)m2);
                            rc->os_p = rc->os_p_n ? 0.5 * rc->os_p + 0.5 * pk : pk;
                            rc->os_p_n = rc->os_p_n + 1;
                        }
                    }
                    if (rc->os_p_n) p = rc->os_p;
                }
                mp = (unsigned)osteal_choose(lf, c.P, c.remote_cost, p, nullptr);
            } else if (active < c.os_thresh) {
                mp = 1;
                if (c.os_epw) {
                    const unsigned long long want = (total_edges + c.os_epw - 1) / c.os_epw;
                    mp = want < 1 ? 1u : (want > (unsigned long long)c.P ? (unsigned)c.P : (unsigned)want);
                }
            }
            if (c.units_dev && mp > rc->mb) {
                // give-back to parked units (device-resident multi-unit loop): they are woken now, rejoin
                // the barriers at the next phase-A barrier and own their fragments from the next control on;
                // this iteration's owners stay within the current members
                grow_to = mp;
                mp = rc->mb;
            }
            if (mp != m) {
                for (int f = 0; f < c.P; f++) rc->owner[f] = (unsigned)f < mp ? (unsigned)f : (unsigned)f % mp;
                m = mp;
                rc->m = mp;
                rc->osteal_iter = k;
                for (int i = 0; i < kMaxW; i++) l[i] = 0;
                for (int f = 0; f < c.P; f++) l[rc->owner[f]] += vload(&c.f[f].ctl->qedges);
            }
        }
        // a7 FSteal gate (P:248 Example 5): max l >= t1 and max l - min l >= t2 over active owners
        unsigned long long mx = 0, mn = ~0ull;
        for (unsigned i = 0; i < m; i++) {
            mx = l[i] > mx ? l[i] : mx;
            mn = l[i] < mn ? l[i] : mn;
        }
        rc->steal_ok = (c.fsteal && m > 1 && mx >= c.t1 && mx - mn >= c.t2) ? 1u : 0u;
        if (c.fsteal == 2 && m == (unsigned)c.P) {
            // NEXT-2 planned FSteal: solve Eq. (1) for this iteration's loads (closed form on a uniform
            // fabric), then carve each queue into consecutive chunk ranges (Alg. 1 l.9-18: prefix sums of
            // the planned edge counts searched in the queue's chunk (edge) prefix): the owner's kept
            // share first, then each thief's share in worker order.
            double X[kMaxW * kMaxW];
            unsigned long long lw[kMaxW];
            for (int f = 0; f < c.P; f++) lw[f] = l[f];
            if (rc->steal_ok) {
                rc->plan_z = fsteal_waterfill(lw, c.P, c.remote_cost, X);
            } else {
                for (int q = 0; q < c.P * c.P; q++) X[q] = 0.0;
                for (int f = 0; f < c.P; f++) X[f * c.P + f] = (double)lw[f];
                rc->plan_z = (double)mx;
            }
            for (int f = 0; f < c.P; f++) {
                const unsigned long long nt = vload(&c.f[f].ctl->ntiles);
                double cum = 0.0;
                unsigned prev = 0;
                for (int q = 0; q < c.P; q++) {
                    const int wk = q == 0 ? f : (q <= f ? q - 1 : q);  // owner first, then others
                    cum += X[f * c.P + wk];
                    unsigned hi = (unsigned)(cum / (double)c.chunk + 0.5);
                    if (q == c.P - 1 || hi > nt) hi = (unsigned)nt;
                    if (hi < prev) hi = prev;
                    rc->plan_lo[f][wk] = prev;
                    rc->plan_hi[f][wk] = hi;
                    prev = hi;
                }
            }
#ifdef GUM_PLAN_DEBUG
            printf("[plan] k=%u loads %llu %llu %llu %llu z=%.1f X0 %.1f %.1f %.1f %.1f lo0 %u %u %u %u hi0 %u %u %u %u nt0 %llu\n", k,
                   lw[0], lw[1], lw[2], lw[3], rc->plan_z, X[0], X[1], X[2], X[3], rc->plan_lo[0][0], rc->plan_lo[0][1],
                   rc->plan_lo[0][2], rc->plan_lo[0][3], rc->plan_hi[0][0], rc->plan_hi[0][1], rc->plan_hi[0][2],
                   rc->plan_hi[0][3], vload(&c.f[0].ctl->ntiles));
#endif
        }
        // frontier density switch: expanding more than V/dense_div edges is expected to activate a
        // dense next frontier -> the advance only sets bitmap bits (fire-and-forget) and the next
        // filter scans the bitmap; otherwise activations are deduplicated and appended to a list.
        rc->next_dense = c.force_mode == 2 ? 1u
                         : c.force_mode == 1 ? 0u
                         : (total_edges * c.dense_div > (unsigned long long)c.num_vertices ? 1u : 0u);
        gum_iter_trace* tr = c.trace[w0];
        if (tr && k < (unsigned)kTraceMax) {
            gum_iter_trace* r = tr + k;
            for (int i = 0; i < kMaxW; i++) {
                r->t_start[i] = ~0ull;
                r->t_end[i] = 0;
                r->edges_own[i] = 0;
                r->edges_stolen[i] = 0;
            }
            r->frontier_vertices = active;
            r->frontier_edges = total_edges;
            r->owners = m;
            r->steal_ok = rc->steal_ok;
        }
        // BFS propagation blocking for dense iterations (single fragment)
        rc->pb = (alg == ALG_BFS && c.pb_shift && c.P == 1 && rc->next_dense) ? 1u : 0u;
        // NEXT-4 direction-optimising BFS (Beamer's rule): go bottom-up when the frontier's out-edges m_f
        // exceed 1/14 of the edges not yet reached m_u; stay while the frontier holds >= V/24 vertices.
        if (alg == ALG_BFS && c.bfs_pull) {
            unsigned long long seen = 0;
            for (int f = 0; f < c.P; f++) seen += vload(&c.f[f].ctl->frontier_edges);
            const unsigned long long mu = c.total_edges > seen ? c.total_edges - seen : 0;
            const bool pull = rc->pull ? active * 24ull >= (unsigned long long)c.num_vertices
                                       : total_edges * 14ull > mu && active * 64ull >= (unsigned long long)c.num_vertices;
            rc->pull = pull ? 1u : 0u;
            if (pull) {
                rc->pb = 0;
                rc->next_dense = 1;  // the bottom-up step writes the next frontier as bits
            }
        }
        // long tail: hand small frontiers to the cooperative tail engine (OSteal m'=1 engine)
        // (OSteal's m'=1 mode: worker 0 owns every fragment while the engine runs)
        rc->tail = 0;
        if (alg != ALG_PR && c.osteal && c.tail_enter && !nf_bump && active <= c.tail_enter &&
            total_edges <= 8ull * c.tail_enter) {
            rc->tail = 1;
            for (int f = 0; f < c.P; f++) {
                // the engine's first next-list counters live in the fragments' (shared) control blocks: only
                // the unit that runs the engine resets them -- another unit's late control would otherwise
                // clear appends the engine already made
                if (w0 == 0) {
                    c.f[f].ctl->tcnt[1] = 0;
                    c.f[f].ctl->tedges[1] = 0;
                }
                rc->owner[f] = 0;
            }
            if (m != 1) rc->osteal_iter = k;
            m = 1;
            rc->m = 1;
            // the engine runs on unit 0 alone: a give-back decided above must not wake parked units now (they
            // would rejoin as members while the engine advances unit 0's iteration count without them)
            grow_to = 0;
            rc->steal_ok = 0;
            rc->pb = 0;
            rc->pull = 0;
            if (tr && k < (unsigned)kTraceMax) tr[k].owners = 1;
        }
        rc->iter = k + 1;
    }
    if (alg == ALG_WCC && !done) {
        // WCC on the blocked static queue: iteration 0 (every vertex active), and later iterations whose
        // frontier (kept as a bitmap by a dense filter) holds >= 1/2 of the graph's entries: one pass over
        // the destination-blocked queue with inactive sources masked keeps the label atomics L2-resident,
        // while the frontier queue would probe a label array larger than L2 at one DRAM sector per edge.
        // The masked pass still stages every queue entry (C4: ~8 ms fixed + ~4 ms per full frontier vs
        // ~19 ms per full frontier for the queue path), hence the 1/2 break-even.
        unsigned blk = rc->skip_filter ? 1u : 0u;
        if (!blk && c.wcc_blocked && rc->m == (unsigned)c.P) {
            bool all_dense = true;
            unsigned long long sq_total = 0;
            for (int f = 0; f < c.P; f++) {
                all_dense = all_dense && vload(&c.f[f].ctl->dense) != 0;
                sq_total += c.f[f].sq_edges;
            }
            if (all_dense && total_edges * 2ull >= sq_total) blk = 2u;
        }
        rc->blocked = blk;
        if (blk) {
            rc->blocked_iters = rc->blocked_iters + 1;
            rc->tail = 0;
        }
    }
    if (c.osteal == 2 && c.os_p_online && !done) {
        const unsigned hs = k & 3u;
        rc->h_tctl[hs] = t_ctl;
        rc->h_edges[hs] = total_edges;
        rc->h_m[hs] = m;
        rc->h_tail[hs] = rc->tail;
        rc->h_adv0[hs] = ~0ull;
        rc->h_adv1[hs] = 0;
    }
    rc->bodies = rc->bodies + 1;
    rc->skip_filter = 0;
    for (int f = 0; f < kMaxW; f++) rc->ticket[f] = 0;
    rc->epoch = rc->epoch + 1;
    if (done) {
        rc->done = 1;
        rc->err = err;
    }
    // device-resident multi-unit loop (a6 across devices, "GPU1 will not participate in
    // synchronization anymore"): the members of the next phase-A barrier are the owners of this iteration
    // (units >= m leave that barrier and park: no launches, no arrivals), plus units being given ownership
    // back; parked units are woken for a give-back or for the end of the run. Every member computes the
    // same membership and wake counts; unit 0 alone copies its run control into each woken unit and then
    // releases the unit's wake word.
    unsigned wk_lo = 0, wk_hi = 0;
    if (c.units_dev) {
        const unsigned mb = rc->mb;
        unsigned nm = mb;
        if (!done) {
            nm = m;
            if (grow_to > nm) nm = grow_to;
        }
        rc->mb_next = nm;
        if (done) {
            wk_lo = mb;
            wk_hi = (unsigned)c.n_units;
        } else if (nm > mb) {
            wk_lo = mb;
            wk_hi = nm;
        }
        for (unsigned u = wk_lo; u < wk_hi; u++) rc->wakes[u] = rc->wakes[u] + 1;
    }
    __threadfence();
    if (c.units_dev && w0 == 0 && wk_hi > wk_lo) {
        constexpr int kWords = (int)(sizeof(RunCtl) / 8);
        const unsigned long long* src = reinterpret_cast<const unsigned long long*>(rc);
        for (unsigned u = wk_lo; u < wk_hi; u++) {
            unsigned long long* dst = reinterpret_cast<unsigned long long*>(c.rctl[u]);
            for (int i = 0; i < kWords; i++) dst[i] = src[i];
        }
        asm volatile("fence.sc.sys;" ::: "memory");
        for (unsigned u = wk_lo; u < wk_hi; u++)
            asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(c.pad[u] + kPadWake),
                         "l"((unsigned long long)rc->wakes[u])
                         : "memory");
    }
    if (use_h) cudaGraphSetConditional(h, done ? 0u : 1u);
}

template <int ALG>
__global__ void k_control(const __grid_constant__ DevCtx c, int w0, int nw, cudaGraphConditionalHandle h, int use_h) {
    if (threadIdx.x != 0) return;
    control_body(c, ALG, w0, nw, h, use_h);
}

// ------------------------------------------------------------------------------------------ advance
template <int ALG>
struct ValT {
    typedef unsigned T;
};
template <>
struct ValT<ALG_PR> {
    typedef double T;
};
template <>
struct ValT<ALG_DPR> {
    typedef double T;
};

// Warp-aggregated append of this thread's activations (bit j of need: slot j) to the owner
// fragments' activation lists: one reservation atomic per warp and target fragment.
// TMA bulk prefetch of [p, p + bytes) into L2 (cp.async.bulk.prefetch: 16-byte granules, no registers held)
#ifndef GUM_ADV_PF
#define GUM_ADV_PF 0
#endif
__device__ __forceinline__ void prefetch_l2_range(const void* p, unsigned bytes) {
    const unsigned long long a = (unsigned long long)p & ~15ull;
    const unsigned long long e = ((unsigned long long)p + bytes + 15ull) & ~15ull;
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"((unsigned)(e - a)));
}

template <bool MULTI>
__device__ __forceinline__ unsigned append_activations(const DevCtx& c, unsigned need, const unsigned char* tfv,
                                                       const unsigned* lvv) {
    unsigned done = 0;
    const int nfrag = MULTI ? c.P : 1;
    for (int g = 0; g < nfrag; g++) {
        unsigned mine = 0;
#pragma unroll
        for (int j = 0; j < kEdgesPerThread; j++) mine += ((need >> j) & 1u) && tfv[j] == g ? 1u : 0u;
        unsigned inc = mine;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned x = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane_id() >= (unsigned)o) inc += x;
        }
        const unsigned total = __shfl_sync(0xffffffffu, inc, 31);
        if (total == 0) continue;  // warp-uniform
        unsigned basepos = 0;
        if (lane_id() == 31) basepos = atomicAdd(&c.f[g].ctl->app_cnt, total);
        basepos = __shfl_sync(0xffffffffu, basepos, 31);
        unsigned pos = basepos + inc - mine;
        unsigned* app = c.f[g].app;
#pragma unroll
        for (int j = 0; j < kEdgesPerThread; j++)
            if (((need >> j) & 1u) && tfv[j] == g) app[pos++] = lvv[j];
        done += mine;
    }
    return done;
}

// NX: the NEXT-1 reducers (mirrors / hub cache) are compiled in; the plain multi-worker instantiation
// leaves them out (their registers cost the default path ~15% on P = 8 virtual workers)
template <int ALG, bool MULTI, bool PB = false, bool NX = false>
#ifndef GUM_ADV_MINB_BFS
#define GUM_ADV_MINB_BFS 4
#endif
__global__ void __launch_bounds__(kAdvThreads, (ALG == ALG_BFS) ? GUM_ADV_MINB_BFS * 256 / kAdvThreads : 4 * 256 / kAdvThreads) k_advance(const __grid_constant__ DevCtx c, int w0, int nw) {
    typedef typename ValT<ALG>::T VT;
    // BFS (no propagation blocking / reducers): the chunk's staging buffers are double-buffered by tile parity
    // (GUM_ADV_DB), so the barrier at the end of a chunk -- it kept the next chunk's staging from overwriting
    // what slow warps still expand -- is not needed (3 CTA barriers per chunk instead of 4)
#ifndef GUM_ADV_DB
#define GUM_ADV_DB 0
#endif
    constexpr int NB = (GUM_ADV_DB && ALG == ALG_BFS && !PB && !NX) ? 2 : 1;
    __shared__ unsigned s_base_b[NB][kTileMax + 1];  // col index of the chunk's first edge of each vertex (E_f < 2^32)
    __shared__ VT s_val[(ALG == ALG_BFS) ? 1 : (kTileMax + 1)];
    static_assert(kTileMax <= 4096, "s_head tags keep the vertex slot in 12 bits");
    __shared__ __align__(16) unsigned s_head_b[NB][kTileMax];  // (tile seq << 12) | vertex slot; untagged after the scan
    unsigned* s_base = s_base_b[0];
    unsigned* s_head = s_head_b[0];
    // BFS propagation blocking: per-chunk counting sort of discovered-candidate ids by destination block
    constexpr int PBB = (ALG == ALG_BFS && !MULTI && PB) ? kPbMaxBins : 1;  // (own instantiation:
    // the shared arrays would otherwise shrink L1, which the random probes of the plain path live on)
    constexpr int PBS = (ALG == ALG_BFS && !MULTI && PB) ? kTileMax : 1;
    __shared__ unsigned s_pbcnt[PBB], s_pboff[PBB], s_pbg[PBB];
    __shared__ unsigned short s_stbin[PBS];
    unsigned* const s_stage = s_head_b[0];  // s_head is dead once the chunk's col ids are loaded (NB == 1 here)
    __shared__ unsigned s_wmax[kAdvThreads / 32];
    // NEXT-1 hub cache: per staged vertex, 1 = its list is expanded from this worker's local copy
    __shared__ unsigned char s_hub[(MULTI && NX) ? kTileMax : 1];
    __shared__ unsigned long long s_ntiles[kMaxW], s_qlen[kMaxW], s_qedges[kMaxW];
    __shared__ unsigned s_owner[kMaxW];
    __shared__ QPtrs s_q[kMaxW];                    // per fragment: where its queue lives (NEXT-3 migration)
    __shared__ unsigned long long s_cnt[kMaxW][4];  // per fragment: edges, chunks, stolen edges, stolen chunks

    // Prologue: thread 0 reads the run-control header once per CTA (per-warp loads of these few shared
    // addresses serialise in their L2 slice), threads < P the fragments' queue sizes.
    __shared__ unsigned s_hdr[7];  // go, m, k, steal_ok, next_dense, pb, blocked
    RunCtl* rc = c.rctl[w0];
    const int w = w0 + (int)(blockIdx.x % (unsigned)nw);
    if (threadIdx.x == 0) {
        const unsigned m_ = vload(&rc->m);
        // tail engine or bottom-up step runs this iteration / evicted by OSteal (the GPU only serves as memory)
        s_hdr[0] = !vload(&rc->done) && !vload(&rc->tail) && !(ALG == ALG_BFS && vload(&rc->pull)) && (unsigned)w < m_;
        s_hdr[1] = m_;
        s_hdr[2] = vload(&rc->iter) - 1;
        s_hdr[3] = vload(&rc->steal_ok);
        s_hdr[4] = vload(&rc->next_dense);
        s_hdr[5] = (ALG == ALG_BFS && !MULTI && PB) ? vload(&rc->pb) : 0u;
        s_hdr[6] = (ALG == ALG_WCC) ? vload(&rc->blocked) : 0u;
    }
    if (threadIdx.x < (unsigned)c.P) {
        FragCtl* ct = c.f[threadIdx.x].ctl;
        const FragPtrs& Fq = c.f[threadIdx.x];
        if (ALG == ALG_WCC && Fq.sq_col && vload(&rc->blocked)) {
            // the static destination-blocked queue (all vertices; inactive ones are masked in staging)
            s_ntiles[threadIdx.x] = (Fq.sq_edges + c.chunk - 1) / c.chunk;
            s_qlen[threadIdx.x] = Fq.sq_len;
            s_qedges[threadIdx.x] = Fq.sq_edges;
        } else {
            s_ntiles[threadIdx.x] = vload(&ct->ntiles);
            s_qlen[threadIdx.x] = vload(&ct->qlen);
            s_qedges[threadIdx.x] = vload(&ct->qedges);
        }
        s_owner[threadIdx.x] = vload(&rc->owner[threadIdx.x]);
        s_q[threadIdx.x] = queue_of(c, threadIdx.x, vload(&ct->qown));  // where the filter put the queue
        s_cnt[threadIdx.x][0] = s_cnt[threadIdx.x][1] = s_cnt[threadIdx.x][2] = s_cnt[threadIdx.x][3] = 0;
    }
    __syncthreads();
    if (!s_hdr[0]) return;
    const unsigned m = s_hdr[1];
    const unsigned k = s_hdr[2];
    const unsigned blk = ALG == ALG_WCC ? s_hdr[6] : 0u;  // 2: masked blocked pass (count valid edges)
    const bool steal = s_hdr[3] != 0;
    const bool next_dense = s_hdr[4] != 0;
    const bool planned = c.fsteal == 2 && m == (unsigned)c.P;  // NEXT-2 plan (else the steal queue)
    const bool pb = (ALG == ALG_BFS && !MULTI && PB) && s_hdr[5] != 0;
    if (pb) {
        for (unsigned b = threadIdx.x; b < (unsigned)PBB; b += kAdvThreads) s_pbcnt[b] = 0;
        __syncthreads();
    }
    const unsigned long long t0 = globaltimer();
    const unsigned CH = c.chunk;
    for (int q = 0; q < NB; q++)
        for (unsigned e = threadIdx.x; e < (unsigned)kTileMax; e += kAdvThreads) s_head_b[q][e] = 0;
    unsigned seq = 0;    // tile sequence number of this CTA (tags s_head entries; no per-tile clearing)
    int own_cursor = 0;  // fragments (w + i) % P for i < own_cursor are drained
    unsigned long long e_own = 0, e_stolen = 0, remote = 0, acts = 0, filtered = 0, hub_e = 0;
    unsigned nval = 0;  // masked blocked pass: this thread's expanded edges of the current chunk
    // NEXT-1 outer-vertex mirrors (this worker's memory): updates to other fragments go through them
    const bool mir = MULTI && NX && c.mirrors;

    // Chunk claims run one chunk ahead of the expansion (thread 0): while chunk n is expanded, chunk n+1
    // is already claimed and its staging data (chunk table entries, degree prefix, col base, source
    // value) is in flight into registers, so a chunk's staging costs no exposed memory round trip. The
    // own-queue claim atomic itself is issued one more chunk ahead (pf_f / pf_t).
    int pf_f = -1;
    unsigned long long pf_t = 0;
    auto claim_next = [&](int& f_out, unsigned long long& t_out, int& stolen_out) {
        int f = -1;
        unsigned long long t = 0;
        int stolen = 0;
        if (planned) {
            // NEXT-2: process the chunk ranges the plan assigned to this worker, queue by queue
            while (own_cursor < c.P) {
                const int g = (w + own_cursor) % c.P;
                const unsigned lo = rc->plan_lo[g][w], hi = rc->plan_hi[g][w];
                if (hi > lo) {
                    const unsigned long long tt = lo + atomicAdd(&c.f[g].ctl->pclaim[w], 1ull);
                    if (tt < hi) {
                        f = g;
                        t = tt;
                        stolen = g != w;
                        break;
                    }
                }
                own_cursor++;
            }
        } else if (pf_f >= 0 && pf_t < s_ntiles[pf_f]) {
            f = pf_f;
            t = pf_t;
        } else {
            if (pf_f >= 0) own_cursor++;  // prefetched claim overflowed: that queue is drained
            while (own_cursor < c.P) {
                int g = (w + own_cursor) % c.P;
                if (s_owner[g] == (unsigned)w) {
                    unsigned long long tt = atomicAdd(&c.f[g].ctl->claim, 1ull);
                    if (tt < s_ntiles[g]) {
                        f = g;
                        t = tt;
                        break;
                    }
                }
                own_cursor++;
            }
        }
        pf_f = -1;
        if (f < 0 && steal && !planned) {
            // FSteal: claim a chunk of the active owner queue with the most remaining chunks
            for (;;) {
                int best = -1;
                unsigned long long best_rem = 0;
                for (int g = 0; g < c.P; g++) {
                    if (s_owner[g] == (unsigned)w) continue;
                    unsigned long long cl = vload(&c.f[g].ctl->claim);
                    unsigned long long rem = s_ntiles[g] > cl ? s_ntiles[g] - cl : 0;
                    if (rem > best_rem) {
                        best_rem = rem;
                        best = g;
                    }
                }
                if (best < 0) break;
                unsigned long long tt = atomicAdd(&c.f[best].ctl->claim, 1ull);
                if (tt < s_ntiles[best]) {
                    f = best;
                    t = tt;
                    stolen = 1;
                    break;
                }
            }
        }
        f_out = f;
        t_out = t;
        stolen_out = stolen;
        if (f >= 0 && !stolen && !planned) {
            pf_f = f;
            pf_t = atomicAdd(&c.f[f].ctl->claim, 1ull);
        }
    };
    // staging descriptor of a claimed chunk (WCC iteration 0 runs on the static destination-blocked
    // queue: edges contiguous in queue order)
    struct ChunkRef {
        int f;
        unsigned long long t;
        int stolen;
        unsigned i0, nv, tlen;
        bool hc;  // NEXT-1: non-local fragment whose hub lists this worker has cached
    };
    auto chunk_ref = [&](int f, unsigned long long t, int stolen) {
        ChunkRef r{f, t, stolen, 0u, 0u, 0u, false};
        if (f < 0) return r;
        r.hc = MULTI && NX && ALG != ALG_PR && ALG != ALG_DPR && c.hub_on && f != w;
        const FragPtrs& F = c.f[f];
        const bool sq = ALG == ALG_WCC && blk && F.sq_col != nullptr;
        const unsigned* const tilep = sq ? F.sq_tile : s_q[f].tile;
        const unsigned long long tb = t * CH, qe = s_qedges[f];
        r.tlen = (unsigned)((qe - tb) < CH ? (qe - tb) : CH);
        r.i0 = __ldg(tilep + t);
        const unsigned i1 = (t + 1 < s_ntiles[f]) ? __ldg(tilep + t + 1) : (unsigned)(s_qlen[f] - 1);
        r.nv = i1 - r.i0 + 1;
        return r;
    };
    // per-vertex staging values of queue entry i of chunk r (vertex slot kk): edge prefix, col base, value
    auto stage_load = [&](const ChunkRef& r, unsigned kk, unsigned long long& off, unsigned& base, unsigned& u,
                          bool& hub) {
        const FragPtrs& F = c.f[r.f];
        const bool sq = ALG == ALG_WCC && blk && F.sq_col != nullptr;
        const unsigned i = r.i0 + kk;
        const unsigned long long tb = r.t * CH;
        off = __ldcs((sq ? F.sq_q_off : s_q[r.f].q_off) + i);
        // PR's (and WCC iteration 0's) blocked queue stores edges contiguously in queue order:
        // col index == q_off + j
        base = (unsigned)((long long)tb + ((ALG == ALG_PR || sq) ? 0ll : __ldcs(s_q[r.f].q_base + i)));
        u = (ALG != ALG_BFS || r.hc) ? __ldcs((sq ? F.sq_q_v : s_q[r.f].q_v) + i) : 0u;
        hub = false;
        if (MULTI && r.hc && !sq) {
            // NEXT-1: a cached hub list is read from the local copy: col index of edge j of
            // the vertex = h + j, i.e. base = tb + h - off (mod 2^32 like the fragment's base)
            const unsigned long long h = __ldg(c.hub[w][r.f].off + u);
            if (h != ~0ull) {
                base = (unsigned)((long long)tb + (long long)h - (long long)off);
                hub = true;
            }
        }
    };
    auto value_of = [&](const ChunkRef& r, unsigned u) -> VT {
        if (ALG == ALG_PR || ALG == ALG_DPR) return (VT)__ldcg(c.f[r.f].cx + u);
        // masked blocked pass: a source outside the frontier (its bit clear in the filter's copy) gets the
        // value INF, and its edges are skipped in the expansion
        if (ALG == ALG_WCC && blk == 2 && !((__ldcg(c.f[r.f].far + (u >> 5)) >> (u & 31)) & 1u)) return (VT)GUM_INF;
        if (ALG != ALG_BFS) return (VT)__ldcg(c.f[r.f].state + u);
        return (VT)0;
    };

    __shared__ int s_nf;
    __shared__ unsigned long long s_nt;
    __shared__ int s_nstolen;
    if (threadIdx.x == 0) {
        int f0;
        unsigned long long t0c;
        int st0;
        claim_next(f0, t0c, st0);
        s_nf = f0;
        s_nt = t0c;
        s_nstolen = st0;
    }
    __syncthreads();
    ChunkRef cur = chunk_ref(s_nf, s_nt, s_nstolen);
    unsigned long long p_off = 0;  // prefetched staging values of vertex slot threadIdx.x
    unsigned p_base = 0, p_u = 0;
    bool p_hub = false;
    VT p_val = (VT)0;
    if (cur.f >= 0 && threadIdx.x < cur.nv) {
        stage_load(cur, threadIdx.x, p_off, p_base, p_u, p_hub);
        p_val = value_of(cur, p_u);
    }
    __syncthreads();  // everyone read s_nf before it is reused
    for (;;) {
        const int f = cur.f;
        if (f < 0) break;
        const unsigned long long t = cur.t;
        const bool stolen = cur.stolen != 0;
        const FragPtrs& F = c.f[f];
        const unsigned long long tb = t * CH;
        const unsigned tlen = cur.tlen;
        const bool sq = ALG == ALG_WCC && blk && F.sq_col != nullptr;
        const unsigned* const colp = sq ? F.sq_col : F.col;
        const unsigned nv = cur.nv;
        if (threadIdx.x == 0) {
            int nf_;
            unsigned long long nt_;
            int ns_;
            claim_next(nf_, nt_, ns_);
            s_nf = nf_;
            s_nt = nt_;
            s_nstolen = ns_;
        }

        // ---- stage the chunk's frontier vertices (merge path over the degree prefix, CTA-local)
        seq++;
        if (NB == 2) {
            s_base = s_base_b[seq & 1u];
            s_head = s_head_b[seq & 1u];
        }
        for (unsigned kk = threadIdx.x; kk < nv; kk += kAdvThreads) {
            unsigned long long off;
            unsigned base, u;
            bool hub;
            VT val;
            if (kk < (unsigned)kAdvThreads) {
                off = p_off;
                base = p_base;
                val = p_val;
                hub = p_hub;
            } else {
                stage_load(cur, kk, off, base, u, hub);
                val = value_of(cur, u);
            }
            s_base[kk] = base;
            if (MULTI && NX) s_hub[kk] = hub ? 1 : 0;
            if (ALG != ALG_BFS) s_val[kk] = val;
            const long long rel = (long long)off - (long long)tb;
            if (rel > 0 && rel < (long long)tlen) s_head[rel] = (seq << 12) | kk;
        }
        __syncthreads();
        // the next chunk's chunk-table entries load while this chunk is scanned
        const ChunkRef nxt = chunk_ref(s_nf, s_nt, s_nstolen);
        // blocked inclusive max-scan of s_head: s_head[e] = index of the vertex owning edge e
        {
            // each thread's 8 consecutive entries move as two 16-byte vectors (a warp touches 1 KB of
            // contiguous shared memory: conflict-free, instead of 8-way bank conflicts per scalar access)
            static_assert(kEdgesPerThread % 4 == 0, "vectorised scan needs kEdgesPerThread % 4 == 0");
            const unsigned b = threadIdx.x * kEdgesPerThread;
            unsigned hv[kEdgesPerThread];
#pragma unroll
            for (int q = 0; q < kEdgesPerThread / 4; q++) {
                const uint4 r4 = *reinterpret_cast<const uint4*>(s_head + b + 4 * q);
                hv[4 * q] = r4.x;
                hv[4 * q + 1] = r4.y;
                hv[4 * q + 2] = r4.z;
                hv[4 * q + 3] = r4.w;
            }
            unsigned run = 0;
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++) {
                const unsigned raw = (b + j < tlen) ? hv[j] : 0u;
                hv[j] = (raw >> 12) == seq ? (raw & 0xFFFu) : 0u;
                run = hv[j] > run ? hv[j] : run;
                hv[j] = run;
            }
            unsigned inc = run;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                unsigned x = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane_id() >= (unsigned)o) inc = x > inc ? x : inc;
            }
            unsigned excl = __shfl_up_sync(0xffffffffu, inc, 1);
            if (lane_id() == 0) excl = 0;
            if (lane_id() == 31) s_wmax[threadIdx.x >> 5] = inc;
            __syncthreads();
            for (unsigned i = 0; i < (threadIdx.x >> 5); i++) excl = s_wmax[i] > excl ? s_wmax[i] : excl;
            // (entries >= tlen are written too: untagged values never match a later sequence tag)
#pragma unroll
            for (int q = 0; q < kEdgesPerThread / 4; q++) {
                uint4 w4;
                w4.x = hv[4 * q] > excl ? hv[4 * q] : excl;
                w4.y = hv[4 * q + 1] > excl ? hv[4 * q + 1] : excl;
                w4.z = hv[4 * q + 2] > excl ? hv[4 * q + 2] : excl;
                w4.w = hv[4 * q + 3] > excl ? hv[4 * q + 3] : excl;
                *reinterpret_cast<uint4*>(s_head + b + 4 * q) = w4;
            }
        }
        __syncthreads();

        // the next chunk's per-vertex staging values load while this chunk is expanded
        if (nxt.f >= 0 && threadIdx.x < nxt.nv) {
            stage_load(nxt, threadIdx.x, p_off, p_base, p_u, p_hub);
            p_val = value_of(nxt, p_u);
        }
        // ---- expand: striped edges, coalesced streaming col/w loads
        unsigned vv[kEdgesPerThread];
        VT cv[kEdgesPerThread];
#pragma unroll
        for (int j = 0; j < kEdgesPerThread; j++) {
            const unsigned e = j * kAdvThreads + threadIdx.x;
            vv[j] = GUM_INF;
            cv[j] = (VT)0;
            if (e < tlen) {
                const unsigned kk = s_head[e];
                if (ALG == ALG_WCC && blk == 2) {
                    if (s_val[kk] == (VT)GUM_INF) continue;  // source not in the frontier
                    nval++;
                }
                const unsigned long long ci = (unsigned)(s_base[kk] + e);  // mod 2^32: the base may wrap
                const bool hv = MULTI && NX && cur.hc && s_hub[kk];
                if (MULTI && NX) hub_e += hv ? 1 : 0;
                vv[j] = __ldcs((hv ? c.hub[w][f].col : colp) + ci);
                if (ALG == ALG_BFS) cv[j] = (VT)(k + 1);  // every frontier vertex has depth k
                if (ALG == ALG_WCC || ALG == ALG_PR || ALG == ALG_DPR) cv[j] = s_val[kk];
                if (ALG == ALG_SSSP) {
                    const unsigned long long nd = (unsigned long long)s_val[kk] + __ldcs((hv ? c.hub[w][f].w : F.w) + ci);
                    if (nd >= (unsigned long long)GUM_INF) {
                        atomicOr(&F.ctl->err, 1u);
                        vv[j] = GUM_INF;
                    }
                    cv[j] = (VT)(unsigned)nd;
                }
            }
        }
        if (GUM_ADV_PF && !(MULTI && NX)) {
            // L2 bulk prefetch of the next chunk's adjacency (col, SSSP w): the next chunk's staging values
            // were issued before this chunk's col loads and have arrived by now; the TMA engine pulls the
            // vertex's run of the next chunk into L2, so its col loads wait for L2 instead of HBM latency
            const unsigned long long n_off = __shfl_down_sync(0xffffffffu, p_off, 1);
            if (nxt.f >= 0 && threadIdx.x < nxt.nv) {
                const unsigned long long ntb = nxt.t * CH;
                const long long r0 = (long long)p_off - (long long)ntb;
                const bool last = lane_id() == 31 || threadIdx.x + 1 >= nxt.nv;
                const long long r1 = last ? (long long)nxt.tlen : (long long)n_off - (long long)ntb;
                const long long a = r0 > 0 ? r0 : 0, b = r1 < (long long)nxt.tlen ? r1 : (long long)nxt.tlen;
                if (b > a) {
                    const FragPtrs& Fn = c.f[nxt.f];
                    const bool nsq = ALG == ALG_WCC && blk && Fn.sq_col != nullptr;
                    const unsigned ci = (unsigned)(p_base + (unsigned)a);
                    prefetch_l2_range((nsq ? Fn.sq_col : Fn.col) + ci, (unsigned)(b - a) * 4u);
                    if (ALG == ALG_SSSP) prefetch_l2_range(Fn.w + ci, (unsigned)(b - a) * 4u);
                }
            }
        }
        if (ALG == ALG_PR) {
            // GAS apply for PR: push x[u]/outdeg(u) into the owner's accumulator (red.global.add.f64)
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++) {
                if (vv[j] != GUM_INF) {
                    const unsigned v = vv[j];
                    int tf = 0;
                    unsigned lv = v;
                    if (MULTI) {
                        tf = frag_of(c, v);
                        lv = v - c.bounds[tf];
                        if (mir && tf != w) {
                            // NEXT-1: early aggregation into this worker's mirror of the outer vertex
                            // (local red.add); the owner's finalize pulls the aggregate once
                            atomicAdd(c.f[w].macc + v, (double)cv[j]);
                            filtered++;
                            continue;
                        }
                        remote += (s_owner[tf] != (unsigned)w) ? 1 : 0;
                    }
                    atomicAdd(c.f[tf].acc + lv, (double)cv[j]);
                }
            }
        } else if (ALG == ALG_DPR) {
            // delta-PR apply (reading #27): add d*delta_u/outdeg(u) to the destination's residual with a
            // returning atom.add.f64; the add that lifts the residual above eps activates v (residuals only
            // grow during an advance, so exactly one add per vertex and round crosses)
            unsigned lvv[kEdgesPerThread];
            unsigned char tfv[kEdgesPerThread];
            double old[kEdgesPerThread];
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++) {
                tfv[j] = 0;
                lvv[j] = vv[j];
                old[j] = 0.0;
                if (vv[j] != GUM_INF) {
                    if (MULTI) {
                        const int tf = frag_of(c, vv[j]);
                        tfv[j] = (unsigned char)tf;
                        lvv[j] = vv[j] - c.bounds[tf];
                        remote += (s_owner[tf] != (unsigned)w) ? 1 : 0;
                    }
                    old[j] = atomicAdd(c.f[tfv[j]].acc + lvv[j], (double)cv[j]);
                }
            }
            const double eps = c.dpr_eps;
            unsigned upd = 0;
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++)
                if (vv[j] != GUM_INF && old[j] <= eps && old[j] + (double)cv[j] > eps) upd |= 1u << j;
            if (next_dense) {
#pragma unroll
                for (int j = 0; j < kEdgesPerThread; j++)
                    if (upd & (1u << j)) atomicOr(c.f[tfv[j]].bm + (lvv[j] >> 5), 1u << (lvv[j] & 31));  // RED.OR
                acts += __popc(upd);
            } else {
                acts += append_activations<MULTI>(c, upd, tfv, lvv);  // (one crossing per vertex: no dedupe)
            }
        } else if (ALG == ALG_BFS && pb) {
            // Propagation blocking (dense BFS iteration): instead of one random visited-bit probe per
            // edge, group the chunk's destination ids by 2^pb_shift-id block (shared-memory counting
            // sort), reserve each block's run with ONE atomic and copy it out coalesced. k_pb_apply then
            // tests and sets the visited bits of one block in shared memory (P:236 message buffers,
            // aggregated on chip instead of serialised).
            const unsigned sh = c.pb_shift, nb = c.pb_nb;
            unsigned rank[kEdgesPerThread];
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++)
                if (vv[j] != GUM_INF) rank[j] = atomicAdd(&s_pbcnt[vv[j] >> sh], 1u);
            __syncthreads();
            {   // exclusive scan of the block counts (4 bins per thread) + one global reservation per bin
                const unsigned b0 = threadIdx.x * 4;
                unsigned cn[4], sum = 0;
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    cn[q] = (b0 + q < nb) ? s_pbcnt[b0 + q] : 0u;
                    sum += cn[q];
                }
                unsigned inc = sum;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const unsigned x = __shfl_up_sync(0xffffffffu, inc, o);
                    if (lane_id() >= (unsigned)o) inc += x;
                }
                if (lane_id() == 31) s_wmax[threadIdx.x >> 5] = inc;
                __syncthreads();
                unsigned run = inc - sum;
                for (unsigned i = 0; i < (threadIdx.x >> 5); i++) run += s_wmax[i];
                unsigned g[4];
#pragma unroll
                for (int q = 0; q < 4; q++)  // four independent reservations in flight per thread
                    g[q] = cn[q] ? atomicAdd(&F.pb_fill[b0 + q], cn[q]) : 0u;
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    if (b0 + q < nb) {
                        s_pboff[b0 + q] = run;
                        s_pbg[b0 + q] = g[q];
                        s_pbcnt[b0 + q] = 0;
                        run += cn[q];
                    }
                }
            }
            __syncthreads();
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++) {
                if (vv[j] != GUM_INF) {
                    const unsigned b = vv[j] >> sh;
                    const unsigned p = s_pboff[b] + rank[j];
                    s_stage[p] = vv[j];
                    s_stbin[p] = (unsigned short)b;
                }
            }
            __syncthreads();
            for (unsigned p = threadIdx.x; p < tlen; p += kAdvThreads) {
                const unsigned b = s_stbin[p];
                F.pb_buf[F.pb_off[b] + s_pbg[b] + (p - s_pboff[b])] = s_stage[p];
                s_stage[p] = 0;  // s_head again: its entries must not look like sequence-tagged heads
            }
        } else if (ALG == ALG_BFS) {
            // BFS: check the visited bit (1 bit/vertex, L1-cacheable) instead of the 4-byte depth.
            // All candidates of iteration k equal k+1, so the depth store needs no atomic.
            unsigned lvv[kEdgesPerThread], wd[kEdgesPerThread];
            unsigned char tfv[kEdgesPerThread];
            unsigned probed = 0;  // NEXT-1: outer vertices whose owner bitmap word was read
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++) {
                tfv[j] = 0;
                lvv[j] = vv[j];
                wd[j] = 0xFFFFFFFFu;
                if (vv[j] != GUM_INF) {
                    if (MULTI) {
                        const int tf = frag_of(c, vv[j]);
                        tfv[j] = (unsigned char)tf;
                        lvv[j] = vv[j] - c.bounds[tf];
                        // NEXT-1 "already sent" filter: an outer vertex this worker has sent to (or
                        // seen visited) before needs no remote probe or update
                        if (mir && tf != w && (c.f[w].msent[vv[j] >> 5] & (1u << (vv[j] & 31)))) {
                            filtered++;
                            continue;  // wd stays all-ones: no update
                        }
                    }
                    wd[j] = c.f[tfv[j]].vis[lvv[j] >> 5];
                    if (mir && tfv[j] != (unsigned char)w) probed |= 1u << j;
                }
            }
            unsigned upd = 0;
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++)
                if (!(wd[j] & (1u << (lvv[j] & 31)))) upd |= 1u << j;
            if (mir) {
                // every probed outer vertex is visited after this iteration (by us or before): cache it
#pragma unroll
                for (int j = 0; j < kEdgesPerThread; j++)
                    if (probed & (1u << j))
                        atomicOr(c.f[w].msent + (vv[j] >> 5), 1u << (vv[j] & 31));  // local RED.OR
            }
            if (next_dense) {
#pragma unroll
                for (int j = 0; j < kEdgesPerThread; j++) {
                    if (upd & (1u << j)) {
                        const FragPtrs& T = c.f[tfv[j]];
                        const unsigned bit = 1u << (lvv[j] & 31);
                        atomicOr(T.vis + (lvv[j] >> 5), bit);  // RED.OR
                        atomicOr(T.bm + (lvv[j] >> 5), bit);   // RED.OR
                        // (the depth k+1 is written by the next filter: BFS state is write-only here)
                        if (MULTI) remote += (s_owner[tfv[j]] != (unsigned)w) ? 1 : 0;
                    }
                }
                acts += __popc(upd);
            } else {
                unsigned ob[kEdgesPerThread];
#pragma unroll
                for (int j = 0; j < kEdgesPerThread; j++) {
                    ob[j] = 0xFFFFFFFFu;
                    if (upd & (1u << j)) ob[j] = atomicOr(c.f[tfv[j]].vis + (lvv[j] >> 5), 1u << (lvv[j] & 31));
                }
                unsigned need = 0;
#pragma unroll
                for (int j = 0; j < kEdgesPerThread; j++) {
                    if (!(ob[j] & (1u << (lvv[j] & 31)))) {
                        need |= 1u << j;
                        if (MULTI) remote += (s_owner[tfv[j]] != (unsigned)w) ? 1 : 0;
                    }
                }
                acts += append_activations<MULTI>(c, need, tfv, lvv);
            }
        } else {
            // GAS apply for min-algorithms: check (plain load) -> red.min on the owner's state ->
            // activation bit. Any thread whose candidate beat the value it read knows v improved in this
            // iteration, so it may set v's bit without waiting for the atomic's return value.
            unsigned lvv[kEdgesPerThread], cur[kEdgesPerThread];
            unsigned char tfv[kEdgesPerThread];
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++) {
                tfv[j] = 0;
                lvv[j] = vv[j];
                cur[j] = 0;
                if (vv[j] != GUM_INF) {
                    if (MULTI) {
                        const int tf = frag_of(c, vv[j]);
                        tfv[j] = (unsigned char)tf;
                        lvv[j] = vv[j] - c.bounds[tf];
                        // NEXT-1 mirror filter: the mirror holds an upper bound of the outer vertex's
                        // value (min of everything this worker sent or read); a candidate that does not
                        // beat it cannot improve the owner's value
                        if (mir && tf != w && (unsigned)cv[j] >= c.f[w].mmin[vv[j]]) {
                            filtered++;
                            vv[j] = GUM_INF;
                            continue;
                        }
                    }
                    cur[j] = c.f[tfv[j]].state[lvv[j]];
                }
            }
            unsigned upd = 0;
#pragma unroll
            for (int j = 0; j < kEdgesPerThread; j++) {
                if (vv[j] != GUM_INF && (unsigned)cv[j] < cur[j]) {
                    upd |= 1u << j;
                    atomicMin(c.f[tfv[j]].state + lvv[j], (unsigned)cv[j]);  // RED.MIN (no return)
                    if (MULTI) remote += (s_owner[tfv[j]] != (unsigned)w) ? 1 : 0;
                }
                if (mir && vv[j] != GUM_INF && tfv[j] != (unsigned char)w) {
                    const unsigned nb = (unsigned)cv[j] < cur[j] ? (unsigned)cv[j] : cur[j];
                    atomicMin(c.f[w].mmin + vv[j], nb);  // local RED.MIN: owner's value <= nb from now on
                }
            }
            if (next_dense) {
#pragma unroll
                for (int j = 0; j < kEdgesPerThread; j++)
                    if (upd & (1u << j)) atomicOr(c.f[tfv[j]].bm + (lvv[j] >> 5), 1u << (lvv[j] & 31));  // RED.OR
                acts += __popc(upd);
            } else {
                // sparse next frontier: dedupe on the bitmap (returning atomics issued back to back) and
                // append with one warp-aggregated reservation per target fragment
                unsigned ob[kEdgesPerThread];
#pragma unroll
                for (int j = 0; j < kEdgesPerThread; j++) {
                    ob[j] = 0xFFFFFFFFu;
                    if (upd & (1u << j)) ob[j] = atomicOr(c.f[tfv[j]].bm + (lvv[j] >> 5), 1u << (lvv[j] & 31));
                }
                unsigned need = 0;
#pragma unroll
                for (int j = 0; j < kEdgesPerThread; j++)
                    if (!(ob[j] & (1u << (lvv[j] & 31)))) need |= 1u << j;
                acts += append_activations<MULTI>(c, need, tfv, lvv);
            }
        }
        if (ALG == ALG_WCC && blk == 2) {
            // masked pass: only the frontier's edges count as expanded (conservation, SURVEY c-6)
            const unsigned long long ws = warp_sum_u64(nval);
            nval = 0;
            if (lane_id() == 0 && ws) {
                atomicAdd(&s_cnt[f][0], ws);
                if (stolen) {
                    atomicAdd(&s_cnt[f][2], ws);
                    e_stolen += ws;
                } else {
                    e_own += ws;
                }
            }
            if (threadIdx.x == 0) {
                s_cnt[f][1] += 1;
                if (stolen) s_cnt[f][3] += 1;
            }
        } else if (threadIdx.x == 0) {
            // conservation counters of the chunk's fragment, accumulated per CTA (flushed at exit: the
            // fragment counters are single addresses)
            s_cnt[f][0] += tlen;
            s_cnt[f][1] += 1;
            if (stolen) {
                s_cnt[f][2] += tlen;
                s_cnt[f][3] += 1;
                e_stolen += tlen;
            } else {
                e_own += tlen;
            }
        }
        if (NB == 1) __syncthreads();  // (double-buffered: the next chunk stages into the other buffers)
        cur = nxt;
    }
    // run counters (warp-reduced) and the per-worker busy window of this iteration
    if (threadIdx.x < (unsigned)c.P && s_cnt[threadIdx.x][1]) {
        FragCtl* ct = c.f[threadIdx.x].ctl;
        atomicAdd(&ct->edges_done, s_cnt[threadIdx.x][0]);
        atomicAdd(&ct->chunks_done, s_cnt[threadIdx.x][1]);
        if (s_cnt[threadIdx.x][3]) {
            atomicAdd(&ct->edges_stolen, s_cnt[threadIdx.x][2]);
            atomicAdd(&ct->chunks_stolen, s_cnt[threadIdx.x][3]);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        remote += __shfl_xor_sync(0xffffffffu, remote, o);
        acts += __shfl_xor_sync(0xffffffffu, acts, o);
        if (MULTI) {
            filtered += __shfl_xor_sync(0xffffffffu, filtered, o);
            hub_e += __shfl_xor_sync(0xffffffffu, hub_e, o);
        }
    }
    if (lane_id() == 0 && (remote | acts | filtered | hub_e)) {
        FragCtl* hc = c.f[w % c.P].ctl;
        if (remote) atomicAdd(&hc->remote_updates, remote);
        if (acts) atomicAdd(&hc->activations, acts);
        if (filtered) atomicAdd(&hc->remote_filtered, filtered);
        if (hub_e) atomicAdd(&hc->hub_edges, hub_e);
    }
    gum_iter_trace* tr = c.trace[w0];
    if (tr && k < (unsigned)kTraceMax) {
        gum_iter_trace* r = tr + k;
        if (threadIdx.x == 0) {
            const unsigned long long t1 = globaltimer();
            atomicMin((unsigned long long*)&r->t_start[w], t0);
            atomicMax((unsigned long long*)&r->t_end[w], t1);
        }
        // (thread 0 holds the per-chunk counts; in a masked WCC pass every warp's lane 0 holds a share)
        if (e_own) atomicAdd((unsigned long long*)&r->edges_own[w], e_own);
        if (e_stolen) atomicAdd((unsigned long long*)&r->edges_stolen[w], e_stolen);
    }
    if (c.os_p_online && c.osteal == 2 && threadIdx.x == 0) {  // NEXT-3 online p: this unit's advance window
        atomicMin(&rc->h_adv0[k & 3u], t0);
        atomicMax(&rc->h_adv1[k & 3u], globaltimer());
    }
}

// ------------------------------------------------------------------------------------------ tail engine
// The OSteal m'=1 engine of SURVEY §3: when the global frontier is small, one cooperative persistent
// kernel runs whole BSP iterations back to back (expand -> one grid barrier -> next), so a long tail of
// latency-bound iterations costs a barrier per iteration instead of three kernel
// launches. Lists alternate between q_v (iteration parity 0; the filter's queue seeds it) and app;
// three per-fragment counters rotate (current / next / reset). Semantics are the regular advance's:
// check -> red.min -> (fence) -> bitmap test-and-set dedupe -> warp-aggregated append; a vertex's bit is
// released (acq) before its value is read, so an improvement after the read re-activates it.
constexpr int kTailThreads = 256;

// Dedupe bit of a next list, set with release semantics (orders the preceding red.min on the state before
// the bit) and released by a local relaxation round with acquire semantics (orders the state read after it):
// if an improvement's OR finds the bit still set, the local round's AND comes later in the bit's coherence
// order and its state read sees that improvement; if the OR comes later, it finds the bit clear and appends.
__device__ __forceinline__ unsigned atom_or_release(unsigned* p, unsigned v) {
    unsigned old;
    asm volatile("atom.release.gpu.global.or.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}
__device__ __forceinline__ unsigned atom_and_acquire(unsigned* p, unsigned v) {
    unsigned old;
    asm volatile("atom.acquire.gpu.global.and.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}

__device__ __forceinline__ void tail_barrier(RunCtl* rc, unsigned nblocks, unsigned& gen) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        if (atomicAdd(&rc->tbar_cnt, 1u) == nblocks - 1) {
            rc->tbar_cnt = 0;
            __threadfence();
            atomicExch(&rc->tbar_gen, gen + 1);
        } else {
            while (vload(&rc->tbar_gen) == gen) __nanosleep(20);
        }
        __threadfence();
    }
    gen++;
    __syncthreads();
}

constexpr unsigned kTailSplit = 256;   // vertices with more out-edges are expanded by all warps
constexpr unsigned kTailSplitCap = 8192;

// Expands edges [e_lo, e_hi) of vertex v (fragment F, value sval) with one warp: check -> red.min ->
// dedupe on this iteration's next-list bitmap -> warp-aggregated append (+ its out-degree).
// tail-engine list append with a capacity check: the lists hold V entries plus kTailSlack (no-dedupe mode may
// list a vertex twice). An append past that keeps the vertex as a bit of the fragment's frontier bitmap
// instead; the reservation counter then exceeds the engine's exit bound, so the engine stops after this
// iteration and hands its frontier back to the regular path as a bitmap (dense), listed vertices included.
__device__ __forceinline__ void tail_put(const DevCtx& c, const FragPtrs& T, unsigned* nxt, unsigned idx, unsigned v) {
    if (idx < T.V + c.tail_slack) nxt[idx] = v;
    else atomicOr(T.bm + (v >> 5), 1u << (v & 31));
}

template <int ALG, bool MULTI>
__device__ __forceinline__ unsigned tail_expand(const DevCtx& c, const FragPtrs& F, unsigned sval,
                                                unsigned long long e_lo, unsigned long long e_hi, unsigned k,
                                                unsigned it, unsigned ns) {
    const unsigned lane = lane_id();
    unsigned acts = 0;
    for (unsigned long long eb = e_lo; eb < e_hi; eb += 32) {
        const unsigned long long e = eb + lane;
        bool need = false;
        int tf = 0;
        unsigned lu = 0;
        if (e < e_hi) {
            const unsigned u = __ldg(F.col + e);
            tf = MULTI ? frag_of(c, u) : 0;
            lu = MULTI ? u - c.bounds[tf] : u;
            const FragPtrs& T = c.f[tf];
            const unsigned bit = 1u << (lu & 31);
            if (ALG == ALG_BFS) {
                if (!(vload(T.vis + (lu >> 5)) & bit)) {
                    const unsigned ob = atomicOr(T.vis + (lu >> 5), bit);
                    if (!(ob & bit)) {
                        T.state[lu] = k + 1;
                        need = true;
                    }
                }
            } else {
                unsigned cand = sval;
                bool ok = true;
                if (ALG == ALG_SSSP) {
                    const unsigned long long nd = (unsigned long long)sval + __ldg(F.w + e);
                    if (nd >= (unsigned long long)GUM_INF) {
                        atomicOr(&F.ctl->err, 1u);
                        ok = false;
                    }
                    cand = (unsigned)nd;
                }
                if (ok && c.tail_nodedupe) {
                    // one returning atomic: whoever lowers the value appends v (the lists may hold a vertex
                    // twice; its second expansion relaxes nothing new)
                    need = cand < atomicMin(T.state + lu, cand);
                } else if (ok && cand < vload(T.state + lu)) {
                    atomicMin(T.state + lu, cand);
                    // the next list of iteration `it` dedupes on bm (it even) / bm2 (it odd)
                    unsigned* const dw = ((it & 1) ? T.bm2 : T.bm) + (lu >> 5);
                    // (release ordering is only needed when local rounds take entries out of the list)
                    const unsigned ob = c.tail_local ? atom_or_release(dw, bit) : atomicOr(dw, bit);
                    need = !(ob & bit);
                }
            }
        }
        const unsigned key = need ? (unsigned)tf : 0xFFFFFFFFu;
        const unsigned grp = MULTI ? __match_any_sync(0xffffffffu, key) : __ballot_sync(0xffffffffu, need);
        if (need) {
            const FragPtrs& T = c.f[tf];
            const unsigned leader = __ffs(grp) - 1;
            unsigned base = 0;
            if (lane == leader) base = atomicAdd(&T.ctl->tcnt[ns], (unsigned)__popc(grp));
            base = __shfl_sync(grp, base, leader);
            unsigned* nxt = (it & 1) ? T.q_v : T.app;
            tail_put(c, T, nxt, base + __popc(grp & lanemask_lt()), lu);
            acts++;
        }
        // out-edges of the appended vertices: one atomic per group (the counter is a single address)
        const unsigned long long deg = need ? __ldg(c.f[tf].row_ptr + lu + 1) - __ldg(c.f[tf].row_ptr + lu) : 0ull;
        if (need) {
            const unsigned hi = __reduce_add_sync(grp, (unsigned)(deg >> 16)), lo = __reduce_add_sync(grp, (unsigned)(deg & 0xFFFFu));
            if (lane == __ffs(grp) - 1) atomicAdd(&c.f[tf].ctl->tedges[ns], ((unsigned long long)hi << 16) + lo);
        }
    }
    return acts;
}

// Phase-1 variant: the warp holds kTailVPW listed vertices at once, kTailG lanes each (gl = lane in the
// group); every group walks its own vertex's edges [s0, s1) kTailG at a time. Low-degree frontiers (road-like
// grids: out-degree <= 4) would otherwise leave 28 of 32 lanes idle and serialise one vertex's dependent
// loads per warp. Appends keep the warp-aggregated reservation of tail_expand.
// (multi-fragment runs keep a warp per vertex: their tails are small frontiers spread over fragments, where
// the 8-lane groups measured slower -- SSSP 2048^2 grid on 8 virtual workers: 90 vs 123 ms of tail engine)
template <bool MULTI>
struct TailGroup {
    static constexpr unsigned G = MULTI ? 32u : 8u;
    static constexpr unsigned VPW = 32u / G;
};
// single fragment: phase-1 appends go to a CTA-local buffer, reserved in the next list with ONE atomic per
// CTA per iteration instead of one returning atomic per warp and round on the same counter address
// (thousands per iteration, serialised in one L2 slice and each on a warp's critical path)
constexpr unsigned kTailAppCap = 2048;
struct TailApp {  // per target fragment f: buf[f * cap ..], n[f], lim[f], edges[f]
    unsigned* buf;
    unsigned* n;
    unsigned* lim;  // reservations past the capacity go to the global list; the first failing base bounds
                    // the buffer's valid prefix (a straddling group leaves [base, cap) unwritten)
    unsigned long long* edges;
    unsigned cap;   // kTailAppCap / fragments
};
template <int ALG, bool MULTI>
__device__ __forceinline__ unsigned tail_expand_g(const DevCtx& c, const FragPtrs& F, bool go, unsigned sval,
                                                  unsigned long long s0, unsigned long long s1, unsigned k,
                                                  unsigned it, unsigned ns, unsigned gl, const TailApp& ta) {
    const unsigned lane = lane_id();
    unsigned acts = 0;
    const unsigned long long d = go ? s1 - s0 : 0ull;
    constexpr unsigned kTailG = TailGroup<MULTI>::G;
    const unsigned rounds = __reduce_max_sync(0xffffffffu, (unsigned)((d + kTailG - 1) / kTailG));
    for (unsigned r = 0; r < rounds; r++) {
        const unsigned long long e = s0 + (unsigned long long)r * kTailG + gl;
        bool need = false;
        int tf = 0;
        unsigned lu = 0;
        unsigned long long rp0 = 0, rp1 = 0;
        if (go && e < s1) {
            const unsigned u = __ldg(F.col + e);
            tf = MULTI ? frag_of(c, u) : 0;
            lu = MULTI ? u - c.bounds[tf] : u;
            const FragPtrs& T = c.f[tf];
            const unsigned bit = 1u << (lu & 31);
            // the neighbour's row bounds (its out-degree, for the next list's edge count) load together with
            // its state instead of after the append decision (one dependent round trip less per round)
            rp0 = __ldg(T.row_ptr + lu);
            rp1 = __ldg(T.row_ptr + lu + 1);
            if (ALG == ALG_BFS) {
                if (!(vload(T.vis + (lu >> 5)) & bit)) {
                    const unsigned ob = atomicOr(T.vis + (lu >> 5), bit);
                    if (!(ob & bit)) {
                        T.state[lu] = k + 1;
                        need = true;
                    }
                }
            } else {
                unsigned cand = sval;
                bool ok = true;
                if (ALG == ALG_SSSP) {
                    const unsigned long long nd = (unsigned long long)sval + __ldg(F.w + e);
                    if (nd >= (unsigned long long)GUM_INF) {
                        atomicOr(&F.ctl->err, 1u);
                        ok = false;
                    }
                    cand = (unsigned)nd;
                }
                if (ok && c.tail_nodedupe) {
                    need = cand < atomicMin(T.state + lu, cand);  // (see tail_expand)
                } else if (ok && cand < vload(T.state + lu)) {
                    atomicMin(T.state + lu, cand);
                    unsigned* const dw = ((it & 1) ? T.bm2 : T.bm) + (lu >> 5);
                    // (release ordering is only needed when local rounds take entries out of the list)
                    const unsigned ob = c.tail_local ? atom_or_release(dw, bit) : atomicOr(dw, bit);
                    need = !(ob & bit);
                }
            }
        }
        const unsigned key = need ? (unsigned)tf : 0xFFFFFFFFu;
        const unsigned grp = MULTI ? __match_any_sync(0xffffffffu, key) : __ballot_sync(0xffffffffu, need);
        const unsigned long long deg = need ? rp1 - rp0 : 0ull;
        if (need) {
            const FragPtrs& T = c.f[tf];
            const unsigned leader = __ffs(grp) - 1;
            const unsigned hi = __reduce_add_sync(grp, (unsigned)(deg >> 16)), lo = __reduce_add_sync(grp, (unsigned)(deg & 0xFFFFu));
            const unsigned long long gdeg = ((unsigned long long)hi << 16) + lo;
            unsigned base = 0;
            bool local = false;
            {
                // (MULTI: grp holds the lanes with the same target fragment -- match_any above)
                if (lane == leader) base = atomicAdd(ta.n + tf, (unsigned)__popc(grp));
                base = __shfl_sync(grp, base, leader);
                local = base + (unsigned)__popc(grp) <= ta.cap;  // group-uniform
                if (!local && lane == leader && base < ta.cap) atomicMin(ta.lim + tf, base);
            }
            if (local) {
                ta.buf[tf * ta.cap + base + __popc(grp & lanemask_lt())] = lu;
                if (lane == leader) atomicAdd(ta.edges + tf, gdeg);
            } else {
                if (lane == leader) base = atomicAdd(&T.ctl->tcnt[ns], (unsigned)__popc(grp));
                base = __shfl_sync(grp, base, leader);
                unsigned* nxt = (it & 1) ? T.q_v : T.app;
                tail_put(c, T, nxt, base + __popc(grp & lanemask_lt()), lu);
                if (lane == leader) atomicAdd(&T.ctl->tedges[ns], gdeg);
            }
            acts++;
        }
    }
    return acts;
}

template <int ALG, bool MULTI>
__global__ void __launch_bounds__(kTailThreads) k_tail(const __grid_constant__ DevCtx c, int w0) {
    __shared__ unsigned s_n[kMaxW], s_nsplit, s_go;
    __shared__ unsigned s_app[kTailAppCap], s_app_n[kMaxW], s_app_na[kMaxW], s_app_lim[kMaxW], s_app_base[kMaxW];
    __shared__ unsigned long long s_app_e[kMaxW];
    const unsigned app_cap = kTailAppCap / (unsigned)(MULTI ? c.P : 1);
    const TailApp ta{s_app, s_app_n, s_app_lim, s_app_e, app_cap};
    if (threadIdx.x < (unsigned)kMaxW) {
        s_app_n[threadIdx.x] = 0;
        s_app_lim[threadIdx.x] = app_cap;
        s_app_e[threadIdx.x] = 0;
    }
    __shared__ unsigned long long s_tn[kMaxW], s_te[kMaxW], s_rep_e;
    __shared__ unsigned s_app_lo;  // local relaxation rounds: buffered entries [0, s_app_lo) are already expanded
    if (threadIdx.x == 0) {
        s_rep_e = 0;
        s_app_lo = 0;
    }
    RunCtl* rc = c.rctl[w0];
    __shared__ unsigned s_hdr[4];  // gen, k0, nfT, fslot
    if (threadIdx.x == 0) {
        s_go = vload(&rc->tail) && !vload(&rc->done) && w0 == 0;  // OSteal's m'=1: unit 0 runs every fragment
        s_hdr[0] = vload(&rc->tbar_gen);
        s_hdr[1] = vload(&rc->iter) - 1;  // control already counted the first tail iteration
        const unsigned long long T = vload(&rc->nf_T);
        s_hdr[2] = (unsigned)(T < 0xFFFFFFFFull ? T : 0xFFFFFFFFull);
        s_hdr[3] = vload(&rc->nf_sweeps) & 1u;
    }
    __syncthreads();
    if (!s_go) return;
    const unsigned lane = lane_id();
    const unsigned nwarps = gridDim.x * (kTailThreads / 32);
    const unsigned gw = blockIdx.x * (kTailThreads / 32) + (threadIdx.x >> 5);
    unsigned gen = s_hdr[0];
    const unsigned k0 = s_hdr[1];
    const bool nf = (ALG == ALG_SSSP) && c.nf_delta != 0;
    const unsigned nfT = nf ? s_hdr[2] : GUM_INF;
    const unsigned fslot = s_hdr[3];
    const int nfrag = MULTI ? c.P : 1;
    gum_iter_trace* tr = c.trace[w0];
    TailSplit* split = c.tsplit[w0];
    // accounting: iteration k0's queue was already counted by the filter (frontier_*); later tail
    // iterations count their own lists. edges_done counts every expanded edge (conservation).
    unsigned long long e_done[kMaxW], e_front[kMaxW], v_front[kMaxW], a_sum = 0, tail_v = 0;
    for (int i = 0; i < kMaxW; i++) e_done[i] = e_front[i] = v_front[i] = 0;
    unsigned it = 0;
    for (;; it++) {
        const unsigned cs = it % 3, ns = (it + 1) % 3, zs = (it + 2) % 3;
        const unsigned k = k0 + it;
        unsigned long long it_edges = 0;
        unsigned long long n_all = 0;
        // list sizes: one load per CTA (per-warp loads of these single addresses serialise in L2)
        if (threadIdx.x < (unsigned)nfrag)
            s_n[threadIdx.x] = it == 0 ? (unsigned)vload(&c.f[threadIdx.x].ctl->qlen) : vload(&c.f[threadIdx.x].ctl->tcnt[cs]);
        __syncthreads();
        // ---- phase 1: kTailG lanes per listed vertex (kTailVPW vertices per warp); high-degree vertices
        // go to the split list
        constexpr unsigned kTailG = TailGroup<MULTI>::G, kTailVPW = TailGroup<MULTI>::VPW;
        const unsigned sub = lane / kTailG, gl = lane % kTailG, src = sub * kTailG;
        // one pass over list entries [lo, n) of `cur`, vertices spread over `nw` warps from warp `gwi`.
        // local = entries of this CTA's own append buffer (a local relaxation round, see below): their
        // next-list dedupe bits stay set (they are flushed to the next list as well)
        auto pass = [&](int f, const unsigned* cur, unsigned lo, unsigned n, unsigned gwi, unsigned nw, bool local) {
            const FragPtrs& F = c.f[f];
            for (unsigned i0 = lo + gwi * kTailVPW; i0 < n; i0 += nw * kTailVPW) {  // warp-uniform trip count
                const unsigned i = i0 + sub;
                const bool have = i < n;
                const unsigned v = have ? cur[i] : 0u;
                const unsigned long long s0 = have ? __ldg(F.row_ptr + v) : 0ull;
                const unsigned long long s1 = have ? __ldg(F.row_ptr + v + 1) : 0ull;
                unsigned sval = (ALG == ALG_BFS) ? k : 0u;
                unsigned slot = 0xFFFFFFFFu;
                bool park = !have;
                if (have && gl == 0) {
                    if (local) atomicAdd(&s_rep_e, s1 - s0);  // (its edges leave the next list's count)
                    if (ALG != ALG_BFS) {
                        // release the cur list's dedupe bit (reused two iterations later); any
                        // improvement of v from now on appends it to the NEXT list (other parity)
                        if (it > 0 && !local && !c.tail_nodedupe) atomicAnd(((it & 1) ? F.bm : F.bm2) + (v >> 5), ~(1u << (v & 31)));
                        // a local round takes v out of the NEXT list: release its bit there first (acquire),
                        // so an improvement after the state read below appends v again (no-dedupe mode: any
                        // later improvement appends v anyway)
                        if (local && !c.tail_nodedupe) atom_and_acquire(((it & 1) ? F.bm2 : F.bm) + (v >> 5), ~(1u << (v & 31)));
                        sval = vload(F.state + v);
                        // v's far bit is only changed by v's own processing: read it with the state (one
                        // round trip) instead of after the near/far decision
                        const unsigned fw = (nf && s1 > s0) ? F.far[v >> 5] : 0u;
                        if (nf && s1 > s0) {  // like the filter, only vertices with out-edges are parked
                            const unsigned bit = 1u << (v & 31);
                            if (sval >= nfT) {
                                park = true;
                                const unsigned ob = atomicOr(F.far + (v >> 5), bit);
                                if (!(ob & bit)) {
                                    atomicAdd(&F.ctl->far_cnt, 1ull);
                                    if (F.farl) F.farl[(size_t)fslot * F.V + atomicAdd(&F.ctl->far_n[fslot], 1u)] = v;
                                }
                                atomicMin(&F.ctl->far_min[fslot], sval);
                            } else if ((fw & bit) && !F.farl) {
                                const unsigned ob = atomicAnd(F.far + (v >> 5), ~bit);
                                if (ob & bit) atomicAdd(&F.ctl->far_cnt, ~0ull);
                            }
                        }
                    }
                    if (!park) {
                        it_edges += s1 - s0;
                        e_done[f] += s1 - s0;
                        if (it > 0 || local) e_front[f] += s1 - s0;
                        if (s1 - s0 > kTailSplit && !local) {
                            slot = atomicAdd(&rc->tsplit_cnt[it & 1], 1u);
                            if (slot < kTailSplitCap) split[slot] = TailSplit{(unsigned)f, v, sval, 0u, s0, s1};
                        }
                    }
                }
                park = __shfl_sync(0xffffffffu, park ? 1u : 0u, src) != 0;
                slot = __shfl_sync(0xffffffffu, slot, src);
                sval = __shfl_sync(0xffffffffu, sval, src);
                // split vertices are expanded cooperatively in phase 2; lists longer than 32 edges by the
                // whole warp, one vertex at a time (8 lanes would need up to 32 rounds for a 256-edge list)
                const bool go = !park && slot >= kTailSplitCap;
                const bool wide = go && s1 - s0 > 32;
                a_sum += tail_expand_g<ALG, MULTI>(c, F, go && !wide, sval, s0, s1, k, it, ns, gl, ta);
                unsigned wmask = __ballot_sync(0xffffffffu, wide && gl == 0);
                while (wmask) {
                    const unsigned ld = __ffs(wmask) - 1;
                    wmask &= wmask - 1;
                    const unsigned wv = __shfl_sync(0xffffffffu, sval, ld);
                    const unsigned long long w0s = __shfl_sync(0xffffffffu, s0, ld), w1s = __shfl_sync(0xffffffffu, s1, ld);
                    a_sum += tail_expand<ALG, MULTI>(c, F, wv, w0s, w1s, k, it, ns);
                }
            }
        };
        for (int f = 0; f < nfrag; f++) {
            const FragPtrs& F = c.f[f];
            const unsigned* cur = (it & 1) ? F.app : (it == 0 ? queue_of(c, f, vload(&F.ctl->qown)).q_v : F.q_v);
            const unsigned n = s_n[f];
            n_all += n;
            if (it > 0 && gw == 0 && lane == 0) v_front[f] += n;
            if (gw == 0 && lane == 0) tail_v += n;
            pass(f, cur, 0, n, gw, nwarps, false);
        }
        // local relaxation rounds (single fragment, min-algorithms): before the grid barrier the CTA expands
        // the vertices it has just activated (its append buffer), up to c.tail_local rounds -- the frontier
        // advances several hops per engine iteration. The entries stay in the buffer and reach the next list
        // anyway (their dedupe bits stay set, so an improvement by another CTA after the local expansion is
        // still expanded next iteration): same min-fixpoint, fewer grid barriers.
        if (!MULTI && ALG != ALG_BFS && c.tail_local) {
            unsigned done_lo = 0;
            for (unsigned lr = 0; lr < c.tail_local; lr++) {
                __syncthreads();
                const unsigned nb = s_app_n[0] < s_app_lim[0] ? s_app_n[0] : s_app_lim[0];
                if (nb <= done_lo) break;  // CTA-uniform (read after the barrier)
                if (threadIdx.x == 0) {
                    tail_v += nb - done_lo;
                    v_front[0] += nb - done_lo;
                }
                pass(0, s_app, done_lo, nb, threadIdx.x >> 5, kTailThreads / 32, true);
                done_lo = nb;
            }
            __syncthreads();
            // the expanded entries leave the buffer: only what the last round activated reaches the next list
            if (threadIdx.x == 0) {
                s_app_lo = done_lo;
                s_app_e[0] -= s_rep_e;
                s_rep_e = 0;
            }
        }
        {
            // the CTA's buffered appends: one reservation per target fragment's next list, then a copy
            __syncthreads();
            unsigned any = 0;
            for (int f = 0; f < nfrag; f++) any |= s_app_n[f];
            if (any)  // CTA-uniform (read after the barrier); nothing buffered: no reservation, no copy
        {
            if (threadIdx.x < (unsigned)nfrag) {
                const unsigned f = threadIdx.x;
                const unsigned lo = f == 0 ? s_app_lo : 0u;  // entries a local round already expanded
                const unsigned nv = s_app_n[f] < s_app_lim[f] ? s_app_n[f] : s_app_lim[f];
                const unsigned na = nv > lo ? nv - lo : 0u;
                if (na) {
                    s_app_base[f] = atomicAdd(&c.f[f].ctl->tcnt[ns], na);
                    atomicAdd(&c.f[f].ctl->tedges[ns], s_app_e[f]);
                }
                s_app_na[f] = na;  // (the valid range to copy; s_app_n stays as read by every thread above)
            }
            __syncthreads();
            for (int f = 0; f < nfrag; f++) {
                const unsigned na = s_app_na[f], lo = f == 0 ? s_app_lo : 0u;
                unsigned* nxt = (it & 1) ? c.f[f].q_v : c.f[f].app;
                for (unsigned i = threadIdx.x; i < na; i += kTailThreads) tail_put(c, c.f[f], nxt, s_app_base[f] + i, s_app[f * app_cap + lo + i]);
            }
            __syncthreads();
            if (threadIdx.x < (unsigned)kMaxW) {
                s_app_n[threadIdx.x] = 0;
                s_app_lim[threadIdx.x] = app_cap;
                s_app_e[threadIdx.x] = 0;
            }
        }
            if (threadIdx.x == 0) s_app_lo = 0;
        }
        if (tr && k < (unsigned)kTraceMax) {
            it_edges = warp_sum_u64(it_edges);  // (group leaders hold the counts)
            if (lane == 0 && it_edges) {
                if (it > 0) atomicAdd((unsigned long long*)&tr[k].frontier_edges, it_edges);
                atomicAdd((unsigned long long*)&tr[k].edges_own[0], it_edges);  // the tail's single owner
            }
            if (it > 0 && blockIdx.x == 0 && threadIdx.x == 0) tr[k].frontier_vertices = n_all;
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            // counters of iteration it+1's next list and split list start empty (nobody touches them
            // before the barrier; their previous users finished before the previous barrier)
            for (int f = 0; f < nfrag; f++) {
                c.f[f].ctl->tcnt[zs] = 0;
                c.f[f].ctl->tedges[zs] = 0;
            }
            rc->tsplit_cnt[(it + 1) & 1] = 0;
        }
        tail_barrier(rc, gridDim.x, gen);
        // ---- phase 2: split vertices, 256-edge segments dealt round-robin over every warp
        if (threadIdx.x == 0) s_nsplit = min(vload(&rc->tsplit_cnt[it & 1]), kTailSplitCap);
        __syncthreads();
        const unsigned nsplit = s_nsplit;
        if (nsplit) {
            for (unsigned sid = gw;; sid += nwarps) {
                // locate segment sid: prefix of segment counts over the split list (warp-parallel)
                unsigned base = 0, j = 0xFFFFFFFFu, seg = 0;
                for (unsigned j0 = 0; j0 < nsplit && j == 0xFFFFFFFFu; j0 += 32) {
                    unsigned cnt = 0;
                    if (j0 + lane < nsplit) {
                        const TailSplit& t = split[j0 + lane];
                        cnt = (unsigned)((t.s1 - t.s0 + kTailSplit - 1) / kTailSplit);
                    }
                    unsigned inc = cnt;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const unsigned x = __shfl_up_sync(0xffffffffu, inc, o);
                        if (lane >= (unsigned)o) inc += x;
                    }
                    const unsigned hit = __ballot_sync(0xffffffffu, cnt && sid < base + inc && sid >= base + inc - cnt);
                    if (hit) {
                        const unsigned l = __ffs(hit) - 1;
                        j = j0 + l;
                        seg = sid - (base + __shfl_sync(0xffffffffu, inc - cnt, l));
                    }
                    base += __shfl_sync(0xffffffffu, inc, 31);
                }
                if (j == 0xFFFFFFFFu) break;  // past the last segment
                const TailSplit t = split[j];
                const unsigned long long lo = t.s0 + (unsigned long long)seg * kTailSplit;
                const unsigned long long hi = lo + kTailSplit < t.s1 ? lo + kTailSplit : t.s1;
                a_sum += tail_expand<ALG, MULTI>(c, c.f[t.f], t.sval, lo, hi, k, it, ns);
            }
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            if (tr && k + 1 < (unsigned)kTraceMax) {  // row of iteration k+1 (accumulated after the barrier)
                gum_iter_trace* r = tr + k + 1;
                for (int i = 0; i < kMaxW; i++) r->t_start[i] = r->t_end[i] = r->edges_own[i] = r->edges_stolen[i] = 0;
                r->frontier_edges = 0;
                r->frontier_vertices = 0;
                r->owners = 1;
                r->steal_ok = 0;
            }
        }
        // appends of phase 2 (and the trace row) must be complete before the counts are read
        if (nsplit || tr) tail_barrier(rc, gridDim.x, gen);
        if (threadIdx.x < (unsigned)nfrag) {
            s_tn[threadIdx.x] = vload(&c.f[threadIdx.x].ctl->tcnt[ns]);
            s_te[threadIdx.x] = vload(&c.f[threadIdx.x].ctl->tedges[ns]);
        }
        __syncthreads();
        unsigned long long total_next = 0, next_edges = 0;
        bool list_ovf = false;  // a next list overflowed into the bitmap (tail_put): hand back now
        for (int f = 0; f < nfrag; f++) {
            total_next += s_tn[f];
            next_edges += s_te[f];
            list_ovf = list_ovf || s_tn[f] > c.f[f].V + c.tail_slack;
        }
        // every CTA must take the same decision: only values that are final after the barrier (next-list
        // counters) enter it -- not the error flag, which next-iteration work of a fast CTA may already
        // set (overflowing candidates are simply not relaxed; control reports GUM_ERANGE afterwards)
        if (total_next == 0 || total_next > c.tail_exit || next_edges > 4ull * c.tail_exit || k + 1 >= c.max_iter ||
            list_ovf)
            break;
    }
    for (int f = 0; f < nfrag; f++) {
        e_done[f] = warp_sum_u64(e_done[f]);  // group leaders (lanes 0, kTailG, ...) hold the counts
        e_front[f] = warp_sum_u64(e_front[f]);
        if (lane == 0 && e_done[f]) {
            atomicAdd(&c.f[f].ctl->edges_done, e_done[f]);
            atomicAdd(&c.f[0].ctl->tail_edges, e_done[f]);
            if (e_front[f]) atomicAdd(&c.f[f].ctl->frontier_edges, e_front[f]);
        }
        // (thread 0 of warp 0 holds the list counts; thread 0 of every CTA its local rounds' entries)
        if (threadIdx.x == 0 && v_front[f]) atomicAdd(&c.f[f].ctl->frontier_vertices, v_front[f]);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) a_sum += __shfl_xor_sync(0xffffffffu, a_sum, o);
    if (lane == 0 && a_sum) {
        atomicAdd(&c.f[0].ctl->activations, a_sum);
        atomicAdd(&c.f[0].ctl->tail_acts, a_sum);
    }
    if (tail_v) atomicAdd(&c.f[0].ctl->tail_vertices, tail_v);
    // hand the last produced list back to the regular path as the sparse activation list (no-dedupe mode after
    // a list overflow: as the frontier bitmap)
    if (blockIdx.x == 0) {
        const unsigned ns = (it + 1) % 3;
        bool ovf = false;
        for (int f = 0; f < nfrag; f++) ovf = ovf || vload(&c.f[f].ctl->tcnt[ns]) > c.f[f].V + c.tail_slack;
        for (int f = 0; f < nfrag; f++) {
            unsigned n = vload(&c.f[f].ctl->tcnt[ns]);
            if (ALG != ALG_BFS && c.tail_nodedupe) {
                // no-dedupe lists may hold a vertex twice: the regular path gets each once, its bm bit set
                // (as a deduplicated activation list); compacted into the other list, then moved to app
                __shared__ unsigned s_hb;
                if (threadIdx.x == 0) s_hb = 0;
                __syncthreads();
                const unsigned* srcl = (it & 1) ? c.f[f].q_v : c.f[f].app;
                unsigned* dstl = (it & 1) ? c.f[f].app : c.f[f].q_v;
                for (unsigned i = threadIdx.x; i < n && i < c.f[f].V + c.tail_slack; i += kTailThreads) {
                    const unsigned v = srcl[i], bit = 1u << (v & 31);
                    if (!(atomicOr(c.f[f].bm + (v >> 5), bit) & bit)) dstl[atomicAdd(&s_hb, 1u)] = v;
                }
                __syncthreads();
                n = s_hb;
                if (!(it & 1))
                    for (unsigned i = threadIdx.x; i < n; i += kTailThreads) c.f[f].app[i] = c.f[f].q_v[i];
                __syncthreads();
                if (threadIdx.x == 0) c.f[f].ctl->app_cnt = n;
                continue;
            }
            if (it & 1) {  // the last next list lives in q_v with its dedupe bits in bm2: move both
                for (unsigned i = threadIdx.x; i < n; i += kTailThreads) {
                    const unsigned v = c.f[f].q_v[i];
                    c.f[f].app[i] = v;
                    if (ALG != ALG_BFS) {
                        atomicAnd(c.f[f].bm2 + (v >> 5), ~(1u << (v & 31)));
                        atomicOr(c.f[f].bm + (v >> 5), 1u << (v & 31));
                    }
                }
            }
            __syncthreads();
            if (threadIdx.x == 0) c.f[f].ctl->app_cnt = n;
        }
        if (threadIdx.x == 0) {
            rc->iter = k0 + it + 1;
            rc->tail_iters += it + 1;
            rc->next_dense = ovf ? 1u : 0u;
            if (ovf) atomicAdd(&c.f[0].ctl->tail_ovf, 1u);
            rc->tail = 0;
            __threadfence();
        }
    }
}

#ifdef GUM_FILTER_TIMING
void dump_filter_timing() {
    static unsigned long long h[1024][8];
    cudaDeviceSynchronize();
    cudaMemcpyFromSymbol(h, g_ftime, sizeof(h));
    unsigned long long t0 = ~0ull;
    for (int i = 0; i < 1024; i++) if (h[i][0] && h[i][0] < t0) t0 = h[i][0];
    for (int i = 0; i < 1024; i++) {
        if (!h[i][0]) continue;
        fprintf(stderr, "cta %4d b=%4llu G=%llu app=%llu start=%7.2f pro=%7.2f p1=%7.2f pre=%7.2f end=%7.2f\n", i, h[i][5], h[i][6], h[i][7],
                (h[i][0] - t0) / 1e3, (h[i][1] - t0) / 1e3, h[i][2] ? (h[i][2] - t0) / 1e3 : -1.0, h[i][3] ? (h[i][3] - t0) / 1e3 : -1.0,
                h[i][4] ? (h[i][4] - t0) / 1e3 : -1.0);
    }
}
#endif

cudaError_t filter_occupancy(int* blocks_per_sm) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k_filter<true>, kThreads, 0);
}

cudaError_t tail_occupancy(int* blocks_per_sm) {
    int a = 0, b = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&a, k_tail<ALG_SSSP, true>, kTailThreads, 0);
    if (e != cudaSuccess) return e;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_tail<ALG_BFS, true>, kTailThreads, 0);
    *blocks_per_sm = a < b ? a : b;
    return e;
}

template <int ALG>
static cudaError_t launch_tail(const DevCtx& c, const LaunchCfg& L, cudaStream_t s) {
    if constexpr (ALG == ALG_PR || ALG == ALG_DPR) {
        return cudaSuccess;  // (no tail engine for the PageRank variants)
    } else {
    if (L.tail_grid <= 0) return cudaSuccess;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(L.tail_grid);
    cfg.blockDim = dim3(kTailThreads);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;  // co-residency guaranteed (grid barrier inside)
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (c.P > 1) return cudaLaunchKernelEx(&cfg, k_tail<ALG, true>, c, L.w0);
    return cudaLaunchKernelEx(&cfg, k_tail<ALG, false>, c, L.w0);
    }
}

// ------------------------------------------------------------------------------------------ bottom-up
// NEXT-4 direction-optimising BFS: in a bottom-up iteration every unvisited vertex of an owned fragment
// looks for a parent at depth k among its in-edges and stops at the first one (a warp per 32-vertex
// visited word, a lane per vertex). New vertices get depth k+1 and their visited and next-frontier bits
// (one word store per warp: each word has a single writer). The frontier's out-edges are counted as
// expanded (the result is the same BFS tree depth); pull_checked records the in-edges inspected.
template <bool MULTI>
__global__ void __launch_bounds__(kThreads) k_bfs_pull(const __grid_constant__ DevCtx c, int w0, int nw) {
    RunCtl* rc = c.rctl[w0];
    const int f = blockIdx.y;
    __shared__ unsigned s_go, s_k;  // prologue by one thread per CTA (hot run-control addresses)
    if (threadIdx.x == 0) {
        const unsigned o = vload(&rc->owner[f]);
        s_go = vload(&rc->pull) && !vload(&rc->done) && !vload(&rc->tail) && (int)o >= w0 && (int)o < w0 + nw;
        s_k = vload(&rc->iter) - 1;
    }
    __syncthreads();
    if (!s_go) return;
    const FragPtrs& F = c.f[f];
    const unsigned k = s_k;
    const unsigned lane = lane_id();
    const unsigned nwords = (F.V + 31) / 32;
    const unsigned warps = gridDim.x * (kThreads / 32);
    unsigned long long checked = 0;
    for (unsigned w = blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5); w < nwords; w += warps) {
        const unsigned vw = F.vis[w];
        const unsigned rem = F.V - w * 32;
        const unsigned valid = rem >= 32 ? 0xFFFFFFFFu : ((1u << rem) - 1u);
        const unsigned todo = ~vw & valid;
        if (!todo) continue;  // warp-uniform
        bool found = false;
        if ((todo >> lane) & 1u) {
            const unsigned v = w * 32 + lane;
            const unsigned long long e1 = __ldg(F.in_row_ptr + v + 1);
            for (unsigned long long e = __ldg(F.in_row_ptr + v); e < e1; e++) {
                const unsigned u = __ldg(F.in_col + e);
                const int tf = MULTI ? frag_of(c, u) : 0;
                const unsigned lu = MULTI ? u - c.bounds[tf] : u;
                checked++;
                if (__ldcg(c.f[tf].state + lu) == k) {
                    found = true;
                    break;
                }
            }
            if (found) F.state[v] = k + 1;
        }
        const unsigned nb = __ballot_sync(0xffffffffu, found);
        if (lane == 0 && nb) {
            F.vis[w] = vw | nb;
            atomicOr(F.bm + w, nb);
        }
    }
#pragma unroll
    for (int q = 16; q > 0; q >>= 1) checked += __shfl_xor_sync(0xffffffffu, checked, q);
    if (lane == 0 && checked) atomicAdd(&F.ctl->pull_checked, checked);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        // conservation: the frontier's out-edges count as expanded in a bottom-up iteration
        atomicAdd(&F.ctl->edges_done, vload(&F.ctl->qedges));
        atomicAdd(&F.ctl->chunks_done, vload(&F.ctl->ntiles));
    }
}

// ------------------------------------------------------------------------------------------ PB apply
// Second half of a propagation-blocked BFS iteration (runs first in the next body, before the filter):
// CTA (block b, part) loads block b's visited bits (2^pb_shift bits) into shared memory, sets the bits of
// its slice of the binned ids there, and publishes the newly set bits as visited + next-frontier bits
// with word-wide red.or, writing depth k+1 for each new vertex. Parts of one block may both discover a
// vertex: the bit ORs and the depth store are idempotent.
constexpr int kPbParts = 8;

__global__ void __launch_bounds__(kThreads) k_pb_apply(const __grid_constant__ DevCtx c, int w0) {
    RunCtl* rc = c.rctl[w0];
    if (!vload(&rc->pb) || vload(&rc->done)) return;
    extern __shared__ unsigned s_pbw[];  // [2 * W]: working bits, original bits
    const unsigned W = 1u << (c.pb_shift - 5);
    unsigned* s_vis = s_pbw;
    unsigned* s_org = s_pbw + W;
    const FragPtrs& F = c.f[0];
    const unsigned b = blockIdx.x / kPbParts, part = blockIdx.x % kPbParts;
    if (b >= c.pb_nb) return;
    const unsigned level = rc->iter;  // the advance of iteration iter-1 discovered depth iter
    const unsigned nwords = (F.V + 31) / 32;
    const unsigned w_lo = b * W;
    for (unsigned w = threadIdx.x; w < W; w += kThreads) {
        const unsigned x = (w_lo + w < nwords) ? F.vis[w_lo + w] : 0xFFFFFFFFu;
        s_vis[w] = x;
        s_org[w] = x;
    }
    __syncthreads();
    const unsigned long long base = F.pb_off[b];
    const unsigned n = vload(&F.pb_fill[b]);
    const unsigned lo = (unsigned)((unsigned long long)n * part / kPbParts);
    const unsigned hi = (unsigned)((unsigned long long)n * (part + 1) / kPbParts);
    for (unsigned i = lo + threadIdx.x; i < hi; i += kThreads) {
        const unsigned v = __ldcs(F.pb_buf + base + i);
        const unsigned lw = (v >> 5) - w_lo, bit = 1u << (v & 31);
        if (!(s_vis[lw] & bit)) atomicOr(&s_vis[lw], bit);
    }
    __syncthreads();
    unsigned acts = 0;
    for (unsigned w = threadIdx.x; w < W; w += kThreads) {
        const unsigned nw = s_vis[w] & ~s_org[w];
        if (!nw) continue;
        atomicOr(F.vis + w_lo + w, nw);
        atomicOr(F.bm + w_lo + w, nw);
        unsigned x = nw;
        while (x) {
            const unsigned bb = __ffs(x) - 1;
            x &= x - 1;
            F.state[(w_lo + w) * 32 + bb] = level;
            acts++;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acts += __shfl_xor_sync(0xffffffffu, acts, o);
    if (lane_id() == 0 && acts) atomicAdd(&F.ctl->activations, (unsigned long long)acts);
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        if (atomicAdd(&F.pb_done[b], 1u) == kPbParts - 1) {  // last part resets the bin for next time
            F.pb_fill[b] = 0;
            F.pb_done[b] = 0;
        }
    }
}

// ------------------------------------------------------------------------------------------ PR push (P = 1)
// The advance of PR's static frontier on one fragment, without CTA barriers: the destination-blocked queue
// is cut at gum_prepare into entries of <= kPrPiece edges, and each warp task takes 32 consecutive entries
// (one per lane: x/outdeg of its source, its col range), scans their lengths with shuffles and walks the
// task's edges 32 at a time -- a warp-level merge path: lane e finds its entry by a 5-step shuffle binary
// search over the lanes' prefixes, loads col (consecutive edges are consecutive in the blocked col array,
// so every round is one coalesced 128-byte load) and issues red.add.f64 of the entry's value into acc.
// The CTA-level merge path of k_advance spends ~27% of its stalls on the per-chunk barriers here (the PR
// push has only 8 edges of work per thread per chunk); warps here are independent. Same sums as k_advance.
// Measured on C5 (opt-in, GUM_PR_PUSH=1): 12.0 ms per iteration vs 10.8 ms for k_advance -- the 8 dependent
// shuffles per 32 edges make it MIO-bound (short_sb 33% + mio 17% of stalls); a static task split was
// worse still (19.1 ms: warps drifted over several acc blocks and thrashed L2).
__global__ void __launch_bounds__(kThreads) k_pr_push(const __grid_constant__ DevCtx c, int w0, int nw) {
    RunCtl* rc = c.rctl[w0];
    __shared__ unsigned s_go;
    if (threadIdx.x == 0) s_go = !vload(&rc->done) && (unsigned)w0 < vload(&rc->m);
    __syncthreads();
    if (!s_go) return;
    const unsigned long long t0 = globaltimer();
    const FragPtrs& F = c.f[0];
    const unsigned lane = lane_id();
    const unsigned long long n = F.pr2_len;
    const unsigned long long tasks = (n + 31) / 32;
    unsigned long long edges = 0;
    // dynamic claims of kPrClaim tasks (one atomic per ~1K edges): every warp works in the same narrow
    // window of the destination-blocked queue, so only the current acc block is live in L2 (a static
    // task split let warps drift over several blocks and thrash L2: 7.5 GB of acc write-backs per launch)
    constexpr unsigned kPrClaim = 4;
    unsigned long long nxt = 0;
    if (lane == 0) nxt = atomicAdd(&F.ctl->claim, (unsigned long long)kPrClaim);
    nxt = __shfl_sync(0xffffffffu, nxt, 0);
    for (;;) {
        const unsigned long long cl = nxt;
        if (cl >= tasks) break;
        if (lane == 0) nxt = atomicAdd(&F.ctl->claim, (unsigned long long)kPrClaim);  // one claim ahead
        nxt = __shfl_sync(0xffffffffu, nxt, 0);
        const unsigned long long tend = cl + kPrClaim < tasks ? cl + kPrClaim : tasks;
    for (unsigned long long task = cl; task < tend; task++) {
        const unsigned long long i = task * 32 + lane;
        unsigned long long off = 0, len = 0;
        double val = 0.0;
        if (i < n) {
            off = __ldcs(F.pr2_q_off + i);
            len = __ldcs(F.pr2_q_off + i + 1) - off;
            val = __ldcg(F.cx + __ldcs(F.pr2_q_v + i));
        }
        // inclusive prefix of the entry lengths over the lanes (len <= kPrPiece: 32-bit sums)
        unsigned inc = (unsigned)len;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned x = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= (unsigned)o) inc += x;
        }
        const unsigned tot = __shfl_sync(0xffffffffu, inc, 31);
        const unsigned excl = inc - (unsigned)len;
        for (unsigned b = 0; b < tot; b += 32) {
            const unsigned e = b + lane;
            // entry of edge e: the last lane j with excl_j <= e (lanes with len 0 share their successor's
            // excl and are never selected past it: the search takes the largest such j)
            unsigned j = 0;
#pragma unroll
            for (unsigned step = 16; step > 0; step >>= 1) {
                const unsigned x = __shfl_sync(0xffffffffu, excl, j + step);
                if (x <= e) j += step;
            }
            const unsigned long long oj = __shfl_sync(0xffffffffu, off, j);
            const double vj = __shfl_sync(0xffffffffu, val, j);
            const unsigned ej = __shfl_sync(0xffffffffu, excl, j);
            if (e < tot) {
                const unsigned v = __ldcs(F.col + oj + (e - ej));
                atomicAdd(F.acc + v, vj);  // RED.ADD.F64
            }
        }
        edges += tot;
    }
    }
    // conservation counters (lane 0 holds the per-task totals) and the worker's busy window
    if (lane == 0 && edges) atomicAdd(&F.ctl->edges_done, edges);
    gum_iter_trace* tr = c.trace[w0];
    const unsigned k = vload(&rc->iter) - 1;
    if (tr && threadIdx.x == 0 && k < (unsigned)kTraceMax) {
        atomicMin((unsigned long long*)&tr[k].t_start[0], t0);
        atomicMax((unsigned long long*)&tr[k].t_end[0], globaltimer());
    }
    if (tr && lane == 0 && edges && k < (unsigned)kTraceMax) atomicAdd((unsigned long long*)&tr[k].edges_own[0], edges);
}

cudaError_t pr_push_occupancy(int* blocks_per_sm) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k_pr_push, kThreads, 0);
}

// ------------------------------------------------------------------------------------------ PR pull
// a8 for PageRank as a pull: pass b gathers, for every vertex v of the fragment, the sum of
// x[u]/outdeg(u) over v's in-edges whose source u lies in source block b (an L2-resident slice of the
// unit's replica of x/outdeg) and adds it to acc[v]; the finalize then forms x' = (1-d)/V + d(acc + D/V)
// as for the push (same terms, summed in another order). Rows and edges of a pass are balanced over CTAs
// by merge path (Merrill & Garland's SpMV): a tile is kPullTile consecutive items of the merge of row ends
// and edge indices. Per tile the CTA first stages, with coalesced loads and every gather of a thread in
// flight at once, the tile's edge values x[u]/outdeg(u), its row ends and its rows' accumulators into
// shared memory; then thread t walks kPullIPT items of the merge. A row that ends in a thread after that
// thread's first row lies entirely inside the thread and is stored once (acc + sum); partial rows are
// carried between threads by a block-wide segmented scan, and only rows that cross a tile boundary use a
// global fp64 atomic: <= 2 atomics per tile instead of one red.add.f64 per edge.
// (A three-stage cp.async pipeline -- ids, then 8-byte async gathers, then the reduction -- measured 2x
// slower on C5: DESIGN.md §6.)
__device__ __forceinline__ unsigned pull_slot(unsigned e) { return e + (e >> 3); }

__global__ void __launch_bounds__(kThreads) k_pr_pull(const __grid_constant__ DevCtx c, int w0, int nw, int pass) {
    __shared__ unsigned s_re[kPullTile + 1];  // row ends (relative to the pass's first edge) of the tile's rows
    // x[u]/outdeg(u) of the tile's edges, one pad slot after every 8 (pull_slot): the walk's lanes read items
    // ~8 apart, i.e. 64 bytes apart unpadded -- a 16-way bank conflict per LDS.64; padded, 72 bytes apart
    __shared__ double s_val[kPullTile + kPullTile / 8];
    __shared__ double s_acc[kPullTile + 1];   // acc of the tile's rows (rows x0 .. x1)
    __shared__ unsigned s_key[kThreads];
    __shared__ double s_inc[kThreads];
    __shared__ unsigned s_wkey[kThreads / 32], s_ckey[kThreads / 32];
    __shared__ double s_wval[kThreads / 32], s_cval[kThreads / 32];
    __shared__ unsigned s_tx[3];
    struct Pro {
        unsigned go, buf, owner, k;
        unsigned long long tb0, ntiles, t0;
    };
    __shared__ Pro s_pro;
    RunCtl* rc = c.rctl[w0];
    const int f = blockIdx.y;
    const FragPtrs& F = c.f[f];
    const unsigned Vf = F.V;
    const unsigned* off = F.pl_off + (size_t)pass * Vf;
    if (threadIdx.x == 0) {
        Pro p{};
        p.owner = vload(&rc->owner[f]);
        p.go = !vload(&rc->done) && (int)p.owner >= w0 && (int)p.owner < w0 + nw;
        if (p.go) {
            p.k = vload(&rc->iter) - 1u;
            p.buf = p.k & 1u;  // iteration k reads x_k/outdeg (control set iter = k+1)
            p.t0 = globaltimer();
            p.tb0 = F.pl_tb[pass];
            p.ntiles = F.pl_tb[pass + 1] - p.tb0 - 1;
        }
        s_pro = p;
    }
    __syncthreads();
    if (!s_pro.go) return;
    const unsigned lane = lane_id(), wid = threadIdx.x >> 5;
    const unsigned ebase = __ldg(off);
    const unsigned long long items = (unsigned long long)Vf + (__ldg(off + Vf) - ebase);
    const double* cx = c.cxw[s_pro.owner] + (size_t)s_pro.buf * c.num_vertices;
    const unsigned* pcol = F.pl_col + ebase;
    double* acc = F.acc;
    const unsigned long long tb0 = s_pro.tb0, ntiles = s_pro.ntiles;
    unsigned long long edges = 0;
    // tile-table entries of the next tile are loaded one tile ahead (threads 0 and 1)
    unsigned nx_tx = 0;
    if (threadIdx.x < 2 && blockIdx.x < ntiles) nx_tx = __ldg(F.pl_tx + tb0 + blockIdx.x + threadIdx.x);
    for (unsigned long long t = blockIdx.x; t < ntiles; t += gridDim.x) {
        if (threadIdx.x < 2) {
            s_tx[threadIdx.x] = nx_tx;
            const unsigned long long tn = t + gridDim.x;
            if (tn < ntiles) nx_tx = __ldg(F.pl_tx + tb0 + tn + threadIdx.x);
        }
        __syncthreads();
        const unsigned x0 = s_tx[0], x1 = s_tx[1];
        const unsigned long long d0 = t * kPullTile;
        const unsigned long long d1 = d0 + kPullTile < items ? d0 + kPullTile : items;
        const unsigned y0 = (unsigned)(d0 - x0), y1 = (unsigned)(d1 - x1);
        const unsigned ne_t = y1 - y0;
        // stage: edge values (coalesced col ids, all gathers of a thread issued back to back), row ends and
        // the accumulators of rows x0 .. min(x1, Vf-1), row x0's start
        {
            unsigned cu[kPullIPT];
#pragma unroll
            for (int j = 0; j < kPullIPT; j++) {
                const unsigned e = threadIdx.x + j * kThreads;
                cu[j] = e < ne_t ? __ldcs(pcol + y0 + e) : 0u;
            }
#pragma unroll
            for (int j = 0; j < kPullIPT; j++) {
                const unsigned e = threadIdx.x + j * kThreads;
                if (e < ne_t) s_val[pull_slot(e)] = __ldg(cx + cu[j]);
            }
        }
        const unsigned nr = (x1 < Vf ? x1 : Vf - 1u) - x0 + 1u;
        for (unsigned i = threadIdx.x; i < nr; i += kThreads) {
            s_re[i] = __ldg(off + x0 + i + 1) - ebase;
            s_acc[i] = __ldcg(acc + x0 + i);
        }
        if (threadIdx.x == kThreads - 1) s_tx[2] = __ldg(off + x0) - ebase;
        __syncthreads();
        edges += ne_t;  // (the same tile total in every thread; thread 0's is flushed)
        // this thread's merge-path coordinate inside the tile
        const unsigned tl = (unsigned)(d1 - d0);
        const unsigned dl = threadIdx.x * kPullIPT < tl ? threadIdx.x * kPullIPT : tl;
        const unsigned ni = tl - dl < (unsigned)kPullIPT ? tl - dl : (unsigned)kPullIPT;
        unsigned lo = dl > ne_t ? dl - ne_t : 0u, hi = dl < x1 - x0 ? dl : x1 - x0;
        while (lo < hi) {
            const unsigned mid = (lo + hi) >> 1;
            if (s_re[mid] <= y0 + (dl - mid) - 1u) lo = mid + 1u;
            else hi = mid;
        }
        const unsigned xs = x0 + lo, ys = y0 + dl - lo;
        // walk: a row that ends in this thread after its first row is complete here -> one store
        double sum = 0.0, first_sum = 0.0;
        bool has_first = false;
        unsigned xi = xs, yi = ys;
#pragma unroll
        for (int k = 0; k < kPullIPT; k++) {
            if ((unsigned)k < ni) {
                if (yi < s_re[xi - x0]) {
                    sum += s_val[pull_slot(yi - y0)];
                    yi++;
                } else {
                    if (!has_first) {
                        has_first = true;
                        first_sum = sum;
                    } else if (sum != 0.0) {
                        acc[xi] = s_acc[xi - x0] + sum;
                    }
                    sum = 0.0;
                    xi++;
                }
            }
        }
        // block-wide inclusive segmented scan of the carry-outs (key = row in progress; keys are monotone)
        unsigned key = xi;
        double val = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const double v2 = __shfl_up_sync(0xffffffffu, val, o);
            const unsigned k2 = __shfl_up_sync(0xffffffffu, key, o);
            if (lane >= (unsigned)o && k2 == key) val += v2;
        }
        if (lane == 31) {
            s_wkey[wid] = key;
            s_wval[wid] = val;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            unsigned ck = 0xFFFFFFFFu;
            double cv = 0.0;
            for (int w = 0; w < kThreads / 32; w++) {
                s_ckey[w] = ck;
                s_cval[w] = cv;
                if (s_wkey[w] == ck) {
                    cv += s_wval[w];
                } else {
                    ck = s_wkey[w];
                    cv = s_wval[w];
                }
            }
        }
        __syncthreads();
        if (key == s_ckey[wid]) val += s_cval[wid];
        s_key[threadIdx.x] = key;
        s_inc[threadIdx.x] = val;
        __syncthreads();
        if (has_first) {
            // this thread's first row: add what earlier threads of the tile carried into it; a row that
            // began in an earlier tile gets the rest from that tile's atomic, so it is added atomically too
            double tot = first_sum;
            if (threadIdx.x > 0 && s_key[threadIdx.x - 1] == xs) tot += s_inc[threadIdx.x - 1];
            if (xs == x0 && s_tx[2] < y0) {
                if (tot != 0.0) atomicAdd(acc + xs, tot);
            } else if (tot != 0.0) {
                acc[xs] = s_acc[xs - x0] + tot;
            }
        }
        if (threadIdx.x == kThreads - 1 && key < Vf && val != 0.0) atomicAdd(acc + key, val);  // continues in t+1
    }
    if (threadIdx.x == 0 && edges) {
        atomicAdd(&F.ctl->edges_done, edges);
        gum_iter_trace* tr = c.trace[w0];
        const unsigned k = s_pro.k, o = s_pro.owner;
        if (tr && k < (unsigned)kTraceMax) {  // per-worker busy window and edges (trace)
            atomicAdd((unsigned long long*)&tr[k].edges_own[o], edges);
            atomicMin((unsigned long long*)&tr[k].t_start[o], s_pro.t0);
            atomicMax((unsigned long long*)&tr[k].t_end[o], globaltimer());
        }
    }
}

cudaError_t pr_pull_occupancy(int* blocks_per_sm) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k_pr_pull, kThreads, 0);
}

// ------------------------------------------------------------------------------------------ PR finalize
__global__ void __launch_bounds__(kThreads) k_pr_finalize(const __grid_constant__ DevCtx c, int w0, int nw) {
    RunCtl* rc = c.rctl[w0];
    const int f = blockIdx.y;
    __shared__ unsigned s_go;  // prologue by one thread per CTA (hot run-control addresses)
    __shared__ double s_D;
    __shared__ unsigned s_nbuf;
    if (threadIdx.x == 0) {
        const unsigned o = vload(&rc->owner[f]);
        s_go = !vload(&rc->done) && (int)o >= w0 && (int)o < w0 + nw;
        s_D = vload(&rc->pr_D);
        s_nbuf = vload(&rc->iter) & 1u;
    }
    __syncthreads();
    if (!s_go) return;
    const FragPtrs& F = c.f[f];
    // PR's frontier queue is static: re-arm its steal-queue head for the next advance (every
    // advance of this iteration has finished: kernel boundary / cross-device barrier)
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        F.ctl->claim = 0;
        for (int q = 0; q < kMaxW; q++) F.ctl->pclaim[q] = 0;
    }
    const double N = (double)c.num_vertices, d = c.pr_d, D = s_D;
    const unsigned nbuf = s_nbuf;  // PR pull replicas: x_{k+1}/outdeg goes to buffer (k+1)&1
    double dang = 0.0, res = 0.0;
    const bool mir = c.mirrors && c.P > 1;
    for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < F.V; i += gridDim.x * blockDim.x) {
        const double xo = F.x[i];
        double a = F.acc[i];
        if (mir) {
            // NEXT-1: the aggregated pushes of every other worker to this (for them outer) vertex are
            // pulled from their mirrors (coalesced peer loads) and the mirror entries cleared
            for (int q = 1; q < c.P; q++) {
                const int g = f + q < c.P ? f + q : f + q - c.P;  // peers in rotated order
                double* m = c.f[g].macc + F.base + i;
                a += *m;
                *m = 0.0;
            }
        }
        const double nx = (1.0 - d) / N + d * (a + D / N);
        res += fabs(nx - xo);
        const unsigned long long od = __ldg(F.row_ptr + i + 1) - __ldg(F.row_ptr + i);
        if (od == 0) dang += nx;
        F.x[i] = nx;
        const double cxv = od ? nx / (double)od : 0.0;  // next iteration's push / pull value x'/outdeg
        F.cx[i] = cxv;
        F.acc[i] = 0.0;
        for (int r = 0; r < c.n_rep; r++) c.cxrep[r][(size_t)nbuf * c.num_vertices + F.base + i] = cxv;
    }
#pragma unroll
    for (int s = 16; s > 0; s >>= 1) {
        dang += __shfl_xor_sync(0xffffffffu, dang, s);
        res += __shfl_xor_sync(0xffffffffu, res, s);
    }
    __shared__ double s_d[kThreads / 32], s_r[kThreads / 32];
    if (lane_id() == 0) {
        s_d[threadIdx.x >> 5] = dang;
        s_r[threadIdx.x >> 5] = res;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double a = 0, b = 0;
        for (int i = 0; i < kThreads / 32; i++) {
            a += s_d[i];
            b += s_r[i];
        }
        const unsigned slot = (rc->iter - 1) & 1;
        atomicAdd(&F.ctl->pr_dang[slot], a);
        atomicAdd(&F.ctl->pr_resid[slot], b);
    }
}

// ------------------------------------------------------------------------------------------ result
template <typename T>
__global__ void k_gather(const __grid_constant__ DevCtx c, int f, T* out, int is_pr) {
    const FragPtrs& F = c.f[f];
    for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i < F.V; i += gridDim.x * blockDim.x) {
        const unsigned ov = F.orig ? F.orig[i] : F.base + i;
        if (is_pr)
            ((double*)out)[ov] = F.x[i];
        else
            ((unsigned*)out)[ov] = F.state[i];
    }
}

// ================================================================================ host launchers
// Phase A / phase B of one iteration; a cross-device barrier separates them (and follows B) when
// the workers live on different GPUs. In single-device mode both phases go into one graph body.
//   BFS/SSSP/WCC: A = filter            B = control, advance
//   PR:           A = control, advance  B = finalize
// Phase A / phase B of one iteration; a cross-device barrier separates them (and follows B) when
// the workers live on different GPUs. In single-device mode both phases go into one graph body.
//   BFS/SSSP/WCC: A = filter            B = control, advance
//   PR:           A = control, advance  B = finalize
template <int ALG>
static cudaError_t launch_kernel_t(int kind, const DevCtx& c, const LaunchCfg& L, cudaStream_t s,
                                   cudaGraphConditionalHandle h, int use_h) {
    switch (kind) {
        case KER_FILTER:
            if (c.nf_delta)
                k_filter<true><<<dim3(L.filter_grid, c.P), kThreads, 0, s>>>(c, L.w0, L.nw, c.fuse_ctl, h, use_h);
            else if (ALG == ALG_DPR)
                k_filter<false, true><<<dim3(L.filter_grid, c.P), kThreads, 0, s>>>(c, L.w0, L.nw, c.fuse_ctl, h, use_h);
            else
                k_filter<false><<<dim3(L.filter_grid, c.P), kThreads, 0, s>>>(c, L.w0, L.nw, c.fuse_ctl, h, use_h);
            break;
        case KER_CONTROL: k_control<ALG><<<1, 32, 0, s>>>(c, L.w0, L.nw, h, use_h); break;
        case KER_ADVANCE:
            if (ALG == ALG_PR && c.pl_B) {
                for (unsigned b = 0; b < c.pl_B; b++) {
                    k_pr_pull<<<dim3(L.pull_grid, c.P), kThreads, 0, s>>>(c, L.w0, L.nw, (int)b);
                    cudaError_t e = cudaGetLastError();
                    if (e != cudaSuccess) return e;
                }
            } else if (ALG == ALG_PR && c.P == 1 && c.f[0].pr2_q_v)
                k_pr_push<<<L.adv_grid_pr, kThreads, 0, s>>>(c, L.w0, L.nw);
            else if (c.P > 1)
                if (c.mirrors || c.hub_on)
                    k_advance<ALG, true, false, true><<<L.adv_grid, kAdvThreads, 0, s>>>(c, L.w0, L.nw);
                else
                    k_advance<ALG, true><<<L.adv_grid, kAdvThreads, 0, s>>>(c, L.w0, L.nw);
            else
                if (ALG == ALG_BFS && c.pb_shift)
                    k_advance<ALG, false, true><<<L.adv_grid, kAdvThreads, 0, s>>>(c, L.w0, L.nw);
                else
                    k_advance<ALG, false><<<L.adv_grid, kAdvThreads, 0, s>>>(c, L.w0, L.nw);
            break;
        case KER_FINALIZE: k_pr_finalize<<<dim3(L.fin_grid, c.P), kThreads, 0, s>>>(c, L.w0, L.nw); break;
        case KER_TAIL: return launch_tail<ALG>(c, L, s);
        case KER_PULL:
            if (ALG == ALG_BFS && c.bfs_pull) {
                if (c.P > 1) k_bfs_pull<true><<<dim3(L.fin_grid, c.P), kThreads, 0, s>>>(c, L.w0, L.nw);
                else k_bfs_pull<false><<<dim3(L.fin_grid, c.P), kThreads, 0, s>>>(c, L.w0, L.nw);
            }
            break;
        case KER_APPLY:
            if (ALG == ALG_BFS && c.pb_shift)
                k_pb_apply<<<c.pb_nb * kPbParts, kThreads, 2u * (1u << (c.pb_shift - 5)) * 4u, s>>>(c, L.w0);
            break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t launch_kernel(int alg, int kind, const DevCtx& c, const LaunchCfg& L, cudaStream_t s,
                          cudaGraphConditionalHandle h, int use_h) {
    switch (alg) {
        case ALG_BFS: return launch_kernel_t<ALG_BFS>(kind, c, L, s, h, use_h);
        case ALG_SSSP: return launch_kernel_t<ALG_SSSP>(kind, c, L, s, h, use_h);
        case ALG_WCC: return launch_kernel_t<ALG_WCC>(kind, c, L, s, h, use_h);
        case ALG_DPR: return launch_kernel_t<ALG_DPR>(kind, c, L, s, h, use_h);
        default: return launch_kernel_t<ALG_PR>(kind, c, L, s, h, use_h);
    }
}

int phase_kernels(int alg, int phase, int* kinds) {
    if (alg != ALG_PR) {
        if (phase == 0) {
            if (alg == ALG_BFS) {
                kinds[0] = KER_APPLY;  // second half of a propagation-blocked advance
                kinds[1] = KER_FILTER;
                return 2;
            }
            kinds[0] = KER_FILTER;
            return 1;
        }
        kinds[0] = KER_CONTROL;
        kinds[1] = KER_ADVANCE;
        kinds[2] = KER_TAIL;
        if (alg == ALG_BFS) {
            kinds[3] = KER_PULL;
            return 4;
        }
        return 3;
    }
    if (phase == 0) {
        kinds[0] = KER_CONTROL;
        kinds[1] = KER_ADVANCE;
        return 2;
    }
    kinds[0] = KER_FINALIZE;
    return 1;
}

cudaError_t launch_phase(int alg, int phase, const DevCtx& c, const LaunchCfg& L, cudaStream_t s,
                         cudaGraphConditionalHandle h, int use_h) {
    int kinds[4];
    const int n = phase_kernels(alg, phase, kinds);
    for (int i = 0; i < n; i++) {
        if (kinds[i] == KER_TAIL && L.tail_grid <= 0) continue;
        if (kinds[i] == KER_PULL && !c.bfs_pull) continue;
        if (kinds[i] == KER_CONTROL && c.fuse_ctl && alg != ALG_PR) continue;  // run by the filter's last CTA
        cudaError_t e = launch_kernel(alg, kinds[i], c, L, s, h, use_h);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

cudaError_t launch_init(int alg, const DevCtx& c, const LaunchCfg& L, cudaStream_t s, int f0, int nf, double D0,
                        int src_frag, unsigned src_local) {
    dim3 g(L.init_grid, nf);
    switch (alg) {
        case ALG_BFS: k_init<ALG_BFS><<<g, kThreads, 0, s>>>(c, f0); break;
        case ALG_SSSP: k_init<ALG_SSSP><<<g, kThreads, 0, s>>>(c, f0); break;
        case ALG_WCC: k_init<ALG_WCC><<<g, kThreads, 0, s>>>(c, f0); break;
        case ALG_DPR: k_init<ALG_DPR><<<g, kThreads, 0, s>>>(c, f0); break;
        default: k_init<ALG_PR><<<g, kThreads, 0, s>>>(c, f0); break;
    }
    // the initial frontier: {source} as a list (BFS/SSSP) or every vertex as a full bitmap (WCC/PR)
    const unsigned nd0 = c.force_mode == 1 ? 0u : ((alg == ALG_WCC || alg == ALG_PR || alg == ALG_DPR) ? 1u : 0u);
    k_init_run<<<1, 1, 0, s>>>(c, L.w0, D0, nd0, (alg == ALG_WCC && c.f[0].sq_col) ? 1u : 0u);
    if (src_frag >= f0 && src_frag < f0 + nf) k_init_source<<<1, 1, 0, s>>>(c, src_frag, src_local);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------- multi-process barrier (a10)
// One thread per unit t: fence.sc.sys orders this rank's completed phase (the previous kernels on the
// stream, incl. their remote atomics into peer memory) before the release-store of `epoch` into
// peer t's pad slot `me`; then spin with acquire loads until peer t has signalled `epoch` into ours.
// The next phase starts after this kernel, so it observes everything the peers did before signalling.
// A peer that never arrives (dead process) trips a 60 s timeout flag instead of hanging the GPU.
__global__ void k_mp_barrier(const MpPads p, int P, int me, unsigned long long epoch) {
    const int t = threadIdx.x;
    if (t >= P) return;
    asm volatile("fence.sc.sys;" ::: "memory");
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p.pad[t] + me), "l"(epoch) : "memory");
    const unsigned long long t0 = globaltimer();
    for (;;) {
        unsigned long long v;
        asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p.pad[me] + t) : "memory");
        if (v >= epoch) break;
        if (globaltimer() - t0 > 60ull * 1000000000ull) {
            atomicExch(p.pad[me] + kMaxW, 1ull);
            break;
        }
        __nanosleep(200);
    }
}

// Device-resident multi-unit loop: the a10 barrier of one unit's CUDA graph, one thread.
// Members are the units {0..mb-1} of the unit's run control (the same on every member). Arrival =
// fence.sc.sys, then st.release.sys of the next epoch into every other member's pad, then an acquire spin
// on this unit's pad until every member has signalled it. At the phase-A barrier (before the filter) the
// membership decided by the previous control takes effect: a unit that is no longer a member (OSteal
// eviction) leaves after this last barrier and parks here -- it launches nothing and arrives
// at no further barrier -- until unit 0 wakes it (give-back, or end of run) after copying its run
// control into it; it then re-evaluates its membership with that state. 60 s without progress sets the
// timeout flag and ends the run (GUM_ENCCL) instead of hanging.
__global__ void k_unit_bar(const __grid_constant__ DevCtx c, int u, int phase) {
    if (threadIdx.x != 0) return;
    RunCtl* rc = c.rctl[u];
    unsigned long long* me = c.pad[u];
    unsigned long long t0 = globaltimer();
    for (;;) {
        if (vload(&rc->done)) return;
        const unsigned mb = vload(&rc->mb);
        unsigned nm = mb, target = 0;
        if (phase == 0) {
            nm = vload(&rc->mb_next);
            target = vload(&rc->wakes[u]) + 1u;  // read before arriving: unit 0 may wake us right after
        }
        // this barrier: the old members (leavers included, so their last writes precede any wake-up) and
        // the joiners woken by the previous control
        const unsigned mem = nm > mb ? nm : mb;
        if ((unsigned)u < mem) {
            const unsigned long long ep = rc->bar_ep + 1;
            rc->bar_ep = ep;
            if (nm != mb) rc->mb = nm;  // later barriers use the new member set
            me[kPadArr] = me[kPadArr] + 1;
            me[kPadLastIt] = rc->iter;
            asm volatile("fence.sc.sys;" ::: "memory");
            for (unsigned t = 0; t < mem; t++)
                if (t != (unsigned)u)
                    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(c.pad[t] + kPadGraph + u), "l"(ep) : "memory");
            for (unsigned t = 0; t < mem; t++) {
                if (t == (unsigned)u) continue;
                for (;;) {
                    unsigned long long v;
                    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(me + kPadGraph + t) : "memory");
                    if (v >= ep) break;
                    if (globaltimer() - t0 > 60ull * 1000000000ull) {
                        atomicExch(me + kPadTimeout, 1ull);
                        rc->err = 2;
                        rc->done = 1;
                        return;
                    }
                    __nanosleep(64);
                }
            }
            if ((unsigned)u < nm) return;
        }
        // parked: wait for unit 0's wake (it wrote our run control first), then re-evaluate
        t0 = globaltimer();
        for (;;) {
            unsigned long long v;
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(me + kPadWake) : "memory");
            if (v >= target) break;
            if (globaltimer() - t0 > 600ull * 1000000000ull) {  // parked units may wait a whole long tail
                atomicExch(me + kPadTimeout, 1ull);
                rc->err = 2;
                rc->done = 1;
                return;
            }
            __nanosleep(256);
        }
        t0 = globaltimer();
    }
}

cudaError_t launch_unit_bar(const DevCtx& c, int u, int phase, cudaStream_t s) {
    k_unit_bar<<<1, 32, 0, s>>>(c, u, phase);
    return cudaGetLastError();
}

cudaError_t launch_mp_barrier(const MpPads& p, int P, int me, unsigned long long epoch, cudaStream_t s) {
    k_mp_barrier<<<1, 32, 0, s>>>(p, P, me, epoch);
    return cudaGetLastError();
}

cudaError_t launch_gather(const DevCtx& c, int f, void* out, int is_pr, cudaStream_t s, int grid) {
    if (is_pr)
        k_gather<double><<<grid, kThreads, 0, s>>>(c, f, (double*)out, 1);
    else
        k_gather<unsigned><<<grid, kThreads, 0, s>>>(c, f, (unsigned*)out, 0);
    return cudaGetLastError();
}

// Shared-memory carveout of the advance: by default the smallest split that still holds the register-bound
// 4 CTAs per SM, so the rest of the unified 256 KB stays L1 for the random visited-bit / state probes (the
// driver's default split left less: C2 advance 1.14 -> 1.10 ms at 35%; a 100% carveout doubles it).
// GUM_SMEM_CARVEOUT (percent) overrides for tuning.
static int g_carveout = -1;
template <typename K>
static void set_carveout(K kern) {
    int pct = g_carveout;
    if (pct < 0) {
        cudaFuncAttributes a;
        if (cudaFuncGetAttributes(&a, kern) != cudaSuccess) {
            cudaGetLastError();
            return;
        }
        const double need = 4.0 * ((double)a.sharedSizeBytes + 1024.0);  // 4 CTAs + 1 KB reserved each
        pct = (int)(need / (228.0 * 1024.0) * 100.0) + 2;
        pct = pct > 100 ? 100 : pct;
    }
    cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
    cudaGetLastError();
}
template <int ALG, bool MULTI>
static void carveout() {
    set_carveout(k_advance<ALG, MULTI>);
    if (MULTI) set_carveout(k_advance<ALG, true, false, true>);
    if (ALG == ALG_BFS && !MULTI) set_carveout(k_advance<ALG_BFS, false, true>);
}

template <int ALG, bool MULTI>
static cudaError_t occ_of(int* n) {
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(n, k_advance<ALG, MULTI>, kAdvThreads, 0);
}

cudaError_t advance_occupancy(int alg, int multi, int* blocks_per_sm) {
    static bool once = false;
    if (!once) {
        once = true;
        if (const char* e = getenv("GUM_SMEM_CARVEOUT")) g_carveout = atoi(e);
        carveout<ALG_BFS, false>();
        carveout<ALG_BFS, true>();
        carveout<ALG_SSSP, false>();
        carveout<ALG_SSSP, true>();
        carveout<ALG_WCC, false>();
        carveout<ALG_WCC, true>();
        carveout<ALG_PR, false>();
        carveout<ALG_PR, true>();
        carveout<ALG_DPR, false>();
        carveout<ALG_DPR, true>();
    }
    switch (alg * 2 + (multi ? 1 : 0)) {
        case 0: return occ_of<ALG_BFS, false>(blocks_per_sm);
        case 1: return occ_of<ALG_BFS, true>(blocks_per_sm);
        case 2: return occ_of<ALG_SSSP, false>(blocks_per_sm);
        case 3: return occ_of<ALG_SSSP, true>(blocks_per_sm);
        case 4: return occ_of<ALG_WCC, false>(blocks_per_sm);
        case 5: return occ_of<ALG_WCC, true>(blocks_per_sm);
        case 6: return occ_of<ALG_PR, false>(blocks_per_sm);
        case 7: return occ_of<ALG_PR, true>(blocks_per_sm);
        case 8: return occ_of<ALG_DPR, false>(blocks_per_sm);
        default: return occ_of<ALG_DPR, true>(blocks_per_sm);
    }
}

}  // namespace gum
