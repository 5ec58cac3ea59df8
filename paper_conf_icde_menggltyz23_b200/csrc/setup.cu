// Setup kernels (untimed): CSR validation, seg bounds, RANDOM relabel, WCC symmetrisation.
// SURVEY.md §8(a) rows a1/a2; PAPER.md P:55-57 (edge-cut partition), P:315/P:382 (seg, random).
#include <cub/cub.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <vector>

#include "kernels.h"

namespace gum {

__host__ __device__ __forceinline__ unsigned long long mix64(unsigned long long z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// Keyed balanced Feistel network on 2h >= ceil(log2 V) bits, cycle-walked into [0, V): a bijection
// of [0, V) (reading #17 "random partitioner = keyed Feistel relabel, then seg").
__host__ __device__ __forceinline__ unsigned feistel(unsigned v, unsigned V, unsigned long long seed) {
    if (V <= 2) return v;
    int bits = 0;
    while ((1ull << bits) < (unsigned long long)V) bits++;
    const int h = (bits + 1) / 2;
    const unsigned long long mask = (1ull << h) - 1;
    const unsigned long long key = mix64(seed ^ 0x5851F42D4C957F2Dull);
    unsigned long long x = v;
    do {
        unsigned long long L = x >> h, R = x & mask;
#pragma unroll
        for (int r = 0; r < 4; r++) {
            unsigned long long nl = R;
            unsigned long long nr = (L ^ mix64(R ^ key ^ ((unsigned long long)r << 56))) & mask;
            L = nl;
            R = nr;
        }
        x = (L << h) | R;
    } while (x >= V);
    return (unsigned)x;
}

unsigned host_feistel(unsigned v, unsigned V, unsigned long long seed) { return feistel(v, V, seed); }

__global__ void k_validate(const unsigned long long* rp, const unsigned* col, unsigned V, unsigned long long E,
                           unsigned* err) {
    const unsigned long long tid = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    if (tid == 0) {
        if (rp[0] != 0) atomicOr(err, 1u);
        if (rp[V] != E) atomicOr(err, 2u);
    }
    for (unsigned long long i = tid; i < V; i += stride)
        if (rp[i] > rp[i + 1]) atomicOr(err, 4u);
    for (unsigned long long e = tid; e < E; e += stride)
        if (col[e] >= V) atomicOr(err, 8u);
}

cudaError_t setup_validate(const unsigned long long* row_ptr, const unsigned* col, unsigned V, unsigned long long E,
                           unsigned* d_err, cudaStream_t s) {
    k_validate<<<1184, 256, 0, s>>>(row_ptr, col, V, E, d_err);
    return cudaGetLastError();
}

__global__ void k_seg_bounds(const unsigned long long* rp, unsigned V, unsigned long long E, int P, unsigned* b) {
    const int g = threadIdx.x;
    if (g > P) return;
    if (g == 0) {
        b[0] = 0;
        return;
    }
    if (g == P) {
        b[P] = V;
        return;
    }
    const unsigned long long target = (E * (unsigned long long)g) / (unsigned long long)P;
    unsigned lo = 0, hi = V;  // first v in [0, V] with rp[v] >= target
    while (lo < hi) {
        unsigned mid = lo + (hi - lo) / 2;
        if (rp[mid] >= target)
            hi = mid;
        else
            lo = mid + 1;
    }
    b[g] = lo;
}

cudaError_t setup_seg_bounds(const unsigned long long* row_ptr, unsigned V, unsigned long long E, int P,
                             unsigned* d_bounds, cudaStream_t s) {
    k_seg_bounds<<<1, 32, 0, s>>>(row_ptr, V, E, P, d_bounds);
    return cudaGetLastError();
}

size_t setup_scan_tmp_bytes(unsigned V) {
    size_t bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, bytes, (unsigned long long*)nullptr, (unsigned long long*)nullptr,
                                  (int)0 + (size_t)V + 1);
    return bytes + 256;
}
size_t setup_relabel_tmp_bytes(unsigned V) {
    return (setup_scan_tmp_bytes(V) + 255) / 256 * 256 + ((size_t)V * 4 + 255) / 256 * 256 + 256;
}

// relabelled rows -> new col/w: short rows by threads, medium rows by warps, hub rows by CTAs
static cudaError_t relabel_move(const unsigned long long* row_ptr, const unsigned* col, const unsigned* w,
                                const unsigned* d_inv, unsigned V, unsigned long long seed, const unsigned* perm,
                                const unsigned long long* r_row_ptr, unsigned* r_col, unsigned* r_w, unsigned* list,
                                unsigned* cnt, cudaStream_t s);

__global__ void k_inv_perm(unsigned V, unsigned long long seed, unsigned* inv) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x)
        inv[feistel(v, V, seed)] = v;
}

__global__ void k_new_deg(const unsigned long long* rp, const unsigned* inv, unsigned V, unsigned long long* out) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v <= V; v += gridDim.x * blockDim.x) {
        if (v == V) {
            out[V] = 0;
        } else {
            unsigned o = inv[v];
            out[v] = rp[o + 1] - rp[o];
        }
    }
}

// rows of <= kShortRow entries: one thread per row (a warp per row would leave most lanes idle and
// serialise the row's dependent loads); longer rows: one warp per row
constexpr unsigned long long kShortRow = 32;
__global__ void k_relabel_short(const unsigned long long* rp, const unsigned* col, const unsigned* w, const unsigned* inv,
                                unsigned V, unsigned long long seed, const unsigned* perm, const unsigned long long* nrp,
                                unsigned* ncol, unsigned* nw) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x) {
        const unsigned long long d0 = nrp[v], n = nrp[v + 1] - d0;
        if (n == 0 || n > kShortRow) continue;
        const unsigned long long s0 = rp[inv[v]];
        for (unsigned long long j = 0; j < n; j++) {
            const unsigned x = col[s0 + j];
            ncol[d0 + j] = perm ? perm[x] : feistel(x, V, seed);
            if (w) nw[d0 + j] = w[s0 + j];
        }
    }
}

constexpr unsigned long long kHugeRow = 4096;  // rows longer than this: one CTA per row (k_relabel_huge)
__global__ void k_relabel_rows(const unsigned long long* rp, const unsigned* col, const unsigned* w, const unsigned* inv,
                               unsigned V, unsigned long long seed, const unsigned* perm, const unsigned long long* nrp,
                               unsigned* ncol, unsigned* nw) {
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long warp = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
    const unsigned long long nwarps = ((unsigned long long)gridDim.x * blockDim.x) >> 5;
    for (unsigned long long v = warp; v < V; v += nwarps) {
        const unsigned long long d0 = nrp[v], n = nrp[v + 1] - d0;
        if (n <= kShortRow || n > kHugeRow) continue;  // k_relabel_short / k_relabel_huge move those
        const unsigned long long s0 = rp[inv[v]];
        for (unsigned long long j = lane; j < n; j += 32) {
            ncol[d0 + j] = perm ? perm[col[s0 + j]] : feistel(col[s0 + j], V, seed);
            if (w) nw[d0 + j] = w[s0 + j];
        }
    }
}

// hub rows (the highest-degree rows hold up to ~0.15% of all edges each on RMAT): collected into a list
// first, then one CTA per listed row (CTAs take list entries round-robin, so the degree-ordered layout's
// hub rows -- all in the first ids -- do not land on one CTA)
__global__ void k_huge_list(const unsigned long long* nrp, unsigned V, unsigned* list, unsigned* cnt) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x)
        if (nrp[v + 1] - nrp[v] > kHugeRow) list[atomicAdd(cnt, 1u)] = v;
}
__global__ void k_relabel_huge(const unsigned long long* rp, const unsigned* col, const unsigned* w, const unsigned* inv,
                               unsigned V, unsigned long long seed, const unsigned* perm, const unsigned long long* nrp,
                               unsigned* ncol, unsigned* nw, const unsigned* list, const unsigned* cnt) {
    const unsigned n = *cnt;
    for (unsigned r = blockIdx.x; r < n; r += gridDim.x) {
        const unsigned hv = list[r];
        const unsigned long long d0 = nrp[hv], m = nrp[hv + 1] - d0, s0 = rp[inv[hv]];
        for (unsigned long long j = threadIdx.x; j < m; j += blockDim.x) {
            ncol[d0 + j] = perm ? perm[col[s0 + j]] : feistel(col[s0 + j], V, seed);
            if (w) nw[d0 + j] = w[s0 + j];
        }
    }
}

cudaError_t setup_relabel(const unsigned long long* row_ptr, const unsigned* col, const unsigned* w, unsigned V,
                          unsigned long long E, unsigned long long seed, unsigned* d_inv, unsigned long long* r_row_ptr,
                          unsigned* r_col, unsigned* r_w, void* tmp, size_t tmp_bytes, cudaStream_t s) {
    (void)E;
    k_inv_perm<<<1184, 256, 0, s>>>(V, seed, d_inv);
    k_new_deg<<<1184, 256, 0, s>>>(row_ptr, d_inv, V, r_row_ptr);
    cudaError_t e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, r_row_ptr, r_row_ptr, (size_t)V + 1, s);
    if (e != cudaSuccess) return e;
    unsigned* list = (unsigned*)((char*)tmp + (setup_scan_tmp_bytes(V) + 255) / 256 * 256);
    unsigned* cnt = list + ((size_t)V * 4 + 255) / 256 * 64;
    return relabel_move(row_ptr, col, w, d_inv, V, seed, nullptr, r_row_ptr, r_col, r_w, list, cnt, s);
}

// DEGREE relabel (layout option): new ids in order of decreasing in-degree (ties by id), so the
// destinations most edges point to share a few KB of the visited bitmap / state array and stay cache-resident.
__global__ void k_indeg(const unsigned* col, unsigned long long E, unsigned* deg) {
    for (unsigned long long e = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; e < E;
         e += (unsigned long long)gridDim.x * blockDim.x)
        atomicAdd(deg + col[e], 1u);
}
__global__ void k_deg_keys(unsigned* deg, unsigned V, unsigned* ids) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x) {
        deg[v] = ~deg[v];  // ascending radix order of ~deg = decreasing degree
        ids[v] = v;
    }
}
__global__ void k_perm_of(const unsigned* inv, unsigned V, unsigned* perm) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x) perm[inv[v]] = v;
}

size_t setup_degree_tmp_bytes(unsigned V) {
    size_t a = 0, b = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, a, (unsigned*)nullptr, (unsigned*)nullptr, (unsigned*)nullptr,
                                    (unsigned*)nullptr, (int)0 + (size_t)V);
    cub::DeviceScan::ExclusiveSum(nullptr, b, (unsigned long long*)nullptr, (unsigned long long*)nullptr,
                                  (int)0 + (size_t)V + 1);
    return (a > b ? a : b) + 2 * ((size_t)V * 4 + 256) + 256;
}

cudaError_t setup_relabel_degree(const unsigned long long* row_ptr, const unsigned* col, const unsigned* w,
                                 unsigned V, unsigned long long E, unsigned* d_perm, unsigned* d_inv,
                                 unsigned long long* r_row_ptr, unsigned* r_col, unsigned* r_w, void* tmp,
                                 size_t tmp_bytes, cudaStream_t s) {
    const size_t vb = ((size_t)V * 4 + 255) & ~(size_t)255;
    unsigned* keys_in = (unsigned*)tmp;
    unsigned* keys_out = (unsigned*)((char*)tmp + vb);
    void* t = (char*)tmp + 2 * vb;
    size_t tb = tmp_bytes - 2 * vb;
    cudaError_t e = cudaMemsetAsync(keys_in, 0, (size_t)V * 4, s);
    if (e != cudaSuccess) return e;
    k_indeg<<<1184, 256, 0, s>>>(col, E, keys_in);
    k_deg_keys<<<1184, 256, 0, s>>>(keys_in, V, d_perm);  // d_perm holds the identity as sort input
    e = cub::DeviceRadixSort::SortPairs(t, tb, keys_in, keys_out, d_perm, d_inv, (size_t)V, 0, 32, s);
    if (e != cudaSuccess) return e;
    k_perm_of<<<1184, 256, 0, s>>>(d_inv, V, d_perm);
    k_new_deg<<<1184, 256, 0, s>>>(row_ptr, d_inv, V, r_row_ptr);
    e = cub::DeviceScan::ExclusiveSum(t, tb, r_row_ptr, r_row_ptr, (size_t)V + 1, s);
    if (e != cudaSuccess) return e;
    // (both key buffers are free after the sort: the hub-row list and its counter go there)
    return relabel_move(row_ptr, col, w, d_inv, V, 0, d_perm, r_row_ptr, r_col, r_w, keys_out, keys_in, s);
}

__global__ void k_sym_deg(const unsigned long long* rp, const unsigned* col, unsigned V, unsigned long long E,
                          unsigned long long* srp) {
    const unsigned long long tid = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long e = tid; e < E; e += stride) atomicAdd(srp + col[e], 1ull);
}

__global__ void k_out_deg_init(const unsigned long long* rp, unsigned V, unsigned long long* srp) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v <= V; v += gridDim.x * blockDim.x)
        srp[v] = (v == V) ? 0 : rp[v + 1] - rp[v];
}

__global__ void k_sym_fill(const unsigned long long* rp, const unsigned* col, unsigned V,
                           const unsigned long long* srp, unsigned* scol, unsigned long long* cursor) {
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long warp = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
    const unsigned long long nwarps = ((unsigned long long)gridDim.x * blockDim.x) >> 5;
    for (unsigned long long u = warp; u < V; u += nwarps) {
        const unsigned long long s0 = rp[u], s1 = rp[u + 1], d0 = srp[u];
        for (unsigned long long j = lane; j < s1 - s0; j += 32) {
            const unsigned v = col[s0 + j];
            scol[d0 + j] = v;                                  // out-neighbour
            scol[atomicAdd(cursor + v, 1ull)] = (unsigned)u;   // u is an in-neighbour of v
        }
    }
}

__global__ void k_cursor_init(const unsigned long long* rp, const unsigned long long* srp, unsigned V,
                              unsigned long long* cursor) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x)
        cursor[v] = srp[v] + (rp[v + 1] - rp[v]);
}

cudaError_t setup_symmetrize(const unsigned long long* row_ptr, const unsigned* col, unsigned V, unsigned long long E,
                             unsigned long long* s_row_ptr, unsigned* s_col, unsigned long long* cursor, void* tmp,
                             size_t tmp_bytes, cudaStream_t s) {
    k_out_deg_init<<<1184, 256, 0, s>>>(row_ptr, V, s_row_ptr);
    k_sym_deg<<<1184, 256, 0, s>>>(row_ptr, col, V, E, s_row_ptr);
    cudaError_t e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, s_row_ptr, s_row_ptr, (size_t)V + 1, s);
    if (e != cudaSuccess) return e;
    k_cursor_init<<<1184, 256, 0, s>>>(row_ptr, s_row_ptr, V, cursor);
    k_sym_fill<<<1184, 256, 0, s>>>(row_ptr, col, V, s_row_ptr, s_col, cursor);
    return cudaGetLastError();
}

// in-CSR (transpose) for bottom-up BFS: in-row of v = sources of its in-edges (any order)
__global__ void k_tr_deg(const unsigned* col, unsigned long long E, unsigned long long* trp) {
    for (unsigned long long e = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; e < E;
         e += (unsigned long long)gridDim.x * blockDim.x)
        atomicAdd(trp + col[e], 1ull);
}

__global__ void k_tr_fill(const unsigned long long* rp, const unsigned* col, unsigned V, unsigned* tcol,
                          unsigned long long* cursor) {
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long warp = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
    const unsigned long long nwarps = ((unsigned long long)gridDim.x * blockDim.x) >> 5;
    for (unsigned long long u = warp; u < V; u += nwarps)
        for (unsigned long long e = rp[u] + lane; e < rp[u + 1]; e += 32)
            tcol[atomicAdd(cursor + col[e], 1ull)] = (unsigned)u;
}

cudaError_t setup_transpose(const unsigned long long* row_ptr, const unsigned* col, unsigned V, unsigned long long E,
                            unsigned long long* t_row_ptr, unsigned* t_col, unsigned long long* cursor, void* tmp,
                            size_t tmp_bytes, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(t_row_ptr, 0, ((size_t)V + 1) * 8, s);
    if (e != cudaSuccess) return e;
    k_tr_deg<<<1184, 256, 0, s>>>(col, E, t_row_ptr);
    e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, t_row_ptr, t_row_ptr, (size_t)V + 1, s);
    if (e != cudaSuccess) return e;
    e = cudaMemcpyAsync(cursor, t_row_ptr, ((size_t)V + 1) * 8, cudaMemcpyDeviceToDevice, s);
    if (e != cudaSuccess) return e;
    k_tr_fill<<<1184, 256, 0, s>>>(row_ptr, col, V, t_col, cursor);
    return cudaGetLastError();
}

__global__ void k_rebase(const unsigned long long* rp, unsigned b0, unsigned b1, unsigned long long* out) {
    const unsigned long long base = rp[b0];
    for (unsigned i = blockIdx.x * blockDim.x + threadIdx.x; i <= b1 - b0; i += gridDim.x * blockDim.x)
        out[i] = rp[b0 + i] - base;
}

cudaError_t setup_rebase_rows(const unsigned long long* row_ptr, unsigned b0, unsigned b1, unsigned long long* out,
                              cudaStream_t s) {
    k_rebase<<<592, 256, 0, s>>>(row_ptr, b0, b1, out);
    return cudaGetLastError();
}

// ---- PR destination-blocked static queue (gum_prepare(PR)) ---------------------------------------
// Destination ids are split into blocks of S ids (an acc block of 8*S bytes sized to stay L2-resident);
// edges are regrouped block-major (rows ascending inside a block, edge order kept inside a row) and the
// static PR frontier becomes the queue of (block, row) pairs with edges, in that order. Consecutive
// chunks then push into one block of acc at a time.
__global__ void k_pr_count(const unsigned long long* rp, const unsigned* col, unsigned Vf, unsigned S, int B,
                           unsigned long long* cnt /* [B*Vf + 1] */) {
    extern __shared__ unsigned s_hist[];  // B counters per warp
    const unsigned lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    unsigned* h = s_hist + wib * B;
    const unsigned long long warp = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
    const unsigned long long nwarps = ((unsigned long long)gridDim.x * blockDim.x) >> 5;
    for (unsigned long long u = warp; u < Vf; u += nwarps) {
        for (int b = lane; b < B; b += 32) h[b] = 0;
        __syncwarp();
        for (unsigned long long e = rp[u] + lane; e < rp[u + 1]; e += 32) atomicAdd(h + col[e] / S, 1u);
        __syncwarp();
        for (int b = lane; b < B; b += 32) cnt[(unsigned long long)b * Vf + u] = h[b];
        __syncwarp();
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) cnt[(unsigned long long)B * Vf] = 0;
}

__global__ void k_pr_scatter(const unsigned long long* rp, const unsigned* col, unsigned Vf, unsigned S, int B,
                             const unsigned long long* off, unsigned* pcol) {
    extern __shared__ unsigned long long s_cur[];  // B cursors per warp
    const unsigned lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    unsigned long long* cur = s_cur + wib * B;
    const unsigned long long warp = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5;
    const unsigned long long nwarps = ((unsigned long long)gridDim.x * blockDim.x) >> 5;
    for (unsigned long long u = warp; u < Vf; u += nwarps) {
        for (int b = lane; b < B; b += 32) cur[b] = off[(unsigned long long)b * Vf + u];
        __syncwarp();
        const unsigned long long e0 = rp[u], e1 = rp[u + 1];
        for (unsigned long long eb = e0; eb < e1; eb += 32) {
            const unsigned long long e = eb + lane;
            const bool ok = e < e1;
            const unsigned v = ok ? col[e] : 0u;
            const unsigned b = ok ? v / S : 0xFFFFFFFFu;
            const unsigned grp = __match_any_sync(0xffffffffu, b);
            const unsigned leader = __ffs(grp) - 1;
            unsigned long long base = 0;
            if (ok) base = cur[b];  // stable: ranks follow the row's edge order
            if (ok) pcol[base + __popc(grp & ((1u << lane) - 1u))] = v;
            __syncwarp();
            if (ok && lane == leader) cur[b] = base + __popc(grp);
            __syncwarp();
        }
    }
}

__global__ void k_pr_flags(const unsigned long long* off, unsigned long long n, unsigned* flag) {
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i <= n;
         i += (unsigned long long)gridDim.x * blockDim.x)
        flag[i] = (i < n && off[i + 1] > off[i]) ? 1u : 0u;
}

__global__ void k_pr_emit(const unsigned long long* off, const unsigned* pos, unsigned long long n, unsigned Vf,
                          unsigned chunk, unsigned* q_v, unsigned long long* q_off, unsigned* tile) {
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
         i += (unsigned long long)gridDim.x * blockDim.x) {
        const unsigned long long o = off[i], d = off[i + 1] - o;
        if (!d) continue;
        const unsigned p = pos[i];
        q_v[p] = (unsigned)(i % Vf);
        q_off[p] = o;
        for (unsigned long long t = (o + chunk - 1) / chunk; t * chunk < o + d; t++) tile[t] = p;
    }
}

size_t setup_pr_tmp_bytes(unsigned Vf, int B) {
    const unsigned long long n = (unsigned long long)B * Vf + 1;
    size_t a = 0, b = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, a, (unsigned long long*)nullptr, (unsigned long long*)nullptr, (size_t)n);
    cub::DeviceScan::ExclusiveSum(nullptr, b, (unsigned*)nullptr, (unsigned*)nullptr, (size_t)n);
    return std::max(a, b) + 256 + n * 8 + n * 4 * 2 + 1024;
}

cudaError_t setup_pr_blocked(const unsigned long long* rp, const unsigned* col, unsigned Vf, unsigned long long Ef,
                             unsigned S, int B, unsigned chunk, unsigned* pcol, unsigned* q_v, unsigned long long* q_off,
                             unsigned* tile, unsigned long long* h_Q, void* tmp, size_t tmp_bytes, cudaStream_t s) {
    const unsigned long long n = (unsigned long long)B * Vf;
    char* t = (char*)tmp;
    unsigned long long* off = (unsigned long long*)t;
    t += ((n + 1) * 8 + 255) / 256 * 256;
    unsigned* flag = (unsigned*)t;
    t += ((n + 1) * 4 + 255) / 256 * 256;
    unsigned* pos = (unsigned*)t;
    t += ((n + 1) * 4 + 255) / 256 * 256;
    void* cub_tmp = t;
    size_t cub_bytes = tmp_bytes - (size_t)(t - (char*)tmp);
    const int warps_per_cta = 8;
    k_pr_count<<<1184, 32 * warps_per_cta, warps_per_cta * B * sizeof(unsigned), s>>>(rp, col, Vf, S, B, off);
    cudaError_t e = cub::DeviceScan::ExclusiveSum(cub_tmp, cub_bytes, off, off, (size_t)n + 1, s);
    if (e != cudaSuccess) return e;
    if (pcol) {
        k_pr_scatter<<<1184, 32 * warps_per_cta, warps_per_cta * B * sizeof(unsigned long long), s>>>(rp, col, Vf, S, B,
                                                                                                      off, pcol);
    }
    k_pr_flags<<<1184, 256, 0, s>>>(off, n, flag);
    e = cub::DeviceScan::ExclusiveSum(cub_tmp, cub_bytes, flag, pos, (size_t)n + 1, s);
    if (e != cudaSuccess) return e;
    k_pr_emit<<<1184, 256, 0, s>>>(off, pos, n, Vf, chunk, q_v, q_off, tile);
    unsigned Q = 0;
    e = cudaMemcpyAsync(&Q, pos + n, 4, cudaMemcpyDeviceToHost, s);
    if (e != cudaSuccess) return e;
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return e;
    *h_Q = Q;
    e = cudaMemcpyAsync(q_off + Q, &Ef, 8, cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) return e;
    e = cudaStreamSynchronize(s);  // Ef is a by-value host local
    (void)e;
    return cudaGetLastError();
}

// ---- PR pull (gum_prepare(PR)): the fragment's in-edges regrouped source-block-major ---------------
// Same counting as the destination-blocked push queue (k_pr_count / k_pr_scatter), applied to the
// fragment's in-CSR: block b holds the in-edges whose SOURCE is in [b*S, (b+1)*S), rows ascending, so a
// pull pass over block b gathers x/outdeg from one L2-sized slice. Offsets narrowed to u32 (the caller
// checks Ein < 2^32); merge-path tile starts precomputed per pass (one binary search per tile, untimed).
__global__ void k_pl_narrow(const unsigned long long* off, unsigned long long n, unsigned* out) {
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i <= n;
         i += (unsigned long long)gridDim.x * blockDim.x)
        out[i] = (unsigned)off[i];
}

// tile t of a pass starts at merge-path diagonal t*tile over (row ends, edges): the first row whose end
// has not been consumed (Merrill & Garland's MergePathSearch)
__global__ void k_pl_tiles(const unsigned* off /* pass rows: [Vf+1] */, unsigned Vf, unsigned long long tile,
                           unsigned long long ntiles, unsigned* tx) {
    const unsigned long long base = off[0], nE = off[Vf] - base, items = (unsigned long long)Vf + nE;
    for (unsigned long long t = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; t <= ntiles;
         t += (unsigned long long)gridDim.x * blockDim.x) {
        const unsigned long long d = t * tile < items ? t * tile : items;
        unsigned long long lo = d > nE ? d - nE : 0, hi = d < Vf ? d : Vf;
        while (lo < hi) {
            const unsigned long long pivot = (lo + hi) >> 1;
            if ((unsigned long long)(off[pivot + 1] - base) <= d - pivot - 1) lo = pivot + 1;
            else hi = pivot;
        }
        tx[t] = (unsigned)lo;
    }
}

cudaError_t setup_pr_pull(const unsigned long long* in_rp, const unsigned* in_col, unsigned Vf, unsigned long long Ein,
                          unsigned S, int B, unsigned tile, unsigned* pl_off, unsigned* pl_col, unsigned* pl_tx,
                          unsigned long long* h_tb, void* tmp, size_t tmp_bytes, cudaStream_t s) {
    (void)Ein;
    const unsigned long long n = (unsigned long long)B * Vf;
    char* t = (char*)tmp;
    unsigned long long* off = (unsigned long long*)t;
    t += ((n + 1) * 8 + 255) / 256 * 256;
    void* cub_tmp = t;
    size_t cub_bytes = tmp_bytes - (size_t)(t - (char*)tmp);
    const int warps_per_cta = 8;
    k_pr_count<<<1184, 32 * warps_per_cta, warps_per_cta * B * sizeof(unsigned), s>>>(in_rp, in_col, Vf, S, B, off);
    cudaError_t e = cub::DeviceScan::ExclusiveSum(cub_tmp, cub_bytes, off, off, (size_t)n + 1, s);
    if (e != cudaSuccess) return e;
    std::vector<unsigned long long> hb(B + 1);
    for (int b = 0; b <= B; b++) {
        e = cudaMemcpyAsync(&hb[b], off + (unsigned long long)b * Vf, 8, cudaMemcpyDeviceToHost, s);
        if (e != cudaSuccess) return e;
    }
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return e;
    unsigned long long acc = 0;
    for (int b = 0; b < B; b++) {
        const unsigned long long items = (unsigned long long)Vf + (hb[b + 1] - hb[b]);
        h_tb[b] = acc;
        acc += (items + tile - 1) / tile + 1;
    }
    h_tb[B] = acc;
    if (!pl_off || !pl_col || !pl_tx) return cudaGetLastError();
    k_pr_scatter<<<1184, 32 * warps_per_cta, warps_per_cta * B * sizeof(unsigned long long), s>>>(in_rp, in_col, Vf, S,
                                                                                                  B, off, pl_col);
    k_pl_narrow<<<1184, 256, 0, s>>>(off, n, pl_off);
    for (int b = 0; b < B; b++) {
        const unsigned long long nt = h_tb[b + 1] - h_tb[b] - 1;
        k_pl_tiles<<<(unsigned)std::min<unsigned long long>((nt + 256) / 256, 4096), 256, 0, s>>>(
            pl_off + (unsigned long long)b * Vf, Vf, tile, nt, pl_tx + h_tb[b]);
    }
    return cudaGetLastError();
}

// ---- BFS propagation blocking: per destination block capacity = in-degree of the block ---------
__global__ void k_pb_hist(const unsigned* col, unsigned long long E, unsigned shift, unsigned long long* cnt) {
    extern __shared__ unsigned s_h[];
    const unsigned nb = blockDim.x * 4;  // caller sizes the block so that 4 * blockDim >= nb
    for (unsigned b = threadIdx.x; b < nb; b += blockDim.x) s_h[b] = 0;
    __syncthreads();
    for (unsigned long long e = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; e < E;
         e += (unsigned long long)gridDim.x * blockDim.x)
        atomicAdd(s_h + (col[e] >> shift), 1u);
    __syncthreads();
    for (unsigned b = threadIdx.x; b < nb; b += blockDim.x)
        if (s_h[b]) atomicAdd(cnt + b, (unsigned long long)s_h[b]);
}

size_t setup_pb_tmp_bytes(unsigned nb) {
    size_t bytes = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, bytes, (unsigned long long*)nullptr, (unsigned long long*)nullptr,
                                  (size_t)nb + 1);
    return bytes + 256;
}

static cudaError_t relabel_move(const unsigned long long* row_ptr, const unsigned* col, const unsigned* w,
                                const unsigned* d_inv, unsigned V, unsigned long long seed, const unsigned* perm,
                                const unsigned long long* r_row_ptr, unsigned* r_col, unsigned* r_w, unsigned* list,
                                unsigned* cnt, cudaStream_t s) {
    k_relabel_short<<<4736, 256, 0, s>>>(row_ptr, col, w, d_inv, V, seed, perm, r_row_ptr, r_col, r_w);
    k_relabel_rows<<<1184, 256, 0, s>>>(row_ptr, col, w, d_inv, V, seed, perm, r_row_ptr, r_col, r_w);
    cudaError_t e = cudaMemsetAsync(cnt, 0, 4, s);
    if (e != cudaSuccess) return e;
    k_huge_list<<<1184, 256, 0, s>>>(r_row_ptr, V, list, cnt);
    k_relabel_huge<<<1184, 256, 0, s>>>(row_ptr, col, w, d_inv, V, seed, perm, r_row_ptr, r_col, r_w, list, cnt);
    return cudaGetLastError();
}

cudaError_t setup_pb_offsets(const unsigned* col, unsigned long long E, unsigned shift, unsigned nb,
                             unsigned long long* pb_off, void* tmp, size_t tmp_bytes, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(pb_off, 0, ((size_t)nb + 1) * 8, s);
    if (e != cudaSuccess) return e;
    k_pb_hist<<<1184, 256, 1024 * sizeof(unsigned), s>>>(col, E, shift, pb_off);
    e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, pb_off, pb_off, (size_t)nb + 1, s);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

__global__ void k_count_dangling(const unsigned long long* rp, unsigned V, unsigned long long* cnt) {
    unsigned long long c = 0;
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x)
        c += (rp[v + 1] == rp[v]) ? 1 : 0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(cnt, c);
}

cudaError_t setup_count_dangling(const unsigned long long* row_ptr, unsigned V, unsigned long long* d_count,
                                 cudaStream_t s) {
    k_count_dangling<<<592, 256, 0, s>>>(row_ptr, V, d_count);
    return cudaGetLastError();
}

// NEXT-1 hub cache (P:274 Example 6): the adjacency lists of global rows [b0, b0+n) with out-degree > t4,
// packed into a worker-local copy. off[v] = position of row b0+v in the copy, ~0 if not cached.
__global__ void k_hub_deg(const unsigned long long* rp, unsigned b0, unsigned n, unsigned t4,
                          unsigned long long* off) {
    for (unsigned v = blockIdx.x * blockDim.x + threadIdx.x; v <= n; v += gridDim.x * blockDim.x) {
        unsigned long long d = 0;
        if (v < n) {
            d = rp[b0 + v + 1] - rp[b0 + v];
            if (d <= t4) d = 0;
        }
        off[v] = d;
    }
}

// one warp per row: copy a cached list, or mark the row as not cached
__global__ void k_hub_fill(const unsigned long long* rp, const unsigned* col, const unsigned* w, unsigned b0,
                           unsigned n, unsigned t4, unsigned long long* off, unsigned* hcol, unsigned* hw) {
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long nwarps = (unsigned long long)gridDim.x * (blockDim.x / 32);
    for (unsigned long long v = blockIdx.x * (unsigned long long)(blockDim.x / 32) + threadIdx.x / 32; v < n;
         v += nwarps) {
        const unsigned long long a = rp[b0 + v], d = rp[b0 + v + 1] - a;
        const unsigned long long o = off[v];
        if (d > t4) {
            for (unsigned long long j = lane; j < d; j += 32) {
                hcol[o + j] = col[a + j];
                if (hw) hw[o + j] = w[a + j];
            }
        }
        __syncwarp();
        if (lane == 0 && d <= t4) off[v] = ~0ull;
    }
}

cudaError_t setup_hub_offsets(const unsigned long long* row_ptr, unsigned b0, unsigned n, unsigned t4,
                              unsigned long long* off, void* tmp, size_t tmp_bytes, cudaStream_t s) {
    k_hub_deg<<<592, 256, 0, s>>>(row_ptr, b0, n, t4, off);
    cudaError_t e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, off, off, (size_t)n + 1, s);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

cudaError_t setup_hub_fill(const unsigned long long* row_ptr, const unsigned* col, const unsigned* w, unsigned b0,
                           unsigned n, unsigned t4, unsigned long long* off, unsigned* hcol, unsigned* hw,
                           cudaStream_t s) {
    k_hub_fill<<<1184, 256, 0, s>>>(row_ptr, col, w, b0, n, t4, off, hcol, hw);
    return cudaGetLastError();
}

// PR pieces: entry i (edges [q_off[i], q_off[i+1])) becomes ceil(len / piece) entries of <= piece edges
__global__ void k_pr_piece_cnt(const unsigned long long* q_off, unsigned long long n, unsigned piece,
                               unsigned long long* cnt) {
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i <= n;
         i += (unsigned long long)gridDim.x * blockDim.x)
        cnt[i] = i < n ? (q_off[i + 1] - q_off[i] + piece - 1) / piece : 0ull;
}
__global__ void k_pr_piece_emit(const unsigned* q_v, const unsigned long long* q_off, unsigned long long n,
                                unsigned piece, const unsigned long long* pos, unsigned* q2_v,
                                unsigned long long* q2_off) {
    for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i <= n;
         i += (unsigned long long)gridDim.x * blockDim.x) {
        if (i == n) {
            q2_off[pos[n]] = q_off[n];
            continue;
        }
        const unsigned long long a = q_off[i], b = q_off[i + 1], p0 = pos[i];
        const unsigned v = q_v[i];
        for (unsigned long long k = 0; a + k * piece < b; k++) {
            q2_v[p0 + k] = v;
            q2_off[p0 + k] = a + k * piece;
        }
    }
}
cudaError_t setup_pr_pieces_count(const unsigned long long* q_off, unsigned long long n, unsigned piece,
                                  unsigned long long* cnt, void* tmp, size_t tmp_bytes, cudaStream_t s) {
    k_pr_piece_cnt<<<1184, 256, 0, s>>>(q_off, n, piece, cnt);
    cudaError_t e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, cnt, cnt, (size_t)n + 1, s);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}
cudaError_t setup_pr_pieces_emit(const unsigned* q_v, const unsigned long long* q_off, unsigned long long n,
                                 unsigned piece, const unsigned long long* pos, unsigned* q2_v,
                                 unsigned long long* q2_off, cudaStream_t s) {
    k_pr_piece_emit<<<1184, 256, 0, s>>>(q_v, q_off, n, piece, pos, q2_v, q2_off);
    return cudaGetLastError();
}

}  // namespace gum
