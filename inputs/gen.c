/*
 * inputs/gen.c -- seeded synthetic graph generators (test/bench INPUT infrastructure).
 *
 * This module produces raw edge lists (src[], dst[], w[]) and nothing else. It holds none of the
 * method's arithmetic: no CSR, no partition, no traversal. Both the CPU oracle (oracle/) and the
 * CUDA path (paper_conf_icde_menggltyz23_b200/) consume its output; neither shares any other code.
 *
 * Generators (recipe in DESIGN.md "Input recipe"; SURVEY.md §8(d) synthetic inputs):
 *   - RMAT (Graph500 a,b,c,d = .57,.19,.19,.05, no noise): every edge i is an independent draw of
 *     `scale` quadrant choices from the counter-based hash h(seed, STREAM_RMAT, i*L + l/2), two
 *     32-bit uniforms per 64-bit hash. Optional vertex-id scramble = keyed Feistel bijection on
 *     [0, 2^scale) (hubs spread over the id space, like Graph500's permutation).
 *   - 2-D n x n 4-neighbour grid, id = r*n + c, both directions, symmetric weights keyed by the
 *     unordered endpoint pair (road-like, high diameter).
 *   - 2-D n x n torus (4-regular, in = out = 4) -- PageRank closed-form pin.
 *   - Weights: w = 1 + (h(seed, STREAM_W, key) mod 255) in [1, 255] (SURVEY.md §8(c) reading #3).
 *
 * Multigraph semantics: duplicates and self-loops are kept.
 * Build: gcc -O3 -fopenmp -shared -fPIC (see Makefile at repo root).
 */
#include <stdint.h>
#include <stddef.h>

#define STREAM_RMAT 1ull
#define STREAM_W 2ull
#define STREAM_GRIDW 3ull
#define STREAM_SCRAMBLE 4ull

static inline uint64_t mix64(uint64_t z) {
    /* splitmix64 finaliser */
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* Counter-based hash: independent of evaluation order, so any thread count yields the same bytes. */
uint64_t gen_hash(uint64_t seed, uint64_t stream, uint64_t ctr) {
    uint64_t k = mix64(seed ^ (stream * 0xD1B54A32D192ED03ull));
    return mix64(k ^ (ctr * 0x9E3779B97F4A7C15ull) ^ (ctr >> 29));
}

/* splitmix64 sequence (used for source selection): x_j = mix64(seed + (j+1)*golden) with the
 * standard splitmix64 increment folded into mix64. */
uint64_t gen_splitmix_seq(uint64_t seed, uint64_t j) { return mix64(seed + j * 0x9E3779B97F4A7C15ull); }

/* Keyed balanced Feistel on 2*h bits with cycle walking down to [0, 2^bits). Bijection. */
static inline uint64_t feistel_round_f(uint64_t x, uint64_t key, int r) {
    return mix64(x ^ key ^ ((uint64_t)r * 0xA24BAED4963EE407ull));
}
uint64_t gen_scramble(uint64_t v, int bits, uint64_t seed) {
    if (bits <= 0) return v;
    int h = (bits + 1) / 2;
    uint64_t mask_h = (h >= 64) ? ~0ull : ((1ull << h) - 1);
    uint64_t lim = 1ull << bits;
    uint64_t key = mix64(seed ^ (STREAM_SCRAMBLE * 0xD1B54A32D192ED03ull));
    uint64_t x = v;
    do {
        uint64_t L = x >> h, R = x & mask_h;
        for (int r = 0; r < 4; r++) {
            uint64_t nl = R;
            uint64_t nr = (L ^ feistel_round_f(R, key, r)) & mask_h;
            L = nl; R = nr;
        }
        x = (L << h) | R;
    } while (x >= lim);
    return x;
}

/* RMAT: writes E edges. Probabilities a, b, c (d = 1-a-b-c). Returns 0. */
int gen_rmat(int scale, uint64_t num_edges, uint64_t seed, double a, double b, double c, int scramble,
             int weighted, uint32_t* src, uint32_t* dst, uint32_t* w) {
    const uint64_t ta = (uint64_t)(a * 4294967296.0);
    const uint64_t tb = (uint64_t)((a + b) * 4294967296.0);
    const uint64_t tc = (uint64_t)((a + b + c) * 4294967296.0);
    const uint64_t L = (uint64_t)((scale + 1) / 2); /* hashes per edge */
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)num_edges; i++) {
        uint64_t s = 0, d = 0, x = 0;
        for (int l = 0; l < scale; l++) {
            if ((l & 1) == 0) x = gen_hash(seed, STREAM_RMAT, (uint64_t)i * L + (uint64_t)(l / 2));
            uint64_t r = (l & 1) ? (x >> 32) : (x & 0xFFFFFFFFull);
            int bit = scale - 1 - l;
            if (r < ta) {
            } else if (r < tb) {
                d |= 1ull << bit;
            } else if (r < tc) {
                s |= 1ull << bit;
            } else {
                s |= 1ull << bit;
                d |= 1ull << bit;
            }
        }
        if (scramble) {
            s = gen_scramble(s, scale, seed);
            d = gen_scramble(d, scale, seed);
        }
        src[i] = (uint32_t)s;
        dst[i] = (uint32_t)d;
        if (weighted) w[i] = 1u + (uint32_t)(gen_hash(seed, STREAM_W, (uint64_t)i) % 255ull);
    }
    return 0;
}

static inline uint32_t grid_weight(uint64_t seed, uint64_t V, uint64_t u, uint64_t v, int unit) {
    if (unit) return 1u;
    uint64_t lo = u < v ? u : v, hi = u < v ? v : u;
    return 1u + (uint32_t)(gen_hash(seed, STREAM_GRIDW, lo * V + hi) % 255ull);
}

/* Number of edges of the n x n grid (torus=0) or torus (torus=1). */
uint64_t gen_grid_num_edges(uint64_t n, int torus) {
    if (torus) return 4ull * n * n;
    return n < 2 ? 0 : 4ull * n * (n - 1);
}

/* Grid / torus edges in vertex order; per vertex neighbours in order up, left, right, down.
 * unit_weights=1 gives all-1 weights (BFS-equivalent SSSP pin). */
int gen_grid(uint64_t n, int torus, uint64_t seed, int unit_weights, uint32_t* src, uint32_t* dst,
             uint32_t* w) {
    const uint64_t V = n * n;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < (int64_t)n; r++) {
        uint64_t off;
        if (torus) {
            off = (uint64_t)r * n * 4ull;
        } else {
            /* edges in rows < r: row 0 has n*(1) vertical + 2(n-1) horizontal ... */
            uint64_t rr = (uint64_t)r;
            uint64_t horiz = rr * 2ull * (n - 1);
            uint64_t vert = 0;
            if (rr > 0) vert = n * (1ull + 2ull * (rr - 1)); /* row0: n (down); rows 1..r-1: 2n each */
            if (n == 1) { horiz = 0; vert = 0; }
            off = horiz + vert;
        }
        for (uint64_t c = 0; c < n; c++) {
            uint64_t u = (uint64_t)r * n + c;
            uint64_t nb[4];
            int k = 0;
            if (torus) {
                nb[k++] = (((uint64_t)r + n - 1) % n) * n + c;
                nb[k++] = (uint64_t)r * n + (c + n - 1) % n;
                nb[k++] = (uint64_t)r * n + (c + 1) % n;
                nb[k++] = (((uint64_t)r + 1) % n) * n + c;
            } else {
                if (r > 0) nb[k++] = u - n;
                if (c > 0) nb[k++] = u - 1;
                if (c + 1 < n) nb[k++] = u + 1;
                if ((uint64_t)r + 1 < n) nb[k++] = u + n;
            }
            for (int j = 0; j < k; j++) {
                src[off] = (uint32_t)u;
                dst[off] = (uint32_t)nb[j];
                if (w) w[off] = grid_weight(seed, V, u, nb[j], unit_weights);
                off++;
            }
        }
    }
    return 0;
}
