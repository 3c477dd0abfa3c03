/*
 * graphgen/gen.c — seeded, counter-based synthetic graph generators.
 *
 * This module is INPUT GENERATION ONLY: it holds none of the MST method's arithmetic.
 * It is the one piece shared by the oracle (oracle/) and the CUDA path
 * (paper_conf_ppopp_nasrebp13_b200/), which otherwise share no code.
 *
 * Workload shapes follow the paper's MST inputs ("randomly generated",
 * Fig. 11: road networks, RMAT, Random4, 2-D grids); the exact recipes are
 * SURVEY.md §8(d) and are restated in DESIGN.md §"Input recipe".
 *
 * Hash: h(seed, i) = mix64(seed*0xD1B54A32D192ED03 + i*0x9E3779B97F4A7C15) (mod 2^64),
 * mix64 = the splitmix64 finaliser. Everything is integer; no floating point.
 * All generators are pure functions of (parameters, seeds): OpenMP only splits the index
 * range, so results do not depend on the thread count.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static inline uint64_t mix64(uint64_t x) {
    x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ULL;
    x ^= x >> 27; x *= 0x94D049BB133111EBULL;
    x ^= x >> 31;
    return x;
}

static inline uint64_t h64(uint64_t seed, uint64_t i) {
    return mix64(seed * 0xD1B54A32D192ED03ULL + i * 0x9E3779B97F4A7C15ULL);
}

void gg_hash_fill(uint64_t seed, int64_t start, int64_t count, uint64_t* out) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < count; ++i) out[i] = h64(seed, (uint64_t)(start + i));
}

/* weight rule shared by grid / uniform / rmat / dense: w = wlo + h(seed_w, i) mod wmod */
static inline uint32_t wmod_rule(uint64_t seed_w, uint64_t i, uint32_t wlo, uint64_t wmod) {
    return (uint32_t)(wlo + h64(seed_w, i) % wmod);
}

/* Grid W x H, v = y*W + x. Emission order: for y, for x: right (v,v+1) if x<W-1, then
 * down (v,v+W) if y<H-1. m = (W-1)*H + W*(H-1). w = wlo + h(seed_w,i) mod wmod.        */
int64_t gg_grid_m(int64_t W, int64_t H) { return (W - 1) * H + W * (H - 1); }

static inline int64_t grid_row_start(int64_t W, int64_t H, int64_t y) {
    (void)H;
    return y * (2 * W - 1);  /* rows 0..H-2 hold 2W-1 edges each; the last row follows */
}

void gg_grid(int64_t W, int64_t H, uint64_t seed_w, uint32_t wlo, uint64_t wmod,
             int32_t* src, int32_t* dst, uint32_t* w) {
    #pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < H; ++y) {
        int64_t e = grid_row_start(W, H, y);
        for (int64_t x = 0; x < W; ++x) {
            int64_t v = y * W + x;
            if (x < W - 1) { src[e] = (int32_t)v; dst[e] = (int32_t)(v + 1);
                             w[e] = wmod_rule(seed_w, (uint64_t)e, wlo, wmod); ++e; }
            if (y < H - 1) { src[e] = (int32_t)v; dst[e] = (int32_t)(v + W);
                             w[e] = wmod_rule(seed_w, (uint64_t)e, wlo, wmod); ++e; }
        }
    }
}

/* Road-like grid (USA-road shape, PAPER.md L421 N=23.9M M=57.7M): the grid's right/down
 * edges as gg_grid (ids 0..mg-1), then for each cell v=(x,y) with x<W-1, y<H-1 in
 * row-major order, the diagonal (v, v+W+1) iff h(seed_diag, v) mod 1000 < thresh.
 * Weight: w = base * (750 + h(seed_w, i) mod 501) / 1000 (integer floor), base 1000 for
 * axis edges and 1414 for diagonals.                                                      */
static inline uint32_t road_w(uint64_t seed_w, uint64_t i, uint64_t base) {
    return (uint32_t)(base * (750 + h64(seed_w, i) % 501) / 1000);
}

int64_t gg_road_m(int64_t W, int64_t H, uint64_t seed_diag, int64_t thresh) {
    int64_t cnt = 0;
    #pragma omp parallel for reduction(+:cnt) schedule(static)
    for (int64_t y = 0; y < H - 1; ++y)
        for (int64_t x = 0; x < W - 1; ++x)
            cnt += (int64_t)((h64(seed_diag, (uint64_t)(y * W + x)) % 1000) < (uint64_t)thresh);
    return gg_grid_m(W, H) + cnt;
}

void gg_road(int64_t W, int64_t H, uint64_t seed_w, uint64_t seed_diag, int64_t thresh,
             int32_t* src, int32_t* dst, uint32_t* w) {
    const int64_t mg = gg_grid_m(W, H);
    #pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < H; ++y) {
        int64_t e = grid_row_start(W, H, y);
        for (int64_t x = 0; x < W; ++x) {
            int64_t v = y * W + x;
            if (x < W - 1) { src[e] = (int32_t)v; dst[e] = (int32_t)(v + 1);
                             w[e] = road_w(seed_w, (uint64_t)e, 1000); ++e; }
            if (y < H - 1) { src[e] = (int32_t)v; dst[e] = (int32_t)(v + W);
                             w[e] = road_w(seed_w, (uint64_t)e, 1000); ++e; }
        }
    }
    /* diagonal ids need a row-major prefix count of the selected cells */
    int64_t rows = H - 1;
    if (rows <= 0 || W < 2) return;
    int64_t* rowcnt = (int64_t*)malloc((size_t)(rows + 1) * sizeof(int64_t));
    #pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < rows; ++y) {
        int64_t c = 0;
        for (int64_t x = 0; x < W - 1; ++x)
            c += (int64_t)((h64(seed_diag, (uint64_t)(y * W + x)) % 1000) < (uint64_t)thresh);
        rowcnt[y + 1] = c;
    }
    rowcnt[0] = 0;
    for (int64_t y = 0; y < rows; ++y) rowcnt[y + 1] += rowcnt[y];
    #pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < rows; ++y) {
        int64_t e = mg + rowcnt[y];
        for (int64_t x = 0; x < W - 1; ++x) {
            int64_t v = y * W + x;
            if ((h64(seed_diag, (uint64_t)v) % 1000) < (uint64_t)thresh) {
                src[e] = (int32_t)v; dst[e] = (int32_t)(v + W + 1);
                w[e] = road_w(seed_w, (uint64_t)e, 1414); ++e;
            }
        }
    }
    free(rowcnt);
}

/* Uniform random multigraph: u = h(seed_u,i) mod n, v = h(seed_v,i) mod n,
 * w = wlo + h(seed_w,i) mod wmod. Self-loops and parallel edges are kept.               */
void gg_uniform(int64_t n, int64_t m, uint64_t seed_u, uint64_t seed_v, uint64_t seed_w,
                uint32_t wlo, uint64_t wmod, int32_t* src, int32_t* dst, uint32_t* w) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i) {
        src[i] = (int32_t)(h64(seed_u, (uint64_t)i) % (uint64_t)n);
        dst[i] = (int32_t)(h64(seed_v, (uint64_t)i) % (uint64_t)n);
        w[i] = wmod_rule(seed_w, (uint64_t)i, wlo, wmod);
    }
}

/* RMAT (Graph500 style): for each edge, `scale` levels MSB-first,
 * q = h(seed_rmat, 32*i + level) mod 100; q < pa -> (0,0), < pa+pb -> (0,1),
 * < pa+pb+pc -> (1,0), else (1,1). Then both endpoints go through the permutation
 * perm (perm[v] = the v-th element of the stable argsort of h(seed_perm, v)), computed
 * by gg_rmat_perm. Duplicates and self-loops are kept.                                  */
typedef struct { uint64_t h; int64_t v; } hv_t;
static int cmp_hv(const void* a, const void* b) {
    const hv_t* x = (const hv_t*)a; const hv_t* y = (const hv_t*)b;
    if (x->h != y->h) return x->h < y->h ? -1 : 1;
    return x->v < y->v ? -1 : (x->v > y->v);
}

void gg_rmat_perm(int64_t n, uint64_t seed_perm, int32_t* perm) {
    hv_t* a = (hv_t*)malloc((size_t)n * sizeof(hv_t));
    #pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; ++v) { a[v].h = h64(seed_perm, (uint64_t)v); a[v].v = v; }
    qsort(a, (size_t)n, sizeof(hv_t), cmp_hv);
    for (int64_t j = 0; j < n; ++j) perm[j] = (int32_t)a[j].v;
    free(a);
}

void gg_rmat(int64_t scale, int64_t m, uint64_t seed_rmat, uint64_t seed_w,
             int64_t pa, int64_t pb, int64_t pc, uint32_t wlo, uint64_t wmod,
             const int32_t* perm, int32_t* src, int32_t* dst, uint32_t* w) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i) {
        uint64_t u = 0, v = 0;
        for (int64_t l = 0; l < scale; ++l) {
            uint64_t q = h64(seed_rmat, (uint64_t)(32 * i + l)) % 100;
            uint64_t bu, bv;
            if (q < (uint64_t)pa) { bu = 0; bv = 0; }
            else if (q < (uint64_t)(pa + pb)) { bu = 0; bv = 1; }
            else if (q < (uint64_t)(pa + pb + pc)) { bu = 1; bv = 0; }
            else { bu = 1; bv = 1; }
            u = (u << 1) | bu; v = (v << 1) | bv;
        }
        src[i] = perm ? perm[u] : (int32_t)u;
        dst[i] = perm ? perm[v] : (int32_t)v;
        w[i] = wmod_rule(seed_w, (uint64_t)i, wlo, wmod);
    }
}
