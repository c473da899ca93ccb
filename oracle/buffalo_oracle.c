/*
 * buffalo_oracle.c — CPU ORACLE for Buffalo's block generation (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load this library.  It shares no code, header, table or constant generator with the
 * CUDA path (paper_conf_hpca_yangzl25_b200/csrc); the Philox generator below is an
 * independent implementation pinned to the Random123 known-answer vectors
 * (tests/test_philox.py).  Plain, single-threaded, obviously-correct code: no blocking,
 * no hashing, no parallelism beyond the optional OpenMP loop over groups used for timing.
 *
 * Paper: Buffalo (HPCA'25), /root/reference/PAPER.md.  Cited as PAPER.md:<line>.
 *
 *  - oracle_philox        : Philox4x32-10 (Salmon et al., SC'11) — DESIGN.md "Philox streams"
 *  - oracle_sample_row    : neighbour sampling of one CSR row, §IV-E PAPER.md:390 ("for each
 *                           CSR row, neighbor sampling for the center nodes is performed");
 *                           mechanism = Floyd's without-replacement algorithm keyed by
 *                           (seed, node, hop)  [DESIGN.md reading R2]
 *  - oracle_build_blocks  : BlockGenerate / MicroBatchGenerator, Alg. 2 l.5 PAPER.md:237,
 *                           Alg. 3 l.11 PAPER.md:279: the L bipartite blocks of one group,
 *                           built top-down from the output layer; local src ids = dst prefix
 *                           then the other neighbours in ascending global id
 *                           [DESIGN.md readings R3, R4]
 *  - oracle_triangles     : the average clustering coefficient C of Eq. 1 (PAPER.md:363,
 *                           :384-386: "C ... obtained by offline graph analysis, utilizing the
 *                           equation presented on page 142 of reference [27]"): the number of
 *                           triangles through every node, T_v = #{(u, w): u < w, u, w in N(v),
 *                           w in N(u)}, by definition (every neighbour pair tested with a binary
 *                           search of the sorted row) [DESIGN.md reading R27]
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------- Philox4x32-10 */
void oracle_philox(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
    uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
    uint32_t k0 = key[0], k1 = key[1];
    for (int r = 0; r < 10; ++r) {
        if (r > 0) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
        uint64_t p0 = (uint64_t)0xD2511F53u * c0;
        uint64_t p1 = (uint64_t)0xCD9E8D57u * c2;
        uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
        uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
        uint32_t n0 = hi1 ^ c1 ^ k0, n1 = lo1, n2 = hi0 ^ c3 ^ k1, n3 = lo0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* Draw t of the sampling stream of node v at hop h: word (t & 3) of
   Philox(key = seed; ctr = (v, h, t >> 2, tag 0)). */
static uint32_t sample_draw(uint64_t seed, int64_t v, int32_t hop, int64_t t) {
    uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    uint32_t ctr[4] = {(uint32_t)v, (uint32_t)hop, (uint32_t)(t >> 2), 0u};
    uint32_t out[4];
    oracle_philox(ctr, key, out);
    return out[t & 3];
}

/* ---------------------------------------------------------------- sampling
 * Writes the sampled neighbours of v (global ids, in ascending CSR position) to out and
 * returns their number D(v).  f <= 0 or deg <= f: all neighbours in CSR order.
 * Otherwise Floyd's algorithm: for t = 0..f-1, j = deg - f + t, r = floor(x_t * (j+1) / 2^32);
 * insert j if r is already chosen, else r.  Then the chosen positions are sorted.        */
int64_t oracle_sample_row(const int64_t* row_ptr, const int32_t* col, int64_t v, int32_t f,
                          uint64_t seed, int32_t hop, int32_t* out) {
    int64_t beg = row_ptr[v], deg = row_ptr[v + 1] - row_ptr[v];
    if (f <= 0 || deg <= f) {
        for (int64_t s = 0; s < deg; ++s) out[s] = col[beg + s];
        return deg;
    }
    int64_t* S = (int64_t*)malloc(sizeof(int64_t) * (size_t)f);
    int64_t n = 0;
    for (int64_t t = 0; t < f; ++t) {
        int64_t j = deg - f + t;
        uint32_t x = sample_draw(seed, v, hop, t);
        int64_t r = (int64_t)(((uint64_t)x * (uint64_t)(j + 1)) >> 32);
        int present = 0;
        for (int64_t q = 0; q < n; ++q) if (S[q] == r) { present = 1; break; }
        S[n++] = present ? j : r;
    }
    /* insertion sort of the f chosen positions */
    for (int64_t a = 1; a < n; ++a) {
        int64_t key = S[a], b = a - 1;
        while (b >= 0 && S[b] > key) { S[b + 1] = S[b]; --b; }
        S[b + 1] = key;
    }
    for (int64_t s = 0; s < n; ++s) out[s] = col[beg + S[s]];
    free(S);
    return n;
}

/* ---------------------------------------------------------------- blocks (Alg. 2 l.5) */
static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}

typedef struct {
    int64_t n_dst, n_src, n_edges;
    int32_t* row_ptr;     /* [n_dst + 1] */
    int32_t* col_local;   /* [n_edges]   position of the neighbour in src_global */
    int32_t* col_global;  /* [n_edges]   the neighbour's global id */
    int32_t* src_global;  /* [n_src]     dst_global is its prefix of length n_dst */
} oracle_block;

void oracle_free_blocks(oracle_block* b, int32_t L) {
    for (int32_t i = 0; i < L; ++i) {
        free(b[i].row_ptr); free(b[i].col_local); free(b[i].col_global); free(b[i].src_global);
        memset(&b[i], 0, sizeof(oracle_block));
    }
}

/* Builds blocks l = L..1 of the micro-batch whose output nodes are seeds[0..n).
 * out[l-1] receives block l.  fanout[l-1] is block l's fanout; the hop of block l is
 * h = L - l + 1.  Returns 0 on success, -1 on allocation failure.                       */
int oracle_build_blocks(int64_t N, const int64_t* row_ptr, const int32_t* col,
                        const int32_t* seeds, int64_t n, int32_t L, const int32_t* fanout,
                        uint64_t seed, oracle_block* out) {
    int64_t* pos = (int64_t*)malloc(sizeof(int64_t) * (size_t)(N > 0 ? N : 1));
    if (!pos) return -1;
    for (int64_t v = 0; v < N; ++v) pos[v] = -1;

    int32_t* dst = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    memcpy(dst, seeds, sizeof(int32_t) * (size_t)n);
    int64_t n_dst = n;
    int64_t max_deg = 0;
    for (int64_t v = 0; v < N; ++v)
        if (row_ptr[v + 1] - row_ptr[v] > max_deg) max_deg = row_ptr[v + 1] - row_ptr[v];
    int32_t* row = (int32_t*)malloc(sizeof(int32_t) * (size_t)(max_deg > 0 ? max_deg : 1));

    for (int32_t l = L; l >= 1; --l) {
        int32_t f = fanout[l - 1];
        int32_t hop = L - l + 1;
        oracle_block* b = &out[l - 1];
        /* pass 1: sampled neighbours of every dst, in dst order then CSR order */
        int64_t cap = 1024, e = 0;
        int32_t* cg = (int32_t*)malloc(sizeof(int32_t) * (size_t)cap);
        int32_t* rp = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_dst + 1));
        rp[0] = 0;
        for (int64_t i = 0; i < n_dst; ++i) {
            int64_t d = oracle_sample_row(row_ptr, col, dst[i], f, seed, hop, row);
            if (e + d > cap) {
                while (e + d > cap) cap *= 2;
                cg = (int32_t*)realloc(cg, sizeof(int32_t) * (size_t)cap);
            }
            memcpy(cg + e, row, sizeof(int32_t) * (size_t)d);
            e += d;
            rp[i + 1] = (int32_t)e;
        }
        /* pass 2: src = dst (prefix, same order), then the distinct neighbours that are not
           dst, in ascending global id (R3) */
        int32_t* src = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_dst + e + 1));
        int64_t n_src = 0;
        for (int64_t i = 0; i < n_dst; ++i) { pos[dst[i]] = n_src; src[n_src++] = dst[i]; }
        for (int64_t k = 0; k < e; ++k) {
            int32_t u = cg[k];
            if (pos[u] == -1) { pos[u] = -2; src[n_src++] = u; }   /* -2: seen, not yet placed */
        }
        qsort(src + n_dst, (size_t)(n_src - n_dst), sizeof(int32_t), cmp_i32);
        for (int64_t j = n_dst; j < n_src; ++j) pos[src[j]] = j;
        int32_t* cl = (int32_t*)malloc(sizeof(int32_t) * (size_t)(e > 0 ? e : 1));
        for (int64_t k = 0; k < e; ++k) cl[k] = (int32_t)pos[cg[k]];
        for (int64_t j = 0; j < n_src; ++j) pos[src[j]] = -1;
        b->n_dst = n_dst; b->n_src = n_src; b->n_edges = e;
        b->row_ptr = rp; b->col_local = cl; b->col_global = cg;
        b->src_global = (int32_t*)realloc(src, sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1));
        /* the next (lower) block's dst are this block's src */
        free(dst);
        dst = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1));
        memcpy(dst, b->src_global, sizeof(int32_t) * (size_t)n_src);
        n_dst = n_src;
    }
    free(row); free(dst); free(pos);
    return 0;
}

/* Layer sizes only (n_0..n_L, e_1..e_L) of the blocks of seeds[0..n) — used for the
 * per-item statistics of Eq. 1 (I, O, D) and the BucketMemEstimator. */
int oracle_block_sizes(int64_t N, const int64_t* row_ptr, const int32_t* col,
                       const int32_t* seeds, int64_t n, int32_t L, const int32_t* fanout,
                       uint64_t seed, int64_t* n_out /*[L+1]*/, int64_t* e_out /*[L]*/) {
    oracle_block* b = (oracle_block*)calloc((size_t)L, sizeof(oracle_block));
    int rc = oracle_build_blocks(N, row_ptr, col, seeds, n, L, fanout, seed, b);
    if (rc == 0) {
        for (int32_t l = 1; l <= L; ++l) {
            n_out[l] = b[l - 1].n_dst;
            e_out[l - 1] = b[l - 1].n_edges;
        }
        n_out[0] = b[0].n_src;
    }
    oracle_free_blocks(b, L);
    free(b);
    return rc;
}

/* ---------------------------------------------------------------- triangles per node (C, R27) */
static int has_edge(const int64_t* row_ptr, const int32_t* col, int32_t u, int32_t w) {
    int64_t lo = row_ptr[u], hi = row_ptr[u + 1];          /* sorted row: binary search */
    while (lo < hi) {
        const int64_t mid = lo + (hi - lo) / 2;
        if (col[mid] < w) lo = mid + 1; else hi = mid;
    }
    return lo < row_ptr[u + 1] && col[lo] == w;
}

/* T[v] for v in [v0, v1): pairs of neighbours of v that are adjacent (each pair once). */
void oracle_triangles(const int64_t* row_ptr, const int32_t* col, int64_t v0, int64_t v1, int64_t* T) {
    for (int64_t v = v0; v < v1; ++v) {
        int64_t t = 0;
        for (int64_t a = row_ptr[v]; a < row_ptr[v + 1]; ++a)
            for (int64_t b = a + 1; b < row_ptr[v + 1]; ++b)
                t += has_edge(row_ptr, col, col[a], col[b]);
        T[v - v0] = t;
    }
}
