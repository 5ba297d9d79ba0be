/* abi_client.c — a plain C client of include/locassm.h (no Python, no C++): builds a tiny batch,
 * runs la_create -> la_load_batch -> la_extend -> la_get_stats -> la_select_reads -> la_destroy on cuda:0 and checks
 * the result against the closed form of SURVEY.md §8(c) pin P2 (error-free tiled reads, Alg 1/2 of
 * P:L404-448): with reads starting at every a in [a_lo, a_hi] (length l, all Q40), the right walk
 * from contig end e is G[e : a_hi + l - V + 1] with code DEADEND; an end without reads is NOREADS
 * (P:L548-549).  Built by __graft_entry__.build(); run by tests/test_gpu_parity.py (-m gpu).
 * Exit 0 = all checks passed, 1 = a check failed, 2 = the library returned an error. */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "locassm.h"

#define GLEN 1200
#define RLEN 150

static uint64_t rng_state = 0x9E3779B97F4A7C15ull;
static uint32_t rnd(void) {   /* xorshift64* */
    rng_state ^= rng_state >> 12;
    rng_state ^= rng_state << 25;
    rng_state ^= rng_state >> 27;
    return (uint32_t)((rng_state * 2685821657736338717ull) >> 32);
}

/* every k-mer of g occurs once (k >= kmin) — brute force; the P2 closed form needs it */
static int unique_kmers(const char *g, int n, int k) {
    for (int i = 0; i + k <= n; ++i)
        for (int j = i + 1; j + k <= n; ++j)
            if (memcmp(g + i, g + j, (size_t)k) == 0) return 0;
    return 1;
}

static char comp(char c) { return c == 'A' ? 'T' : (c == 'C' ? 'G' : (c == 'G' ? 'C' : 'A')); }

/* every k-mer of g occurs once counting both strands (N4's closed form needs unique seeds) */
static int unique_kmers_both(const char *g, int n, int k) {
    char *r = (char *)malloc((size_t)n);
    for (int i = 0; i < n; ++i) r[i] = comp(g[n - 1 - i]);
    int ok = unique_kmers(g, n, k);
    for (int i = 0; ok && i + k <= n; ++i)
        for (int j = 0; j + k <= n; ++j)
            if (memcmp(g + i, r + j, (size_t)k) == 0) { ok = 0; break; }
    free(r);
    return ok;
}

#define CHECK(cond, ...)                                            \
    do {                                                            \
        if (!(cond)) {                                              \
            fprintf(stderr, "abi_client: check failed: " __VA_ARGS__); \
            fprintf(stderr, "\n");                                  \
            return 1;                                               \
        }                                                           \
    } while (0)

int main(void) {
    char g[GLEN + 1];
    do {
        for (int i = 0; i < GLEN; ++i) g[i] = "ACGT"[rnd() & 3u];
        g[GLEN] = 0;
    } while (!unique_kmers(g, GLEN, 21) || !unique_kmers_both(g, GLEN, 16));
    /* one contig G[300:500); its right end e = 500 has reads starting at a = 200..600 (a_hi = 600),
       its left end has none */
    const int cs = 300, e = 500, a_lo = 200, a_hi = 600, V = 2;
    const int n_reads = a_hi - a_lo + 1;
    char *rseq = (char *)malloc((size_t)n_reads * RLEN), *rqual = (char *)malloc((size_t)n_reads * RLEN);
    int64_t *roff = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n_reads + 1));
    for (int i = 0; i < n_reads; ++i) {
        memcpy(rseq + (size_t)i * RLEN, g + a_lo + i, RLEN);
        memset(rqual + (size_t)i * RLEN, 'I', RLEN);
        roff[i] = (int64_t)i * RLEN;
    }
    roff[n_reads] = (int64_t)n_reads * RLEN;
    int64_t coff[2] = {0, e - cs};
    int64_t eoff[3] = {0, 0, n_reads};
    la_batch b;
    memset(&b, 0, sizeof b);
    b.mem = LA_MEM_HOST;
    b.n_contigs = 1;
    b.contig_seq = g + cs;
    b.contig_off = coff;
    b.n_reads = n_reads;
    b.read_seq = rseq;
    b.read_qual = rqual;
    b.read_off = roff;
    b.end_read_off = eoff;
    la_params p = {33, 21, 99, 8, 300, 33, 10, 20, V, 20};

    la_ctx *ctx = NULL;
    la_status s = la_create(&ctx, 0, NULL);
    if (s != LA_OK) { fprintf(stderr, "abi_client: la_create -> %d\n", (int)s); return 2; }
    la_result r;
    if ((s = la_load_batch(ctx, &b, &p)) != LA_OK || (s = la_extend(ctx, &r)) != LA_OK) {
        fprintf(stderr, "abi_client: %d: %s\n", (int)s, la_last_error(ctx));
        la_destroy(ctx);
        return 2;
    }
    la_stats st;
    la_get_stats(ctx, &st);
    /* P2: walk length a_hi + l - V + 1 - e, the genome continuation, DEADEND, k_used = k_start,
       floor((k_start - k_min) / shift) + 1 attempts (every downshift ties) */
    const int want_len = a_hi + RLEN - V + 1 - e;
    const int64_t got_len = r.ext_off[2] - r.ext_off[1];
    CHECK(r.n_ends == 2, "n_ends %lld", (long long)r.n_ends);
    CHECK(r.term[0] == LA_TERM_NOREADS && r.ext_off[1] == 0, "left end: term %d", r.term[0]);
    CHECK(got_len == want_len, "right extension length %lld, closed form %d", (long long)got_len, want_len);
    CHECK(memcmp(r.ext_seq + r.ext_off[1], g + e, (size_t)want_len) == 0, "right extension != genome continuation");
    CHECK(r.term[1] == LA_TERM_DEADEND, "right term %d", r.term[1]);
    CHECK(r.k_used[1] == 33 && r.n_attempts[1] == (33 - 21) / 8 + 1, "k_used %d attempts %d", r.k_used[1],
          r.n_attempts[1]);
    CHECK(st.ext_bases == want_len, "stats.ext_bases %lld", (long long)st.ext_bases);
    /* results are library-owned: read them before la_destroy */
    printf("abi_client ok: right extension %lld bases (closed form %d), DEADEND, k %d, %d attempts\n",
           (long long)got_len, want_len, r.k_used[1], r.n_attempts[1]);

    /* NEXT N4 (la_select_reads, readings S1-S6): FR pairs from fragments [a, a+350), a = a_lo..a_hi,
       mate 0 = G[a, a+150), mate 1 = rc(G[a+200, a+350)).  With unique 16-mers on both strands the
       selection has a closed form: the RIGHT end (window G[350, 500)) takes every pair whose forward
       read overlaps the window by >= 20 (a in [220, 480]) or whose reverse read does and reaches past
       500 (a in [200, 280]): a in [200, 480], 281 pairs; the LEFT end (window G[300, 450)) takes the
       pairs whose reverse read overlaps it by >= 20 (a <= 230) or whose forward read does and starts
       before 300 (a in [200, 299]): 100 pairs.  The selected batch, loaded on the device and extended,
       tiles starts 200..680 (forward reads and mates): the right walk passes W = 300 bases (P2 closed
       form 680 + 150 - V + 1 - 500 = 329 > W): MAXLEN with G[500, 800). */
    CHECK(unique_kmers_both(g, GLEN, 16), "the genome repeats a 16-mer (on either strand)");
    {
        const int np = a_hi - a_lo + 1;
        char *ps = (char *)malloc((size_t)np * 2 * RLEN), *pq = (char *)malloc((size_t)np * 2 * RLEN);
        int64_t *po = (int64_t *)malloc(sizeof(int64_t) * (size_t)(2 * np + 1));
        for (int i = 0; i < np; ++i) {
            const int a = a_lo + i;
            memcpy(ps + (size_t)(2 * i) * RLEN, g + a, RLEN);
            for (int j = 0; j < RLEN; ++j) ps[(size_t)(2 * i + 1) * RLEN + j] = comp(g[a + 349 - j]);
        }
        memset(pq, 'I', (size_t)np * 2 * RLEN);
        for (int i = 0; i <= 2 * np; ++i) po[i] = (int64_t)i * RLEN;
        la_pool pool;
        memset(&pool, 0, sizeof pool);
        pool.mem = LA_MEM_HOST;
        pool.n_contigs = 1;
        pool.contig_seq = g + cs;
        pool.contig_off = coff;
        pool.n_pairs = np;
        pool.read_seq = ps;
        pool.read_qual = pq;
        pool.read_off = po;
        la_sel_params sp = {150, 16, 4, 20, 4};
        la_selection sel;
        if ((s = la_select_reads(ctx, &pool, &sp, &sel)) != LA_OK) {
            fprintf(stderr, "abi_client: la_select_reads %d: %s\n", (int)s, la_last_error(ctx));
            la_destroy(ctx);
            return 2;
        }
        CHECK(sel.n_sel == 281 + 100, "selected (end, pair) records %lld, closed form 381", (long long)sel.n_sel);
        CHECK(sel.batch.mem == LA_MEM_DEVICE && sel.batch.n_reads == 2 * sel.n_sel, "selection batch");
        if ((s = la_load_batch(ctx, &sel.batch, &p)) != LA_OK || (s = la_extend(ctx, &r)) != LA_OK) {
            fprintf(stderr, "abi_client: select -> extend %d: %s\n", (int)s, la_last_error(ctx));
            la_destroy(ctx);
            return 2;
        }
        CHECK(r.ext_off[2] - r.ext_off[1] == 300 && r.term[1] == LA_TERM_MAXLEN, "selected right end: %lld bases, term %d",
              (long long)(r.ext_off[2] - r.ext_off[1]), r.term[1]);
        CHECK(memcmp(r.ext_seq + r.ext_off[1], g + e, 300) == 0, "selected right end != genome continuation");
        printf("abi_client ok: la_select_reads %lld pairs (closed form 381); extended right end MAXLEN, 300 bases\n",
               (long long)sel.n_sel);
        free(ps);
        free(pq);
        free(po);
    }
    CHECK(la_destroy(ctx) == LA_OK, "la_destroy");
    free(rseq);
    free(rqual);
    free(roff);
    return 0;
}
