/* abi_client.c — a plain C client of include/locassm.h (no Python, no C++): builds a tiny batch,
 * runs la_create -> la_load_batch -> la_extend -> la_get_stats -> la_destroy on cuda:0 and checks
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
    } while (!unique_kmers(g, GLEN, 21));
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
    CHECK(la_destroy(ctx) == LA_OK, "la_destroy");
    free(rseq);
    free(rqual);
    free(roff);
    return 0;
}
