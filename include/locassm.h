/*
 * locassm.h — C ABI of the B200 (sm_100a) local-assembly library.
 *
 * The operation (paper = /root/reference/PAPER.md, "P:L<line>"):
 *   MetaHipMer local assembly extends every contig end using only the reads that map to that end
 *   (§2.3).  For each end: build a k-mer -> extension hash table from the end's
 *   candidate reads (Alg 1; the value is the following base with its quality and count,
 *   P:L450-457), then mer-walk from the contig's last k-mer until a dead end, a fork, a loop or
 *   max_walk_len (Alg 2), and retry with k up-shifted after a fork and down-shifted
 *   after a dead end, stopping on a fork after a down-shift or a dead end after an up-shift
 *   (Fig 5).  Reads of the left and right side are kept separate and the same
 *   algorithm runs on both sides (Fig 4); a left end is computed as the right end of the
 *   reverse-complement problem and its extension is returned in contig-forward orientation.
 *   Where the paper is silent the readings listed in DESIGN.md §3 apply (vote rule, quality tiers,
 *   loop handling, choice of the returned walk, N handling, ...).
 *
 * Results are deterministic and equal, per end, to the CPU oracle (oracle/oracle.cpp) bit for bit:
 * extension string, termination code, k of the returned walk and number of attempts.
 *
 * Conventions: every call returns la_status; nothing is thrown across the ABI; no C++ types.
 * A context is bound to one CUDA device and one stream and is NOT thread-safe.
 */
#ifndef LOCASSM_H
#define LOCASSM_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct la_ctx la_ctx; /* opaque */

typedef enum {
    LA_OK = 0,
    LA_ERR_INVALID_ARG = -1, /* bad pointer, offsets, characters, lengths or parameters; the
                                context is unchanged */
    LA_ERR_OOM = -2,         /* device or pinned host allocation failed                       */
    LA_ERR_CUDA = -3,        /* CUDA error; sticky: the caller must la_destroy the context     */
    LA_ERR_STATE = -4,       /* la_extend before a successful la_load_batch                    */
    LA_ERR_CAPACITY = -5     /* an internal bound was exceeded (never a silent drop)           */
} la_status;

typedef enum {
    LA_TERM_DEADEND = 0, /* lookup found no usable extension (Alg 2 line 10, "end")           */
    LA_TERM_FORK = 1,    /* two or more candidate extensions (Alg 2 line 10, "fork")          */
    LA_TERM_LOOP = 2,    /* the next k-mer was already visited in this walk (Alg 2 line 6)    */
    LA_TERM_MAXLEN = 3,  /* max_walk_len bases appended (Alg 2 line 5 bound)                  */
    LA_TERM_NOREADS = 4, /* the end has no candidate reads (bin 1): not extended  */
    LA_TERM_SHORT = 5    /* contig shorter than k_start: no start k-mer                       */
} la_term;

typedef enum { LA_MEM_HOST = 0, LA_MEM_DEVICE = 1 } la_mem;

#define LA_HIST 16
#define LA_N_CLASSES 7

typedef struct {
    int32_t k_start, k_min, k_max, k_shift; /* 1 <= k_min <= k_start <= k_max <= 128; k_shift >= 1 */
    int32_t max_walk_len;                   /* W: 0 <= W <= 1024 (paper: walks up to 300) */
    int32_t qual_offset;                    /* Phred offset of read_qual characters, e.g. 33      */
    int32_t q_lo, q_hi;                     /* 0 <= q_lo <= q_hi <= 93: a base of quality q gives a
                                               low-tier vote if q >= q_lo and also a high-tier vote
                                               if q >= q_hi (reading #2)                          */
    int32_t min_votes;                      /* V >= 1 (reading #3)                                */
    int32_t min_frac_pct;                   /* F in 0..100 (reading #3)                           */
} la_params;

/* Input batch.  Caller-owned, read only during la_load_batch, may be freed after it returns.
 * mem = LA_MEM_HOST: all pointers are host memory (pinned memory is fastest);
 * mem = LA_MEM_DEVICE: all pointers are device memory of the context's device (e.g. torch tensor
 * data_ptr()); the loader reads them on the context stream.
 * Offsets start at 0 and are non-decreasing. */
typedef struct {
    int32_t mem;
    int32_t n_contigs;
    const char *contig_seq;       /* uppercase A,C,G,T,N                                      */
    const int64_t *contig_off;    /* [n_contigs+1]                                            */
    int64_t n_reads;
    const char *read_seq;         /* A,C,G,T,N; each read in its end's contig-forward orientation */
    const char *read_qual;        /* one quality character per base, >= qual_offset           */
    const int64_t *read_off;      /* [n_reads+1]; every read 0 <= len <= 300     */
    const int64_t *end_read_off;  /* [2*n_contigs+1]; end 2c = LEFT of contig c, 2c+1 = RIGHT;
                                     end e owns reads end_read_off[e] .. end_read_off[e+1]-1;
                                     end_read_off[2*n_contigs] == n_reads                       */
} la_batch;

/* Results.  Library-owned host memory, valid until the next la_load_batch / la_extend /
 * la_destroy on the same context. */
typedef struct {
    int64_t n_ends;               /* 2*n_contigs                                               */
    const int64_t *ext_off;       /* [n_ends+1]; extension of end e is ext_seq[ext_off[e]..ext_off[e+1]) */
    const char *ext_seq;          /* LEFT ends: contig-forward orientation, to prepend; RIGHT: to append */
    const uint8_t *term;          /* la_term of the returned walk                               */
    const uint8_t *k_used;        /* k of the returned walk (0 for NOREADS / SHORT)             */
    const uint8_t *n_attempts;    /* number of table builds + walks made for the end            */
} la_result;

typedef struct {
    double ms_total;          /* device time of the last la_extend (CUDA events on the ctx stream) */
    double ms_smem;           /* device time of the shared-memory-table kernel                  */
    double ms_global;         /* device time of the global-memory-table rounds                  */
    double ms_emit;           /* device time of result compaction                               */
    int64_t inserts;          /* sum over attempts of k-mer occurrences with a following base    */
    int64_t inserts_smem;     /* ... of which made by the shared-memory-table kernel             */
    int64_t walk_steps;       /* table lookups made by walks                                     */
    int64_t attempts;         /* table builds                                                    */
    int64_t ext_bases;        /* total extension length                                          */
    int64_t ends_by_class[5]; /* NOREADS, SHORT, SMEM, GLOBAL, SMEM->GLOBAL (smem table overflow) */
    int64_t kernel_launches;  /* kernels launched by the last la_extend                          */
    int64_t smem_bytes_per_cta;  /* small-table kernel                                          */
    int32_t smem_ctas_per_sm;
    int32_t global_rounds;
    int64_t ends_medium;         /* ends routed to the medium (one CTA per SM) kernel             */
    double ms_smem_medium;       /* summed kernel times of the XL, 2- and 1-CTA/SM classes          */
    int64_t ends_xl;             /* ends whose table lived in the XL class's global scratch        */
    int64_t xl_scratch_bytes;
    /* per table class (LA_N_CLASSES): 0..4 shared memory (64x12, 128x6, 256x3, 512x2, 1024x1 threads x
       CTAs per SM), 5 = XL (table in L2-resident global scratch), 6 = XLC (table split over a 2-CTA
       cluster's shared memory, reached through DSMEM) */
    int64_t cls_ends[LA_N_CLASSES], cls_inserts[LA_N_CLASSES], cls_attempts[LA_N_CLASSES],
        cls_filtered[LA_N_CLASSES];
    double cls_ms[LA_N_CLASSES];            /* device time of each class kernel (serial by default; spans if
                                    LA_CONCURRENT_CLASSES=1 launches them together)                */
    /* LA_PROFILE=1 only: per class, summed clock64 cycles of the builders' leader (wait for the
       walker, prefix, clear, filter pass, build pass, link) and of the walker (wait, walk) */
    uint64_t prof_cycles[LA_N_CLASSES][8];
    /* hash-build / walk split (SURVEY.md §8(b), §8(d) timing step 5), set by la_replay_build
       (-1 until then): ms_build = device time of the build-only replay of the table-class kernels,
       ms_walk = ms_smem - ms_build (link pass, walk and hand-offs); per class likewise */
    double ms_build, ms_walk;
    double cls_build_ms[LA_N_CLASSES];
    int64_t cls_build_inserts[LA_N_CLASSES];
    /* per class: attempts built with inline keys (k <= 63) and with pointer keys (k >= 64) */
    int64_t cls_inl_attempts[LA_N_CLASSES], cls_ref_attempts[LA_N_CLASSES];
    int64_t attempts_hist[LA_HIST]; /* ends by number of attempts (last bin: >= LA_HIST-1)       */
    int64_t cls_dead0[LA_N_CLASSES];   /* per class: attempts decided after the filter pass (the start k-mer has
                               < 2 voting occurrences: DEADEND at step 0 without building the table) */
    /* NEXT N3 co-execution (la_set_coexec): ends extended on host threads and their work (included in
       the totals above) */
    int64_t cpu_ends, cpu_inserts, cpu_walk_steps, cpu_attempts;
} la_stats;

la_status la_create(la_ctx **out, int device, void *cuda_stream /* cudaStream_t; NULL: own stream */);
la_status la_load_batch(la_ctx *ctx, const la_batch *batch, const la_params *params);
/* Runs the extension on the device and blocks until the results are in host memory. */
la_status la_extend(la_ctx *ctx, la_result *out);
/* Same, but leaves the results on the device only (no device-to-host copy); for device-resident
 * pipelines and the kernel-only benchmark.  Device pointers are returned in *out. */
la_status la_extend_device(la_ctx *ctx, la_result *out);
/* Streamed load + extend of a HOST batch (the batched pipeline of Fig 4
 * L558-563 and the host-to-device staging of P:L480-484).  The batch is cut into up to n_chunks
 * contiguous contig ranges of ~equal read bytes; chunk i+1's host-to-device copy runs on a second
 * stream while chunk i is validated, encoded and extended on the context stream, so the copy of a
 * batch overlaps its extension and device memory holds two chunks of raw input instead of all of it.
 * batch->mem must be LA_MEM_HOST (pinned memory gives full PCIe bandwidth); n_chunks in 1..4096
 * (more chunks than contigs is allowed).  Results are identical to la_load_batch + la_extend on the
 * same batch and are returned like la_extend's (library-owned host memory, valid until the next call
 * on the context); la_get_stats then reports the work and device time summed over chunks.
 * Errors: as la_load_batch (an invalid chunk aborts the call with LA_ERR_INVALID_ARG; unlike
 * la_load_batch, the context's loaded batch is then unspecified until the next la_load_batch). */
la_status la_extend_streamed(la_ctx *ctx, const la_batch *batch, const la_params *params, int32_t n_chunks,
                             la_result *out);
/* On-device append of extensions to contigs (the "Append extensions to contigs"
 * step of Fig 4; "appended to the end of contig", left ends by symmetry P:L399-402).
 * Extended contig c = ext(2c) + contig c + ext(2c+1), where ext(e) = ext_seq[ext_off[e]..ext_off[e+1])
 * (LEFT extensions are already in contig-forward orientation, see la_result) — e.g. the ext_off /
 * ext_seq that la_extend_device returns together with the batch's contig arrays.
 * ALL pointers are device memory of the context's device; the call runs on the context stream and
 * returns when the result is complete.  contig_off [n_contigs+1] and ext_off [2*n_contigs+1] are
 * non-decreasing (their first elements need not be 0: offsets are taken relative to them).
 * Outputs (caller-owned device memory): out_off [n_contigs+1], out_off[0] = 0, and out_seq of
 * (contig_off[n]-contig_off[0]) + (ext_off[2n]-ext_off[0]) bytes.  The offsets are not validated
 * on the device (inconsistent offsets are undefined behaviour).  Errors: LA_ERR_INVALID_ARG for
 * n_contigs < 0 or NULL offset pointers, LA_ERR_CUDA (sticky) for a failed launch. */
la_status la_append_extensions(la_ctx *ctx, int32_t n_contigs, const char *contig_seq, const int64_t *contig_off,
                               const int64_t *ext_off, const char *ext_seq, char *out_seq, int64_t *out_off);
/* Build-only replay of the last la_extend (SURVEY.md §8(d) timing protocol step 5, "the hash-build
 * phase"): reruns, on the device, exactly the (end, k) table builds that la_extend made in its
 * shared-memory / XL table classes — read staging, per-read prefix, table clear, filter and build
 * passes of Alg 1 — with the link pass and the walk disabled, and records the device
 * time in la_stats.ms_build / cls_build_ms and the replayed inserts in cls_build_inserts.  Results
 * of the last la_extend are unchanged.  Errors: LA_ERR_STATE if no la_extend completed since the
 * last la_load_batch; LA_ERR_CUDA (sticky). */
la_status la_replay_build(la_ctx *ctx);
/* CPU+GPU co-execution (the paper's co-scheduling of LA on CPU cores and
 * GPUs, §4.3, Fig 11): with n_threads > 0 and cpu_share > 0, every following la_extend /
 * la_extend_device / la_extend_streamed gives the lightest round(cpu_share x n) ends of the smallest
 * table class (n ends; by the planner's work estimate) to n_threads host threads, which extend them
 * (a host implementation of the same method, in this library) while the GPU's kernels run; the
 * results are identical and are returned with the GPU's.  n_threads = 0 or cpu_share = 0 turns it
 * off (the default).  Errors: LA_ERR_INVALID_ARG unless 0 <= n_threads <= 1024, 0 <= cpu_share <= 1. */
la_status la_set_coexec(la_ctx *ctx, int32_t n_threads, double cpu_share);

/* ---- NEXT N4: candidate-read selection ----
 * The step before local assembly: "contigs are aligned against reads to find reads that can be used
 * to further extend the contigs. The reads that align to the ends of contigs are then used for
 * extending the contigs" (§2.2), left and right sides separately.  The paper
 * gives no alignment rule; DESIGN.md §10d's readings S1-S6 define it:
 *   S1 end window: the last `window` bases of the contig (RIGHT end 2c+1) / the first (LEFT end 2c);
 *   S2 read x aligns to end e on strand σ (y = x or rc(x)) at diagonal d (y[j] faces C[d+j]) iff
 *      (a) a stride seed y[j, j+seed_len), j = 0, seed_stride, 2*seed_stride, ..., lies inside the
 *      window and equals the contig there (no N), (b) |[d, d+|y|) ∩ window| >= min_overlap,
 *      (c) 100 x mismatches <= max_mism_pct x L over the whole contig overlap of length L (N mismatches);
 *   S3 outward: RIGHT end: σ = + or the read reaches past the contig end; LEFT end: σ = - or it
 *      starts before the contig start;
 *   S4 pair i (reads 2i, 2i+1; an FR library) is a candidate of end e iff a mate aligns to e with
 *      S2 and S3; the first such alignment (mate 0 first, + first, smallest d) orients the pair;
 *   S5-S6 end e's reads: its pairs in ascending pair index, mate 0 then mate 1, each in contig-forward
 *      orientation (the mate on the - strand reverse-complemented, its qualities reversed).
 * Input: contigs and a pool of reads as sequenced (la_pool; mem = LA_MEM_HOST or LA_MEM_DEVICE on the
 * context's device; read length is not limited here).  Output (*out): the selected (end, pair, flip)
 * records, sorted by (end, pair), flip = 1 when mate 0 is the reverse-complemented one, and `batch`,
 * an la_batch with mem = LA_MEM_DEVICE that la_load_batch takes directly (its contig arrays are the
 * library's device copy of the pool's contigs).  All output pointers are device memory owned by the
 * context, valid until the next la_select_reads or la_destroy on it.  The call runs on the context
 * stream and returns when the selection is complete.
 * Errors: LA_ERR_INVALID_ARG for NULL pointers, n_contigs < 0, n_pairs < 0, non-monotone offsets, or
 * parameters out of range (1 <= seed_len <= 31, seed_stride >= 1, seed_len <= window <= 65535,
 * min_overlap >= 0, 0 <= max_mism_pct <= 100); LA_ERR_OOM; LA_ERR_CUDA (sticky). */
typedef struct {
    int32_t mem;                                          /* LA_MEM_HOST or LA_MEM_DEVICE */
    int32_t n_contigs;
    const char *contig_seq; const int64_t *contig_off;    /* [n_contigs+1] */
    int64_t n_pairs;                                      /* reads 2i, 2i+1 are the mates of pair i */
    const char *read_seq, *read_qual; const int64_t *read_off;   /* [2*n_pairs+1] */
} la_pool;
typedef struct {
    int32_t window;         /* S1, default 150 */
    int32_t seed_len;       /* S2(a), default 16 */
    int32_t seed_stride;    /* S2(a), default 4 */
    int32_t min_overlap;    /* S2(b), default 20 */
    int32_t max_mism_pct;   /* S2(c), default 4 */
} la_sel_params;
typedef struct {
    int64_t n_sel;                                        /* selected (end, pair) records */
    const int64_t *sel_end, *sel_pair;                    /* device [n_sel] */
    const uint8_t *sel_flip;                              /* device [n_sel] */
    la_batch batch;                                       /* device; n_reads = 2 * n_sel */
} la_selection;
la_status la_select_reads(la_ctx *ctx, const la_pool *pool, const la_sel_params *sp, la_selection *out);

la_status la_get_stats(const la_ctx *ctx, la_stats *out);
la_status la_destroy(la_ctx *ctx);                /* NULL is a no-op */
const char *la_last_error(const la_ctx *ctx);     /* message of the last non-OK status */

/* Host-side helper (no GPU needed): table capacity the planner reserves for an end whose reads
 * hold `inserts` k-mer occurrences with a following base, and the paper's load-factor bound
 * (l-k+1)/l for table size l*r.  Exposed for tests. */
int64_t la_plan_global_capacity(int64_t inserts);
double la_paper_load_factor(int32_t max_read_len, int32_t k);

#ifdef __cplusplus
}
#endif
#endif
