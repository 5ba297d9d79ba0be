/*
 * oracle.h — plain, slow, single-threaded CPU oracle of MetaHipMer local assembly.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_sc_awanhedbdoy21_b200/) never links, imports or calls it, and shares
 * no code, header, table or constant with it.
 *
 * What it computes (paper = /root/reference/PAPER.md, cited P:L<line>):
 *   for every contig end e: build a k-mer -> extension-vote table from the end's
 *   candidate reads (Alg 1; value semantics P:L450-457, L716-723),
 *   mer-walk from the contig's last k-mer (Alg 2), retry with the
 *   k up/down-shift rule (Fig 5); right ends are
 *   walked directly, left ends through the reverse complement (Fig 4).
 *   Where the paper is silent the readings of SURVEY.md §8(c) / DESIGN.md §3 apply.
 *
 * Parity status: pinned by tests/test_oracle_pins.py (closed forms P2-P8, RC and
 * permutation invariance P9-P10, vote truth table P12, brute force P11).  Agreement
 * with MetaHipMer2's own code is UNPINNED (no code or worked example in the paper).
 */
#ifndef LA_ORACLE_H
#define LA_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
    int32_t k_start, k_min, k_max, k_shift; /* k schedule (reading #9)          */
    int32_t max_walk_len;                   /* Alg 2 line 5; "up to 300 steps" P:L878      */
    int32_t qual_offset;                    /* Phred offset (reading #2)                   */
    int32_t q_lo, q_hi;                     /* low/high quality vote thresholds (#2)       */
    int32_t min_votes;                      /* V (#3)                                      */
    int32_t min_frac_pct;                   /* F (#3)                                      */
    int32_t loop_accepts;                   /* 0: LOOP upshifts like FORK (#8); 1: accept  */
} orc_params;

enum { ORC_DEADEND = 0, ORC_FORK = 1, ORC_LOOP = 2, ORC_MAXLEN = 3, ORC_NOREADS = 4, ORC_SHORT = 5 };

/*
 * Extend the selected ends.  All pointers are host memory owned by the caller.
 *   contig_seq/contig_off[n_contigs+1]      uppercase ACGTN
 *   read_seq/read_qual/read_off[n_reads+1]  reads in contig-forward orientation
 *   end_read_off[2*n_contigs+1]             end 2c = LEFT of contig c, 2c+1 = RIGHT
 *   ends[n_sel]                             end ids to compute (NULL: all 2*n_contigs, in order)
 * Outputs, one per selected end:
 *   ext_len[i], ext_buf[i*max_walk_len ..] (LEFT: contig-forward, to prepend; RIGHT: to append)
 *   term[i], k_used[i], n_attempts[i]
 *   inserts[i]    (may be NULL) Σ over attempts of k-mer occurrences that carry a vote candidate
 *                 (p+k < len), i.e. Σ_attempts Σ_reads max(0, len-k): the algorithmic unit
 *   walk_steps[i] (may be NULL) Σ over attempts of table lookups made by the walk
 * Returns 0, or -1 on invalid arguments.
 */
int orc_extend(int32_t n_contigs, const char *contig_seq, const int64_t *contig_off,
               int64_t n_reads, const char *read_seq, const char *read_qual,
               const int64_t *read_off, const int64_t *end_read_off,
               const orc_params *p, const int64_t *ends, int64_t n_sel,
               int64_t *ext_len, char *ext_buf, uint8_t *term, uint8_t *k_used,
               uint8_t *n_attempts, int64_t *inserts, int64_t *walk_steps);

/* The vote rule ext(lo, hi) of reading #1, exposed for the truth-table pin P12.
 * Returns 0..3 for A,C,G,T, -1 for FORK, -2 for DEADEND. */
int orc_ext_rule(const uint32_t lo[4], const uint32_t hi[4], const orc_params *p);

#ifdef __cplusplus
}
#endif
#endif
