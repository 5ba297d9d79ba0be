/*
 * select.cpp — plain single-threaded CPU oracle of candidate-read selection.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h; same rules: loaded by tests/, smoke() and bench.py's
 * baseline legs only, shares nothing with the CUDA path).
 *
 * The paper places this step before local assembly: "the alignment stage, where contigs are aligned
 * against reads to find reads that can be used to further extend the contigs. The reads that align
 * to the ends of contigs are then used for extending the contigs in both directions" (P:L308-311,
 * §2.2; reads for the left and right sides kept separate; the GPU aligner of [3],
 * P:L289-290, L367-368).  It gives no alignment rule, so the definition below is DESIGN.md §10d's
 * reading S1-S6, written out literally: std::string::find for the seeds, a character loop for the
 * mismatches, no index, no hashing, no sorting beyond std::sort of the final records.
 *
 *   S1  end window W_e: RIGHT end of contig C: [max(0,|C|-w), |C|); LEFT end: [0, min(w,|C|)).
 *   S2  a read x aligns to end e with strand σ and diagonal d (y = x if σ=+, rc(x) if σ=-;
 *       y[j] faces C[d+j]) iff
 *         (a) seed: some j ≡ 0 (mod t), 0 <= j <= |y|-s, with [d+j, d+j+s) inside W_e and
 *             y[j, j+s) == C[d+j, d+j+s), neither containing N;
 *         (b) window overlap |[d, d+|y|) ∩ W_e| >= o;
 *         (c) M = mismatches of y against C over their whole overlap [max(0,d), min(|C|, d+|y|))
 *             (an N on either side is a mismatch), L = that overlap's length: 100*M <= mm_pct*L.
 *   S3  outward: RIGHT end: σ = + (the mate lies downstream, past the end) or d+|y| > |C|;
 *       LEFT end: σ = - or d < 0.
 *   S4  pair i (reads 2i, 2i+1, an FR library) is a candidate of end e iff one of its mates has an
 *       alignment to e satisfying S2 and S3; the first such alignment in the order (mate 0 before
 *       mate 1, σ=+ before σ=-, d ascending) decides the pair's orientation: if it has mate a on
 *       strand σ, mate a is written as y and the other mate on the opposite strand (rc if σ=+).
 *   S5  reads are written in contig-forward orientation (rc'd bases, reversed qualities), as
 *       la_load_batch expects (reading #14).
 *   S6  end e's reads: its candidate pairs in ascending pair index, mate 0 then mate 1.
 */
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <string>
#include <vector>

namespace {

char comp(char c) {
    switch (c) {
        case 'A': return 'T';
        case 'C': return 'G';
        case 'G': return 'C';
        case 'T': return 'A';
        default: return 'N';
    }
}

std::string rc(const std::string &s) {
    std::string o(s.rbegin(), s.rend());
    for (auto &c : o) c = comp(c);
    return o;
}

struct Hit {            // one qualifying alignment of a pair to an end (S4 order key)
    int64_t end, pair;
    int mate, strand;   // strand 0 = +, 1 = -
    int64_t d;
};

bool key_less(const Hit &a, const Hit &b) {
    if (a.end != b.end) return a.end < b.end;
    if (a.pair != b.pair) return a.pair < b.pair;
    if (a.mate != b.mate) return a.mate < b.mate;
    if (a.strand != b.strand) return a.strand < b.strand;
    return a.d < b.d;
}

}  // namespace

extern "C" {

/* Select candidate reads (S1-S6).
 *   contigs: contig_seq / contig_off[n_contigs+1]; pool: read_seq / read_qual / read_off[2*n_pairs+1]
 *   w, s (1..32), t (>= 1), o, mm_pct: the parameters of S1-S2.
 * Output (caller-allocated, capacity max_sel records): per selected (end, pair), sorted by (end, pair):
 *   sel_end[i], sel_pair[i], sel_flip[i] (0: mate 0 written as is, mate 1 rc'd; 1: the opposite).
 * Returns the number of selected (end, pair) records, -1 on invalid arguments, -2 if max_sel is
 * too small. */
int64_t orc_select(int32_t n_contigs, const char *contig_seq, const int64_t *contig_off, int64_t n_pairs,
                   const char *read_seq, const int64_t *read_off, int32_t w, int32_t s, int32_t t, int32_t o,
                   int32_t mm_pct, int64_t max_sel, int64_t *sel_end, int64_t *sel_pair, uint8_t *sel_flip) {
    if (n_contigs < 0 || n_pairs < 0 || w < 1 || s < 1 || s > 32 || t < 1 || o < 0 || mm_pct < 0) return -1;
    std::vector<std::string> C(n_contigs);
    for (int32_t c = 0; c < n_contigs; ++c)
        C[c].assign(contig_seq + contig_off[c], contig_seq + contig_off[c + 1]);
    std::vector<Hit> hits;
    for (int64_t i = 0; i < n_pairs; ++i) {
        for (int mate = 0; mate < 2; ++mate) {
            const int64_t rid = 2 * i + mate;
            const std::string x(read_seq + read_off[rid], read_seq + read_off[rid + 1]);
            for (int strand = 0; strand < 2; ++strand) {
                const std::string y = strand == 0 ? x : rc(x);
                const int64_t ly = (int64_t)y.size();
                for (int32_t c = 0; c < n_contigs; ++c) {
                    const std::string &Cs = C[c];
                    const int64_t lc = (int64_t)Cs.size();
                    for (int side = 0; side < 2; ++side) {   // 0 = LEFT (end 2c), 1 = RIGHT (end 2c+1)
                        // S1
                        const int64_t wlo = side ? std::max<int64_t>(0, lc - w) : 0;
                        const int64_t whi = side ? lc : std::min<int64_t>(w, lc);
                        const std::string win = Cs.substr(wlo, whi - wlo);
                        // S2(a): every stride seed of y found anywhere in the window -> diagonal
                        std::vector<int64_t> diags;
                        for (int64_t j = 0; j + s <= ly; j += t) {
                            const std::string seed = y.substr(j, s);
                            if (seed.find('N') != std::string::npos) continue;
                            for (size_t f = win.find(seed); f != std::string::npos; f = win.find(seed, f + 1))
                                diags.push_back(wlo + (int64_t)f - j);
                        }
                        std::sort(diags.begin(), diags.end());
                        diags.erase(std::unique(diags.begin(), diags.end()), diags.end());
                        for (int64_t d : diags) {
                            // S2(b)
                            const int64_t ov = std::min(d + ly, whi) - std::max(d, wlo);
                            if (ov < o) continue;
                            // S2(c)
                            const int64_t a0 = std::max<int64_t>(0, d), a1 = std::min(lc, d + ly);
                            int64_t M = 0;
                            for (int64_t p = a0; p < a1; ++p) {
                                const char u = y[p - d], v = Cs[p];
                                if (u == 'N' || v == 'N' || u != v) ++M;
                            }
                            if (100 * M > (int64_t)mm_pct * (a1 - a0)) continue;
                            // S3
                            const bool outward = side ? (strand == 0 || d + ly > lc) : (strand == 1 || d < 0);
                            if (!outward) continue;
                            hits.push_back(Hit{2 * (int64_t)c + side, i, mate, strand, d});
                        }
                    }
                }
            }
        }
    }
    // S4: the first qualifying alignment per (end, pair) decides; S6: (end, pair) order
    std::sort(hits.begin(), hits.end(), key_less);
    int64_t n = 0;
    for (size_t h = 0; h < hits.size(); ++h) {
        if (h > 0 && hits[h].end == hits[h - 1].end && hits[h].pair == hits[h - 1].pair) continue;
        if (n >= max_sel) return -2;
        sel_end[n] = hits[h].end;
        sel_pair[n] = hits[h].pair;
        // mate a on strand + -> mate 0 forward iff a == 0; on strand - -> the opposite
        sel_flip[n] = (uint8_t)((hits[h].mate == 0) == (hits[h].strand == 1));
        ++n;
    }
    return n;
}

}  // extern "C"
