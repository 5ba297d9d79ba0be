/*
 * oracle.cpp — plain single-threaded CPU oracle of MetaHipMer local assembly.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h).  Written from the paper, step by step,
 * with std::string keys and std::unordered_map; no packing, no SIMD, no threads,
 * nothing shared with the CUDA path.  Each function cites the passage it follows
 * (P:L<line> = /root/reference/PAPER.md line).  Readings where the paper is silent
 * are numbered as in DESIGN.md §3 / SURVEY.md §8(c).
 */
#include "oracle.h"

#include <algorithm>
#include <array>
#include <cstring>
#include <string>
#include <unordered_map>
#include <unordered_set>
#include <vector>

namespace {

/* Extension object: votes for the base that follows the k-mer,
 * split by the quality of that base (reading #2): lo[b] counts q >= q_lo, hi[b] q >= q_hi. */
struct Votes {
    std::array<uint32_t, 4> lo{{0, 0, 0, 0}};
    std::array<uint32_t, 4> hi{{0, 0, 0, 0}};
};

int base_index(char c) {
    switch (c) {
        case 'A': return 0;
        case 'C': return 1;
        case 'G': return 2;
        case 'T': return 3;
        default: return -1; /* 'N' */
    }
}

const char BASES[4] = {'A', 'C', 'G', 'T'};

char complement(char c) {
    switch (c) {
        case 'A': return 'T';
        case 'C': return 'G';
        case 'G': return 'C';
        case 'T': return 'A';
        default: return 'N';
    }
}

/* Reverse complement; N <-> N.  Left ends are walked on rc(contig) (reading #14). */
std::string rc(const std::string &s) {
    std::string r(s.rbegin(), s.rend());
    for (char &c : r) c = complement(c);
    return r;
}

struct Read {
    std::string seq;
    std::string qual;
};

typedef std::unordered_map<std::string, Votes> KmerTable; /* kmer_ht */

/* Alg 1: for each read, for each k-mer, kmer_ht.insert(k).  The value is the
 * extension: the following base with its quality and count.  Reading #4: all
 * |s|-k+1 k-mers are inserted; the last one has no following base and so gets no vote.
 * Reading #5: k-mers containing N are skipped; an N following base gives no vote.
 * Reading #16: every listed read votes (multiset). */
KmerTable build(const std::vector<Read> &reads, int k, const orc_params &P, int64_t *inserts) {
    KmerTable T;
    for (const Read &r : reads) {
        const std::string &s = r.seq;
        const int len = (int)s.size();
        for (int p = 0; p + k <= len; ++p) {
            if (p + k < len) ++*inserts; /* work unit: an occurrence with a following base */
            std::string K = s.substr(p, k);
            if (K.find('N') != std::string::npos) continue;
            Votes &v = T[K];
            if (p + k < len) {
                int b = base_index(s[p + k]);
                if (b < 0) continue;
                int q = (int)(unsigned char)r.qual[p + k] - P.qual_offset;
                if (q >= P.q_lo) v.lo[b] += 1;
                if (q >= P.q_hi) v.hi[b] += 1;
            }
        }
    }
    return T;
}

const int EXT_FORK = -1;
const int EXT_DEADEND = -2;

/* Reading #1 (the paper does not state how an extension is chosen from the votes; P:L437-441
 * only says lookup returns a base, "end" or "fork"): high-quality votes decide; low-quality
 * votes are the fallback.  A base qualifies with >= V votes and >= F% of its tier's total. */
int ext_rule(const Votes &v, const orc_params &P) {
    uint64_t H = 0, L = 0;
    for (int b = 0; b < 4; ++b) {
        H += v.hi[b];
        L += v.lo[b];
    }
    std::vector<int> S;
    for (int b = 0; b < 4; ++b)
        if (v.hi[b] >= (uint32_t)P.min_votes && 100ull * v.hi[b] >= (uint64_t)P.min_frac_pct * H)
            S.push_back(b);
    if (S.size() == 1) return S[0];
    if (S.size() >= 2) return EXT_FORK;
    std::vector<int> A;
    for (int b = 0; b < 4; ++b)
        if (v.lo[b] >= (uint32_t)P.min_votes && 100ull * v.lo[b] >= (uint64_t)P.min_frac_pct * L)
            A.push_back(b);
    if (A.size() == 1) return A[0];
    if (A.size() >= 2) return EXT_FORK;
    return EXT_DEADEND;
}

struct WalkResult {
    std::string walk;
    int state;
};

/* Alg 2.  kmer <- get_kmer(c): the last k bases of the oriented contig (reading #6).
 * for i < max_walk_len: loop check BEFORE lookup (lines 6-8; reading #12; the visited set is the
 * paper's second table), lookup (line 9), stop on end/fork (lines 10-13), append
 * (line 14), next_kmer (line 15).  Leaving the loop by its bound is MAXLEN (reading #7). */
WalkResult walk(const std::string &C, const KmerTable &T, int k, const orc_params &P,
                int64_t *steps) {
    std::string K = C.substr(C.size() - k, k);
    std::string w;
    std::unordered_set<std::string> visited;
    for (int i = 0; i < P.max_walk_len; ++i) {
        if (visited.count(K)) return {w, ORC_LOOP};
        visited.insert(K);
        ++*steps;
        int e;
        auto it = T.find(K);
        if (it == T.end())
            e = EXT_DEADEND;
        else
            e = ext_rule(it->second, P);
        if (e == EXT_DEADEND) return {w, ORC_DEADEND};
        if (e == EXT_FORK) return {w, ORC_FORK};
        w.push_back(BASES[e]);
        K = K.substr(1) + BASES[e];
    }
    return {w, ORC_MAXLEN};
}

struct EndResult {
    std::string ext;
    int term;
    int k_used;
    int attempts;
};

/* The k up/down-shift iteration (Fig 5):
 *   fork -> upshift k and rebuild; dead-end -> downshift k and rebuild; stop on a fork after a
 *   downshift or a dead-end after an upshift.  Readings: #8 (LOOP shifts like FORK; MAXLEN is
 *   accepted), #10 (out-of-range k stops), #11 (the longest walk over attempts is returned, the
 *   earliest on ties), #18 (NOREADS / SHORT). */
EndResult extend_end(const std::string &C, const std::vector<Read> &R, const orc_params &P,
                     int64_t *inserts, int64_t *steps) {
    if (R.empty()) return {"", ORC_NOREADS, 0, 0}; /* bin 1 */
    const int kmax_eff = std::min<int>(P.k_max, (int)C.size());
    if (P.k_start > kmax_eff) return {"", ORC_SHORT, 0, 0};
    int k = P.k_start;
    int shift = 0;
    bool have_best = false;
    EndResult best{"", ORC_DEADEND, 0, 0};
    int attempts = 0;
    for (;;) {
        KmerTable T = build(R, k, P, inserts);
        WalkResult wr = walk(C, T, k, P, steps);
        attempts += 1;
        if (!have_best || wr.walk.size() > best.ext.size()) {
            best = {wr.walk, wr.state, k, 0};
            have_best = true;
        }
        if (wr.state == ORC_MAXLEN) break;
        if (wr.state == ORC_LOOP && P.loop_accepts) break;
        if (wr.state == ORC_DEADEND) {
            if (shift > 0) break;   /* dead-end after upshift */
            shift = -P.k_shift;     /* downshift */
        } else {                    /* FORK or LOOP */
            if (shift < 0) break;   /* fork after downshift */
            shift = +P.k_shift;     /* upshift */
        }
        k += shift;
        if (k < P.k_min || k > kmax_eff) break;
    }
    best.attempts = attempts;
    return best;
}

bool valid_params(const orc_params &P) {
    return P.k_min >= 1 && P.k_min <= P.k_start && P.k_start <= P.k_max && P.k_max <= 128 &&
           P.k_shift >= 1 && P.max_walk_len >= 0 && P.q_lo >= 0 && P.q_lo <= P.q_hi &&
           P.min_votes >= 1 && P.min_frac_pct >= 0 && P.min_frac_pct <= 100;
}

} // namespace

extern "C" int orc_ext_rule(const uint32_t lo[4], const uint32_t hi[4], const orc_params *p) {
    Votes v;
    for (int b = 0; b < 4; ++b) {
        v.lo[b] = lo[b];
        v.hi[b] = hi[b];
    }
    return ext_rule(v, *p);
}

extern "C" int orc_extend(int32_t n_contigs, const char *contig_seq, const int64_t *contig_off,
                          int64_t n_reads, const char *read_seq, const char *read_qual,
                          const int64_t *read_off, const int64_t *end_read_off,
                          const orc_params *p, const int64_t *ends, int64_t n_sel,
                          int64_t *ext_len, char *ext_buf, uint8_t *term, uint8_t *k_used,
                          uint8_t *n_attempts, int64_t *inserts, int64_t *walk_steps) {
    if (!p || !valid_params(*p) || n_contigs < 0 || n_reads < 0) return -1;
    if (!contig_off || !read_off || !end_read_off) return -1;
    if (end_read_off[2 * (int64_t)n_contigs] > n_reads) return -1;
    const orc_params &P = *p;
    if (!ends) n_sel = 2 * (int64_t)n_contigs;
    for (int64_t i = 0; i < n_sel; ++i) {
        const int64_t e = ends ? ends[i] : i;
        if (e < 0 || e >= 2 * (int64_t)n_contigs) return -1;
        const int64_t c = e / 2;
        const bool right = (e % 2) == 1;
        std::string C(contig_seq + contig_off[c], contig_seq + contig_off[c + 1]);
        std::vector<Read> R;
        for (int64_t r = end_read_off[e]; r < end_read_off[e + 1]; ++r) {
            Read rd;
            rd.seq.assign(read_seq + read_off[r], read_seq + read_off[r + 1]);
            rd.qual.assign(read_qual + read_off[r], read_qual + read_off[r + 1]);
            R.push_back(rd);
        }
        int64_t ins = 0, st = 0;
        EndResult res;
        if (right) {
            res = extend_end(C, R, P, &ins, &st);
        } else {
            /* left end: the same algorithm on the reverse-complement problem */
            std::vector<Read> Rrc;
            for (const Read &rd : R) {
                Read x;
                x.seq = rc(rd.seq);
                x.qual = std::string(rd.qual.rbegin(), rd.qual.rend());
                Rrc.push_back(x);
            }
            res = extend_end(rc(C), Rrc, P, &ins, &st);
            res.ext = rc(res.ext);
        }
        ext_len[i] = (int64_t)res.ext.size();
        if (!res.ext.empty())
            std::memcpy(ext_buf + i * (int64_t)P.max_walk_len, res.ext.data(), res.ext.size());
        term[i] = (uint8_t)res.term;
        k_used[i] = (uint8_t)res.k_used;
        n_attempts[i] = (uint8_t)res.attempts;
        if (inserts) inserts[i] = ins;
        if (walk_steps) walk_steps[i] = st;
    }
    return 0;
}
