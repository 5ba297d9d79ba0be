// la_cpu.cpp — host implementation of local assembly for the CPU+GPU co-execution mode (NEXT N3).
//
// Per end (oriented so that the end to extend is on the right; LEFT ends arrive reverse-complemented
// from the device encoder, reading #14): for each k of the schedule build the k-mer -> votes table from
// the end's reads (Alg 1; the vote goes to the following base with its quality tier,
// P:L450-457, reading #2), mer-walk from the last k bases of the contig (Alg 2: loop check
// before the lookup, fork / dead end from the vote rule, reading #1) and shift k (readings
// #8, #10), keeping the longest walk (reading #11).  Only occurrences with a voting following base are
// inserted (reading #4); k-mers or following bases with an N give no vote (reading #5).
// Tables are per-thread open-addressing arrays reused across ends; ends are scheduled dynamically over
// std::threads.
#include "la_cpu.h"

#include <algorithm>
#include <atomic>
#include <cstring>
#include <thread>
#include <vector>

namespace la_cpu {
namespace {

enum { T_DEADEND = 0, T_FORK = 1, T_LOOP = 2, T_MAXLEN = 3, T_NOREADS = 4, T_SHORT = 5 };
enum { C_FORK = 4, C_DEADEND = 5 };

struct Key {
    uint64_t w[4];
};

inline uint64_t funnel(uint64_t hi, uint64_t lo, int s) { return s ? ((hi << s) | (lo >> (64 - s))) : hi; }

// k-mer at base p of a packed row (base j at bit 62 - 2*(j%32) of word j/32), left aligned
inline Key kmer_at(const uint64_t *R, int p, int k, int KW) {
    Key K;
    const int q = p >> 5, s = (p & 31) << 1;
    for (int w = 0; w < 4; ++w) {
        const int bits = 2 * k - 64 * w;
        const uint64_t m = bits >= 64 ? ~0ull : (bits > 0 ? (~0ull << (64 - bits)) : 0ull);
        K.w[w] = w < KW ? (funnel(R[q + w], R[q + w + 1], s) & m) : 0ull;
    }
    return K;
}

inline uint32_t code_at(const uint64_t *R, int i) { return (uint32_t)(R[i >> 5] >> (62 - 2 * (i & 31))) & 3u; }

// next_kmer (Alg 2 line 15): drop base 0, append base b at position k-1
inline void roll(Key &K, int k, int KW, uint32_t b) {
    for (int w = 0; w < KW; ++w) K.w[w] = (K.w[w] << 2) | (w + 1 < KW ? (K.w[w + 1] >> 62) : 0ull);
    const int wl = (k - 1) >> 5;
    K.w[wl] |= (uint64_t)b << (62 - 2 * ((k - 1) & 31));
}

inline uint64_t hash_key(const Key &K, int KW) {
    uint64_t h = K.w[0] * 0x9E3779B97F4A7C15ull;
    for (int w = 1; w < KW; ++w) h = (h ^ (h >> 29) ^ K.w[w]) * 0xBF58476D1CE4E5B9ull;
    h ^= h >> 31;
    h *= 0x94D049BB133111EBull;
    return h ^ (h >> 32);
}

inline bool same(const Key &a, const Key &b, int KW) {
    for (int w = 0; w < KW; ++w)
        if (a.w[w] != b.w[w]) return false;
    return true;
}

// Reading #1: two-tier vote rule on exact integer counts -> base 0..3, C_FORK or C_DEADEND.
inline int ext_rule(const uint32_t *lo, const uint32_t *hi, int V, int F) {
    uint64_t H = 0, L = 0;
    for (int b = 0; b < 4; ++b) {
        H += hi[b];
        L += lo[b];
    }
    uint32_t mh = 0, ml = 0;
    for (int b = 0; b < 4; ++b) {
        if (hi[b] >= (uint32_t)V && 100ull * hi[b] >= (uint64_t)F * H) mh |= 1u << b;
        if (lo[b] >= (uint32_t)V && 100ull * lo[b] >= (uint64_t)F * L) ml |= 1u << b;
    }
    const uint32_t m = mh ? mh : ml;   // the high tier decides when it has a candidate
    if (m == 0) return C_DEADEND;
    if (m & (m - 1)) return C_FORK;
    int b = 0;
    while (!((m >> b) & 1u)) ++b;
    return b;
}

// The k shift rule (readings #8, #10): true when the end is done
inline bool next_k(int term, int &k, int &shift, int kmax_eff, const Params &P) {
    if (term == T_MAXLEN) return true;
    if (term == T_DEADEND) {
        if (shift > 0) return true;
        shift = -P.k_shift;
    } else {
        if (shift < 0) return true;
        shift = P.k_shift;
    }
    k += shift;
    return k < P.k_min || k > kmax_eff;
}

// open-addressing table: key -> lo[4], hi[4], visited (one per thread, reused)
struct Table {
    std::vector<Key> key;
    std::vector<uint32_t> cnt;   // 8 per slot: lo[4], hi[4]
    std::vector<uint8_t> used, vis;
    uint64_t mask = 0;

    void reset(uint64_t U) {
        uint64_t cap = 64;
        while (cap < 2 * U + 16) cap <<= 1;
        if (key.size() < cap) {
            key.resize(cap);
            cnt.resize(8 * cap);
            used.resize(cap);
            vis.resize(cap);
        }
        mask = cap - 1;
        std::fill(used.begin(), used.begin() + cap, 0);
    }
    int64_t find(const Key &K, int KW) const {
        for (uint64_t s = hash_key(K, KW) & mask;; s = (s + 1) & mask) {
            if (!used[s]) return -1;
            if (same(key[s], K, KW)) return (int64_t)s;
        }
    }
    uint64_t insert(const Key &K, int KW) {
        for (uint64_t s = hash_key(K, KW) & mask;; s = (s + 1) & mask) {
            if (!used[s]) {
                used[s] = 1;
                vis[s] = 0;
                key[s] = K;
                std::memset(&cnt[8 * s], 0, 8 * sizeof(uint32_t));
                return s;
            }
            if (same(key[s], K, KW)) return s;
        }
    }
};

struct Worker {
    Table T;
    std::vector<int> nN;            // N prefix count of one read
    std::vector<uint8_t> cur, best;
    int64_t inserts = 0, steps = 0, attempts = 0;
};

void extend_one(const Input &in, int i, const Params &P, Worker &wk, Output &out) {
    const int64_t r0 = in.roff[i], r = in.roff[i + 1] - r0;
    const int clen = in.clen[i];
    const int kmax_eff = std::min(P.k_max, clen);
    uint8_t *walk = out.walk + (size_t)i * (size_t)std::max(P.W, 1);
    if (r == 0 || P.k_start > kmax_eff) {   // NOREADS (bin 1) / SHORT (reading #18)
        out.len[i] = 0;
        out.term[i] = r == 0 ? T_NOREADS : T_SHORT;
        out.k_used[i] = 0;
        out.att[i] = 0;
        out.dir[i] = 0;
        return;
    }
    const uint64_t *tail = in.tail + 5 * (size_t)i;
    const uint64_t tn0 = in.tailN[2 * (size_t)i], tn1 = in.tailN[2 * (size_t)i + 1];
    const int Tn = std::min(clen, 128);
    wk.cur.resize(std::max(P.W, 1));
    wk.best.resize(std::max(P.W, 1));
    int k = P.k_start, shift = 0, attempts = 0, best_len = -1, best_term = T_DEADEND, best_k = 0;
    for (;;) {
        const int KW = (2 * k + 63) >> 6;
        uint64_t U = 0;
        for (int64_t j = r0; j < r0 + r; ++j) U += in.rlen[j] > k ? (uint64_t)(in.rlen[j] - k) : 0ull;
        // ---- Alg 1: every occurrence with a voting following base ----
        wk.T.reset(U);
        for (int64_t j = r0; j < r0 + r; ++j) {
            const int L = in.rlen[j];
            if (L <= k) continue;
            const uint64_t *R = in.rseq + (size_t)j * in.SW, *Q = in.rqc + (size_t)j * in.SW;
            wk.nN.resize(L + 1);
            wk.nN[0] = 0;
            for (int t = 0; t < L; ++t) wk.nN[t + 1] = wk.nN[t] + (code_at(Q, t) == 3u);
            for (int p = 0; p + k < L; ++p) {
                const uint32_t qc = code_at(Q, p + k);
                if (qc != 1u && qc != 2u) continue;        // no vote: q < q_lo, or an N
                if (wk.nN[p + k] != wk.nN[p]) continue;    // an N inside the k-mer
                const uint64_t s = wk.T.insert(kmer_at(R, p, k, KW), KW);
                const uint32_t b = code_at(R, p + k);
                uint32_t *c = &wk.T.cnt[8 * s];
                ++c[b];
                if (qc == 2u) ++c[4 + b];
            }
        }
        wk.inserts += (int64_t)U;
        // ---- Alg 2: walk from the last k bases of the oriented contig (reading #6) ----
        const int p0 = Tn - k;
        bool hasN = false;
        for (int t = p0; t < Tn; ++t) hasN |= ((t < 64 ? tn0 >> t : tn1 >> (t - 64)) & 1ull) != 0;
        Key K = kmer_at(tail, p0, k, KW);
        int len = 0, term = T_MAXLEN;
        int64_t steps = 0;
        for (int s = 0; s < P.W; ++s) {
            ++steps;
            const int64_t slot = (hasN && s == 0) ? -1 : wk.T.find(K, KW);
            if (slot < 0) {
                term = T_DEADEND;
                break;
            }
            if (wk.T.vis[slot]) {   // loop check before the lookup (reading #12)
                term = T_LOOP;
                --steps;
                break;
            }
            wk.T.vis[slot] = 1;
            const uint32_t *c = &wk.T.cnt[8 * slot];
            const int code = ext_rule(c, c + 4, P.V, P.F);
            if (code == C_FORK) {
                term = T_FORK;
                break;
            }
            if (code == C_DEADEND) {
                term = T_DEADEND;
                break;
            }
            wk.cur[len++] = "ACGT"[code];
            roll(K, k, KW, (uint32_t)code);
        }
        wk.steps += steps;
        ++attempts;
        if (len > best_len) {   // longest walk, earliest on ties (reading #11)
            best_len = len;
            best_term = term;
            best_k = k;
            std::copy(wk.cur.begin(), wk.cur.begin() + len, wk.best.begin());
        }
        if (next_k(term, k, shift, kmax_eff, P)) break;
    }
    wk.attempts += attempts;
    std::copy(wk.best.begin(), wk.best.begin() + best_len, walk);
    out.len[i] = best_len;
    out.term[i] = (uint8_t)best_term;
    out.k_used[i] = (uint8_t)best_k;
    out.att[i] = (uint8_t)attempts;
    out.dir[i] = (int8_t)(shift > 0 ? 1 : (shift < 0 ? -1 : 0));
}

}  // namespace

void extend(const Input &in, const Params &P, int threads, Output &out) {
    out.inserts = out.walk_steps = out.attempts = 0;
    if (in.n <= 0) return;
    threads = std::max(1, std::min(threads, in.n));
    std::vector<Worker> wk(threads);
    std::atomic<int> next{0};
    auto run = [&](int t) {
        for (int i; (i = next.fetch_add(16)) < in.n;)
            for (int j = i; j < std::min(in.n, i + 16); ++j) extend_one(in, j, P, wk[t], out);
    };
    std::vector<std::thread> pool;
    for (int t = 1; t < threads; ++t) pool.emplace_back(run, t);
    run(0);
    for (auto &th : pool) th.join();
    for (const Worker &w : wk) {
        out.inserts += w.inserts;
        out.walk_steps += w.steps;
        out.attempts += w.attempts;
    }
}

}  // namespace la_cpu
