// la_smem.cuh — planner and the shared-memory-table kernel.
//
// One CTA extends one contig end at a time (persistent CTAs pull ends from a work counter, largest
// first).  Per end: the end's packed reads are staged in shared memory once; per attempt (k):
//   [filter pass]  only when the unfiltered table may not fit: every voting k-mer occurrence sets a
//                  bit in B1 (atomicOr); a second sighting sets the bit in B2.  k-mers with fewer
//                  than two voting occurrences can never reach min_votes >= 2, so they extend like
//                  absent k-mers (DEADEND) and may be left out of the table (reading #4's argument);
//                  hash collisions only let extra k-mers in, never keep one out.
//   [build, Alg 1] every voting occurrence (of a k-mer that passed the filter) is inserted into an
//                  open-addressing table in shared memory: slot = tag|read|pos (pointer-encoded key,
//                  P:L670-691), claimed with a 64-bit atomicCAS, equality verified against the staged
//                  read; the vote goes to packed 8-bit counters lo[4] | hi[4] of the slot
//                  (32-bit atomicAdds; an 8-bit carry is detected from the returned old value -> redone in
//                  the global path with 32-bit counters).
//   [ext rule + successor links]  per slot: ext(lo, hi) (reading #1) and, for a base, the slot of
//                  the successor k-mer (next_kmer, Alg 2 line 15) -> info word.
//   [walk, Alg 2]  one thread follows the info words from the start k-mer with a visited bit per slot
//                  (the paper's loop-check table), then applies the k-shift rule.
// Table overflow (claims above 70% of capacity) also sends the end to the global path; nothing is
// ever dropped.
#pragma once
#include "la_device.cuh"

namespace la {

enum : int { CLS_NOREADS = 0, CLS_SHORT = 1, CLS_S = 2, CLS_GLOBAL = 7 };   // CLS_S + class index
constexpr float SMEM_MAX_LOAD = 0.70f;

// ---- shared-memory layout ------------------------------------------------------------------------
struct SmemFixed {            // per end: staged reads, lengths (+ has-N bit 15), walk buffers
    uint32_t off_qc, off_len, off_walk, off_var, var_bytes;
};

__host__ __device__ __forceinline__ SmemFixed smem_fixed(int r, int SW, int W, uint32_t bytes) {
    SmemFixed F;
    const uint32_t rs = (uint32_t)r * (uint32_t)SW * 8u;
    F.off_qc = rs;
    F.off_len = 2u * rs;
    F.off_walk = (F.off_len + 2u * (uint32_t)r + 15u) & ~15u;
    F.off_var = (F.off_walk + 2u * (((uint32_t)W + 15u) & ~15u) + 15u) & ~15u;
    F.var_bytes = bytes > F.off_var + 64u ? bytes - F.off_var - 64u : 0u;
    return F;
}

// Two slot formats.  INLINE (k <= 63): the 2-bit k-mer itself, 16 B, claimed with one 128-bit CAS;
// REF (k >= 64): 8 B tag|read|pos, verified against the staged read.  Both + 8 B counters.
__host__ __device__ __forceinline__ bool inline_keys(int k) { return k <= 63; }
__host__ __device__ __forceinline__ uint32_t key_bytes(int k) { return inline_keys(k) ? 16u : 8u; }

struct SmemTab {              // per attempt: [vis bits][B1][B2][keys][cnts u64]
    uint32_t off_vis, off_b1, off_b2, off_keys, off_cnts, cap, mwords;
};

// U = voting-occurrence upper bound (sum over reads of max(0, len-k)).
__host__ __device__ __forceinline__ SmemTab smem_tab(uint32_t off_var, uint32_t var_bytes, uint32_t U,
                                                     bool allow_filter, uint32_t kbytes) {
    SmemTab T;
    const uint32_t per_slot_bits = 8u * (kbytes + 8u) + 1u;   // key + counters + 1 visited bit
    uint32_t cap_nf = (uint32_t)(((uint64_t)var_bytes * 8u) / per_slot_bits) & ~1u;
    uint32_t mwords = 0;
    uint32_t cap = cap_nf;
    if (allow_filter && (float)U > SMEM_MAX_LOAD * (float)cap_nf) {
        // two bitmaps of ~4 bits per occurrence each, at most a quarter of the region each
        mwords = (4u * U + 31u) / 32u;
        const uint32_t maxw = var_bytes / 16u;
        if (mwords > maxw) mwords = maxw;
        mwords = (mwords + 3u) & ~3u;
        const uint32_t rem = var_bytes > 8u * mwords ? var_bytes - 8u * mwords : 0u;
        cap = (uint32_t)(((uint64_t)rem * 8u) / per_slot_bits) & ~1u;
    }
    T.cap = cap;
    T.mwords = mwords;
    T.off_vis = off_var;
    T.off_b1 = (off_var + ((cap + 31u) / 32u) * 4u + 15u) & ~15u;
    T.off_b2 = T.off_b1 + mwords * 4u;
    T.off_keys = (T.off_b2 + mwords * 4u + 15u) & ~15u;
    T.off_cnts = T.off_keys + cap * kbytes;
    return T;
}

// ---- plan ------------------------------------------------------------------------------------
// Routing estimate of the filtered table: distinct k-mers with >= 2 voting occurrences plus filter
// false positives, as a fraction of the occurrences (measured on C2/C4 samples: 0.05-0.2, higher for
// ends with few reads).  A wrong guess only costs a redo in the global path.
__host__ __device__ __forceinline__ float filtered_fraction(int64_t r) {
    return r < 50 ? 0.30f : (r < 200 ? 0.16f : 0.10f);
}

__device__ __forceinline__ bool fits(int64_t r, int64_t U, int SW, const DevParams &P, uint32_t bytes,
                                     uint32_t min_cap) {
    if (bytes == 0) return false;
    const SmemFixed F = smem_fixed((int)r, SW, P.W, bytes);
    if (F.var_bytes == 0) return false;
    const SmemTab T = smem_tab(F.off_var, F.var_bytes, (uint32_t)U, P.V >= 2, key_bytes(P.k_min));
    if (T.cap < min_cap) return false;
    if (T.mwords == 0) return true;   // U <= 0.7 cap: cannot overflow
    return filtered_fraction(r) * (float)U + 64.f <= SMEM_MAX_LOAD * (float)T.cap;
}

// Shared-memory classes, smallest CTA first: (threads, CTAs/SM) = (64, 12), (128, 6), (256, 3),
// (256, 2), (512, 1).  Smaller ends get smaller CTAs, so the single-thread walk idles fewer warps;
// the first class whose table is predicted to fit wins; G = global-memory rounds.
constexpr int N_SMEM_CLASSES = 5;
struct PlanBytes {
    uint32_t b[N_SMEM_CLASSES];   // dynamic shared memory per CTA
    uint32_t t[N_SMEM_CLASSES];   // threads per CTA
};

__global__ void k_plan(const int64_t *__restrict__ eoff, const int64_t *__restrict__ roff,
                       const int32_t *__restrict__ clen, int64_t n_ends, DevParams P, int SW, PlanBytes pb,
                       int32_t *__restrict__ cls, int32_t *__restrict__ out_len, uint8_t *__restrict__ out_term,
                       uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att, int32_t *__restrict__ lists,
                       uint32_t *__restrict__ keys, int32_t *__restrict__ list_G, int *__restrict__ ctr) {
    // ctr: [0..4] n per smem class, [5] n_G, [6] NOREADS, [7] SHORT
    const int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (e >= n_ends) return;
    const int64_t r = eoff[e + 1] - eoff[e];
    int c;
    if (r == 0) c = CLS_NOREADS;
    else if (clen[e] < P.k_start) c = CLS_SHORT;
    else {
        const int64_t sumlen = roff[eoff[e + 1]] - roff[eoff[e]];
        int64_t U = sumlen - r * (int64_t)P.k_min;   // occurrences at the smallest k of the schedule
        if (U < 0) U = 0;
        c = CLS_GLOBAL;
        int sc = -1;
        if (r < 65536 && U < (1ll << 30))
            for (int i = 0; i < N_SMEM_CLASSES && sc < 0; ++i)
                if (fits(r, U, SW, P, pb.b[i], 4u * pb.t[i])) sc = i;
        int64_t U0 = sumlen - r * (int64_t)P.k_start;   // LPT key: occurrences at k_start
        U0 = U0 < 0 ? 0 : (U0 > 0xffffffffll ? 0xffffffffll : U0);
        if (sc >= 0) {
            c = CLS_S + sc;
            const int i = atomicAdd(&ctr[sc], 1);
            lists[sc * n_ends + i] = (int32_t)e;
            keys[sc * n_ends + i] = (uint32_t)U0;
        } else {
            list_G[atomicAdd(&ctr[N_SMEM_CLASSES], 1)] = (int32_t)e;
        }
    }
    cls[e] = c;
    if (c == CLS_NOREADS || c == CLS_SHORT) {
        atomicAdd(&ctr[N_SMEM_CLASSES + (c == CLS_NOREADS ? 1 : 2)], 1);
        out_len[e] = 0;
        out_term[e] = c == CLS_NOREADS ? T_NOREADS : T_SHORT;
        out_k[e] = 0;
        out_att[e] = 0;
    }
}

// ---- table operations ------------------------------------------------------------------------------
constexpr uint32_t NEXT_NONE = 0x0FFFFFFFu;   // info word: next slot (28 bits) << 4 | visited << 3 | code

struct SmemCtl {
    int end_idx, overflow, nclaim;
    int k, shift, kmax_eff, done, attempts;
    int best_len, best_term, best_k, best_buf;
    int maxlen;
    unsigned long long U;
    unsigned long long end_ins, end_steps;
    uint32_t start_slot;
};

struct GlobalStats {
    unsigned long long inserts, steps, attempts;
};

__device__ __forceinline__ uint32_t filt_index(uint64_t h, uint32_t mbits) {
    return (uint32_t)(((h >> 32) * (uint64_t)mbits) >> 32);
}

// 128-bit compare-and-swap in shared memory (ATOMS.CAS.128, sm_90+).  Returns the old value.
__device__ __forceinline__ void cas128_shared(void *p, uint64_t c0, uint64_t c1, uint64_t n0, uint64_t n1,
                                              uint64_t &o0, uint64_t &o1) {
    const unsigned addr = (unsigned)__cvta_generic_to_shared(p);
    asm volatile(
        "{\n .reg .b128 d, b, c;\n mov.b128 b, {%2, %3};\n mov.b128 c, {%4, %5};\n"
        " atom.shared.cas.b128 d, [%6], b, c;\n mov.b128 {%0, %1}, d;\n}"
        : "=l"(o0), "=l"(o1)
        : "l"(c0), "l"(c1), "l"(n0), "l"(n1), "r"(addr)
        : "memory");
}

__device__ __forceinline__ void ld128_volatile(const uint64_t *p, uint64_t &x, uint64_t &y) {
    asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];"
                 : "=l"(x), "=l"(y)
                 : "r"((unsigned)__cvta_generic_to_shared(p))
                 : "memory");
}

// Stored form of an inline key: word 1 is complemented, so a real key never reads (0, 0) = empty
// (k <= 63 leaves at least two zero pad bits in word 1).
__device__ __forceinline__ void inline_form(const Kmer &K, int KW, uint64_t &a, uint64_t &b) {
    a = K.w[0];
    b = ~(KW >= 2 ? K.w[1] : 0ull);
}

struct TabCtx {   // what a table operation needs
    uint64_t *keys;
    uint32_t *c32;   // per slot: word 0 = lo[4] (8 bits each), word 1 = hi[4]
    uint32_t cap;
    const uint64_t *sseq;
    uint32_t rbase;
    int SW, k, KW;
};

template <bool INL>
__device__ __forceinline__ uint32_t tab_lookup(const TabCtx &T, const Kmer &K, uint64_t h) {
    uint32_t s = slot_of(h, T.cap);
    if (INL) {
        uint64_t a, b;
        inline_form(K, T.KW, a, b);
        const ulonglong2 *kk = (const ulonglong2 *)T.keys;
        for (uint32_t n = 0; n < T.cap; ++n) {
            const ulonglong2 w = kk[s];
            if (w.y == 0) return NONE;
            if (w.x == a && w.y == b) return s;
            s = (s + 1 == T.cap) ? 0 : s + 1;
        }
    } else {
        const uint64_t tag = tag_of(h);
        for (uint32_t n = 0; n < T.cap; ++n) {
            const uint64_t w = T.keys[s];
            if (w == 0) return NONE;
            if ((w & TAG_MASK) == tag) {
                const Kmer K2 = extract_kmer(T.sseq + (size_t)(slot_read(w) - T.rbase) * T.SW, slot_pos(w), T.k, T.KW);
                if (kmer_eq(K, K2, T.KW)) return s;
            }
            s = (s + 1 == T.cap) ? 0 : s + 1;
        }
    }
    return NONE;
}

// Alg 1 line 5 (kmer_ht.insert) with the vote of the following base.
template <bool INL>
__device__ __forceinline__ void tab_insert(const TabCtx &T, const Kmer &K, uint64_t h, uint32_t rid, int pos,
                                           uint32_t b, bool hi, int *nclaim, int claim_limit, volatile int *ovf) {
    uint32_t s = slot_of(h, T.cap);
    bool hit = false;
    if (INL) {
        uint64_t a, bb;
        inline_form(K, T.KW, a, bb);
        for (;;) {
            uint64_t x, y;
            ld128_volatile(&T.keys[2 * s], x, y);
            if (y == 0) {   // looks empty: the CAS either claims it or returns its true content
                if (*ovf) return;
                cas128_shared((void *)&T.keys[2 * s], 0ull, 0ull, a, bb, x, y);
                if (y == 0) {   // claimed
                    if (atomicAdd(nclaim, 1) >= claim_limit) *ovf = 1;
                    break;
                }
            } else if (y == bb && x != a) {
                // a 16 B load is not guaranteed single-copy atomic: if it raced with the claiming CAS,
                // word 0 may be stale — re-read it (the slot never changes once claimed)
                x = *(volatile uint64_t *)&T.keys[2 * s];
            }
            if (x == a && y == bb) break;
            s = (s + 1 == T.cap) ? 0 : s + 1;
        }
    } else {
        const uint64_t tag = tag_of(h);
        volatile uint64_t *vk = T.keys;
        for (;;) {
            uint64_t w = vk[s];
            if (w == 0) {
                if (*ovf) return;
                const uint64_t mine = make_slot(tag, rid, (uint32_t)pos);
                const uint64_t old = atomicCAS((unsigned long long *)&T.keys[s], 0ull, (unsigned long long)mine);
                if (old == 0) {
                    if (atomicAdd(nclaim, 1) >= claim_limit) *ovf = 1;
                    break;
                }
                w = old;
            }
            if ((w & TAG_MASK) == tag) {
                const Kmer K2 = extract_kmer(T.sseq + (size_t)(slot_read(w) - T.rbase) * T.SW, slot_pos(w), T.k, T.KW);
                if (kmer_eq(K, K2, T.KW)) break;
            }
            s = (s + 1 == T.cap) ? 0 : s + 1;
        }
    }
    (void)hit;
    // 32-bit ATOMS.ADD (a 64-bit shared-memory add compiles to a CAS loop)
    const uint32_t old = atomicAdd(&T.c32[2 * s], 1u << (8 * b));
    if (((old >> (8 * b)) & 0xffu) == 0xffu) *ovf = 1;   // an 8-bit lo counter would carry
    if (hi) atomicAdd(&T.c32[2 * s + 1], 1u << (8 * b));  // hi <= lo: cannot carry first
}

// Every voting occurrence of the staged reads: thread per (read, 16-position segment), rolling k-mer,
// the following base / quality class read from a two-word window.  f(K, j, p, nb, nq2) per occurrence.
template <int BLOCK, typename F>
__device__ __forceinline__ unsigned long long for_each_vote(const uint64_t *sseq, const uint64_t *sqc,
                                                            const uint16_t *slen, int r, int SW, int k, int KW,
                                                            int maxlen, const volatile int *stop, F &&f) {
    unsigned long long n = 0;
    if (maxlen <= k) return 0;
    const int nseg = (maxlen - k + 15) >> 4;
    const int items = r * nseg;
    for (int it = threadIdx.x; it < items; it += BLOCK) {
        if (*stop) break;
        const int j = it / nseg;
        const int sg = it - j * nseg;
        const uint32_t lf = slen[j];
        const int len = (int)(lf & 0x7fffu);
        const int p0 = sg << 4;
        const int p1 = min(p0 + 16, len - k);
        if (p0 >= p1) continue;
        n += (unsigned)(p1 - p0);
        const uint64_t *R = sseq + (size_t)j * SW;
        const uint64_t *Q = sqc + (size_t)j * SW;
        Kmer K = extract_kmer(R, p0, k, KW);
        int lastN = -1;
        if (lf & 0x8000u)   // this read has an N
            for (int i = p0; i < p0 + k; ++i)
                if (get2(Q, i) == 3u) lastN = i;
        const int q0 = (p0 + k) >> 5;
        const uint64_t Ra = R[q0], Rb = R[q0 + 1], Qa = Q[q0], Qb = Q[q0 + 1];
        for (int p = p0; p < p1; ++p) {
            const int i = p + k;
            const bool second = (i >> 5) != q0;
            const int sh = 62 - ((i & 31) << 1);
            const uint32_t nb = (uint32_t)((second ? Rb : Ra) >> sh) & 3u;
            const uint32_t nq = (uint32_t)((second ? Qb : Qa) >> sh) & 3u;
            if (nq - 1u < 2u && lastN < p) f(K, j, p, nb, nq == 2u);
            if (nq == 3u) lastN = i;
            roll_kmer(K, k, KW, nb);
        }
    }
    return n;
}

// Build (filter pass when planned, then insert) and link one attempt.  Returns via C.overflow.
template <int BLOCK, bool INL>
__device__ __forceinline__ void build_and_link(SmemCtl &C, const TabCtx &T, uint32_t *B1, uint32_t *B2,
                                               uint32_t mbits, const uint16_t *slen, const uint64_t *sqc, int r,
                                               int maxlen, uint32_t r0, const DevParams &P,
                                               unsigned long long &my_ins) {
    const volatile int *stop = &C.overflow;
    const int k = T.k, KW = T.KW;
    // ---- filter pass: B1 = seen once, B2 = seen at least twice (readings #4) ----
    if (mbits) {
        for_each_vote<BLOCK>(T.sseq, sqc, slen, r, T.SW, k, KW, maxlen, stop,
                             [&](const Kmer &K, int, int, uint32_t, bool) {
                                 const uint32_t fi = filt_index(hash_kmer(K, KW), mbits);
                                 const uint32_t bit = 1u << (fi & 31);
                                 if (!(B2[fi >> 5] & bit)) {
                                     const uint32_t old = atomicOr(&B1[fi >> 5], bit);
                                     if (old & bit) atomicOr(&B2[fi >> 5], bit);
                                 }
                             });
        __syncthreads();
    }
    // ---- build (Alg 1) ----
    const int claim_limit = (int)(SMEM_MAX_LOAD * (float)T.cap);
    my_ins = for_each_vote<BLOCK>(T.sseq, sqc, slen, r, T.SW, k, KW, maxlen, stop,
                                  [&](const Kmer &K, int j, int p, uint32_t nb, bool hi) {
                                      const uint64_t h = hash_kmer(K, KW);
                                      if (mbits) {
                                          const uint32_t fi = filt_index(h, mbits);
                                          if (!((B2[fi >> 5] >> (fi & 31)) & 1u)) return;
                                      }
                                      tab_insert<INL>(T, K, h, r0 + (uint32_t)j, p, nb, hi, &C.nclaim,
                                                      claim_limit, &C.overflow);
                                  });
    __syncthreads();
    if (C.overflow) return;
    // ---- ext rule + successor links (a5) ----
    for (uint32_t s = threadIdx.x; s < T.cap; s += BLOCK) {
        Kmer K;
        if (INL) {
            const ulonglong2 w = ((const ulonglong2 *)T.keys)[s];
            if (w.y == 0) continue;
            K.w[0] = w.x;
            K.w[1] = KW >= 2 ? ~w.y : 0ull;
            K.w[2] = K.w[3] = 0;
        } else {
            const uint64_t w = T.keys[s];
            if (w == 0) continue;
            K = extract_kmer(T.sseq + (size_t)(slot_read(w) - T.rbase) * T.SW, slot_pos(w), k, KW);
        }
        const uint32_t lw = T.c32[2 * s], hw = T.c32[2 * s + 1];
        uint32_t lo[4], hi[4];
#pragma unroll
        for (int b = 0; b < 4; ++b) {
            lo[b] = (lw >> (8 * b)) & 0xffu;
            hi[b] = (hw >> (8 * b)) & 0xffu;
        }
        const int code = ext_rule(lo, hi, P.V, P.F);
        uint32_t nxt = NEXT_NONE;
        if (code < 4) {
            roll_kmer(K, k, KW, (uint32_t)code);
            const uint32_t t = tab_lookup<INL>(T, K, hash_kmer(K, KW));
            nxt = t == NONE ? NEXT_NONE : t;
        }
        T.c32[2 * s] = (nxt << 4) | (uint32_t)code;
    }
}

template <int BLOCK>
__global__ void __launch_bounds__(BLOCK, 768 / BLOCK > 0 ? 768 / BLOCK : 1) k_smem(
    const int32_t *__restrict__ list, int n_list, int *__restrict__ work_ctr,
    const uint64_t *__restrict__ rseq, const uint64_t *__restrict__ rqc,
    const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag,
    const int64_t *__restrict__ eoff, const uint64_t *__restrict__ tail,
    const uint64_t *__restrict__ tailN, const int32_t *__restrict__ clen, int SW, DevParams P,
    uint32_t smem_bytes, uint8_t *__restrict__ walk_buf, int32_t *__restrict__ out_len,
    uint8_t *__restrict__ out_term, uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att,
    int32_t *__restrict__ ovf_list, int *__restrict__ n_ovf, GlobalStats *__restrict__ gstats) {
    extern __shared__ __align__(16) unsigned char sm[];
    __shared__ SmemCtl C;
    __shared__ unsigned long long acc_ins, acc_steps, acc_att;
    const int tid = threadIdx.x;
    const int lane = tid & 31;
    if (tid == 0) { acc_ins = 0; acc_steps = 0; acc_att = 0; }

    for (;;) {
        __syncthreads();
        if (tid == 0) C.end_idx = atomicAdd(work_ctr, 1);
        __syncthreads();
        const int idx = C.end_idx;
        if (idx >= n_list) break;
        const int e = list[idx];
        const int64_t r0 = eoff[e];
        const int r = (int)(eoff[e + 1] - r0);
        const SmemFixed FX = smem_fixed(r, SW, P.W, smem_bytes);
        if (FX.var_bytes < 4096u) {   // reads do not fit: the global path takes this end
            if (tid == 0) ovf_list[atomicAdd(n_ovf, 1)] = e;
            continue;
        }
        uint64_t *sseq = (uint64_t *)sm;
        uint64_t *sqc = (uint64_t *)(sm + FX.off_qc);
        uint16_t *slen = (uint16_t *)(sm + FX.off_len);
        uint8_t *swalk = sm + FX.off_walk;   // two buffers of Wp bytes
        const int Wp = (P.W + 15) & ~15;

        // stage the end's packed reads (contiguous in HBM): coalesced 16 B loads
        {
            const int nw = r * SW;
            const uint4 *gs = (const uint4 *)(rseq + r0 * SW);
            const uint4 *gq = (const uint4 *)(rqc + r0 * SW);
            uint4 *ss = (uint4 *)sseq;
            uint4 *sq = (uint4 *)sqc;
            for (int i = tid; i < nw / 2; i += BLOCK) { ss[i] = gs[i]; sq[i] = gq[i]; }   // SW is even
            int ml = 0;
            for (int i = tid; i < r; i += BLOCK) {
                const int l = rlen[r0 + i];
                slen[i] = (uint16_t)(l | (rflag[r0 + i] ? 0x8000 : 0));
                ml = max(ml, l);
            }
            for (int o = 16; o; o >>= 1) ml = max(ml, __shfl_xor_sync(0xffffffffu, ml, o));
            if (tid == 0) {
                C.maxlen = 0;
                C.kmax_eff = min(P.k_max, (int)clen[e]);
                C.k = P.k_start;
                C.shift = 0;
                C.done = 0;
                C.attempts = 0;
                C.best_len = -1;
                C.best_term = T_DEADEND;
                C.best_k = 0;
                C.best_buf = 1;
                C.overflow = 0;
                C.end_ins = 0;
                C.end_steps = 0;
            }
            __syncthreads();
            if (lane == 0) atomicMax(&C.maxlen, ml);
        }
        __syncthreads();
        const int maxlen = C.maxlen;

        // ---------------- retry loop ----------------
        for (;;) {
            const int k = C.k;
            const int KW = kwords(k);
            const bool INL = inline_keys(k);
            // voting-occurrence bound at this k -> table plan
            {
                unsigned long long u = 0;
                for (int i = tid; i < r; i += BLOCK) u += (unsigned)max(0, (int)(slen[i] & 0x7fff) - k);
                for (int o = 16; o; o >>= 1) u += __shfl_xor_sync(0xffffffffu, u, o);
                if (tid == 0) C.U = 0;
                __syncthreads();
                if (lane == 0 && u) atomicAdd(&C.U, u);
                __syncthreads();
            }
            const SmemTab TB = smem_tab(FX.off_var, FX.var_bytes, (uint32_t)C.U, P.V >= 2, key_bytes(k));
            const uint32_t cap = TB.cap;
            if (cap < 4u * BLOCK) {   // no room for a table at this k (keeps claims + in-flight < cap)
                if (tid == 0) C.overflow = 1;
                __syncthreads();
                break;
            }
            const uint32_t mbits = TB.mwords * 32u;
            uint32_t *svis = (uint32_t *)(sm + TB.off_vis);
            (void)svis;
            uint32_t *B1 = (uint32_t *)(sm + TB.off_b1);
            uint32_t *B2 = (uint32_t *)(sm + TB.off_b2);
            TabCtx T;
            T.keys = (uint64_t *)(sm + TB.off_keys);
            T.c32 = (uint32_t *)(sm + TB.off_cnts);
            T.cap = cap;
            T.sseq = sseq;
            T.rbase = (uint32_t)r0;
            T.SW = SW;
            T.k = k;
            T.KW = KW;
            // clear keys + counters (contiguous) and the filters
            {
                const uint4 z = make_uint4(0, 0, 0, 0);
                uint4 *a = (uint4 *)T.keys;
                const uint32_t n16 = (cap * (key_bytes(k) + 8u)) / 16u;
                for (uint32_t i = tid; i < n16; i += BLOCK) a[i] = z;
                for (uint32_t i = tid; i < 2u * TB.mwords; i += BLOCK) B1[i] = 0;   // B1, B2 contiguous
                if (tid == 0) C.nclaim = 0;
            }
            __syncthreads();
            unsigned long long my_ins = 0;
            if (INL) build_and_link<BLOCK, true>(C, T, B1, B2, mbits, slen, sqc, r, maxlen, (uint32_t)r0, P, my_ins);
            else build_and_link<BLOCK, false>(C, T, B1, B2, mbits, slen, sqc, r, maxlen, (uint32_t)r0, P, my_ins);
            if (C.overflow) break;   // uniform: read after build_and_link's barrier
            for (int o = 16; o; o >>= 1) my_ins += __shfl_xor_sync(0xffffffffu, my_ins, o);
            if (lane == 0 && my_ins) atomicAdd(&C.end_ins, my_ins);
            if (tid == 0) {
                // start k-mer: last k bases of the oriented contig (Alg 2 line 4; reading #6)
                const uint64_t *Tl = tail + (size_t)e * TAIL_W;
                const int Tn = min((int)clen[e], 128);
                const int p = Tn - k;
                const uint64_t n0 = tailN[2 * (size_t)e], n1 = tailN[2 * (size_t)e + 1];
                bool hasN = false;
                for (int i = p; i < Tn; ++i) hasN |= ((i < 64 ? n0 >> i : n1 >> (i - 64)) & 1ull) != 0;
                C.start_slot = NONE;
                if (!hasN) {
                    uint64_t Tw[TAIL_W];
#pragma unroll
                    for (int i = 0; i < TAIL_W; ++i) Tw[i] = Tl[i];
                    const Kmer K = extract_kmer(Tw, p, k, KW);
                    const uint64_t h = hash_kmer(K, KW);
                    C.start_slot = INL ? tab_lookup<true>(T, K, h) : tab_lookup<false>(T, K, h);
                }
            }
            __syncthreads();

            // ---- walk (Alg 2) over the successor links + retry decision, one thread ----
            if (tid == 0) {
                uint8_t *wb = swalk + (C.best_buf ^ 1) * Wp;
                uint32_t *info = T.c32;   // info word of slot s at info[2 s]
                uint32_t node = C.start_slot == NONE ? NEXT_NONE : C.start_slot;
                int len = 0, term = T_MAXLEN;
                unsigned long long steps = 0;
                for (int i = 0; i < P.W; ++i) {
                    ++steps;   // a lookup (the loop check of a present k-mer precedes it, below)
                    if (node == NEXT_NONE) { term = T_DEADEND; break; }
                    const uint32_t inf = info[2 * node];
                    if (inf & 8u) { term = T_LOOP; --steps; break; }   // visited: loop check before lookup
                    info[2 * node] = inf | 8u;
                    const uint32_t code = inf & 7u;
                    if (code == CODE_FORK) { term = T_FORK; break; }
                    if (code == CODE_DEADEND) { term = T_DEADEND; break; }
                    wb[len++] = "ACGT"[code];
                    node = inf >> 4;
                }
                C.attempts += 1;
                C.end_steps += steps;
                if (len > C.best_len) {   // longest walk, earliest on ties (reading #11)
                    C.best_len = len;
                    C.best_term = term;
                    C.best_k = k;
                    C.best_buf ^= 1;
                }
                int kk = C.k, sh = C.shift;
                C.done = next_k(term, kk, sh, C.kmax_eff, P) ? 1 : 0;
                C.k = kk;
                C.shift = sh;
            }
            __syncthreads();
            if (C.done) break;
        }

        if (C.overflow) {   // table or counter overflow: the global path redoes this end from scratch
            if (tid == 0) ovf_list[atomicAdd(n_ovf, 1)] = e;
            continue;
        }
        // ---- write the selected walk ----
        const int bl = C.best_len;
        const uint8_t *bw = swalk + C.best_buf * Wp;
        uint8_t *dst = walk_buf + (size_t)e * P.W;
        for (int i = tid; i < bl; i += BLOCK) dst[i] = bw[i];
        if (tid == 0) {
            acc_ins += C.end_ins;
            acc_steps += C.end_steps;
            acc_att += C.attempts;
            out_len[e] = bl;
            out_term[e] = (uint8_t)C.best_term;
            out_k[e] = (uint8_t)C.best_k;
            out_att[e] = (uint8_t)C.attempts;
        }
    }
    if (tid == 0) {
        atomicAdd(&gstats->inserts, acc_ins);
        atomicAdd(&gstats->steps, acc_steps);
        atomicAdd(&gstats->attempts, acc_att);
    }
}

}  // namespace la
