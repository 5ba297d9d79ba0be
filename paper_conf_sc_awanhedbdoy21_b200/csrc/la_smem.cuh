// la_smem.cuh — planner and the shared-memory-table kernel.
//
// k_smem: persistent CTAs; each CTA = one walker warp + (BLOCK-32) builder threads and keeps TWO
// contig ends in flight, so the serial mer-walk of one end overlaps the table build of the other.
//   builders, per attempt (k) of an end:
//     [filter pass]  only when the unfiltered table may not fit: every voting k-mer occurrence sets a
//                    bit in B1 (atomicOr); a second sighting sets its bit in B2.  k-mers with fewer
//                    than two voting occurrences cannot reach min_votes >= 2, so they extend exactly
//                    like absent k-mers (DEADEND) and may be left out (reading #4); bitmap collisions
//                    only admit extra k-mers, never exclude one.
//     [build, Alg 1] every voting occurrence of a k-mer that passed the filter is
//                    inserted into an open-addressing table in shared memory.  k <= 63: the slot holds
//                    the 2-bit k-mer itself (16 B) and is claimed with one 128-bit CAS; k >= 64: the slot
//                    holds tag|read|pos (pointer-encoded key) verified against the read.
//                    The vote for the following base goes to packed 8-bit counters lo[4],
//                    hi[4] (32-bit atomicAdds; an 8-bit carry is detected -> redo in the global path).
//     [link]         per slot: ext(lo, hi) (reading #1) and, for a base, the slot of the successor
//                    k-mer (next_kmer, Alg 2 line 15) -> an info word in the end's own info buffer.
//   walker (lane 0 of warp 0): follows the info words from the start k-mer (Alg 2) with a
//     visited bit per slot (the loop-check table), then applies the k-shift rule
//      and hands the end back to the builders (next k) or writes its result.
// Reads are not staged: builders stream them from HBM/L2 (up to 2 passes per attempt).  Table
// overflow (claims above 70% of capacity) or a counter carry re-routes the end to the global path.
#pragma once
#include "la_device.cuh"

namespace la {

enum : int { CLS_NOREADS = 0, CLS_SHORT = 1, CLS_S = 2, CLS_GLOBAL = 8 };   // CLS_S + class index (5 = XL)
constexpr float SMEM_MAX_LOAD = 0.70f;

// ---- shared-memory layout ------------------------------------------------------------------------
// [info0: icap u32][info1: icap u32][walk strings: 4 x Wp][table region: B1 | B2 | keys | cnts]
// Two slot formats.  INLINE (k <= 63): 16 B key; REF (k >= 64): 8 B tag|read|pos.  + 8 B counters.
__host__ __device__ __forceinline__ bool inline_keys(int k) { return k <= 63; }
__host__ __device__ __forceinline__ uint32_t key_bytes(int k) { return inline_keys(k) ? 16u : 8u; }

struct SmemFixed {
    uint32_t icap;        // slots an info buffer can describe (max table capacity)
    uint32_t off_info1, off_walk, off_tab, tab_bytes;
};

// gt_stride > 0: the table region lives in a per-CTA global-memory scratch of gt_stride bytes (XL
// class); shared memory then holds only the two info buffers and the walk strings.
__host__ __device__ __forceinline__ SmemFixed smem_fixed(int W, uint32_t bytes, uint32_t gt_stride = 0) {
    SmemFixed F;
    const uint32_t Wp = ((uint32_t)W + 15u) & ~15u;
    const uint32_t fixed = 4u * Wp + 128u;
    const uint32_t rem = bytes > fixed ? bytes - fixed : 0u;
    F.icap = (gt_stride ? rem / 8u : rem / 32u) & ~3u;   // (24 B inline slot +) 2 x 4 B info
    F.off_info1 = F.icap * 4u;
    F.off_walk = F.off_info1 + F.icap * 4u;
    if (gt_stride) {
        F.off_tab = 0u;   // relative to the CTA's global scratch
        F.tab_bytes = gt_stride;
    } else {
        F.off_tab = (F.off_walk + 4u * Wp + 15u) & ~15u;
        F.tab_bytes = bytes > F.off_tab + 32u ? bytes - F.off_tab - 32u : 0u;
    }
    return F;
}

struct SmemTab {
    uint32_t off_pref, off_b1, off_b2, off_keys, off_cnts, cap, mwords;
};

__host__ __device__ __forceinline__ uint32_t pref_bytes(int r) { return (((uint32_t)r + 1u) * 4u + 15u) & ~15u; }

// U = voting-occurrence upper bound (sum over reads of max(0, len-k)); the table region starts with
// the per-read position prefix array (pref_bytes(r)).
__host__ __device__ __forceinline__ SmemTab smem_tab(const SmemFixed &F, uint32_t U, bool allow_filter,
                                                     uint32_t kbytes, int r) {
    SmemTab T;
    const uint32_t pb = pref_bytes(r);
    const uint32_t tab = F.tab_bytes > pb ? F.tab_bytes - pb : 0u;
    const uint32_t per_slot = kbytes + 8u;
    uint32_t cap_nf = tab / per_slot;
    if (cap_nf > F.icap) cap_nf = F.icap;
    cap_nf &= ~1u;
    uint32_t mwords = 0, cap = cap_nf;
    if (allow_filter && (float)U > SMEM_MAX_LOAD * (float)cap_nf) {
        // two bitmaps of ~4 bits per occurrence each, at most a quarter of the region each
        mwords = (4u * U + 31u) / 32u;
        const uint32_t maxw = tab / 16u;
        if (mwords > maxw) mwords = maxw;
        mwords = (mwords + 3u) & ~3u;
        const uint32_t rem = tab > 8u * mwords + 16u ? tab - 8u * mwords - 16u : 0u;
        cap = rem / per_slot;
        if (cap > F.icap) cap = F.icap;
        cap &= ~1u;
    }
    T.cap = cap;
    T.mwords = mwords;
    T.off_pref = F.off_tab;
    T.off_b1 = F.off_tab + pb;
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

__device__ __forceinline__ bool fits(int64_t r, int64_t U, const DevParams &P, uint32_t bytes, uint32_t min_cap) {
    if (bytes == 0) return false;
    const SmemFixed F = smem_fixed(P.W, bytes);
    if (F.tab_bytes == 0) return false;
    if (r > 16384) return false;
    const SmemTab T = smem_tab(F, (uint32_t)U, P.V >= 2, key_bytes(P.k_min), (int)r);
    if (T.cap < min_cap) return false;
    if (T.mwords == 0) return true;   // U <= 0.7 cap: cannot overflow
    return filtered_fraction(r) * (float)U + 64.f <= SMEM_MAX_LOAD * (float)T.cap;
}

// Shared-memory classes, smallest CTA first: (threads, CTAs/SM) = (64, 12), (128, 6), (256, 3),
// (256, 2), (512, 1); one warp of each CTA walks, the others build.  The first class whose table is
// predicted to fit wins; G = global-memory rounds.
constexpr int N_SMEM_CLASSES = 5;
struct PlanBytes {
    uint32_t b[N_SMEM_CLASSES];   // dynamic shared memory per CTA
    uint32_t t[N_SMEM_CLASSES];   // threads per CTA
};

__host__ __device__ __forceinline__ uint32_t min_table_cap(uint32_t threads) { return 4u * threads; }

// XL class: 512-thread CTAs (1 per SM) whose tables live in a per-CTA global-memory scratch (L2-resident
// for the paper-shaped batch); shared memory keeps the info buffers (so the walk stays on-chip).
constexpr int XL_THREADS = 512;
constexpr int64_t XL_MAX_U = 1 << 21;
__host__ __device__ __forceinline__ uint32_t xl_needed_cap(int64_t r, int64_t U, bool filter) {
    const float need = filter ? (filtered_fraction(r) * (float)U + 1024.f) : (float)U;
    return (uint32_t)(need / SMEM_MAX_LOAD) + 16u;
}
// bytes of one CTA's global scratch for the largest XL end (U_max occurrences, r_max reads)
__host__ __device__ __forceinline__ uint32_t xl_stride(int64_t r_max, int64_t U_max, bool filter, uint32_t icap) {
    uint32_t cap = xl_needed_cap(r_max, U_max, filter);
    if (cap > icap) cap = icap;
    const uint32_t mwords = filter ? (uint32_t)(((4 * U_max + 31) / 32 + 3) & ~3ll) : 0u;
    return (pref_bytes((int)r_max) + 8u * mwords + 32u + cap * 24u + 255u) & ~255u;
}

__global__ void k_plan(const int64_t *__restrict__ eoff, const int64_t *__restrict__ roff,
                       const int32_t *__restrict__ clen, int64_t n_ends, DevParams P, PlanBytes pb, uint32_t xl_bytes,
                       int32_t *__restrict__ cls, int32_t *__restrict__ out_len, uint8_t *__restrict__ out_term,
                       uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att, int32_t *__restrict__ lists,
                       uint32_t *__restrict__ keys, int32_t *__restrict__ list_G, int *__restrict__ ctr) {
    // ctr: [0..4] n per smem class, [5] n_G, [6] NOREADS, [7] SHORT, [8] n_XL, [9] max U_XL, [10] max r_XL
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
        if (U < (1ll << 30))
            for (int i = 0; i < N_SMEM_CLASSES && sc < 0; ++i)
                if (fits(r, U, P, pb.b[i], min_table_cap(pb.t[i]))) sc = i;
        int64_t U0 = sumlen - r * (int64_t)P.k_start;   // LPT key: occurrences at k_start
        U0 = U0 < 0 ? 0 : (U0 > 0xffffffffll ? 0xffffffffll : U0);
        if (sc < 0 && xl_bytes && r <= 16384 && U <= XL_MAX_U &&
            xl_needed_cap(r, U, P.V >= 2) <= smem_fixed(P.W, xl_bytes, 1u).icap)
            sc = N_SMEM_CLASSES;   // XL: table in global scratch
        if (sc >= 0) {
            c = CLS_S + sc;
            const int i = atomicAdd(&ctr[sc == N_SMEM_CLASSES ? 8 : sc], 1);
            lists[sc * n_ends + i] = (int32_t)e;
            keys[sc * n_ends + i] = (uint32_t)U0;
            if (sc == N_SMEM_CLASSES) {
                atomicMax(&ctr[9], (int)U);
                atomicMax(&ctr[10], (int)r);
            }
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

struct GlobalStats {
    unsigned long long inserts, steps, attempts;
};

__device__ __forceinline__ uint32_t filt_index(uint64_t h, uint32_t mbits) {
    return (uint32_t)(((h >> 32) * (uint64_t)mbits) >> 32);
}

// 128-bit compare-and-swap (ATOMS.CAS.128 / ATOMG.CAS.128, sm_90+) on a shared-memory (GT = false)
// or global-memory (GT = true) slot.  Returns the old value.
template <bool GT>
__device__ __forceinline__ void cas128(void *p, uint64_t c0, uint64_t c1, uint64_t n0, uint64_t n1, uint64_t &o0,
                                       uint64_t &o1) {
    if (GT) {
        asm volatile(
            "{\n .reg .b128 d, b, c;\n mov.b128 b, {%2, %3};\n mov.b128 c, {%4, %5};\n"
            " atom.global.cas.b128 d, [%6], b, c;\n mov.b128 {%0, %1}, d;\n}"
            : "=l"(o0), "=l"(o1)
            : "l"(c0), "l"(c1), "l"(n0), "l"(n1), "l"(p)
            : "memory");
    } else {
        const unsigned addr = (unsigned)__cvta_generic_to_shared(p);
        asm volatile(
            "{\n .reg .b128 d, b, c;\n mov.b128 b, {%2, %3};\n mov.b128 c, {%4, %5};\n"
            " atom.shared.cas.b128 d, [%6], b, c;\n mov.b128 {%0, %1}, d;\n}"
            : "=l"(o0), "=l"(o1)
            : "l"(c0), "l"(c1), "l"(n0), "l"(n1), "r"(addr)
            : "memory");
    }
}

template <bool GT>
__device__ __forceinline__ void ld128v(const uint64_t *p, uint64_t &x, uint64_t &y) {
    if (GT)
        asm volatile("ld.volatile.global.v2.u64 {%0, %1}, [%2];" : "=l"(x), "=l"(y) : "l"(p) : "memory");
    else
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
    const uint64_t *rseq;   // packed reads (global), for REF-format key verification
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
                const Kmer K2 = extract_kmer(T.rseq + (size_t)slot_read(w) * T.SW, slot_pos(w), T.k, T.KW);
                if (kmer_eq(K, K2, T.KW)) return s;
            }
            s = (s + 1 == T.cap) ? 0 : s + 1;
        }
    }
    return NONE;
}

// Alg 1 line 5 (kmer_ht.insert) with the vote of the following base.
template <bool INL, bool GT>
__device__ __forceinline__ void tab_insert(const TabCtx &T, const Kmer &K, uint64_t h, uint32_t rid, int pos,
                                           uint32_t b, bool hi, int *nclaim, int claim_limit, volatile int *ovf) {
    uint32_t s = slot_of(h, T.cap);
    if (INL) {
        uint64_t a, bb;
        inline_form(K, T.KW, a, bb);
        for (;;) {
            uint64_t x, y;
            ld128v<GT>(&T.keys[2 * s], x, y);
            if (y == 0) {   // looks empty: the CAS either claims it or returns its true content
                if (*ovf) return;
                cas128<GT>((void *)&T.keys[2 * s], 0ull, 0ull, a, bb, x, y);
                if (y == 0) {   // claimed
                    if (atomicAdd(nclaim, 1) >= claim_limit) *ovf = 1;
                    break;
                }
            } else if (y == bb && x != a) {
                // a 16 B load is not guaranteed single-copy atomic: if it raced with the claiming CAS,
                // word 0 may be stale — re-read it (a slot never changes once claimed)
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
                const Kmer K2 = extract_kmer(T.rseq + (size_t)slot_read(w) * T.SW, slot_pos(w), T.k, T.KW);
                if (kmer_eq(K, K2, T.KW)) break;
            }
            s = (s + 1 == T.cap) ? 0 : s + 1;
        }
    }
    // 32-bit ATOMS.ADD (a 64-bit shared-memory add compiles to a CAS loop)
    const uint32_t old = atomicAdd(&T.c32[2 * s], 1u << (8 * b));
    if (((old >> (8 * b)) & 0xffu) == 0xffu) *ovf = 1;   // an 8-bit lo counter would carry
    if (hi) atomicAdd(&T.c32[2 * s + 1], 1u << (8 * b));  // hi <= lo: cannot carry first
}

// Every voting occurrence of the end's reads (streamed from global memory).  The end's positions with a
// following base are numbered 0..total-1 read by read (pref[j] = first number of read j); builder bt
// takes the contiguous range [bt*total/NB, (bt+1)*total/NB), so work is balanced to one position and a
// thread extracts a k-mer only where its range enters a read, then rolls it; the following base and
// its quality class come from one 64-bit word per 32 positions.  f(K, rid, p, nb, hi) per vote.
template <typename F>
__device__ __forceinline__ void for_each_vote(const uint64_t *__restrict__ rseq, const uint64_t *__restrict__ rqc,
                                              const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag,
                                              const uint32_t *pref, int64_t r0, int r, int SW, int k, int KW,
                                              int bt, int NB, const volatile int *stop, F &&f) {
    const uint32_t total = pref[r];
    uint32_t cur = (uint32_t)(((uint64_t)total * (uint32_t)bt) / (uint32_t)NB);
    const uint32_t end = (uint32_t)(((uint64_t)total * (uint32_t)(bt + 1)) / (uint32_t)NB);
    if (cur >= end) return;
    int lo = 0, hi = r;   // read j with pref[j] <= cur < pref[j+1]
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (pref[mid] <= cur) lo = mid; else hi = mid;
    }
    int j = lo;
    while (pref[j + 1] <= cur) ++j;   // skip reads without positions
    int p = (int)(cur - pref[j]);
    while (cur < end) {
        if (*stop) return;
        const int64_t rid = r0 + j;
        const int npos = (int)(pref[j + 1] - pref[j]);   // = len - k > 0
        const int pe = min(npos, p + (int)(end - cur));
        const uint64_t *R = rseq + rid * SW;
        const uint64_t *Q = rqc + rid * SW;
        Kmer K = extract_kmer(R, p, k, KW);
        int lastN = -1;
        if (__ldg(&rflag[rid]))   // this read has an N
            for (int i = p; i < p + k; ++i)
                if (get2(Q, i) == 3u) lastN = i;
        int wi = (p + k) >> 5;
        uint64_t wR = __ldg(&R[wi]), wQ = __ldg(&Q[wi]);
        for (int q = p; q < pe; ++q) {
            const int i = q + k;
            if ((i >> 5) != wi) {
                wi = i >> 5;
                wR = __ldg(&R[wi]);
                wQ = __ldg(&Q[wi]);
            }
            const int sh = 62 - ((i & 31) << 1);
            const uint32_t nb = (uint32_t)(wR >> sh) & 3u;
            const uint32_t nq = (uint32_t)(wQ >> sh) & 3u;
            if (nq - 1u < 2u && lastN < q) f(K, (uint32_t)rid, q, nb, nq == 2u);
            if (nq == 3u) lastN = i;
            roll_kmer(K, k, KW, nb);
        }
        cur += (uint32_t)(pe - p);
        ++j;
        p = 0;
        while (cur < end && pref[j + 1] == pref[j]) ++j;
    }
}

// ---- the kernel --------------------------------------------------------------------------------
enum : int { ST_EMPTY = 0, ST_BUILD = 1, ST_WALK = 2 };

struct EndSlot {            // one contig end in flight
    int e, r;
    long long r0;
    int k, shift, kmax_eff, attempts;
    int best_len, best_term, best_k, best_buf;
    int status;             // ST_*; written after a fence, polled with volatile loads
    uint32_t start;         // the start k-mer's slot (NONE if absent) of the last build
    unsigned long long ins, steps;
};

struct BuildCtl {           // builders' shared scratch
    int slot;               // end slot chosen by the builders' leader (-1: exit)
    int overflow, nclaim;
    uint32_t start;
    uint32_t wsum[16];      // per builder warp: prefix-scan totals
};

__device__ __forceinline__ void builders_sync(int NB) { asm volatile("bar.sync 1, %0;" ::"r"(NB) : "memory"); }

template <bool INL, bool GT>
__device__ __forceinline__ void build_link(BuildCtl &B, const TabCtx &T, uint32_t *B1, uint32_t *B2, uint32_t mbits,
                                           uint32_t *info, const uint64_t *__restrict__ rqc,
                                           const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag,
                                           const uint32_t *pref, long long r0, int r, const DevParams &P,
                                           const uint64_t *tail_e, int Tn, uint64_t n0, uint64_t n1, int bt, int NB) {
    const volatile int *stop = &B.overflow;
    const int k = T.k, KW = T.KW;
    // ---- filter pass: B1 = seen once, B2 = seen at least twice (reading #4) ----
    if (mbits) {
        for_each_vote(T.rseq, rqc, rlen, rflag, pref, r0, r, T.SW, k, KW, bt, NB, stop,
                      [&](const Kmer &K, uint32_t, int, uint32_t, bool) {
                          const uint32_t fi = filt_index(hash_kmer(K, KW), mbits);
                          const uint32_t bit = 1u << (fi & 31);
                          if (!(B2[fi >> 5] & bit)) {
                              const uint32_t old = atomicOr(&B1[fi >> 5], bit);
                              if (old & bit) atomicOr(&B2[fi >> 5], bit);
                          }
                      });
        builders_sync(NB);
    }
    // ---- build (Alg 1) ----
    const int claim_limit = (int)(SMEM_MAX_LOAD * (float)T.cap);
    for_each_vote(T.rseq, rqc, rlen, rflag, pref, r0, r, T.SW, k, KW, bt, NB, stop,
                      [&](const Kmer &K, uint32_t rid, int p, uint32_t nb, bool hi) {
                          const uint64_t h = hash_kmer(K, KW);
                          if (mbits) {
                              const uint32_t fi = filt_index(h, mbits);
                              if (!((B2[fi >> 5] >> (fi & 31)) & 1u)) return;
                          }
                          tab_insert<INL, GT>(T, K, h, rid, p, nb, hi, &B.nclaim, claim_limit, &B.overflow);
                      });
    builders_sync(NB);
    if (B.overflow) return;
    // ---- ext rule + successor links (a5) into the end's info buffer ----
    for (uint32_t s = bt; s < T.cap; s += NB) {
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
            K = extract_kmer(T.rseq + (size_t)slot_read(w) * T.SW, slot_pos(w), k, KW);
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
        info[s] = (nxt << 4) | (uint32_t)code;
    }
    if (bt == 0) {
        // start k-mer: last k bases of the oriented contig (Alg 2 line 4; reading #6)
        const int p = Tn - k;
        bool hasN = false;
        for (int i = p; i < Tn; ++i) hasN |= ((i < 64 ? n0 >> i : n1 >> (i - 64)) & 1ull) != 0;
        uint32_t st = NONE;
        if (!hasN) {
            uint64_t Tw[TAIL_W];
#pragma unroll
            for (int i = 0; i < TAIL_W; ++i) Tw[i] = tail_e[i];
            const Kmer K = extract_kmer(Tw, p, k, KW);
            st = tab_lookup<INL>(T, K, hash_kmer(K, KW));
        }
        B.start = st;
    }
}

template <int BLOCK, bool GT>
__global__ void __launch_bounds__(BLOCK, 768 / BLOCK > 0 ? 768 / BLOCK : 1) k_smem(
    const int32_t *__restrict__ list, int n_list, int *__restrict__ work_ctr,
    const uint64_t *__restrict__ rseq, const uint64_t *__restrict__ rqc,
    const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag,
    const int64_t *__restrict__ eoff, const uint64_t *__restrict__ tail,
    const uint64_t *__restrict__ tailN, const int32_t *__restrict__ clen, int SW, DevParams P,
    uint32_t smem_bytes, uint8_t *__restrict__ walk_buf, int32_t *__restrict__ out_len,
    uint8_t *__restrict__ out_term, uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att,
    int32_t *__restrict__ ovf_list, int *__restrict__ n_ovf, GlobalStats *__restrict__ gstats,
    unsigned char *__restrict__ gscratch, uint32_t gstride) {
    static_assert(BLOCK >= 64, "one walker warp + at least one builder warp");
    constexpr int NB = BLOCK - 32;   // builder threads
    extern __shared__ __align__(16) unsigned char sm[];
    __shared__ EndSlot S[2];
    __shared__ BuildCtl B;
    __shared__ int builders_done;
    const int tid = threadIdx.x;
    const SmemFixed FX = smem_fixed(P.W, smem_bytes, GT ? gstride : 0u);
    // table region: shared memory, or this CTA's slice of the global scratch (XL class)
    unsigned char *tbase = GT ? gscratch + (size_t)blockIdx.x * gstride : sm;
    const int Wp = (P.W + 15) & ~15;
    uint8_t *wstr = sm + FX.off_walk;   // end slot s: buffers 2s, 2s+1 (current / best)
    if (tid == 0) {
        S[0].status = ST_EMPTY;
        S[1].status = ST_EMPTY;
        builders_done = 0;
    }
    __syncthreads();

    if (tid < 32) {
        // ============================ walker warp ============================
        const int lane = tid;
        unsigned long long acc_ins = 0, acc_steps = 0, acc_att = 0;
        int pref = 0;
        for (;;) {
            int s = -1;
            if (lane == 0) {
                for (;;) {
                    if (*(volatile int *)&S[pref].status == ST_WALK) { s = pref; break; }
                    if (*(volatile int *)&S[pref ^ 1].status == ST_WALK) { s = pref ^ 1; break; }
                    // builders finish only when both end slots are empty, so nothing is left to walk
                    if (*(volatile int *)&builders_done) break;
                    __nanosleep(32);
                }
                __threadfence_block();
            }
            s = __shfl_sync(0xffffffffu, s, 0);
            if (s < 0) break;
            pref = s ^ 1;
            EndSlot &E = S[s];
            int done = 0, bl = 0, bb = 0;
            if (lane == 0) {
                // ---- walk (Alg 2) over the successor links ----
                uint32_t *info = (uint32_t *)(sm + (s ? FX.off_info1 : 0u));
                uint8_t *wb = wstr + (2 * s + (E.best_buf ^ 1)) * Wp;
                uint32_t node = E.start == NONE ? NEXT_NONE : E.start;
                int len = 0, term = T_MAXLEN;
                unsigned long long steps = 0;
                for (int i = 0; i < P.W; ++i) {
                    ++steps;   // a lookup; the loop check of a present k-mer precedes it (below)
                    if (node == NEXT_NONE) { term = T_DEADEND; break; }
                    const uint32_t inf = info[node];
                    if (inf & 8u) { term = T_LOOP; --steps; break; }   // visited: loop check before lookup
                    info[node] = inf | 8u;
                    const uint32_t code = inf & 7u;
                    if (code == CODE_FORK) { term = T_FORK; break; }
                    if (code == CODE_DEADEND) { term = T_DEADEND; break; }
                    wb[len++] = "ACGT"[code];
                    node = inf >> 4;
                }
                E.attempts += 1;
                E.steps += steps;
                if (len > E.best_len) {   // longest walk, earliest on ties (reading #11)
                    E.best_len = len;
                    E.best_term = term;
                    E.best_k = E.k;
                    E.best_buf ^= 1;
                }
                int kk = E.k, sh = E.shift;
                done = next_k(term, kk, sh, E.kmax_eff, P) ? 1 : 0;
                E.k = kk;
                E.shift = sh;
                bl = E.best_len;
                bb = E.best_buf;
            }
            done = __shfl_sync(0xffffffffu, done, 0);
            bl = __shfl_sync(0xffffffffu, bl, 0);
            bb = __shfl_sync(0xffffffffu, bb, 0);
            if (done) {
                // ---- the selected walk -> HBM ----
                const int e = E.e;
                const uint8_t *bw = wstr + (2 * s + bb) * Wp;
                uint8_t *dst = walk_buf + (size_t)e * P.W;
                for (int i = lane; i < bl; i += 32) dst[i] = bw[i];
                if (lane == 0) {
                    out_len[e] = bl;
                    out_term[e] = (uint8_t)E.best_term;
                    out_k[e] = (uint8_t)E.best_k;
                    out_att[e] = (uint8_t)E.attempts;
                    acc_ins += E.ins;
                    acc_steps += E.steps;
                    acc_att += E.attempts;
                }
            }
            __syncwarp();
            if (lane == 0) {
                __threadfence_block();
                *(volatile int *)&E.status = done ? ST_EMPTY : ST_BUILD;
            }
        }
        if (lane == 0) {
            atomicAdd(&gstats->inserts, acc_ins);
            atomicAdd(&gstats->steps, acc_steps);
            atomicAdd(&gstats->attempts, acc_att);
        }
        return;
    }

    // ============================ builders ============================
    const int bt = tid - 32;
    int pref = 0;
    bool no_more = false;
    for (;;) {
        if (bt == 0) {
            int s = -1;
            for (;;) {
                for (int c = 0; c < 2 && s < 0; ++c) {
                    const int cand = pref ^ c;
                    const int st = *(volatile int *)&S[cand].status;
                    if (st == ST_BUILD) {
                        __threadfence_block();
                        s = cand;
                    } else if (st == ST_EMPTY && !no_more) {
                        const int idx = atomicAdd(work_ctr, 1);
                        if (idx >= n_list) { no_more = true; continue; }
                        const int e = list[idx];
                        EndSlot &E = S[cand];
                        E.e = e;
                        E.r0 = eoff[e];
                        E.r = (int)(eoff[e + 1] - E.r0);
                        E.kmax_eff = min(P.k_max, (int)clen[e]);
                        E.k = P.k_start;
                        E.shift = 0;
                        E.attempts = 0;
                        E.best_len = -1;
                        E.best_term = T_DEADEND;
                        E.best_k = 0;
                        E.best_buf = 1;
                        E.ins = 0;
                        E.steps = 0;
                        s = cand;
                    }
                }
                if (s >= 0) break;
                if (no_more && *(volatile int *)&S[0].status == ST_EMPTY && *(volatile int *)&S[1].status == ST_EMPTY)
                    break;
                __nanosleep(32);
            }
            B.slot = s;
            B.overflow = 0;
            B.nclaim = 0;
            if (s >= 0) pref = s ^ 1;
        }
        builders_sync(NB);
        const int s = B.slot;
        if (s < 0) break;
        EndSlot &E = S[s];
        const int k = E.k;
        const int KW = kwords(k);
        const bool INL = inline_keys(k);
        const long long r0 = E.r0;
        const int r = E.r;
        // positions with a following base, per read (exclusive prefix, pref[r] = U) -> table plan
        uint32_t *pref = (uint32_t *)(tbase + FX.off_tab);
        {
            const int per = (r + NB - 1) / NB;
            const int j0 = min(r, bt * per), j1 = min(r, j0 + per);
            uint32_t loc = 0;
            for (int j = j0; j < j1; ++j) loc += (uint32_t)max(0, (int)__ldg(&rlen[r0 + j]) - k);
            const int lane = bt & 31, w = bt >> 5;
            uint32_t inc = loc;
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t v = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o) inc += v;
            }
            if (lane == 31) B.wsum[w] = inc;
            builders_sync(NB);
            uint32_t off = inc - loc;
            for (int i = 0; i < w; ++i) off += B.wsum[i];
            for (int j = j0; j < j1; ++j) {
                pref[j] = off;
                off += (uint32_t)max(0, (int)__ldg(&rlen[r0 + j]) - k);
            }
            if (bt == NB - 1) pref[r] = off;   // the last builder covers the last read (or none)
            builders_sync(NB);
        }
        const uint32_t U = pref[r];
        const SmemTab TB = smem_tab(FX, U, P.V >= 2, key_bytes(k), r);
        bool ovf = TB.cap < min_table_cap(BLOCK);   // no room at this k (claims + in-flight < cap)
        if (!ovf) {
            const uint32_t mbits = TB.mwords * 32u;
            uint32_t *B1 = (uint32_t *)(tbase + TB.off_b1);
            uint32_t *B2 = (uint32_t *)(tbase + TB.off_b2);
            TabCtx T;
            T.keys = (uint64_t *)(tbase + TB.off_keys);
            T.c32 = (uint32_t *)(tbase + TB.off_cnts);
            T.cap = TB.cap;
            T.rseq = rseq;
            T.SW = SW;
            T.k = k;
            T.KW = KW;
            // clear keys + counters (contiguous) and the filters
            {
                const uint4 z = make_uint4(0, 0, 0, 0);
                uint4 *a = (uint4 *)T.keys;
                const uint32_t n16 = (TB.cap * (key_bytes(k) + 8u)) / 16u;
                for (uint32_t i = bt; i < n16; i += NB) a[i] = z;
                for (uint32_t i = bt; i < 2u * TB.mwords; i += NB) B1[i] = 0;   // B1, B2 contiguous
            }
            builders_sync(NB);
            const int e = E.e;
            const int Tn = min((int)clen[e], 128);
            const uint64_t *tail_e = tail + (size_t)e * TAIL_W;
            const uint64_t n0 = tailN[2 * (size_t)e], n1 = tailN[2 * (size_t)e + 1];
            uint32_t *info = (uint32_t *)(sm + (s ? FX.off_info1 : 0u));
            if (INL)
                build_link<true, GT>(B, T, B1, B2, mbits, info, rqc, rlen, rflag, pref, r0, r, P, tail_e, Tn, n0, n1, bt, NB);
            else
                build_link<false, GT>(B, T, B1, B2, mbits, info, rqc, rlen, rflag, pref, r0, r, P, tail_e, Tn, n0, n1, bt, NB);
            ovf = B.overflow != 0;   // uniform: last written before build_link's last barrier
        }
        builders_sync(NB);   // info buffer complete; the table is free for the next build
        if (bt == 0) {
            if (ovf) {   // table or counter overflow: the global path redoes this end from scratch
                ovf_list[atomicAdd(n_ovf, 1)] = E.e;
                __threadfence_block();
                *(volatile int *)&E.status = ST_EMPTY;
            } else {
                E.start = B.start;
                E.ins += U;
                __threadfence_block();
                *(volatile int *)&E.status = ST_WALK;
            }
        }
    }
    if (bt == 0) {
        __threadfence_block();
        *(volatile int *)&builders_done = 1;
    }
}

}  // namespace la
