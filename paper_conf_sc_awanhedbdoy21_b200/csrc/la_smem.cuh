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

enum : int { CLS_NOREADS = 0, CLS_SHORT = 1, CLS_S = 2, CLS_M = 3, CLS_GLOBAL = 4 };
constexpr float SMEM_MAX_LOAD = 0.70f;

// ---- shared-memory layout ------------------------------------------------------------------------
struct SmemFixed {            // per end: staged reads, lengths, walk buffers
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

struct SmemTab {              // per attempt: [vis bits][B1][B2][keys u64][cnts u64]
    uint32_t off_vis, off_b1, off_b2, off_keys, off_cnts, cap, mwords;
};

// U = voting-occurrence upper bound (sum over reads of max(0, len-k)).
__host__ __device__ __forceinline__ SmemTab smem_tab(uint32_t off_var, uint32_t var_bytes, uint32_t U,
                                                     bool allow_filter) {
    SmemTab T;
    // unfiltered: 16 B per slot + 1 visited bit
    uint32_t cap_nf = (uint32_t)(((uint64_t)var_bytes * 8u) / 129u) & ~1u;
    uint32_t mwords = 0;
    uint32_t cap = cap_nf;
    if (allow_filter && (float)U > SMEM_MAX_LOAD * (float)cap_nf) {
        // two bitmaps of ~4 bits per occurrence each, at most a quarter of the region each
        mwords = (4u * U + 31u) / 32u;
        const uint32_t maxw = var_bytes / 16u;
        if (mwords > maxw) mwords = maxw;
        mwords = (mwords + 3u) & ~3u;
        const uint32_t rem = var_bytes > 8u * mwords ? var_bytes - 8u * mwords : 0u;
        cap = (uint32_t)(((uint64_t)rem * 8u) / 129u) & ~1u;
    }
    T.cap = cap;
    T.mwords = mwords;
    T.off_vis = off_var;
    T.off_b1 = (off_var + ((cap + 31u) / 32u) * 4u + 15u) & ~15u;
    T.off_b2 = T.off_b1 + mwords * 4u;
    T.off_keys = (T.off_b2 + mwords * 4u + 15u) & ~15u;
    T.off_cnts = T.off_keys + cap * 8u;
    return T;
}

// ---- plan ------------------------------------------------------------------------------------
// Routing estimate of the filtered table: distinct k-mers with >= 2 voting occurrences plus filter
// false positives, as a fraction of the occurrences (measured on C2/C4 samples: 0.05-0.2, higher for
// ends with few reads).  A wrong guess only costs a redo in the global path.
__host__ __device__ __forceinline__ float filtered_fraction(int64_t r) {
    return r < 50 ? 0.30f : (r < 200 ? 0.16f : 0.10f);
}

__device__ __forceinline__ bool fits(int64_t r, int64_t U, int SW, const DevParams &P, uint32_t bytes) {
    if (bytes == 0) return false;
    const SmemFixed F = smem_fixed((int)r, SW, P.W, bytes);
    if (F.var_bytes == 0) return false;
    const SmemTab T = smem_tab(F.off_var, F.var_bytes, (uint32_t)U, P.V >= 2);
    if (T.cap < 512) return false;
    if (T.mwords == 0) return true;   // U <= 0.7 cap: cannot overflow
    return filtered_fraction(r) * (float)U + 64.f <= SMEM_MAX_LOAD * (float)T.cap;
}

__global__ void k_plan(const int64_t *__restrict__ eoff, const int64_t *__restrict__ roff,
                       const int32_t *__restrict__ clen, int64_t n_ends, DevParams P, int SW,
                       uint32_t bytes_S, uint32_t bytes_M, int32_t *__restrict__ cls,
                       int32_t *__restrict__ out_len, uint8_t *__restrict__ out_term,
                       uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att,
                       int32_t *__restrict__ list_S, uint32_t *__restrict__ key_S,
                       int32_t *__restrict__ list_M, uint32_t *__restrict__ key_M,
                       int32_t *__restrict__ list_G, int *__restrict__ ctr) {
    // ctr: [0] n_S [1] n_M [2] n_G [3] NOREADS [4] SHORT
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
        if (r < 65536 && U < (1ll << 31)) {
            if (fits(r, U, SW, P, bytes_S)) c = CLS_S;
            else if (fits(r, U, SW, P, bytes_M)) c = CLS_M;
        }
        int64_t U0 = sumlen - r * (int64_t)P.k_start;   // LPT key: occurrences at k_start
        U0 = U0 < 0 ? 0 : (U0 > 0xffffffffll ? 0xffffffffll : U0);
        const uint32_t key = (uint32_t)U0;
        if (c == CLS_S) { int i = atomicAdd(&ctr[0], 1); list_S[i] = (int32_t)e; key_S[i] = key; }
        else if (c == CLS_M) { int i = atomicAdd(&ctr[1], 1); list_M[i] = (int32_t)e; key_M[i] = key; }
        else { int i = atomicAdd(&ctr[2], 1); list_G[i] = (int32_t)e; }
    }
    cls[e] = c;
    if (c == CLS_NOREADS || c == CLS_SHORT) {
        atomicAdd(&ctr[c == CLS_NOREADS ? 3 : 4], 1);
        out_len[e] = 0;
        out_term[e] = c == CLS_NOREADS ? T_NOREADS : T_SHORT;
        out_k[e] = 0;
        out_att[e] = 0;
    }
}

// ---- table operations ------------------------------------------------------------------------------
struct SmemCtl {
    int end_idx, overflow, nclaim;
    int k, shift, kmax_eff, done, attempts;
    int best_len, best_term, best_k, best_buf;
    int maxlen, hasN_any;
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

__device__ __forceinline__ uint32_t tab_lookup(const uint64_t *keys, uint32_t cap, const Kmer &K, uint64_t h,
                                               int k, int KW, const uint64_t *sseq, uint32_t rbase, int SW) {
    const uint64_t tag = tag_of(h);
    uint32_t s = slot_of(h, cap);
    for (uint32_t n = 0; n < cap; ++n) {
        const uint64_t w = keys[s];
        if (w == 0) return NONE;
        if ((w & TAG_MASK) == tag) {
            const Kmer K2 = extract_kmer(sseq + (size_t)(slot_read(w) - rbase) * SW, slot_pos(w), k, KW);
            if (kmer_eq(K, K2, KW)) return s;
        }
        s = (s + 1 == cap) ? 0 : s + 1;
    }
    return NONE;
}

// Alg 1 line 5 (kmer_ht.insert) with the vote of the following base.
__device__ __forceinline__ void tab_insert(uint64_t *keys, unsigned long long *cnts, uint32_t cap,
                                           const Kmer &K, uint64_t h, int k, int KW, uint32_t rid, int pos,
                                           uint32_t b, bool hi, const uint64_t *sseq, uint32_t rbase,
                                           int SW, int *nclaim, int claim_limit, volatile int *ovf) {
    const uint64_t tag = tag_of(h);
    uint32_t s = slot_of(h, cap);
    volatile uint64_t *vk = keys;
    uint32_t *c32 = (uint32_t *)cnts;   // per slot: word 0 = lo[4] (8 bits each), word 1 = hi[4]
    for (;;) {
        uint64_t w = vk[s];
        bool hit = false;
        if (w == 0) {
            if (*ovf) return;
            const uint64_t mine = make_slot(tag, rid, (uint32_t)pos);
            const uint64_t old = atomicCAS((unsigned long long *)&keys[s], 0ull, (unsigned long long)mine);
            if (old == 0) {
                hit = true;
                if (atomicAdd(nclaim, 1) >= claim_limit) *ovf = 1;
            } else {
                w = old;
            }
        }
        if (!hit && (w & TAG_MASK) == tag) {
            const Kmer K2 = extract_kmer(sseq + (size_t)(slot_read(w) - rbase) * SW, slot_pos(w), k, KW);
            hit = kmer_eq(K, K2, KW);
        }
        if (hit) {   // 32-bit ATOMS.ADD (a 64-bit smem add would be a CAS loop)
            const uint32_t old = atomicAdd(&c32[2 * s], 1u << (8 * b));
            if (((old >> (8 * b)) & 0xffu) == 0xffu) *ovf = 1;   // 8-bit lo counter would carry
            if (hi) atomicAdd(&c32[2 * s + 1], 1u << (8 * b));    // hi <= lo: cannot carry first
            return;
        }
        s = (s + 1 == cap) ? 0 : s + 1;
    }
}

template <int BLOCK>
__global__ void __launch_bounds__(BLOCK, BLOCK >= 512 ? 1 : 3) k_smem(
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
        uint64_t *sseq = (uint64_t *)sm;
        uint64_t *sqc = (uint64_t *)(sm + FX.off_qc);
        uint16_t *slen = (uint16_t *)(sm + FX.off_len);
        uint8_t *swalk = sm + FX.off_walk;   // two buffers of Wp bytes
        const int Wp = (P.W + 15) & ~15;
        if (FX.var_bytes < 2048u) {   // reads do not fit at all: the global path takes this end
            if (tid == 0) ovf_list[atomicAdd(n_ovf, 1)] = e;
            continue;
        }

        // stage the end's packed reads (contiguous in HBM): coalesced 16 B loads
        {
            const int nw = r * SW;
            if ((SW & 1) == 0) {
                const uint4 *gs = (const uint4 *)(rseq + r0 * SW);
                const uint4 *gq = (const uint4 *)(rqc + r0 * SW);
                uint4 *ss = (uint4 *)sseq;
                uint4 *sq = (uint4 *)sqc;
                for (int i = tid; i < nw / 2; i += BLOCK) { ss[i] = gs[i]; sq[i] = gq[i]; }
            } else {
                for (int i = tid; i < nw; i += BLOCK) { sseq[i] = rseq[r0 * SW + i]; sqc[i] = rqc[r0 * SW + i]; }
            }
            int ml = 0, hn = 0;
            for (int i = tid; i < r; i += BLOCK) {
                const int l = rlen[r0 + i];
                slen[i] = (uint16_t)l;
                ml = max(ml, l);
                hn |= rflag[r0 + i];
            }
            for (int o = 16; o; o >>= 1) {
                ml = max(ml, __shfl_xor_sync(0xffffffffu, ml, o));
                hn |= __shfl_xor_sync(0xffffffffu, hn, o);
            }
            if (tid == 0) {
                C.maxlen = 0;
                C.hasN_any = 0;
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
            if (lane == 0) { atomicMax(&C.maxlen, ml); atomicOr(&C.hasN_any, hn); }
        }
        __syncthreads();
        const int maxlen = C.maxlen;
        const bool anyN = C.hasN_any != 0;

        // ---------------- retry loop ----------------
        for (;;) {
            const int k = C.k;
            const int KW = kwords(k);
            // voting-occurrence bound at this k -> table plan
            {
                unsigned long long u = 0;
                for (int i = tid; i < r; i += BLOCK) u += (unsigned)max(0, (int)slen[i] - k);
                for (int o = 16; o; o >>= 1) u += __shfl_xor_sync(0xffffffffu, u, o);
                if (tid == 0) C.U = 0;
                __syncthreads();
                if (lane == 0 && u) atomicAdd(&C.U, u);
                __syncthreads();
            }
            const uint32_t U = (uint32_t)C.U;
            const SmemTab T = smem_tab(FX.off_var, FX.var_bytes, U, P.V >= 2);
            const uint32_t cap = T.cap;
            if (cap < 128u) {   // no room for a table at this k
                if (tid == 0) C.overflow = 1;
                __syncthreads();
                break;
            }
            const uint32_t mbits = T.mwords * 32u;
            uint32_t *svis = (uint32_t *)(sm + T.off_vis);
            uint32_t *B1 = (uint32_t *)(sm + T.off_b1);
            uint32_t *B2 = (uint32_t *)(sm + T.off_b2);
            uint64_t *keys = (uint64_t *)(sm + T.off_keys);
            unsigned long long *cnts = (unsigned long long *)(sm + T.off_cnts);
            // clear keys, counters, visited bits and filters
            {
                const uint4 z = make_uint4(0, 0, 0, 0);
                uint4 *a = (uint4 *)keys;
                for (uint32_t i = tid; i < cap; i += BLOCK) a[i] = z;   // keys + cnts: 16 B per slot
                for (uint32_t i = tid; i < (cap + 31u) / 32u; i += BLOCK) svis[i] = 0;
                for (uint32_t i = tid; i < 2u * T.mwords; i += BLOCK) B1[i] = 0;   // B1, B2 contiguous
                if (tid == 0) C.nclaim = 0;
            }
            __syncthreads();

            const int nseg = maxlen > k ? ((maxlen - k + 15) >> 4) : 0;
            const int items = r * nseg;

            // ---- filter pass: B1 = seen once, B2 = seen at least twice ----
            if (mbits) {
                for (int it = tid; it < items; it += BLOCK) {
                    const int j = it / nseg;
                    const int sg = it - j * nseg;
                    const int len = slen[j];
                    const int p0 = sg << 4;
                    const int p1 = min(p0 + 16, len - k);
                    if (p0 >= p1) continue;
                    const uint64_t *R = sseq + (size_t)j * SW;
                    const uint64_t *Q = sqc + (size_t)j * SW;
                    Kmer K = extract_kmer(R, p0, k, KW);
                    int lastN = -1;
                    if (anyN)
                        for (int i = p0; i < p0 + k; ++i)
                            if (get2(Q, i) == 3u) lastN = i;
                    for (int p = p0; p < p1; ++p) {
                        const uint32_t nb = get2(R, p + k);
                        const uint32_t nq = get2(Q, p + k);
                        if ((nq == 1u || nq == 2u) && lastN < p) {
                            const uint32_t fi = filt_index(hash_kmer(K, KW), mbits);
                            const uint32_t bit = 1u << (fi & 31);
                            if (!(B2[fi >> 5] & bit)) {
                                const uint32_t old = atomicOr(&B1[fi >> 5], bit);
                                if (old & bit) atomicOr(&B2[fi >> 5], bit);
                            }
                        }
                        if (nq == 3u) lastN = p + k;
                        roll_kmer(K, k, KW, nb);
                    }
                }
                __syncthreads();
            }

            // ---- build (Alg 1) ----
            unsigned long long my_ins = 0;
            {
                const int claim_limit = (int)(SMEM_MAX_LOAD * (float)cap);
                for (int it = tid; it < items; it += BLOCK) {
                    if (*(volatile int *)&C.overflow) break;
                    const int j = it / nseg;
                    const int sg = it - j * nseg;
                    const int len = slen[j];
                    const int p0 = sg << 4;
                    const int p1 = min(p0 + 16, len - k);
                    if (p0 >= p1) continue;
                    my_ins += (unsigned)(p1 - p0);
                    const uint64_t *R = sseq + (size_t)j * SW;
                    const uint64_t *Q = sqc + (size_t)j * SW;
                    Kmer K = extract_kmer(R, p0, k, KW);
                    int lastN = -1;
                    if (anyN)
                        for (int i = p0; i < p0 + k; ++i)
                            if (get2(Q, i) == 3u) lastN = i;
                    for (int p = p0; p < p1; ++p) {
                        const uint32_t nb = get2(R, p + k);
                        const uint32_t nq = get2(Q, p + k);
                        if ((nq == 1u || nq == 2u) && lastN < p) {
                            const uint64_t h = hash_kmer(K, KW);
                            bool keep = true;
                            if (mbits) {
                                const uint32_t fi = filt_index(h, mbits);
                                keep = (B2[fi >> 5] >> (fi & 31)) & 1u;
                            }
                            if (keep)
                                tab_insert(keys, cnts, cap, K, h, k, KW, (uint32_t)(r0 + j), p, nb, nq == 2u, sseq,
                                           (uint32_t)r0, SW, &C.nclaim, claim_limit, &C.overflow);
                        }
                        if (nq == 3u) lastN = p + k;
                        roll_kmer(K, k, KW, nb);
                    }
                }
            }
            for (int o = 16; o; o >>= 1) my_ins += __shfl_xor_sync(0xffffffffu, my_ins, o);
            if (lane == 0 && my_ins) atomicAdd(&C.end_ins, my_ins);
            __syncthreads();
            if (C.overflow) break;

            // ---- ext rule + successor links (a5): info = next_slot << 3 | code ----
            for (uint32_t s = tid; s < cap; s += BLOCK) {
                const uint64_t w = keys[s];
                if (w == 0) continue;
                const unsigned long long c8 = cnts[s];
                uint32_t lo[4], hi[4];
#pragma unroll
                for (int b = 0; b < 4; ++b) {
                    lo[b] = (uint32_t)(c8 >> (8 * b)) & 0xffu;
                    hi[b] = (uint32_t)(c8 >> (32 + 8 * b)) & 0xffu;
                }
                const int code = ext_rule(lo, hi, P.V, P.F);
                uint32_t nxt = NONE;
                if (code < 4) {
                    Kmer K = extract_kmer(sseq + (size_t)(slot_read(w) - (uint32_t)r0) * SW, slot_pos(w), k, KW);
                    roll_kmer(K, k, KW, (uint32_t)code);
                    nxt = tab_lookup(keys, cap, K, hash_kmer(K, KW), k, KW, sseq, (uint32_t)r0, SW);
                }
                cnts[s] = (unsigned long long)((nxt << 3) | (uint32_t)code);
            }
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
                    C.start_slot = tab_lookup(keys, cap, K, hash_kmer(K, KW), k, KW, sseq, (uint32_t)r0, SW);
                }
            }
            __syncthreads();

            // ---- walk (Alg 2) + retry decision, one thread ----
            if (tid == 0) {
                uint8_t *wb = swalk + (C.best_buf ^ 1) * Wp;
                uint32_t node = C.start_slot;
                int len = 0, term = T_MAXLEN;
                unsigned long long steps = 0;
                const uint32_t *info = (const uint32_t *)cnts;   // low word of each 8 B counter slot
                for (int i = 0; i < P.W; ++i) {
                    if (node != NONE) {   // loop check before lookup (Alg 2 lines 6-8)
                        const uint32_t bit = 1u << (node & 31);
                        const uint32_t v = svis[node >> 5];
                        if (v & bit) { term = T_LOOP; break; }
                        svis[node >> 5] = v | bit;
                    }
                    ++steps;
                    if (node == NONE) { term = T_DEADEND; break; }
                    const uint32_t inf = info[2 * node];
                    const uint32_t code = inf & 7u;
                    if (code == CODE_FORK) { term = T_FORK; break; }
                    if (code == CODE_DEADEND) { term = T_DEADEND; break; }
                    wb[len++] = "ACGT"[code];
                    node = inf >> 3;
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
