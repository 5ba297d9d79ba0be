// la_kernels.cuh — sm_100a kernels of the local-assembly hot path.
//
//   encode:   ASCII reads/quals -> 2-bit bases + 2-bit quality class, oriented per end (a2, a8)
//   plan:     per end: NOREADS / SHORT / SMEM / GLOBAL class (a3, bins of P:L508-556)
//   smem:     persistent CTA per end: table in shared memory, Alg 1 build (a4), ext rule and
//             successor links (a5), single-thread mer-walk (a6), k-shift retry (a7) in-kernel
//   global:   round-synchronous path for ends whose table exceeds shared memory: L2/HBM table,
//             many CTAs per end, one thread per end walks
//   emit:     compaction of the walks into ext_off / ext_seq, reverse complement of LEFT ends (a9)
#pragma once
#include "la_device.cuh"

namespace la {

// ------------------------------------------------------------------------------------------------
// validation + encode (la_load_batch)
// ------------------------------------------------------------------------------------------------
enum : uint32_t {
    ERR_OFFSETS = 1u,       // non-monotone offsets
    ERR_READ_LEN = 2u,      // read longer than 300
    ERR_READ_CHAR = 4u,     // read base outside ACGTN
    ERR_QUAL_CHAR = 8u,     // quality below qual_offset
    ERR_CONTIG_CHAR = 16u,  // contig base outside ACGTN
};

__device__ __forceinline__ int base_code(unsigned char c) {
    switch (c) {
        case 'A': return 0;
        case 'C': return 1;
        case 'G': return 2;
        case 'T': return 3;
        case 'N': return 4;
        default: return -1;
    }
}

// offsets monotone; per-read length <= 300; max length
__global__ void k_check_offsets(const int64_t *__restrict__ off, int64_t n, int is_reads,
                                uint32_t *err, int *maxlen) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int len = 0;
    if (i < n) {
        int64_t d = off[i + 1] - off[i];
        if (d < 0) atomicOr(err, ERR_OFFSETS);
        if (is_reads && d > MAX_READ_LEN) atomicOr(err, ERR_READ_LEN);
        len = d > 0 ? (int)(d > 1000000 ? 1000000 : d) : 0;
    }
    if (maxlen) {
        for (int o = 16; o; o >>= 1) len = max(len, __shfl_xor_sync(0xffffffffu, len, o));
        if ((threadIdx.x & 31) == 0 && len) atomicMax(maxlen, len);
    }
}

// read -> end id (binary search in end_read_off); stored as side bit + end
__global__ void k_read_end(const int64_t *__restrict__ eoff, int64_t n_ends, int64_t n_reads,
                           int32_t *__restrict__ read_end) {
    int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (j >= n_reads) return;
    int64_t lo = 0, hi = n_ends;  // find e with eoff[e] <= j < eoff[e+1]
    while (hi - lo > 1) {
        int64_t mid = (lo + hi) >> 1;
        if (eoff[mid] <= j) lo = mid; else hi = mid;
    }
    read_end[j] = (int32_t)lo;
}

// one thread per (read, 32-base word): oriented 2-bit bases and quality classes.
// LEFT-end reads are reverse complemented with reversed qualities (reading #14).
__global__ void k_encode_reads(const char *__restrict__ seq, const char *__restrict__ qual,
                               const int64_t *__restrict__ roff, const int32_t *__restrict__ read_end,
                               int64_t n_reads, int SW, DevParams P, uint64_t *__restrict__ rseq,
                               uint64_t *__restrict__ rqc, uint16_t *__restrict__ rlen,
                               uint8_t *__restrict__ rflag, uint32_t *err) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t j = t / SW;
    int w = (int)(t - j * SW);
    if (j >= n_reads) return;
    const int64_t o = roff[j];
    const int len = (int)(roff[j + 1] - o);
    const bool left = (read_end[j] & 1) == 0;
    uint64_t sb = 0, qb = 0;
    uint32_t e = 0;
    bool hasN = false;
    for (int i = 0; i < 32; ++i) {
        int ib = w * 32 + i;
        uint32_t code = 0, qc = 0;
        if (ib < len) {
            int64_t src = left ? o + len - 1 - ib : o + ib;
            int c = base_code((unsigned char)seq[src]);
            int q = (int)(unsigned char)qual[src] - P.qual_offset;
            if (c < 0) { e |= ERR_READ_CHAR; c = 4; }
            if (q < 0) e |= ERR_QUAL_CHAR;
            if (c == 4) { code = 0; qc = 3; hasN = true; }
            else {
                code = left ? 3 - c : c;
                qc = q >= P.q_hi ? 2 : (q >= P.q_lo ? 1 : 0);
            }
        }
        sb |= (uint64_t)code << (62 - 2 * i);
        qb |= (uint64_t)qc << (62 - 2 * i);
    }
    rseq[j * SW + w] = sb;
    rqc[j * SW + w] = qb;
    if (e) atomicOr(err, e);
    if (w == 0) rlen[j] = (uint16_t)len;
    if (hasN) rflag[j] = 1;   // rflag zeroed before launch
}

__global__ void k_check_contigs(const char *__restrict__ cseq, int64_t n, uint32_t *err) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n && base_code((unsigned char)cseq[i]) < 0) atomicOr(err, ERR_CONTIG_CHAR);
}

// per end: the oriented contig tail (last <= 128 bases of the oriented contig), packed, + N mask
constexpr int TAIL_W = 5;   // 4 words of bases + 1 pad word
__global__ void k_encode_tails(const char *__restrict__ cseq, const int64_t *__restrict__ coff,
                               int64_t n_ends, uint64_t *__restrict__ tail, uint64_t *__restrict__ tailN,
                               int32_t *__restrict__ clen) {
    int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (e >= n_ends) return;
    const int64_t c = e >> 1;
    const int64_t o = coff[c];
    const int64_t L = coff[c + 1] - o;
    const int T = (int)(L < 128 ? L : 128);
    const bool left = (e & 1) == 0;
    uint64_t w[TAIL_W] = {0, 0, 0, 0, 0};
    uint64_t nm[2] = {0, 0};
    for (int i = 0; i < T; ++i) {
        // oriented contig: RIGHT = C, LEFT = rc(C); its last T bases
        int c2;
        if (left) {
            int cc = base_code((unsigned char)cseq[o + T - 1 - i]);
            c2 = (cc < 0 || cc == 4) ? 4 : 3 - cc;
        } else {
            int cc = base_code((unsigned char)cseq[o + L - T + i]);
            c2 = cc < 0 ? 4 : cc;
        }
        if (c2 == 4) { nm[i >> 6] |= 1ull << (i & 63); c2 = 0; }
        w[i >> 5] |= (uint64_t)c2 << (62 - 2 * (i & 31));
    }
    for (int i = 0; i < TAIL_W; ++i) tail[e * TAIL_W + i] = w[i];
    tailN[2 * e] = nm[0];
    tailN[2 * e + 1] = nm[1];
    clen[e] = (int32_t)(L > 0x7fffffff ? 0x7fffffff : L);
}

// ------------------------------------------------------------------------------------------------
// plan (la_extend)
// ------------------------------------------------------------------------------------------------
enum : int { CLS_NOREADS = 0, CLS_SHORT = 1, CLS_SMEM = 2, CLS_GLOBAL = 3 };

struct SmemLayout {   // per-end shared memory layout of the SMEM kernel
    uint32_t off_qc, off_len, off_walk, off_vis, off_slots, off_cnt, cap;
};

__host__ __device__ __forceinline__ SmemLayout smem_layout(int r, int SW, int W, uint32_t bytes) {
    SmemLayout L;
    uint32_t rs = (uint32_t)r * SW * 8u;
    L.off_qc = rs;
    L.off_len = 2 * rs;
    L.off_walk = (L.off_len + 2u * r + 15u) & ~15u;
    L.off_vis = (L.off_walk + 2u * (((uint32_t)W + 15u) & ~15u) + 15u) & ~15u;
    uint32_t fixed = L.off_vis + 64u;
    uint32_t rem = bytes > fixed ? bytes - fixed : 0u;
    uint32_t cap = (uint32_t)(((uint64_t)rem * 8u) / 193u) & ~1u;   // 8 B slot + 16 B counts + 1 bit
    L.cap = cap;
    uint32_t visb = ((cap + 31u) / 32u) * 4u;
    L.off_slots = (L.off_vis + visb + 15u) & ~15u;
    L.off_cnt = L.off_slots + cap * 8u;
    if (L.off_cnt + cap * 16u > bytes) {   // rounding slack
        L.cap = cap > 16 ? cap - 16 : 0;   // stays even
        L.off_cnt = L.off_slots + L.cap * 8u;
    }
    return L;
}

constexpr float SMEM_MAX_LOAD = 0.70f;   // claims beyond this fraction of cap -> overflow

__global__ void k_plan(const int64_t *__restrict__ eoff, const int64_t *__restrict__ roff,
                       const int32_t *__restrict__ clen, int64_t n_ends, DevParams P, int SW,
                       uint32_t smem_bytes, float pred_distinct, int32_t *__restrict__ cls,
                       int32_t *__restrict__ out_len, uint8_t *__restrict__ out_term,
                       uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att,
                       int32_t *smem_list, uint32_t *smem_key, int *n_smem, int32_t *glob_list,
                       int *n_glob, int *n_special) {
    int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (e >= n_ends) return;
    const int64_t r = eoff[e + 1] - eoff[e];
    int c;
    if (r == 0) c = CLS_NOREADS;
    else if (clen[e] < P.k_start) c = CLS_SHORT;
    else {
        const int64_t sumlen = roff[eoff[e + 1]] - roff[eoff[e]];
        int64_t U = sumlen - r * (int64_t)P.k_start;
        if (U < 0) U = 0;
        c = CLS_GLOBAL;
        if (sumlen < 65536 && r < 4096) {   // 16-bit counters are exact while inserts < 65536
            SmemLayout L = smem_layout((int)r, SW, P.W, smem_bytes);
            if (L.cap >= 1024 && (float)U * pred_distinct <= SMEM_MAX_LOAD * (float)L.cap) c = CLS_SMEM;
        }
        if (c == CLS_SMEM) {
            int i = atomicAdd(n_smem, 1);
            smem_list[i] = (int32_t)e;
            smem_key[i] = (uint32_t)U;
        } else {
            int i = atomicAdd(n_glob, 1);
            glob_list[i] = (int32_t)e;
        }
    }
    cls[e] = c;
    if (c == CLS_NOREADS || c == CLS_SHORT) {
        atomicAdd(&n_special[c], 1);
        out_len[e] = 0;
        out_term[e] = c == CLS_NOREADS ? T_NOREADS : T_SHORT;
        out_k[e] = 0;
        out_att[e] = 0;
    }
}

// ------------------------------------------------------------------------------------------------
// shared-memory table kernel
// ------------------------------------------------------------------------------------------------
struct SmemCtl {
    int end_idx;
    int overflow;
    int nclaim;
    int k, shift, kmax_eff, done, attempts;
    int best_len, best_term, best_k, best_buf;
    int r, maxlen, hasN_any;
    unsigned long long inserts;                 // this attempt
    unsigned long long end_ins, end_steps;      // this end (counted only if it completes here)
    uint32_t start_slot;
};

struct GlobalStats {
    unsigned long long inserts, steps, attempts;
};

__device__ __forceinline__ uint32_t smem_lookup(const uint64_t *slots, uint32_t cap, const Kmer &K,
                                                int k, int KW, const uint64_t *sseq, uint32_t rbase,
                                                int SW) {
    const uint64_t h = hash_kmer(K, KW);
    const uint64_t tag = tag_of(h);
    uint32_t s = slot_of(h, cap);
    for (uint32_t n = 0; n < cap; ++n) {
        const uint64_t w = slots[s];
        if (w == 0) return NONE;
        if ((w & TAG_MASK) == tag) {
            Kmer K2 = extract_kmer(sseq + (size_t)(slot_read(w) - rbase) * SW, slot_pos(w), k, KW);
            if (kmer_eq(K, K2, KW)) return s;
        }
        s = (s + 1 == cap) ? 0 : s + 1;
    }
    return NONE;
}

// Alg 1 line 5, kmer_ht.insert(k) with the vote for the following base.
__device__ __forceinline__ void smem_insert(uint64_t *slots, uint32_t *cnt, uint32_t cap,
                                            const Kmer &K, int k, int KW, uint32_t rid, int pos,
                                            uint32_t b, uint32_t inc, const uint64_t *sseq,
                                            uint32_t rbase, int SW, int *nclaim, int claim_limit,
                                            volatile int *ovf) {
    const uint64_t h = hash_kmer(K, KW);
    const uint64_t tag = tag_of(h);
    uint32_t s = slot_of(h, cap);
    volatile uint64_t *vs = slots;
    for (;;) {
        uint64_t w = vs[s];
        if (w == 0) {
            if (*ovf) return;
            const uint64_t mine = make_slot(tag, rid, (uint32_t)pos);
            const uint64_t old = atomicCAS((unsigned long long *)&slots[s], 0ull, (unsigned long long)mine);
            if (old == 0) {
                atomicAdd(&cnt[4 * s + b], inc);
                if (atomicAdd(nclaim, 1) >= claim_limit) *ovf = 1;
                return;
            }
            w = old;
        }
        if ((w & TAG_MASK) == tag) {
            Kmer K2 = extract_kmer(sseq + (size_t)(slot_read(w) - rbase) * SW, slot_pos(w), k, KW);
            if (kmer_eq(K, K2, KW)) {
                atomicAdd(&cnt[4 * s + b], inc);
                return;
            }
        }
        s = (s + 1 == cap) ? 0 : s + 1;
    }
}

template <int BLOCK>
__global__ void __launch_bounds__(BLOCK) k_smem(
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
        const SmemLayout L = smem_layout(r, SW, P.W, smem_bytes);
        uint64_t *sseq = (uint64_t *)sm;
        uint64_t *sqc = (uint64_t *)(sm + L.off_qc);
        uint16_t *slen = (uint16_t *)(sm + L.off_len);
        uint8_t *swalk = sm + L.off_walk;   // two buffers of Wp bytes
        const int Wp = (P.W + 15) & ~15;
        uint32_t *svis = (uint32_t *)(sm + L.off_vis);
        uint64_t *slots = (uint64_t *)(sm + L.off_slots);
        uint32_t *cnt = (uint32_t *)(sm + L.off_cnt);
        const uint32_t cap = L.cap;

        // stage the end's packed reads (contiguous in HBM): coalesced 16 B loads
        {
            const uint4 *gs = (const uint4 *)(rseq + r0 * SW);
            const uint4 *gq = (const uint4 *)(rqc + r0 * SW);
            uint4 *ss = (uint4 *)sseq;
            uint4 *sq = (uint4 *)sqc;
            const int nv = r * SW / 2;   // SW even
            for (int i = tid; i < nv; i += BLOCK) { ss[i] = gs[i]; sq[i] = gq[i]; }
            int ml = 0, hn = 0;
            for (int i = tid; i < r; i += BLOCK) {
                int l = rlen[r0 + i];
                slen[i] = (uint16_t)l;
                ml = max(ml, l);
                hn |= rflag[r0 + i];
            }
            for (int o = 16; o; o >>= 1) {
                ml = max(ml, __shfl_xor_sync(0xffffffffu, ml, o));
                hn |= __shfl_xor_sync(0xffffffffu, hn, o);
            }
            if (tid == 0) { C.maxlen = 0; C.hasN_any = 0; }
            __syncthreads();
            if ((tid & 31) == 0) { atomicMax(&C.maxlen, ml); atomicOr(&C.hasN_any, hn); }
        }
        if (tid == 0) {
            const int kmax_eff = min(P.k_max, (int)clen[e]);
            C.kmax_eff = kmax_eff;
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
        const int maxlen = C.maxlen;
        const bool anyN = C.hasN_any != 0;

        // ---------------- retry loop ----------------
        for (;;) {
            const int k = C.k;
            const int KW = kwords(k);
            // clear the table, the visited bits
            {
                uint4 z = make_uint4(0, 0, 0, 0);
                uint4 *a = (uint4 *)slots;
                const uint32_t n8 = (cap * 8u) / 16u;
                for (uint32_t i = tid; i < n8; i += BLOCK) a[i] = z;
                if ((cap & 1u) && tid == 0) slots[cap - 1] = 0;
                uint4 *b4 = (uint4 *)cnt;
                for (uint32_t i = tid; i < cap; i += BLOCK) b4[i] = z;
                for (uint32_t i = tid; i < (cap + 31) / 32; i += BLOCK) svis[i] = 0;
                if (tid == 0) { C.nclaim = 0; C.inserts = 0; }
            }
            __syncthreads();

            // ---- build (Alg 1): thread per (read, 16-position segment) ----
            const int npos_max = maxlen - k;   // positions with a following base
            unsigned long long my_ins = 0;
            if (npos_max > 0) {
                const int nseg = (npos_max + 15) >> 4;
                const int items = r * nseg;
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
                    int lastN = -1;   // last N position among bases < p + k
                    if (anyN) {
                        for (int i = p0; i < p0 + k; ++i)
                            if (get2(Q, i) == 3u) lastN = i;
                    }
                    for (int p = p0; p < p1; ++p) {
                        const uint32_t nb = get2(R, p + k);
                        const uint32_t nq = get2(Q, p + k);
                        if ((nq == 1u || nq == 2u) && lastN < p) {
                            const uint32_t inc = nq == 2u ? 0x00010001u : 0x00000001u;
                            smem_insert(slots, cnt, cap, K, k, KW, (uint32_t)(r0 + j), p, nb, inc,
                                        sseq, (uint32_t)r0, SW, &C.nclaim, claim_limit, &C.overflow);
                        }
                        if (nq == 3u) lastN = p + k;
                        roll_kmer(K, k, KW, nb);
                    }
                }
            }
            for (int o = 16; o; o >>= 1) my_ins += __shfl_xor_sync(0xffffffffu, my_ins, o);
            if ((tid & 31) == 0 && my_ins) atomicAdd(&C.inserts, my_ins);
            __syncthreads();
            if (C.overflow) break;

            // ---- ext rule + successor links (a5): info = next_slot << 3 | code ----
            for (uint32_t s = tid; s < cap; s += BLOCK) {
                const uint64_t w = slots[s];
                if (w == 0) continue;
                const uint4 c4 = ((const uint4 *)cnt)[s];
                const uint32_t lo[4] = {c4.x & 0xffffu, c4.y & 0xffffu, c4.z & 0xffffu, c4.w & 0xffffu};
                const uint32_t hi[4] = {c4.x >> 16, c4.y >> 16, c4.z >> 16, c4.w >> 16};
                const int code = ext_rule(lo, hi, P.V, P.F);
                uint32_t nxt = NONE;
                if (code < 4) {
                    Kmer K = extract_kmer(sseq + (size_t)(slot_read(w) - (uint32_t)r0) * SW, slot_pos(w), k, KW);
                    roll_kmer(K, k, KW, (uint32_t)code);
                    nxt = smem_lookup(slots, cap, K, k, KW, sseq, (uint32_t)r0, SW);
                }
                cnt[4 * s] = (nxt << 3) | (uint32_t)code;
            }
            if (tid == 0) {
                // start k-mer: last k bases of the oriented contig (Alg 2 line 4; reading #6)
                const uint64_t *T = tail + (size_t)e * TAIL_W;
                const int Tn = min((int)clen[e], 128);
                const int p = Tn - k;
                const uint64_t n0 = tailN[2 * (size_t)e], n1 = tailN[2 * (size_t)e + 1];
                bool hasN = false;
                for (int i = p; i < Tn; ++i) hasN |= ((i < 64 ? n0 >> i : n1 >> (i - 64)) & 1ull) != 0;
                C.start_slot = NONE;
                if (!hasN) {
                    uint64_t Tw[TAIL_W];
                    for (int i = 0; i < TAIL_W; ++i) Tw[i] = T[i];
                    Kmer K = extract_kmer(Tw, p, k, KW);
                    C.start_slot = smem_lookup(slots, cap, K, k, KW, sseq, (uint32_t)r0, SW);
                }
            }
            __syncthreads();

            // ---- walk (Alg 2) + retry decision, one thread ----
            if (tid == 0) {
                uint8_t *wb = swalk + (C.best_buf ^ 1) * Wp;
                uint32_t node = C.start_slot;
                int len = 0, term = T_MAXLEN;
                unsigned long long steps = 0;
                for (int i = 0; i < P.W; ++i) {
                    if (node != NONE) {   // loop check before lookup (Alg 2 lines 6-8)
                        const uint32_t bit = 1u << (node & 31);
                        if (svis[node >> 5] & bit) { term = T_LOOP; break; }
                        svis[node >> 5] |= bit;
                    }
                    ++steps;
                    if (node == NONE) { term = T_DEADEND; break; }
                    const uint32_t info = cnt[4 * node];
                    const uint32_t code = info & 7u;
                    if (code == CODE_FORK) { term = T_FORK; break; }
                    if (code == CODE_DEADEND) { term = T_DEADEND; break; }
                    wb[len++] = "ACGT"[code];
                    node = info >> 3;
                }
                C.attempts += 1;
                C.end_steps += steps;
                C.end_ins += C.inserts;
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

        if (C.overflow) {   // table did not fit: the GLOBAL path redoes this end from scratch
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

// ------------------------------------------------------------------------------------------------
// global-memory path (round-synchronous)
// ------------------------------------------------------------------------------------------------
struct GState {
    int k, shift, kmax_eff, attempts, best_len, best_term, best_k, done;
};

__global__ void k_g_init(const int32_t *__restrict__ glist, int n, const int32_t *__restrict__ clen,
                         DevParams P, GState *__restrict__ st, int32_t *__restrict__ active) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    GState s;
    s.k = P.k_start;
    s.shift = 0;
    s.kmax_eff = min(P.k_max, (int)clen[glist[i]]);
    s.attempts = 0;
    s.best_len = -1;
    s.best_term = T_DEADEND;
    s.best_k = 0;
    s.done = 0;
    st[i] = s;
    active[i] = i;
}

// table capacity of an end: inserts / 0.7 (+ slack), so the load factor stays <= 0.7
__host__ __device__ __forceinline__ int64_t global_capacity(int64_t inserts) {
    return (inserts * 10 + 6) / 7 + 16;
}

// block per active end: exact insert count at its current k -> capacity; read count
__global__ void k_g_caps(const int32_t *__restrict__ active, int n_act, const int32_t *__restrict__ glist,
                         const GState *__restrict__ st, const int64_t *__restrict__ eoff,
                         const uint16_t *__restrict__ rlen, int64_t *__restrict__ cap,
                         int64_t *__restrict__ nrd) {
    const int i = blockIdx.x;
    if (i >= n_act) return;
    const int g = active[i];
    const int e = glist[g];
    const int k = st[g].k;
    const int64_t a = eoff[e], b = eoff[e + 1];
    long long U = 0;
    for (int64_t j = a + threadIdx.x; j < b; j += blockDim.x) U += max(0, (int)rlen[j] - k);
    for (int o = 16; o; o >>= 1) U += __shfl_xor_sync(0xffffffffu, U, o);
    __shared__ long long part[32];
    if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = U;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long t = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += part[w];
        cap[i] = global_capacity(t);
        nrd[i] = b - a;
    }
}

__device__ __forceinline__ int upper_idx(const int64_t *off, int n, int64_t x) {
    // largest i in [0, n) with off[i] <= x   (off[0] = 0, non-decreasing)
    int lo = 0, hi = n;
    while (hi - lo > 1) {
        int mid = (lo + hi) >> 1;
        if (off[mid] <= x) lo = mid; else hi = mid;
    }
    return lo;
}

__device__ __forceinline__ uint32_t g_lookup(const uint64_t *slots, uint64_t cap, const Kmer &K,
                                             int k, int KW, const uint64_t *rseq, int SW) {
    const uint64_t h = hash_kmer(K, KW);
    const uint64_t tag = tag_of(h);
    uint64_t s = ((uint64_t)(uint32_t)h * cap) >> 32;
    for (uint64_t n = 0; n < cap; ++n) {
        const uint64_t w = slots[s];
        if (w == 0) return NONE;
        if ((w & TAG_MASK) == tag) {
            Kmer K2 = extract_kmer(rseq + (size_t)slot_read(w) * SW, slot_pos(w), k, KW);
            if (kmer_eq(K, K2, KW)) return (uint32_t)s;
        }
        s = (s + 1 == cap) ? 0 : s + 1;
    }
    return NONE;
}

constexpr int GSEG = 16;

// thread per (read, 16-position segment) of every active end; table in global memory with
// 8 x u32 counters per slot (lo[4], hi[4]).
__global__ void k_g_build(const int32_t *__restrict__ active, int n_act, const int32_t *__restrict__ glist,
                          const GState *__restrict__ st, const int64_t *__restrict__ eoff,
                          const int64_t *__restrict__ rd_off, const int64_t *__restrict__ cap_off,
                          int nseg, const uint64_t *__restrict__ rseq, const uint64_t *__restrict__ rqc,
                          const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag, int SW,
                          uint64_t *__restrict__ slots, uint32_t *__restrict__ cnt,
                          unsigned long long *ins_ctr) {
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t item = t / nseg;
    const int sg = (int)(t - item * nseg);
    if (item >= rd_off[n_act]) return;
    const int i = upper_idx(rd_off, n_act, item);
    const int g = active[i];
    const int e = glist[g];
    const int k = st[g].k;
    const int KW = kwords(k);
    const int64_t rid = eoff[e] + (item - rd_off[i]);
    const int len = rlen[rid];
    const int p0 = sg * GSEG;
    const int p1 = min(p0 + GSEG, len - k);
    unsigned long long ins = 0;
    if (p0 < p1) {
        ins = (unsigned)(p1 - p0);
        const uint64_t *R = rseq + rid * SW;
        const uint64_t *Q = rqc + rid * SW;
        uint64_t *tslots = slots + cap_off[i];
        uint32_t *tcnt = cnt + 8 * cap_off[i];
        const uint64_t cap = (uint64_t)(cap_off[i + 1] - cap_off[i]);
        Kmer K = extract_kmer(R, p0, k, KW);
        int lastN = -1;
        if (rflag[rid])
            for (int q = p0; q < p0 + k; ++q)
                if (get2(Q, q) == 3u) lastN = q;
        for (int p = p0; p < p1; ++p) {
            const uint32_t nb = get2(R, p + k);
            const uint32_t nq = get2(Q, p + k);
            if ((nq == 1u || nq == 2u) && lastN < p) {
                const uint64_t h = hash_kmer(K, KW);
                const uint64_t tag = tag_of(h);
                uint64_t s = ((uint64_t)(uint32_t)h * cap) >> 32;
                volatile uint64_t *vs = tslots;
                for (;;) {
                    uint64_t w = vs[s];
                    bool hit = false;
                    if (w == 0) {
                        const uint64_t mine = make_slot(tag, (uint32_t)rid, (uint32_t)p);
                        const uint64_t old = atomicCAS((unsigned long long *)&tslots[s], 0ull, (unsigned long long)mine);
                        if (old == 0) hit = true;
                        else w = old;
                    }
                    if (!hit && (w & TAG_MASK) == tag) {
                        Kmer K2 = extract_kmer(rseq + (size_t)slot_read(w) * SW, slot_pos(w), k, KW);
                        hit = kmer_eq(K, K2, KW);
                    }
                    if (hit) {
                        atomicAdd(&tcnt[8 * s + nb], 1u);
                        if (nq == 2u) atomicAdd(&tcnt[8 * s + 4 + nb], 1u);
                        break;
                    }
                    s = (s + 1 == cap) ? 0 : s + 1;
                }
            }
            if (nq == 3u) lastN = p + k;
            roll_kmer(K, k, KW, nb);
        }
    }
    for (int o = 16; o; o >>= 1) ins += __shfl_xor_sync(0xffffffffu, ins, o);
    if ((threadIdx.x & 31) == 0 && ins) atomicAdd(ins_ctr, ins);
}

// thread per slot: ext rule + successor link, written over lo[0]
__global__ void k_g_graph(const int32_t *__restrict__ active, int n_act, const int32_t *__restrict__ glist,
                          const GState *__restrict__ st, const int64_t *__restrict__ cap_off,
                          const uint64_t *__restrict__ rseq, int SW, DevParams P,
                          const uint64_t *__restrict__ slots, uint32_t *__restrict__ cnt) {
    const int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (s >= cap_off[n_act]) return;
    const uint64_t w = slots[s];
    if (w == 0) return;
    const int i = upper_idx(cap_off, n_act, s);
    const int k = st[active[i]].k;
    const int KW = kwords(k);
    uint32_t lo[4], hi[4];
    const uint4 a = ((const uint4 *)(cnt + 8 * s))[0];
    const uint4 b = ((const uint4 *)(cnt + 8 * s))[1];
    lo[0] = a.x; lo[1] = a.y; lo[2] = a.z; lo[3] = a.w;
    hi[0] = b.x; hi[1] = b.y; hi[2] = b.z; hi[3] = b.w;
    const int code = ext_rule(lo, hi, P.V, P.F);
    uint32_t nxt = NONE;
    if (code < 4) {
        Kmer K = extract_kmer(rseq + (size_t)slot_read(w) * SW, slot_pos(w), k, KW);
        roll_kmer(K, k, KW, (uint32_t)code);
        const uint64_t base = cap_off[i];
        nxt = g_lookup(slots + base, (uint64_t)(cap_off[i + 1] - base), K, k, KW, rseq, SW);
    }
    cnt[8 * s] = (nxt << 3) | (uint32_t)code;
}

// thread per active end: start lookup, walk, retry decision, results when done
__global__ void k_g_walk(const int32_t *__restrict__ active, int n_act, const int32_t *__restrict__ glist,
                         GState *__restrict__ st, const int64_t *__restrict__ cap_off,
                         const uint64_t *__restrict__ rseq, int SW, const uint64_t *__restrict__ tail,
                         const uint64_t *__restrict__ tailN, const int32_t *__restrict__ clen, DevParams P,
                         const uint64_t *__restrict__ slots, const uint32_t *__restrict__ cnt,
                         uint32_t *__restrict__ vis, uint8_t *__restrict__ cur_buf,
                         uint8_t *__restrict__ walk_buf, int32_t *__restrict__ out_len,
                         uint8_t *__restrict__ out_term, uint8_t *__restrict__ out_k,
                         uint8_t *__restrict__ out_att, int32_t *__restrict__ still,
                         unsigned long long *steps_ctr) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_act) return;
    const int g = active[i];
    const int e = glist[g];
    GState S = st[g];
    const int k = S.k;
    const int KW = kwords(k);
    const uint64_t base = cap_off[i];
    const uint64_t cap = (uint64_t)(cap_off[i + 1] - base);
    const uint64_t *tslots = slots + base;
    const uint32_t *tcnt = cnt + 8 * base;
    uint32_t *tvis = vis + (base >> 5) + i;   // visited bits: cap bits + 1 pad word per table
    // start k-mer
    const int Tn = min((int)clen[e], 128);
    const int p = Tn - k;
    bool hasN = false;
    const uint64_t n0 = tailN[2 * (size_t)e], n1 = tailN[2 * (size_t)e + 1];
    for (int q = p; q < Tn; ++q) hasN |= ((q < 64 ? n0 >> q : n1 >> (q - 64)) & 1ull) != 0;
    uint32_t node = NONE;
    if (!hasN) {
        uint64_t Tw[TAIL_W];
        for (int q = 0; q < TAIL_W; ++q) Tw[q] = tail[(size_t)e * TAIL_W + q];
        Kmer K = extract_kmer(Tw, p, k, KW);
        node = g_lookup(tslots, cap, K, k, KW, rseq, SW);
    }
    uint8_t *wb = cur_buf + (size_t)g * P.W;
    int len = 0, term = T_MAXLEN;
    unsigned long long steps = 0;
    for (int it = 0; it < P.W; ++it) {
        if (node != NONE) {
            const uint32_t bit = 1u << (node & 31);
            if (tvis[node >> 5] & bit) { term = T_LOOP; break; }
            tvis[node >> 5] |= bit;
        }
        ++steps;
        if (node == NONE) { term = T_DEADEND; break; }
        const uint32_t info = tcnt[8 * (size_t)node];
        const uint32_t code = info & 7u;
        if (code == CODE_FORK) { term = T_FORK; break; }
        if (code == CODE_DEADEND) { term = T_DEADEND; break; }
        wb[len++] = "ACGT"[code];
        node = info >> 3;
    }
    S.attempts += 1;
    if (len > S.best_len) {
        S.best_len = len;
        S.best_term = term;
        S.best_k = k;
        uint8_t *dst = walk_buf + (size_t)e * P.W;
        for (int q = 0; q < len; ++q) dst[q] = wb[q];
    }
    int kk = S.k, sh = S.shift;
    S.done = next_k(term, kk, sh, S.kmax_eff, P) ? 1 : 0;
    S.k = kk;
    S.shift = sh;
    st[g] = S;
    still[i] = S.done ? 0 : 1;
    if (S.done) {
        out_len[e] = S.best_len;
        out_term[e] = (uint8_t)S.best_term;
        out_k[e] = (uint8_t)S.best_k;
        out_att[e] = (uint8_t)S.attempts;
    }
    atomicAdd(steps_ctr, steps);
}

__global__ void k_g_compact(const int32_t *__restrict__ active, int n_act, const int32_t *__restrict__ still,
                            int32_t *__restrict__ next_active, int *n_next) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_act || !still[i]) return;
    next_active[atomicAdd(n_next, 1)] = active[i];
}

// ------------------------------------------------------------------------------------------------
// emit (a9)
// ------------------------------------------------------------------------------------------------
__global__ void k_len64(const int32_t *__restrict__ len, int64_t n, int64_t *__restrict__ out) {
    int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) out[i] = len[i];
    if (i == n) out[n] = 0;
}

// warp per end: copy the walk, reverse-complemented for LEFT ends (reading #14)
__global__ void k_emit(const uint8_t *__restrict__ walk_buf, int W, const int64_t *__restrict__ ext_off,
                       int64_t n_ends, char *__restrict__ ext_seq) {
    const int64_t e = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (e >= n_ends) return;
    const int64_t o = ext_off[e];
    const int len = (int)(ext_off[e + 1] - o);
    const uint8_t *src = walk_buf + (size_t)e * W;
    const bool left = (e & 1) == 0;
    for (int i = lane; i < len; i += 32) {
        if (left) {
            const uint8_t c = src[len - 1 - i];
            ext_seq[o + i] = c == 'A' ? 'T' : c == 'C' ? 'G' : c == 'G' ? 'C' : 'A';
        } else {
            ext_seq[o + i] = (char)src[i];
        }
    }
}

}  // namespace la
