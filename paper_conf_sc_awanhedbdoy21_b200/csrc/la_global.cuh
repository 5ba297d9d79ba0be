#pragma once
#include "la_device.cuh"

namespace la {

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

}  // namespace la
