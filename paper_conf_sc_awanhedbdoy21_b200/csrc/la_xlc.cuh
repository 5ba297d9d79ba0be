// la_xlc.cuh — the XLC table class: one contig end per 2-CTA thread-block cluster, its k-mer table
// split across the two SMs' shared memory and reached through distributed shared memory (DSMEM).
//
// Ends whose filtered table does not fit one SM's shared memory (the largest shared-memory class) but
// fits two: r01/r02's XL class kept those tables in an L2-resident global scratch (~300-cycle L2
// round trips on every probe, and every table written back to DRAM: 3 GB per C4S step).  Here slot s
// lives in CTA s / half's shared memory (half = cap / 2, even, so a probed slot pair never straddles
// the two CTAs); probes, 128-bit CAS claims, vote atomics and the filter bitmaps use shared::cluster
// addresses (38 cycles local, ~215 remote, B300_MICROARCH.md), nothing touches L2 but the reads.
// Both CTAs' 2 x 1024 threads build one end (positions split over 64 warps); CTA rank 0 fetches the
// ends, holds the link words (info) and walks (thread 0) while the cluster waits.  Phases are separated
// by cluster barriers.  Keys: inline (k <= 63, la_inl32.cuh formats); counters: 16-bit fields
// (4 x u32 per slot, RED without return): the planner routes here only ends with U(k_min) < 65536
// voting occurrences, so no field can carry.  An attempt at k >= 64 (pointer keys) or a table that
// overflows sends the end to the global rounds, as the other classes do.
#pragma once
#include "la_inl32.cuh"

namespace la {


__device__ __forceinline__ uint32_t cl_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cl_map(uint32_t shared_addr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(shared_addr), "r"(rank));
    return r;
}
__device__ __forceinline__ void cl_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t cl_ld32(uint32_t a) {
    uint32_t v;
    asm volatile("ld.relaxed.cluster.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ void cl_st32(uint32_t a, uint32_t v) {
    asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint4 cl_ld128(uint32_t a) {
    uint4 v;
    asm volatile("ld.relaxed.cluster.shared::cluster.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "r"(a)
                 : "memory");
    return v;
}
__device__ __forceinline__ uint4 cl_cas128(uint32_t a, const uint4 f) {
    const uint64_t n0 = (uint64_t)f.x | ((uint64_t)f.y << 32), n1 = (uint64_t)f.z | ((uint64_t)f.w << 32);
    uint64_t o0, o1;
    asm volatile(
        "{\n .reg .b128 d, b, c;\n mov.b128 b, {%2, %3};\n mov.b128 c, {%4, %5};\n"
        " atom.relaxed.cluster.shared::cluster.cas.b128 d, [%6], b, c;\n mov.b128 {%0, %1}, d;\n}"
        : "=l"(o0), "=l"(o1)
        : "l"(0ull), "l"(0ull), "l"(n0), "l"(n1), "r"(a)
        : "memory");
    return make_uint4((uint32_t)o0, (uint32_t)(o0 >> 32), (uint32_t)o1, (uint32_t)(o1 >> 32));
}
__device__ __forceinline__ uint32_t cl_or(uint32_t a, uint32_t v) {
    uint32_t o;
    asm volatile("atom.relaxed.cluster.shared::cluster.or.b32 %0, [%1], %2;" : "=r"(o) : "r"(a), "r"(v) : "memory");
    return o;
}
__device__ __forceinline__ void cl_red_add(uint32_t a, uint32_t v) {
    asm volatile("red.relaxed.cluster.shared::cluster.add.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

// the cluster's table: slot s in rank s / half; counters 4 x u32 of 16-bit fields per slot
struct TabC {
    uint32_t keys[2], cnts[2];   // shared::cluster addresses of each rank's key / counter halves
    uint32_t bm1[2], bm2[2];     // filter bitmaps B1 / B2, split the same way (hw words per rank)
    uint32_t half, cap, hw;
    uint32_t info;               // rank 0's link words (shared::cluster address)
    uint16_t *list;              // this CTA's claim list (its own shared memory)
};
// (selects, not indexed arrays: a runtime index would put the table descriptor in local memory)
__device__ __forceinline__ uint32_t slot_addr(const TabC &T, uint32_t s) {
    const bool hi = s >= T.half;
    return (hi ? T.keys[1] : T.keys[0]) + 16u * (hi ? s - T.half : s);
}
__device__ __forceinline__ uint32_t cnt_addr(const TabC &T, uint32_t s) {
    const bool hi = s >= T.half;
    return (hi ? T.cnts[1] : T.cnts[0]) + 16u * (hi ? s - T.half : s);
}
__device__ __forceinline__ uint32_t bm_word(const uint32_t bm[2], uint32_t hw, uint32_t fi) {
    const uint32_t w = fi >> 5;
    const bool hi = w >= hw;
    return (hi ? bm[1] : bm[0]) + 4u * (hi ? w - hw : w);
}
__device__ __forceinline__ int cmp_slot_c(uint32_t a, uint4 v, const uint4 f) {
    if (v.w == 0u) return 2;
    if (v.w != f.w) return 1;
    if (v.x == f.x && v.y == f.y && v.z == f.z) return 0;
    v = cl_ld128(a);   // a 16 B load racing the claiming CAS: re-read once
    return (v.x == f.x && v.y == f.y && v.z == f.z) ? 0 : 1;
}
__device__ __forceinline__ void vote_c(const TabC &T, uint32_t s, uint32_t b, bool hi) {
    cl_red_add(cnt_addr(T, s) + 4u * ((hi ? 2u : 0u) + (b >> 1)), 1u << (16 * (b & 1u)));
}
__device__ __forceinline__ void votes_c(const TabC &T, uint32_t s, uint32_t lo[4], uint32_t hi[4]) {
    const uint4 a = cl_ld128(cnt_addr(T, s));
    hi[0] = a.z & 0xffffu; hi[1] = a.z >> 16; hi[2] = a.w & 0xffffu; hi[3] = a.w >> 16;
    lo[0] = (a.x & 0xffffu) + hi[0]; lo[1] = (a.x >> 16) + hi[1];
    lo[2] = (a.y & 0xffffu) + hi[2]; lo[3] = (a.y >> 16) + hi[3];
}

// convergent insert over the cluster table (warp_insert32's protocol: slot-pair rounds, 128-bit CAS
// claims, claims appended to this CTA's list)
__device__ __forceinline__ void warp_insert_c(const TabC &T, bool want, const uint4 f, uint32_t h, uint32_t nb,
                                              bool hi, int *nclaim, int claim_limit, volatile int *ovf) {
    uint32_t s = slot32(h, T.cap), hit = 0, n = 0;
    bool pend = want, found = false;
    while (__any_sync(0xffffffffu, pend)) {
        bool claimed = false;
        if (pend && (n += 2) > T.cap + 2u) {   // a whole table's worth of probes: full (the other CTA
            *ovf = 1;                          // can still be claiming) -> the end overflows
            pend = false;
        }
        if (pend) {
            const uint32_t s1 = s + 1, a0 = slot_addr(T, s), a1 = a0 + 16u;
            const uint4 v0 = cl_ld128(a0), v1 = cl_ld128(a1);
            int st = cmp_slot_c(a0, v0, f);
            uint32_t at = s, aa = a0;
            if (st == 1) {
                st = cmp_slot_c(a1, v1, f);
                at = s1;
                aa = a1;
            }
            if (st == 0) {
                hit = at;
                pend = false;
                found = true;
            } else if (st == 2) {
                if (*ovf) {
                    pend = false;
                } else {
                    const uint4 o = cl_cas128(aa, f);
                    if (o.w == 0u) {
                        claimed = found = true;
                        hit = at;
                        pend = false;
                    } else if (same4(o, f)) {
                        found = true;
                        hit = at;
                        pend = false;
                    } else if (at == s) {
                        const int st1 = cmp_slot_c(a1, cl_ld128(a1), f);
                        if (st1 == 0) {
                            found = true;
                            hit = s1;
                            pend = false;
                        } else if (st1 == 1) {
                            s = s1 + 1 == T.cap ? 0 : s1 + 1;
                        }
                    }
                }
            } else {
                s = s1 + 1 == T.cap ? 0 : s1 + 1;
            }
        }
        if (claimed) {
            const int idx = atomicAdd(nclaim, 1);
            if (idx >= claim_limit) *ovf = 1;
            T.list[idx] = (uint16_t)hit;
        }
    }
    if (found) vote_c(T, hit, nb, hi);
}

__device__ __forceinline__ uint32_t warp_lookup_c(const TabC &T, bool want, const uint4 f, uint32_t h) {
    uint32_t s = slot32(h, T.cap), res = NONE, n = 0;
    bool pend = want;
    while (__any_sync(0xffffffffu, pend)) {
        if (pend) {
            const uint32_t a0 = slot_addr(T, s);
            const uint4 v0 = cl_ld128(a0), v1 = cl_ld128(a0 + 16u);
            const int x = cmp_slot_c(a0, v0, f);
            if (x == 0) {
                res = s;
                pend = false;
            } else if (x == 2) {
                pend = false;
            } else {
                const int y = cmp_slot_c(a0 + 16u, v1, f);
                if (y == 0) {
                    res = s + 1;
                    pend = false;
                } else if (y == 2) {
                    pend = false;
                } else {
                    s = s + 2 == T.cap ? 0 : s + 2;
                    n += 2;
                    if (n >= T.cap) pend = false;
                }
            }
        }
    }
    return res;
}

__device__ __forceinline__ uint32_t lookup_c(const TabC &T, const uint4 f, uint32_t h) {
    uint32_t s = slot32(h, T.cap);
    for (uint32_t n = 0; n < T.cap; ++n) {
        const uint32_t a = slot_addr(T, s);
        const int c = cmp_slot_c(a, cl_ld128(a), f);
        if (c == 0) return s;
        if (c == 2) return NONE;
        s = s + 1 == T.cap ? 0 : s + 1;
    }
    return NONE;
}

// push this CTA's end slot to the peer CTA (one thread; the cluster barrier that follows publishes it)
__device__ __forceinline__ void push_end(const EndSlot &E, uint32_t E_peer) {
    const uint32_t *w = (const uint32_t *)&E;
#pragma unroll 4
    for (int i = 0; i < (int)(sizeof(EndSlot) / 4); ++i) cl_st32(E_peer + 4u * i, w[i]);
}

// One attempt's filter, dead-start check, build and link passes over the cluster table (NW 32-bit
// words per k-mer).  Every thread of both CTAs calls it; returns through B (start, dead0, overflow).
template <int NW>
__device__ __forceinline__ void xlc_passes(BuildCtl &B, const TabC &T, uint32_t mbits, const uint64_t *R64,
                                           const uint64_t *Q64, const uint8_t *gF, const uint32_t *pref,
                                           long long lr0, int r, int SW, int k, int ulen, const DevParams &P,
                                           const uint64_t *tail_e, int Tn, uint64_t n0, uint64_t n1, uint32_t rank,
                                           int tid, int gw, int NWT, uint32_t flag_local, uint32_t flag_peer,
                                           int claim_limit, bool replay, bool anyN) {
    const int lane = tid & 31;
    const uint32_t *R32 = (const uint32_t *)R64, *Q32 = (const uint32_t *)Q64;
    const int SW2 = 2 * SW;
    const volatile int *stop = &B.overflow;
    K32<NW> Kst;
    if (tid == 0) {   // start k-mer: last k bases of the oriented contig (Alg 2 line 4; reading #6)
        const int p = Tn - k;
        bool hasN = false;
        hasN = any_n_range(n0, n1, p, Tn);
        uint32_t Tw[2 * TAIL_W];
#pragma unroll
        for (int i = 0; i < TAIL_W; ++i) {
            const uint64_t x = tail_e[i];
            Tw[2 * i] = (uint32_t)x;
            Tw[2 * i + 1] = (uint32_t)(x >> 32);
        }
        Kst = extract32<NW>(Tw, p, kmask32<NW>(k));
        B.start_h = hash32<NW>(Kst);
        B.start_ok = !hasN;
    }
    // ---- filter pass (reading #4): B1 = seen once, B2 = seen at least twice, bitmaps split ----
    if (mbits) {
        warp_positions32<NW, 2>(R32, Q32, anyN ? gF : nullptr, pref, lr0, r, SW2, k, ulen, gw, NWT, lane, stop,
                                [&](bool, bool act, uint32_t, const K32<NW> &, uint32_t h, uint32_t, bool) {
                                    if (!act) return;
                                    const uint32_t fi = filt32(h, mbits), bit = 1u << (fi & 31);
                                    const uint32_t w2 = bm_word(T.bm2, T.hw, fi);
                                    if (!(cl_ld32(w2) & bit)) {
                                        const uint32_t old = cl_or(bm_word(T.bm1, T.hw, fi), bit);
                                        if (old & bit) cl_or(w2, bit);
                                    }
                                });
    }
    cl_sync();
    // dead start (reading #4): decided identically in both CTAs (thread 0 of each)
    if (tid == 0) {
        bool dead = false;
        if (mbits && LA_DEAD0) {
            const uint32_t fs = filt32(B.start_h, mbits);
            dead = !B.start_ok || !((cl_ld32(bm_word(T.bm2, T.hw, fs)) >> (fs & 31)) & 1u);
        }
        B.dead0 = dead ? 1 : 0;
    }
    __syncthreads();
    if (!B.dead0) {
        // ---- build (Alg 1) into the cluster table ----
        warp_positions32<NW>(R32, Q32, anyN ? gF : nullptr, pref, lr0, r, SW2, k, ulen, gw, NWT, lane, stop,
                             [&](bool, bool act, uint32_t, const K32<NW> &K, uint32_t h, uint32_t nb, bool hi) {
                                 bool want = act;
                                 if (mbits) {
                                     const uint32_t fi = filt32(h, mbits);
                                     want = want && ((cl_ld32(bm_word(T.bm2, T.hw, fi)) >> (fi & 31)) & 1u);
                                 }
                                 warp_insert_c(T, want, key_form<NW>(K, h), h, nb, hi, &B.nclaim, claim_limit,
                                               &B.overflow);
                             });
    }
    __syncthreads();
    if (tid == 0) cl_st32(flag_local, (uint32_t)B.overflow);
    cl_sync();   // every insert of both CTAs done; both overflow flags published
    if (tid == 0 && cl_ld32(flag_peer)) B.overflow = 1;
    __syncthreads();
    if (B.overflow || replay) return;
    if (!B.dead0) {
        // ---- ext rule + successor links (a5) over this CTA's claimed slots -> rank 0's info ----
        const uint32_t nocc = min((uint32_t)B.nclaim, T.cap);
        for (uint32_t base = (uint32_t)(tid >> 5) * 32u; base < nocc; base += (uint32_t)XLC_THREADS) {
            const uint32_t i = base + lane;
            const bool has = i < nocc;
            const uint32_t s = has ? (uint32_t)T.list[i] : 0u;
            K32<NW> K;
#pragma unroll
            for (int w = 0; w < NW; ++w) K.w[w] = 0u;
            int code = CODE_DEADEND;
            if (has) {
                K = key_of<NW>(cl_ld128(slot_addr(T, s)));
                uint32_t lo[4], hi[4];
                votes_c(T, s, lo, hi);
                code = ext_rule(lo, hi, P.V, P.F);
                if (code < 4) roll32<NW>(K, k, (uint32_t)code);
            }
            const uint32_t h = hash32<NW>(K);
            const uint32_t t = warp_lookup_c(T, has && code < 4, key_form<NW>(K, h), h);
            if (has) cl_st32(T.info + 4u * s, link_info(code, t));
        }
    }
    if (rank == 0 && tid == 0)
        B.start = (B.dead0 || !B.start_ok) ? NONE : lookup_c(T, key_form<NW>(Kst, B.start_h), B.start_h);
}

// The XLC class kernel (launched with 2-CTA clusters, one cluster per 2 SMs, persistent over its list)
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(XLC_THREADS, 1) k_xlc(
    const int32_t *__restrict__ list, int n_list, int *__restrict__ work_ctr, const uint64_t *__restrict__ rseq,
    const uint64_t *__restrict__ rqc, const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag,
    const int64_t *__restrict__ eoff, const uint64_t *__restrict__ tail, const uint64_t *__restrict__ tailN,
    const int32_t *__restrict__ clen, int SW, DevParams P, uint32_t smem_bytes, uint8_t *__restrict__ walk_buf,
    int32_t *__restrict__ out_len, uint8_t *__restrict__ out_term, uint8_t *__restrict__ out_k,
    uint8_t *__restrict__ out_att, int8_t *__restrict__ out_dir, int32_t *__restrict__ ovf_list,
    int *__restrict__ n_ovf, GlobalStats *__restrict__ gstats) {
    constexpr int NB = XLC_THREADS;
    extern __shared__ __align__(16) unsigned char sm[];
    __shared__ EndSlot E;
    __shared__ BuildCtl B;
    __shared__ uint32_t s_flag, s_umax;
    __shared__ unsigned long long s_acc[GSTATS_WORDS];
    const uint32_t rank = cl_rank(), peer = rank ^ 1u;
    const int tid = threadIdx.x, wid = tid >> 5;
    const int gw = (int)rank * (NB / 32) + wid, NWT = 2 * (NB / 32);
    const uint32_t base = smem_addr(sm);
    const uint32_t base_r0 = cl_map(base, 0), base_r1 = cl_map(base, 1);
    const uint32_t E_peer = cl_map(smem_addr(&E), peer);
    const uint32_t flag_local = cl_map(smem_addr(&s_flag), rank), flag_peer = cl_map(smem_addr(&s_flag), peer);
    const int Wp = ((P.W > 0 ? P.W : 1) + 15) & ~15;
    if (tid < GSTATS_WORDS) s_acc[tid] = 0;
    for (;;) {
        // ---- rank 0 fetches the next end and pushes its slot to rank 1 ----
        if (tid == 0) s_umax = 0;
        if (rank == 0 && tid == 0) {
            int idx, e = 0, lv = 0;
            do {   // replay: ends that left this kernel (overflow) in the extension are not replayed
                idx = atomicAdd(work_ctr, 1);
                if (idx < n_list) {
                        lv = list[idx];
                        e = list_end(lv);
                    }
            } while (P.replay && idx < n_list && out_dir[e] == OVF_DIR);
            E.dead = idx >= n_list;
            if (!E.dead) {
                E.e = e;
                E.anyN = list_anyn(lv);
                E.r0 = eoff[e];
                E.r = (int)(eoff[e + 1] - E.r0);
                E.ulen = list_uniform(lv) ? P.maxlen : -1;
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
                E.done = 0;
                E.ovf = 0;
                if (P.replay) {
                    E.rec_att = out_att[e];
                    E.shift = out_dir[e] * P.k_shift;
                }
            }
            push_end(E, E_peer);
        }
        cl_sync();
        if (E.dead) break;
        const int e = E.e, r = E.r;
        const long long r0 = E.r0;
        // stage the reads in both CTAs if the largest attempt's layout leaves room (U at k_min)
        {
            uint32_t part = 0;
            for (int j = tid; j < r; j += NB) part += (uint32_t)max(0, (int)rlen[r0 + j] - P.k_min);
            for (int o = 16; o; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
            if ((tid & 31) == 0 && part) atomicAdd(&s_umax, part);
            __syncthreads();
        }
        const bool stage = xlc_layout(smem_bytes, r, SW, s_umax, P.W, true).fits;
        uint64_t *sR = (uint64_t *)sm;
        uint64_t *sQ = sR + (size_t)r * SW;
        uint16_t *sL = (uint16_t *)(sQ + (size_t)r * SW);
        uint8_t *sF = (uint8_t *)(sL + r);
        if (stage) {
            const uint4 *a4 = (const uint4 *)(rseq + r0 * SW);
            const uint4 *b4 = (const uint4 *)(rqc + r0 * SW);
            for (int i = tid; i < r * SW / 2; i += NB) {
                ((uint4 *)sR)[i] = __ldg(&a4[i]);
                ((uint4 *)sQ)[i] = __ldg(&b4[i]);
            }
            for (int i = tid; i < r; i += NB) {
                sL[i] = __ldg(&rlen[r0 + i]);
                sF[i] = __ldg(&rflag[r0 + i]);
            }
            __syncthreads();
        }
        const uint64_t *gR = stage ? sR : rseq, *gQ = stage ? sQ : rqc;
        const uint16_t *gL = stage ? sL : rlen;
        const uint8_t *gF = stage ? sF : rflag;
        const long long lr0 = stage ? 0 : r0;
        const int Tn = min((int)clen[e], 128);
        const uint64_t *tail_e = tail + (size_t)e * TAIL_W;
        const uint64_t n0 = tailN[2 * (size_t)e], n1 = tailN[2 * (size_t)e + 1];
        uint8_t *wstr = sm + xlc_layout(smem_bytes, r, SW, 0u, P.W, stage).off_walk;   // two walk strings
        bool ovf = false;
        for (;;) {   // attempts (k schedule)
            const int k = E.k;
            if (!inline_keys(k)) {   // pointer-key attempts are not done here: the global rounds redo the end
                ovf = true;
                break;
            }
            const XlcLayout L0 = xlc_layout(smem_bytes, r, SW, 0u, P.W, stage);
            uint32_t *pref = (uint32_t *)(sm + L0.off_pref);
            read_prefix(B, E, pref, gL, lr0, r, k, E.ulen, tid, NB);
            const uint32_t U = pref[r];
            const XlcLayout L = xlc_layout(smem_bytes, r, SW, U, P.W, stage);
            if (!L.fits || P.V < 2) {   // no room (or an unfiltered table): the global rounds
                ovf = true;
                break;
            }
            TabC T;
            T.keys[0] = base_r0 + L.off_keys;
            T.keys[1] = base_r1 + L.off_keys;
            T.cnts[0] = base_r0 + L.off_cnts;
            T.cnts[1] = base_r1 + L.off_cnts;
            T.bm1[0] = base_r0 + L.off_b1;
            T.bm1[1] = base_r1 + L.off_b1;
            T.bm2[0] = base_r0 + L.off_b2;
            T.bm2[1] = base_r1 + L.off_b2;
            T.half = L.half;
            T.cap = L.cap;
            T.hw = L.hw;
            T.info = base_r0 + L.off_info;
            T.list = (uint16_t *)(sm + L.off_list);
            // clear this CTA's halves of the table and of the bitmaps
            {
                uint4 *a = (uint4 *)(sm + L.off_keys);
                for (uint32_t i = tid; i < L.half * 2u; i += NB) a[i] = make_uint4(0, 0, 0, 0);   // keys + counters
                uint32_t *b1 = (uint32_t *)(sm + L.off_b1);
                for (uint32_t i = tid; i < 2u * L.hw; i += NB) b1[i] = 0;   // B1 half, B2 half
            }
            if (tid == 0) {
                B.overflow = 0;
                B.nclaim = 0;
                B.dead0 = 0;
            }
            cl_sync();
            const int NW = kw32(k);
            const int lim = (int)(0.45f * (float)L.cap);
            const uint32_t mbits = L.mwords * 32u;
            if (NW <= 2)
                xlc_passes<2>(B, T, mbits, gR, gQ, gF, pref, lr0, r, SW, k, E.ulen, P, tail_e, Tn, n0, n1, rank, tid,
                              gw, NWT, flag_local, flag_peer, lim, P.replay != 0, E.anyN != 0);
            else if (NW == 3)
                xlc_passes<3>(B, T, mbits, gR, gQ, gF, pref, lr0, r, SW, k, E.ulen, P, tail_e, Tn, n0, n1, rank, tid,
                              gw, NWT, flag_local, flag_peer, lim, P.replay != 0, E.anyN != 0);
            else
                xlc_passes<4>(B, T, mbits, gR, gQ, gF, pref, lr0, r, SW, k, E.ulen, P, tail_e, Tn, n0, n1, rank, tid,
                              gw, NWT, flag_local, flag_peer, lim, P.replay != 0, E.anyN != 0);
            if (B.overflow) {   // identical in both CTAs (flags exchanged)
                ovf = true;
                break;
            }
            cl_sync();   // link words complete in rank 0
            if (rank == 0 && tid == 0) {
                s_acc[3] += 1;
                s_acc[4] += 1;
                s_acc[6] += B.dead0;
                E.ins += U;
                if (P.replay) {
                    E.attempts += 1;
                    E.done = E.attempts >= E.rec_att;
                    E.k += E.shift;
                } else {
                    // ---- walk (Alg 2) over the link words, as k_small ----
                    uint32_t *info = (uint32_t *)(sm + L.off_info);
                    uint8_t *wb = wstr + (E.best_buf ^ 1) * Wp;
                    int term;
                    unsigned long long steps;
                    const int len = walk_links(info, B.start == NONE ? NEXT_NONE : B.start, P.W, wb, term, steps);
                    E.attempts += 1;
                    E.steps += steps;
                    if (len > E.best_len) {   // longest walk, earliest on ties (reading #11)
                        E.best_len = len;
                        E.best_term = term;
                        E.best_k = E.k;
                        E.best_buf ^= 1;
                    }
                    int kk = E.k, sh = E.shift;
                    E.done = next_k(term, kk, sh, E.kmax_eff, P) ? 1 : 0;
                    E.k = kk;
                    E.shift = sh;
                }
                push_end(E, E_peer);
            }
            cl_sync();
            if (E.done) break;
        }
        if (rank == 0) {
            if (ovf) {
                if (tid == 0 && !P.replay) {
                    ovf_list[atomicAdd(n_ovf, 1)] = e;
                    out_dir[e] = OVF_DIR;
                }
            } else if (P.replay) {
                if (tid == 0) {
                    s_acc[0] += E.ins;
                    s_acc[2] += E.attempts;
                }
            } else {
                const int bl = E.best_len;
                const uint8_t *bw = wstr + E.best_buf * Wp;
                uint8_t *dst = walk_buf + (size_t)e * P.W;
                for (int i = tid; i < bl; i += NB) dst[i] = bw[i];
                if (tid == 0) {
                    out_len[e] = bl;
                    out_term[e] = (uint8_t)E.best_term;
                    out_k[e] = (uint8_t)E.best_k;
                    out_att[e] = (uint8_t)E.attempts;
                    out_dir[e] = shift_dir(E.shift);
                    s_acc[0] += E.ins;
                    s_acc[1] += E.steps;
                    s_acc[2] += E.attempts;
                }
            }
        }
        __syncthreads();   // E, staged reads and walk strings are reused by the next end
    }
    if (rank == 0 && tid == 0) {
        unsigned long long *g = &gstats->inserts;
        for (int i = 0; i < GSTATS_WORDS; ++i) atomicAdd(&g[i], s_acc[i]);
    }
}

}  // namespace la
