// la_inl32.cuh — the inline-key (k <= 63) table path on 32-bit words (DESIGN.md §7 "r02").
//
// The packed rows (rseq / rqc, 64-bit words, base i at bit 62 - 2*(i%32) of word i/32) are read
// through a 32-bit view: 32-bit word j holds bases 16j..16j+15 big-endian (base i at bit
// 30 - 2*(i%16)), i.e. the high half of 64-bit word j/2 for even j — at address 4*(j ^ 1) in
// little-endian memory.  A k-mer is NW = ceil(2k/32) such words, left aligned; extracting it at base p
// is NW+1 loads and NW one-instruction funnel shifts (SHF.L.W), and the hash is 32-bit arithmetic
// only (r01's 64-bit funnels and 64-bit mixing took ~100 instructions per position, ncu/SASS r01).
//
// Table slot (16 B, claimed with one 128-bit CAS): NW <= 3: [w0, w1, w2, tag] with tag = hash | 1
// (never 0: the occupancy marker, and a cheap first comparison); NW = 4 (49 <= k <= 63): [w0, w1, w2,
// ~w3] (2k <= 126 leaves pad bits in w3, so ~w3 is never 0).  Empty slot: word 3 == 0.
#pragma once
#include "la_device.cuh"

// LA_ABL_* (timing ablations only; results are NOT correct with any of them set): tools/ab.sh
#ifndef LA_ABL_NOVOTE
#define LA_ABL_NOVOTE 0
#endif
#ifndef LA_ABL_NOCAS
#define LA_ABL_NOCAS 0
#endif
#ifndef LA_ABL_NOCLAIM
#define LA_ABL_NOCLAIM 0
#endif
#ifndef LA_ABL_NOFILTATOM
#define LA_ABL_NOFILTATOM 0
#endif
namespace la {

#ifdef LA_PROBE_STATS
// debug build only (tools/probe_stats.py): [0] warp_insert32 calls (per warp), [1] their probe rounds,
// [2] inserting lanes, [3] claims, [4] warp_lookup32 calls, [5] their rounds, [6] looking-up lanes,
// [7] unused, [8] filter-pass warp iterations, [9] their voting lanes, [10] 128-bit CAS issued,
// [11] slot re-reads after a racing claim
__device__ unsigned long long g_probe_stats[12];
#define LA_PSTAT(i, v) atomicAdd(&g_probe_stats[i], (unsigned long long)(v))
#else
#define LA_PSTAT(i, v) ((void)0)
#endif

template <int NW>
struct K32 {
    uint32_t w[NW];
};

__host__ __device__ __forceinline__ int kw32(int k) { return (2 * k + 31) >> 5; }

// masks of the k-mer's bits in words NW-2 and NW-1 (hoisted per attempt)
struct KMask {
    uint32_t m2, m1;
};
template <int NW>
__device__ __forceinline__ KMask kmask32(int k) {
    KMask m;
    const int b1 = 2 * k - 32 * (NW - 1), b2 = 2 * k - 32 * (NW - 2);
    m.m1 = b1 >= 32 ? ~0u : (b1 <= 0 ? 0u : (~0u << (32 - b1)));
    m.m2 = NW < 2 ? ~0u : (b2 >= 32 ? ~0u : (b2 <= 0 ? 0u : (~0u << (32 - b2))));
    return m;
}

// 32-bit word j of a packed row (64-bit big-endian words in memory)
__device__ __forceinline__ uint32_t rw32(const uint32_t *R, int j) { return R[j ^ 1]; }

template <int NW>
__device__ __forceinline__ K32<NW> extract32(const uint32_t *R, int p, const KMask &m) {
    const int q = p >> 4, s = (p & 15) << 1;
    uint32_t x[NW + 1];
#pragma unroll
    for (int i = 0; i <= NW; ++i) x[i] = rw32(R, q + i);
    K32<NW> K;
#pragma unroll
    for (int i = 0; i < NW; ++i) K.w[i] = __funnelshift_l(x[i + 1], x[i], s);
    if (NW >= 2) K.w[NW - 2] &= m.m2;
    K.w[NW - 1] &= m.m1;
    return K;
}

// 2-bit code of base i of a packed row
__device__ __forceinline__ uint32_t base32(const uint32_t *R, int i) {
    return (rw32(R, i >> 4) >> (30 - ((i & 15) << 1))) & 3u;
}

// next_kmer (Alg 2 line 15): drop base 0, append base b at position k-1
template <int NW>
__device__ __forceinline__ void roll32(K32<NW> &K, int k, uint32_t b) {
#pragma unroll
    for (int i = 0; i < NW; ++i) K.w[i] = (K.w[i] << 2) | (i + 1 < NW ? (K.w[i + 1 < NW ? i + 1 : i] >> 30) : 0u);
    const int wl = (k - 1) >> 4, sh = 30 - (((k - 1) & 15) << 1);
#pragma unroll
    for (int i = 0; i < NW; ++i)
        if (i == wl) K.w[i] |= b << sh;
}

// 32-bit hash (multiply-xor of the words + the murmur3 finaliser); never 0.  The hash function does
// not affect results (reading #17), only probe lengths and filter false positives.
#ifndef LA_HASH_LITE
#define LA_HASH_LITE 1   // a shorter finaliser: fewer instructions, same probe lengths (r02 A/B: -0.5%)
#endif
template <int NW>
__device__ __forceinline__ uint32_t hash32(const K32<NW> &K) {
    uint32_t h = K.w[0] * 0xCC9E2D51u;
#pragma unroll
    for (int i = 1; i < NW; ++i) h = (h ^ (h >> 15) ^ K.w[i]) * (i == 1 ? 0x1B873593u : (i == 2 ? 0x85EBCA6Bu : 0xC2B2AE35u));
    h ^= h >> 16;
    h *= 0x85EBCA6Bu;
    h ^= h >> 13;
#if !LA_HASH_LITE
    h *= 0xC2B2AE35u;
    h ^= h >> 16;
#endif
    return h | 1u;
}
// the slot (high bits of h x cap: multiply-shift) and the filter bit (high bits of a second mix)
__device__ __forceinline__ uint32_t slot32(uint32_t h, uint32_t cap) { return __umulhi(h, cap) & ~1u; }
__device__ __forceinline__ uint32_t filt32(uint32_t h, uint32_t mbits) { return __umulhi(h * 0x9E3779B9u, mbits); }

// stored form of a key (see the header comment)
template <int NW>
__device__ __forceinline__ uint4 key_form(const K32<NW> &K, uint32_t h) {
    uint4 f;
    f.x = K.w[0];
    f.y = NW > 1 ? K.w[NW > 1 ? 1 : 0] : 0u;
    f.z = NW > 2 ? K.w[NW > 2 ? 2 : 0] : 0u;
    f.w = NW > 3 ? ~K.w[NW > 3 ? 3 : 0] : h;
    return f;
}
template <int NW>
__device__ __forceinline__ K32<NW> key_of(const uint4 f) {
    K32<NW> K;
    K.w[0] = f.x;
    if (NW > 1) K.w[NW > 1 ? 1 : 0] = f.y;
    if (NW > 2) K.w[NW > 2 ? 2 : 0] = f.z;
    if (NW > 3) K.w[NW > 3 ? 3 : 0] = ~f.w;
    return K;
}
__device__ __forceinline__ bool same4(const uint4 a, const uint4 b) {
    return a.x == b.x && a.y == b.y && a.z == b.z && a.w == b.w;
}

// ---- 128-bit slot access: shared memory (GT = false, 32-bit shared address) or global (XL) ----
struct Tab32 {
    unsigned char *keys;    // slot array (generic pointer: the XL class's global scratch)
    uint32_t ks;            // shared-memory address of the slot array (shared tables)
    uint32_t *c32;          // counters: per slot two u32 of four 8-bit fields (shared) / 8 x u32 (XL)
    uint16_t *list;         // claimed slots in claim order
    uint32_t cap;           // even
    int wide;               // XL: 32-bit counter fields (else 16-bit)
};

template <bool GT>
__device__ __forceinline__ uint4 ld_slot(const Tab32 &T, uint32_t s) {
    uint4 v;
    if (GT) {
        asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                     : "l"(T.keys + 16 * (size_t)s)
                     : "memory");
    } else {
        asm volatile("ld.volatile.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                     : "r"(T.ks + 16u * s)
                     : "memory");
    }
    return v;
}
// claim an empty slot: 128-bit CAS (0 -> f); returns the slot's previous content (0 = claimed)
template <bool GT>
__device__ __forceinline__ uint4 cas_slot(const Tab32 &T, uint32_t s, const uint4 f) {
    const uint64_t n0 = (uint64_t)f.x | ((uint64_t)f.y << 32), n1 = (uint64_t)f.z | ((uint64_t)f.w << 32);
    uint64_t o0, o1;
    if (LA_ABL_NOCAS && !GT) {
        asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(T.ks + 16u * s), "r"(f.x), "r"(f.y), "r"(f.z),
                     "r"(f.w)
                     : "memory");
        return make_uint4(0u, 0u, 0u, 0u);
    }
    if (GT) {
        asm volatile(
            "{\n .reg .b128 d, b, c;\n mov.b128 b, {%2, %3};\n mov.b128 c, {%4, %5};\n"
            " atom.global.cas.b128 d, [%6], b, c;\n mov.b128 {%0, %1}, d;\n}"
            : "=l"(o0), "=l"(o1)
            : "l"(0ull), "l"(0ull), "l"(n0), "l"(n1), "l"(T.keys + 16 * (size_t)s)
            : "memory");
    } else {
        asm volatile(
            "{\n .reg .b128 d, b, c;\n mov.b128 b, {%2, %3};\n mov.b128 c, {%4, %5};\n"
            " atom.shared.cas.b128 d, [%6], b, c;\n mov.b128 {%0, %1}, d;\n}"
            : "=l"(o0), "=l"(o1)
            : "l"(0ull), "l"(0ull), "l"(n0), "l"(n1), "r"(T.ks + 16u * s)
            : "memory");
    }
    return make_uint4((uint32_t)o0, (uint32_t)(o0 >> 32), (uint32_t)o1, (uint32_t)(o1 >> 32));
}

// One vote for base b of slot s: high-tier (q >= q_hi) and low-only (q_lo <= q < q_hi)
// votes in separate counter words; the low tier of reading #1 is their sum.  Shared memory: 8-bit
// fields, a field about to carry flags the end for the global path (reading #15); XL: 8 x u32.
// Counters.  Shared-memory tables: per slot two u32 of four 8-bit fields (low-only votes, high
// votes); a field about to carry flags the end for the global path (reading #15).  XL tables (global
// scratch, GT): no carry check (a global atomic's return trip is slow), fire-and-forget RED.ADD on
// fields wide enough for the attempt: 16-bit fields (4 x u32 per slot) when the attempt has fewer than
// 65536 voting occurrences (a field counts at most all of them), else 8 x u32 (`wide`).
template <bool GT>
__device__ __forceinline__ void vote32(const Tab32 &T, uint32_t s, uint32_t b, bool hi, volatile int *ovf) {
    if (LA_ABL_NOVOTE) {
        if (s == 0xFFFFFFFFu) *ovf = 1;
        return;
    }
    if (GT) {
        if (T.wide) atomicAdd(&T.c32[8 * (size_t)s + (hi ? 4u : 0u) + b], 1u);
        else atomicAdd(&T.c32[4 * (size_t)s + (hi ? 2u : 0u) + (b >> 1)], 1u << (16 * (b & 1u)));
    } else {
        const uint32_t old = atomicAdd(&T.c32[2 * s + (hi ? 1u : 0u)], 1u << (8 * b));
        if (((old >> (8 * b)) & 0xffu) == 0xffu) *ovf = 1;
    }
}
// Same vote with the carry check of the PREVIOUS vote of this lane (pend: its old counter word shifted
// to the voted field): the atomic's return value is first used one insert later, so the warp does not
// wait for the shared-memory atomic's round trip on every insert.  flush_vote32 checks the last one.
#ifndef LA_DEFER_VOTE
#define LA_DEFER_VOTE 1
#endif
template <bool GT>
__device__ __forceinline__ void vote32d(const Tab32 &T, uint32_t s, uint32_t b, bool hi, volatile int *ovf,
                                        uint32_t &pend) {
    if (GT || LA_ABL_NOVOTE || !LA_DEFER_VOTE) {
        vote32<GT>(T, s, b, hi, ovf);
        return;
    }
    if ((pend & 0xffu) == 0xffu) *ovf = 1;
    pend = atomicAdd(&T.c32[2 * s + (hi ? 1u : 0u)], 1u << (8 * b)) >> (8 * b);
}
__device__ __forceinline__ void flush_vote32(uint32_t &pend, volatile int *ovf) {
    if ((pend & 0xffu) == 0xffu) *ovf = 1;
    pend = 0;
}

template <bool GT>
__device__ __forceinline__ void votes32(const Tab32 &T, uint32_t s, uint32_t lo[4], uint32_t hi[4]) {
    if (GT && T.wide) {
        const uint4 a = ((const uint4 *)T.c32)[2 * (size_t)s], c = ((const uint4 *)T.c32)[2 * (size_t)s + 1];
        hi[0] = c.x; hi[1] = c.y; hi[2] = c.z; hi[3] = c.w;
        lo[0] = a.x + c.x; lo[1] = a.y + c.y; lo[2] = a.z + c.z; lo[3] = a.w + c.w;
    } else if (GT) {
        const uint4 a = ((const uint4 *)T.c32)[s];
        hi[0] = a.z & 0xffffu; hi[1] = a.z >> 16; hi[2] = a.w & 0xffffu; hi[3] = a.w >> 16;
        lo[0] = (a.x & 0xffffu) + hi[0]; lo[1] = (a.x >> 16) + hi[1];
        lo[2] = (a.y & 0xffffu) + hi[2]; lo[3] = (a.y >> 16) + hi[3];
    } else {
        const uint2 w = ((const uint2 *)T.c32)[s];
#pragma unroll
        for (int b = 0; b < 4; ++b) {
            hi[b] = (w.y >> (8 * b)) & 0xffu;
            lo[b] = ((w.x >> (8 * b)) & 0xffu) + hi[b];
        }
    }
}

// Compare a loaded slot with the lane's key form.  0 = match, 1 = another key, 2 = empty.  A 16 B
// load racing the claiming 128-bit CAS is re-read once when its occupancy word matches but the rest
// does not (a slot never changes after its claim).
template <bool GT>
__device__ __forceinline__ int cmp_slot(const Tab32 &T, uint32_t s, uint4 v, const uint4 f) {
    if (v.w == 0u) return 2;
    if (v.w != f.w) return 1;
    if (v.x == f.x && v.y == f.y && v.z == f.z) return 0;
    LA_PSTAT(11, 1);
    v = ld_slot<GT>(T, s);
    return (v.x == f.x && v.y == f.y && v.z == f.z) ? 0 : 1;
}

// Convergent insert (Alg 1 line 5 + the vote): every probe round is entered by the whole warp and
// tests a slot pair (s, s+1) with two 16 B loads; an empty slot is claimed with one 128-bit CAS;
// claims are appended to the claim list once per warp (ballot + one atomic).
template <bool GT>
__device__ __forceinline__ void warp_insert32(const Tab32 &T, bool want, const uint4 f, uint32_t h, uint32_t nb,
                                              bool hi, int lane, int *nclaim, int claim_limit, volatile int *ovf,
                                              uint32_t &vpend) {
    uint32_t s = slot32(h, T.cap), hit = 0;
    bool pend = want, found = false;
#ifdef LA_PROBE_STATS
    {
        const unsigned wm = __ballot_sync(0xffffffffu, want);
        if (lane == 0) { LA_PSTAT(0, 1); LA_PSTAT(2, __popc(wm)); }
    }
#endif
    while (__any_sync(0xffffffffu, pend)) {
        if (lane == 0) LA_PSTAT(1, 1);
        bool claimed = false;
        if (pend) {
            const uint32_t s1 = s + 1;   // s even, cap even
            const uint4 v0 = ld_slot<GT>(T, s), v1 = ld_slot<GT>(T, s1);
            int st = cmp_slot<GT>(T, s, v0, f);
            uint32_t at = s;
            if (st == 1) {
                st = cmp_slot<GT>(T, s1, v1, f);
                at = s1;
            }
            if (st == 0) {
                hit = at;
                pend = false;
                found = true;
            } else if (st == 2) {   // empty: claim it, or learn what the winner wrote
                if (*ovf) {
                    pend = false;
                } else {
                    LA_PSTAT(10, 1);
                    const uint4 o = cas_slot<GT>(T, at, f);
                    if (o.w == 0u) {
                        claimed = found = true;
                        hit = at;
                        pend = false;
                    } else if (same4(o, f)) {
                        found = true;
                        hit = at;
                        pend = false;
                    } else if (at == s) {   // lost slot s to another key: slot s1 is still to test
                        const int st1 = cmp_slot<GT>(T, s1, ld_slot<GT>(T, s1), f);
                        if (st1 == 0) {
                            found = true;
                            hit = s1;
                            pend = false;
                        } else if (st1 == 1) {
                            s = s1 + 1 == T.cap ? 0 : s1 + 1;
                        } else {
                            s = s1 & ~1u;   // s1 empty: the next round starts at its pair (s, s1) again
                        }
                    }
                    // lost slot s1: the next round re-probes the pair (s, s1) — both now occupied
                }
            } else {
                s = s1 + 1 == T.cap ? 0 : s1 + 1;
            }
        }
        if (claimed) LA_PSTAT(3, 1);
        if (claimed) {   // claim list: one shared atomic per claim (claims <= cap: no overflow)
            const int idx = LA_ABL_NOCLAIM ? (int)(hit & 1023u) : atomicAdd(nclaim, 1);
            if (idx >= claim_limit) *ovf = 1;
            T.list[idx] = (uint16_t)hit;
        }
    }
    if (found) vote32d<GT>(T, hit, nb, hi, ovf, vpend);
}

// Convergent lookup (no insert): slot of the key or NONE
template <bool GT>
__device__ __forceinline__ uint32_t warp_lookup32(const Tab32 &T, bool want, const uint4 f, uint32_t h) {
    uint32_t s = slot32(h, T.cap), res = NONE, n = 0;
    bool pend = want;
#ifdef LA_PROBE_STATS
    {
        const unsigned wm = __ballot_sync(0xffffffffu, want);
        if ((threadIdx.x & 31) == 0) { LA_PSTAT(4, 1); LA_PSTAT(6, __popc(wm)); }
    }
#endif
    while (__any_sync(0xffffffffu, pend)) {
        if ((threadIdx.x & 31) == 0) LA_PSTAT(5, 1);
        if (pend) {
            const uint4 v0 = ld_slot<GT>(T, s), v1 = ld_slot<GT>(T, s + 1);
            const int a = cmp_slot<GT>(T, s, v0, f);
            if (a == 0) {
                res = s;
                pend = false;
            } else if (a == 2) {
                pend = false;
            } else {
                const int b = cmp_slot<GT>(T, s + 1, v1, f);
                if (b == 0) {
                    res = s + 1;
                    pend = false;
                } else if (b == 2) {
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

// Scalar lookup (one thread: the start k-mer)
template <bool GT>
__device__ __forceinline__ uint32_t lookup32(const Tab32 &T, const uint4 f, uint32_t h) {
    uint32_t s = slot32(h, T.cap);
    for (uint32_t n = 0; n < T.cap; ++n) {
        const int c = cmp_slot<GT>(T, s, ld_slot<GT>(T, s), f);
        if (c == 0) return s;
        if (c == 2) return NONE;
        s = s + 1 == T.cap ? 0 : s + 1;
    }
    return NONE;
}

__device__ __forceinline__ uint32_t nmask32(uint32_t q) { return q & (q >> 1) & 0x55555555u; }

// Lane-per-position traversal over the end's numbered positions (pref, read by read): builder warp
// `wid` owns [wid*U/nw, (wid+1)*U/nw) and its lanes take 32 consecutive positions per iteration, so
// the hash / probe / vote code runs with the whole warp.  ulen > 0: every read of the end has length
// ulen, so the (read, offset) of a position is one multiply-high (no prefix walk).
// f(inr, act, g, K, h, nb, hi): inr = this lane has a position g this iteration; act = it is a voting
// occurrence (q >= q_lo, no N in the window and in the following base).  rflag = nullptr: no read of
// the end has an N (the class list entry says so), so the k-mer windows are not tested for N.
// SM = true: rseq / rqc are the end's reads staged in shared memory; the word loads then go through
// 32-bit shared-window addresses (LDS) — through the generic pointers nvcc emitted LD.E with 64-bit
// address arithmetic (r02b ncu of k_smem<256>: the extraction loads' line was 14% of the instructions)
__device__ __forceinline__ uint32_t lds32(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
template <int NW>
__device__ __forceinline__ K32<NW> extract32s(uint32_t rowb, int p, const KMask &m) {
    const int q = p >> 4, s = (p & 15) << 1;
    uint32_t x[NW + 1];
#pragma unroll
    for (int i = 0; i <= NW; ++i) x[i] = lds32(rowb + 4u * (uint32_t)((q + i) ^ 1));
    K32<NW> K;
#pragma unroll
    for (int i = 0; i < NW; ++i) K.w[i] = __funnelshift_l(x[i + 1], x[i], s);
    if (NW >= 2) K.w[NW - 2] &= m.m2;
    K.w[NW - 1] &= m.m1;
    return K;
}
__device__ __forceinline__ uint32_t base32s(uint32_t rowb, int i) {
    return (lds32(rowb + 4u * (uint32_t)((i >> 4) ^ 1)) >> (30 - ((i & 15) << 1))) & 3u;
}

template <int NW, int UNR = 1, bool SM = false, typename F>
__device__ __forceinline__ void warp_positions32(const uint32_t *__restrict__ rseq, const uint32_t *__restrict__ rqc,
                                                 const uint8_t *__restrict__ rflag, const uint32_t *pref,
                                                 long long r0, int r, int SW2, int k, int ulen, int wid, int nwarps,
                                                 int lane, const volatile int *stop, F &&f) {
    const uint32_t total = pref[r];
    const uint32_t wb = (uint32_t)(((uint64_t)total * (uint32_t)wid) / (uint32_t)nwarps);
    const uint32_t we = (uint32_t)(((uint64_t)total * (uint32_t)(wid + 1)) / (uint32_t)nwarps);
    if (wb >= we) return;
    const KMask m = kmask32<NW>(k);
    const uint32_t sR = SM ? (uint32_t)__cvta_generic_to_shared(rseq) : 0u;   // staged reads (r0 == 0)
    const uint32_t sQ = SM ? (uint32_t)__cvta_generic_to_shared(rqc) : 0u;
    const uint32_t np = ulen > k ? (uint32_t)(ulen - k) : 1u;
    const uint32_t magic = 0xFFFFFFFFu / np;
    uint32_t g = wb + lane;
    int j = 0;
    uint32_t pj0 = 0, pj1 = 0;
    if (ulen <= 0) {   // mixed read lengths: binary search once, then walk the prefix
        const uint32_t gg = min(g, we - 1);
        int lo = 0, hi = r;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (pref[mid] <= gg) lo = mid; else hi = mid;
        }
        j = lo;
        pj0 = pref[j];
        pj1 = pref[j + 1];
    }
    // UNR > 1 (uniform read lengths only): a lane takes positions g, g+32, ... per iteration, so the
    // independent load -> hash -> filter chains of UNR positions overlap (the filter pass)
    if (UNR > 1 && ulen > 0) {
        for (uint32_t base = wb; base < we; base += 32u * UNR, g += 32u * UNR) {
#pragma unroll
            for (int u = 0; u < UNR; ++u) {
                const uint32_t gu = g + 32u * u;
                const bool act = gu < we;
                uint32_t jj = __umulhi(gu, magic);
                uint32_t pp = gu - jj * np;
                if (pp >= np) { ++jj; pp -= np; }
                const int p = act ? (int)pp : 0;
                const long long row = (r0 + (act ? (int)jj : 0)) * (long long)SW2;
                const uint32_t *R = rseq + row, *Q = rqc + row;
                K32<NW> K;
                uint32_t nb, nq;
                if (SM) {
                    const uint32_t rowo = 4u * (uint32_t)row;
                    K = extract32s<NW>(sR + rowo, p, m);
                    nb = base32s(sR + rowo, p + k);
                    nq = base32s(sQ + rowo, p + k);
                } else {
                    K = extract32<NW>(R, p, m);
                    nb = base32(R, p + k);
                    nq = base32(Q, p + k);
                }
                bool vote = act && (nq - 1u < 2u);
                if (vote && rflag && rflag[r0 + jj]) {
                    const int q = p >> 4, s = (p & 15) << 1;
                    uint32_t any = 0;
#pragma unroll
                    for (int w = 0; w < NW; ++w) {
                        const uint32_t mw = w == NW - 1 ? m.m1 : (w == NW - 2 ? m.m2 : ~0u);
                        any |= __funnelshift_l(nmask32(rw32(Q, q + w + 1)), nmask32(rw32(Q, q + w)), s) & mw;
                    }
                    if (any) vote = false;
                }
                f(act, vote, gu, K, hash32<NW>(K), nb, nq == 2u);
            }
        }
        return;
    }
    for (uint32_t base = wb; base < we; base += 32u, g += 32u) {
        if (((base - wb) & 127u) == 0 && __shfl_sync(0xffffffffu, *stop, 0)) return;   // every 4th iteration
        const bool act = g < we;
        int p;
        if (ulen > 0) {
            uint32_t jj = __umulhi(g, magic);
            uint32_t pp = g - jj * np;
            if (pp >= np) { ++jj; pp -= np; }
            j = (int)jj;
            p = (int)pp;
        } else {
            if (act && g >= pj1) {   // crossed into a later read (skips reads without positions)
                do {
                    pj0 = pj1;
                    pj1 = pref[++j + 1];
                } while (g >= pj1);
            }
            p = (int)(g - pj0);
        }
        const long long row = (r0 + (act ? j : 0)) * (long long)SW2;
        const uint32_t *R = rseq + row, *Q = rqc + row;
        const int i = p + k;
        K32<NW> K;
        uint32_t nb, nq;
        if (SM) {
            const uint32_t rowo = 4u * (uint32_t)row;
            K = extract32s<NW>(sR + rowo, act ? p : 0, m);
            nb = base32s(sR + rowo, act ? i : 0);
            nq = base32s(sQ + rowo, act ? i : 0);
        } else {
            K = extract32<NW>(R, act ? p : 0, m);
            nb = base32(R, act ? i : 0);
            nq = base32(Q, act ? i : 0);
        }
        bool vote = act && (nq - 1u < 2u);
        if (vote && rflag && rflag[r0 + j]) {   // reading #5: a k-mer with an N has no entry (rare)
            const int q = p >> 4, s = (p & 15) << 1;
            uint32_t any = 0;
#pragma unroll
            for (int w = 0; w < NW; ++w) {
                const uint32_t mw = w == NW - 1 ? m.m1 : (w == NW - 2 ? m.m2 : ~0u);
                any |= __funnelshift_l(nmask32(rw32(Q, q + w + 1)), nmask32(rw32(Q, q + w)), s) & mw;
            }
            if (any) vote = false;
        }
        f(act, vote, g, K, hash32<NW>(K), nb, nq == 2u);
    }
}

// Dynamic version for ends whose reads all have length ulen > 0: warps take chunks of 32 * UNR
// consecutive positions from a shared counter (one atomic per chunk) instead of a fixed 1/nwarps
// range, so no warp waits at the pass's closing barrier for a slower one (probe rounds differ).
template <int NW, int UNR, bool SM = false, typename F>
__device__ __forceinline__ void warp_positions32_dyn(const uint32_t *__restrict__ rseq, const uint32_t *__restrict__ rqc,
                                                     const uint8_t *__restrict__ rflag, uint32_t total, long long r0,
                                                     int SW2, int k, int ulen, int lane, const volatile int *stop,
                                                     int *ctr, F &&f) {
    const KMask m = kmask32<NW>(k);
    const uint32_t np = (uint32_t)(ulen - k);
    const uint32_t magic = 0xFFFFFFFFu / np;
    const uint32_t sR = SM ? (uint32_t)__cvta_generic_to_shared(rseq) : 0u;
    const uint32_t sQ = SM ? (uint32_t)__cvta_generic_to_shared(rqc) : 0u;
    for (;;) {
        uint32_t base = 0;
        if (lane == 0) base = (uint32_t)atomicAdd(ctr, 32 * UNR);
        base = __shfl_sync(0xffffffffu, base, 0);
        if (base >= total || __shfl_sync(0xffffffffu, *stop, 0)) return;
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            const uint32_t gu = base + 32u * u + lane;
            const bool act = gu < total;
            uint32_t jj = __umulhi(gu, magic);
            uint32_t pp = gu - jj * np;
            if (pp >= np) { ++jj; pp -= np; }
            const int p = act ? (int)pp : 0;
            const long long row = (r0 + (act ? (int)jj : 0)) * (long long)SW2;
            const uint32_t *R = rseq + row, *Q = rqc + row;
            K32<NW> K;
            uint32_t nb, nq;
            if (SM) {   // r0 == 0 for staged reads: 32-bit row offsets
                const uint32_t rowo = 4u * (uint32_t)row;
                K = extract32s<NW>(sR + rowo, p, m);
                nb = base32s(sR + rowo, p + k);
                nq = base32s(sQ + rowo, p + k);
            } else {
                K = extract32<NW>(R, p, m);
                nb = base32(R, p + k);
                nq = base32(Q, p + k);
            }
            bool vote = act && (nq - 1u < 2u);
            if (vote && rflag && rflag[r0 + jj]) {   // reading #5: a k-mer with an N has no entry (rare)
                const int q = p >> 4, s = (p & 15) << 1;
                uint32_t any = 0;
#pragma unroll
                for (int w = 0; w < NW; ++w) {
                    const uint32_t mw = w == NW - 1 ? m.m1 : (w == NW - 2 ? m.m2 : ~0u);
                    any |= __funnelshift_l(nmask32(rw32(Q, q + w + 1)), nmask32(rw32(Q, q + w)), s) & mw;
                }
                if (any) vote = false;
            }
            f(act, vote, gu, K, hash32<NW>(K), nb, nq == 2u);
        }
    }
}

// (read, offset) of position g of the end (pref: positions per read, exclusive prefix)
__device__ __forceinline__ void pos_of(uint32_t g, const uint32_t *pref, int r, int ulen, int k, int &j, int &p) {
    if (ulen > 0) {
        const uint32_t np = ulen > k ? (uint32_t)(ulen - k) : 1u;
        uint32_t jj = __umulhi(g, 0xFFFFFFFFu / np);
        uint32_t pp = g - jj * np;
        if (pp >= np) { ++jj; pp -= np; }
        j = (int)jj;
        p = (int)pp;
    } else {
        int lo = 0, hi = r;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (pref[mid] <= g) lo = mid; else hi = mid;
        }
        j = lo;
        p = (int)(g - pref[lo]);
    }
}

}  // namespace la
