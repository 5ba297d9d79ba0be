// la_device.cuh — device-side building blocks of the sm_100a local-assembly path.
//
// Encodings (DESIGN.md §6 "Data layout in HBM"):
//  * bases: 2 bits (A0 C1 G2 T3), big-endian inside u64 words: base i of a read sits in word i/32
//    at bit 62 - 2*(i%32).  Every read owns SW words (zero padded) in `rseq`.
//  * quality class, same layout in `rqc`: 0 = no vote (q < q_lo), 1 = low-tier vote
//    (q_lo <= q < q_hi), 2 = both tiers (q >= q_hi), 3 = the base is N (reading #2, #5).
//  * k-mers: KW = ceil(2k/64) u64 words, left aligned (base 0 in the top bits of word 0), the
//    2*(32*KW-k) low bits of the last word zero.
//  * table slot: u64 = tag(23) | read(32) | pos(9); 0 = empty.  The key is NOT stored: it is the
//    k-mer of read `read` at `pos` (pointer-encoded key, Fig 6), verified against the
//    packed read on every tag match, so equality is exact.
#pragma once
#include <cstdint>

namespace la {

constexpr int MAX_KW = 4;            // k <= 128
constexpr int MAX_READ_LEN = 300;
constexpr uint32_t NONE = 0x1FFFFFFFu;
enum : int { CODE_FORK = 4, CODE_DEADEND = 5 };
enum : int { T_DEADEND = 0, T_FORK = 1, T_LOOP = 2, T_MAXLEN = 3, T_NOREADS = 4, T_SHORT = 5 };

struct DevParams {
    int k_start, k_min, k_max, k_shift, W, qual_offset, q_lo, q_hi, V, F;
    int replay;   // 1: build-only replay of the recorded attempts (la_replay_build); 0: extension
    int maxlen;   // longest read of the batch (LIST_UNIFORM ends: every read has this length)
};

__host__ __device__ __forceinline__ int kwords(int k) { return (2 * k + 63) >> 6; }

// A k-mer with at most NW words (NW = 2 covers k <= 64: the inline-key path keeps half the registers).
template <int NW>
struct KmerN {
    uint64_t w[NW];
};
using Kmer = KmerN<MAX_KW>;

__device__ __forceinline__ uint64_t funnel64(uint64_t hi, uint64_t lo, int s) {
    return s ? ((hi << s) | (lo >> (64 - s))) : hi;
}

// k-mer of length k starting at base p of the packed sequence R (words in any address space).
// Written with per-word selects only (no "if (w == KW - 1)" updates): that form lets the compiler turn
// the unrolled loop into one dynamically indexed store, which puts the k-mer in local memory.
template <int NW = MAX_KW, typename P>
__device__ __forceinline__ KmerN<NW> extract_kmer(const P *R, int p, int k, int KW) {
    KmerN<NW> K;
    const int q = p >> 5, s = (p & 31) << 1;
#pragma unroll
    for (int w = 0; w < NW; ++w) {
        const int bits = 2 * k - 64 * w;   // bits of word w that belong to the k-mer (> 0 iff w < KW)
        const uint64_t m = bits >= 64 ? ~0ull : (~0ull << (64 - bits));
        K.w[w] = w < KW ? (funnel64(R[q + w], R[q + w + 1], s) & m) : 0ull;
    }
    return K;
}

// next_kmer (Alg 2 line 15): drop base 0, append base b (the new base k-1 lands in word (k-1)/32).
template <int NW>
__device__ __forceinline__ void roll_kmer(KmerN<NW> &K, int k, int KW, uint32_t b) {
    (void)KW;
    const int wl = (k - 1) >> 5;
    const uint64_t nb = ((uint64_t)b * 0x5555555555555555ull) & (3ull << (62 - 2 * ((k - 1) & 31)));
#pragma unroll
    for (int w = 0; w < NW; ++w) {
        const uint64_t carry = (w + 1 < NW) ? (K.w[(w + 1 < NW) ? w + 1 : w] >> 62) : 0ull;
        K.w[w] = (K.w[w] << 2) | carry | (w == wl ? nb : 0ull);
    }
}

template <int NW>
__device__ __forceinline__ bool kmer_eq(const KmerN<NW> &a, const KmerN<NW> &b, int KW) {
    bool eq = true;
#pragma unroll
    for (int w = 0; w < NW; ++w)
        if (w < KW) eq &= (a.w[w] == b.w[w]);
    return eq;
}

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
    x ^= x >> 30;
    x *= 0xbf58476d1ce4e5b9ull;
    x ^= x >> 27;
    x *= 0x94d049bb133111ebull;
    x ^= x >> 31;
    return x;
}

// Hash of a k-mer: polynomial combine of the words + murmur3 fmix64.  The hash function does not
// affect results (reading #17), only probe lengths and filter false positives.
template <int NW>
__device__ __forceinline__ uint64_t hash_kmer(const KmerN<NW> &K, int KW) {
    if (NW <= 2) {
        // k <= 64: a 32-bit multiply-xorshift mix of the four 32-bit halves (fewer instructions than
        // 64-bit arithmetic); the high word (filter index, tag) is a second multiplicative mix.
        const uint64_t w1 = (NW > 1 && KW > 1) ? K.w[NW > 1 ? 1 : 0] : 0ull;
        uint32_t h = ((uint32_t)K.w[0] ^ ((uint32_t)(K.w[0] >> 32) * 0x85EBCA6Bu)) * 0xCC9E2D51u;
        h ^= ((uint32_t)w1 ^ ((uint32_t)(w1 >> 32) * 0x27D4EB2Fu)) * 0x1B873593u;
        h ^= h >> 15;
        h *= 0x2C1B3C6Du;
        h ^= h >> 12;
        const uint32_t g = (h ^ (h >> 16)) * 0x9E3779B9u;
        return ((uint64_t)(g | 1u) << 32) | h;
    }
    uint64_t h = K.w[0];
#pragma unroll
    for (int w = 1; w < NW; ++w)
        if (w < KW) h = h * 0x9E3779B97F4A7C15ull + K.w[w];
    h ^= h >> 33;
    h *= 0xff51afd7ed558ccdull;
    h ^= h >> 33;
    h *= 0xc4ceb9fe1a85ec53ull;
    h ^= h >> 33;
    return h;
}

__device__ __forceinline__ uint32_t slot_of(uint64_t h, uint32_t cap) {
    return (uint32_t)(((uint64_t)(uint32_t)h * cap) >> 32);
}
__device__ __forceinline__ uint64_t tag_of(uint64_t h) { return ((h >> 41) | 1ull) << 41; }
__device__ __forceinline__ uint64_t make_slot(uint64_t tag, uint32_t read, uint32_t pos) {
    return tag | ((uint64_t)read << 9) | pos;
}
__device__ __forceinline__ uint32_t slot_read(uint64_t w) { return (uint32_t)(w >> 9); }
__device__ __forceinline__ uint32_t slot_pos(uint64_t w) { return (uint32_t)(w & 511u); }
constexpr uint64_t TAG_MASK = ~((1ull << 41) - 1);

__device__ __forceinline__ uint32_t get2(const uint64_t *R, int i) {
    return (uint32_t)(R[i >> 5] >> (62 - ((i & 31) << 1))) & 3u;
}

// Reading #1: two-tier vote rule on exact integer counts.  Returns 0..3 (base), CODE_FORK or
// CODE_DEADEND.  Branch-free (selects only): it runs slot-parallel in the link pass, where data-
// dependent branches split the warp.
__device__ __forceinline__ int ext_rule(const uint32_t lo[4], const uint32_t hi[4], int V, int F) {
    const uint64_t H = (uint64_t)hi[0] + hi[1] + hi[2] + hi[3];
    const uint64_t L = (uint64_t)lo[0] + lo[1] + lo[2] + lo[3];
    uint32_t mh = 0, ml = 0;
#pragma unroll
    for (int b = 0; b < 4; ++b) {
        mh |= (hi[b] >= (uint32_t)V && 100ull * hi[b] >= (uint64_t)F * H) ? (1u << b) : 0u;
        ml |= (lo[b] >= (uint32_t)V && 100ull * lo[b] >= (uint64_t)F * L) ? (1u << b) : 0u;
    }
    const uint32_t m = mh ? mh : ml;   // the high tier decides when it has a candidate
    const int one = __ffs(m) - 1;
    return m == 0 ? CODE_DEADEND : ((m & (m - 1)) ? CODE_FORK : one);
}

// Same rule in 32-bit arithmetic, for tables whose counters are bounded well below 2^32 / 100 (the
// shared-memory classes' 8-bit fields, the XL class's fields for at most XL_MAX_U = 2^21 occurrences):
// 100 x count and F x total then fit in 32 bits, exactly as the 64-bit products above.
__device__ __forceinline__ int ext_rule32(const uint32_t lo[4], const uint32_t hi[4], int V, int F) {
    const uint32_t H = hi[0] + hi[1] + hi[2] + hi[3];
    const uint32_t L = lo[0] + lo[1] + lo[2] + lo[3];
    uint32_t mh = 0, ml = 0;
#pragma unroll
    for (int b = 0; b < 4; ++b) {
        mh |= (hi[b] >= (uint32_t)V && 100u * hi[b] >= (uint32_t)F * H) ? (1u << b) : 0u;
        ml |= (lo[b] >= (uint32_t)V && 100u * lo[b] >= (uint32_t)F * L) ? (1u << b) : 0u;
    }
    const uint32_t m = mh ? mh : ml;   // the high tier decides when it has a candidate
    const int one = __ffs(m) - 1;
    return m == 0 ? CODE_DEADEND : ((m & (m - 1)) ? CODE_FORK : one);
}

// N in bases [lo, hi) of a contig tail whose N mask is the 128-bit pair (n0, n1) (bit i = base i):
// two masked ANDs instead of a per-base loop (reading #5, the start k-mer's N test)
__device__ __forceinline__ bool any_n_range(uint64_t n0, uint64_t n1, int lo, int hi) {
    auto rng = [](int a, int b) -> uint64_t {   // bits [a, b) of one 64-bit word, a and b clamped to [0, 64]
        a = a < 0 ? 0 : (a > 64 ? 64 : a);
        b = b < 0 ? 0 : (b > 64 ? 64 : b);
        if (a >= b) return 0ull;
        const uint64_t upto = b >= 64 ? ~0ull : ((1ull << b) - 1ull);
        return upto & ~((1ull << a) - 1ull);
    };
    return ((n0 & rng(lo, hi)) | (n1 & rng(lo - 64, hi - 64))) != 0ull;
}

// The k up/down-shift rule (readings #8, #10).  Returns true when the end is done,
// else updates k / shift for the next attempt.
__device__ __forceinline__ bool next_k(int term, int &k, int &shift, int kmax_eff, const DevParams &P) {
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

}  // namespace la
