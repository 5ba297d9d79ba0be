// la_select.cuh — NEXT N4: candidate-read selection on the device (la_select_reads).
//
// The step before local assembly in MetaHipMer: contigs are aligned against the reads and "the reads
// that align to the ends of contigs are then used for extending the contigs" (§2.2; left
// and right sides separately; the paper's GPU aligner is [3]).  The
// paper states no alignment rule; this implements DESIGN.md §10d's readings S1-S6 (the oracle,
// oracle/select.cpp, writes the same definition out with string searches):
//   index  every seed (s-mer without N) of every end window W_e (S1) -> (end, offset), sorted by
//          key (CUB radix sort), one hash-table entry per distinct key -> its run of entries;
//   query  one thread per (read, strand): the stride seeds j = 0, t, 2t, ... of y (the read or its
//          reverse complement) are looked up; a hit (end, offset) gives the diagonal d; the hit is
//          kept only if no earlier stride seed of y matches the same diagonal inside W_e (so every
//          (read, strand, end, d) is examined once), then S2(b) window overlap, S2(c) mismatch rate
//          over the whole contig overlap, S3 outward -> one record (end, pair | mate, strand, d);
//   select records sorted by (end, pair) and, among equal keys, by (mate, strand, d) (two stable
//          radix sorts); the first of each (end, pair) decides the orientation (S4);
//   batch  end_read_off by binary search, read offsets by scan, reads copied in contig-forward
//          orientation (S5-S6), ready for la_load_batch (LA_MEM_DEVICE).
#pragma once
#include <cstdint>

namespace la {
namespace sel {

__device__ __forceinline__ uint32_t code_of(char c) {
    return c == 'A' ? 0u : (c == 'C' ? 1u : (c == 'G' ? 2u : (c == 'T' ? 3u : 4u)));
}
__device__ __forceinline__ char comp_of(char c) {
    return c == 'A' ? 'T' : (c == 'C' ? 'G' : (c == 'G' ? 'C' : (c == 'T' ? 'A' : 'N')));
}
// base j of y = x (strand 0) or rc(x) (strand 1), x = X[0..ly)
__device__ __forceinline__ char y_at(const char *X, int ly, int strand, int j) {
    return strand ? comp_of(X[ly - 1 - j]) : X[j];
}

__device__ __forceinline__ void window_of(const int64_t *coff, int64_t e, int w, int64_t &wl, int64_t &wh,
                                          int64_t &lc) {
    const int64_t c = e >> 1;
    lc = coff[c + 1] - coff[c];
    if (e & 1) {
        wl = lc - w > 0 ? lc - w : 0;
        wh = lc;
    } else {
        wl = 0;
        wh = w < lc ? w : lc;
    }
}

constexpr uint64_t KEY_NONE = ~0ull;

// S1: number of seeds of each end window
__global__ void k_sel_wcount(int64_t n_ends, const int64_t *__restrict__ coff, int w, int s, int64_t *__restrict__ cnt) {
    const int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (e >= n_ends) return;
    int64_t wl, wh, lc;
    window_of(coff, e, w, wl, wh, lc);
    const int64_t n = wh - wl - s + 1;
    cnt[e] = n > 0 ? n : 0;
}

// the index entries: key = 1 << 2s | 2-bit code of the seed (KEY_NONE if it has an N), value = end << 16 | offset
__global__ void k_sel_index(int64_t n_ends, const char *__restrict__ cseq, const int64_t *__restrict__ coff,
                            const int64_t *__restrict__ woff, int w, int s, uint64_t *__restrict__ key,
                            uint64_t *__restrict__ val) {
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (warp >= n_ends) return;
    const int64_t e = warp;
    int64_t wl, wh, lc;
    window_of(coff, e, w, wl, wh, lc);
    const char *C = cseq + coff[e >> 1];
    const int64_t n = woff[e + 1] - woff[e];
    for (int64_t i = lane; i < n; i += 32) {
        uint64_t k = 1ull << (2 * s);
        bool bad = false;
        for (int q = 0; q < s; ++q) {
            const uint32_t b = code_of(C[wl + i + q]);
            bad |= b > 3u;
            k |= (uint64_t)(b & 3u) << (2 * (s - 1 - q));
        }
        key[woff[e] + i] = bad ? KEY_NONE : k;
        val[woff[e] + i] = ((uint64_t)e << 16) | (uint64_t)i;
    }
}

// first entry of each run of equal (valid) keys
__global__ void k_sel_runs(int64_t n, const uint64_t *__restrict__ key, int64_t *__restrict__ flag) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    flag[i] = (key[i] != KEY_NONE && (i == 0 || key[i] != key[i - 1])) ? 1 : 0;
}

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
    x ^= x >> 33;
    x *= 0xff51afd7ed558ccdull;
    x ^= x >> 33;
    x *= 0xc4ceb9fe1a85ec53ull;
    x ^= x >> 33;
    return x;
}

// hash table of the distinct keys: slot = key (0 = empty) + the key's first entry
__global__ void k_sel_hash(int64_t n, const uint64_t *__restrict__ key, const int64_t *__restrict__ flag,
                           const int64_t *__restrict__ uidx, int64_t *__restrict__ ustart, uint64_t cap_mask,
                           unsigned long long *__restrict__ hkey, int64_t *__restrict__ hval) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n || !flag[i]) return;
    const uint64_t k = key[i];
    ustart[uidx[i]] = i;
    uint64_t h = mix64(k) & cap_mask;
    for (;;) {
        const unsigned long long old = atomicCAS(&hkey[h], 0ull, (unsigned long long)k);
        if (old == 0ull) {
            hval[h] = uidx[i];
            return;
        }
        h = (h + 1) & cap_mask;
    }
}

// the number of valid entries (the position of the first KEY_NONE in the sorted keys)
__global__ void k_sel_nvalid(int64_t n, const uint64_t *__restrict__ key, int64_t *__restrict__ out) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    if (key[i] != KEY_NONE && (i == n - 1 || key[i + 1] == KEY_NONE)) *out = i + 1;
}

__device__ __forceinline__ int64_t sel_lookup(const unsigned long long *__restrict__ hkey, const int64_t *__restrict__ hval,
                                              uint64_t cap_mask, uint64_t k) {
    uint64_t h = mix64(k) & cap_mask;
    for (;;) {
        const unsigned long long v = hkey[h];
        if (v == k) return hval[h];
        if (v == 0ull) return -1;
        h = (h + 1) & cap_mask;
    }
}

// S2-S3 for one (read, strand) per thread; records: rkey = end << 32 | pair, rord = mate << 31 | strand << 30 |
// (d + 2^29)
__global__ void k_sel_query(int64_t n_reads, const char *__restrict__ rseq, const int64_t *__restrict__ roff,
                            const char *__restrict__ cseq, const int64_t *__restrict__ coff, int w, int s, int t,
                            int o, int mm, const unsigned long long *__restrict__ hkey, const int64_t *__restrict__ hval,
                            uint64_t cap_mask, const int64_t *__restrict__ ustart, const uint64_t *__restrict__ val,
                            unsigned long long *__restrict__ n_rec, int64_t cap_rec, uint64_t *__restrict__ rkey,
                            uint32_t *__restrict__ rord) {
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (tid >= 2 * n_reads) return;
    const int64_t r = tid >> 1;
    const int strand = (int)(tid & 1);
    const char *X = rseq + roff[r];
    const int ly = (int)(roff[r + 1] - roff[r]);
    for (int j = 0; j + s <= ly; j += t) {
        uint64_t k = 1ull << (2 * s);
        bool bad = false;
        for (int q = 0; q < s; ++q) {
            const uint32_t b = code_of(y_at(X, ly, strand, j + q));
            bad |= b > 3u;
            k |= (uint64_t)(b & 3u) << (2 * (s - 1 - q));
        }
        if (bad) continue;
        const int64_t u = sel_lookup(hkey, hval, cap_mask, k);
        if (u < 0) continue;
        for (int64_t q = ustart[u]; q < ustart[u + 1]; ++q) {
            const uint64_t v = val[q];
            const int64_t e = (int64_t)(v >> 16);
            int64_t wl, wh, lc;
            window_of(coff, e, w, wl, wh, lc);
            const int64_t d = wl + (int64_t)(v & 0xffffu) - j;
            const char *C = cseq + coff[e >> 1];
            // examined once: skip if an earlier stride seed of y hits the same diagonal in the window
            bool dup = false;
            for (int j2 = j - t; j2 >= 0 && d + j2 >= wl && !dup; j2 -= t) {
                if (d + j2 + s > wh) continue;
                bool eq = true;
                for (int q2 = 0; q2 < s && eq; ++q2) {
                    const char a = y_at(X, ly, strand, j2 + q2), b = C[d + j2 + q2];
                    eq = a == b && code_of(a) < 4u;
                }
                dup = eq;
            }
            if (dup) continue;
            // S2(b): window overlap
            const int64_t ov = (d + ly < wh ? d + ly : wh) - (d > wl ? d : wl);
            if (ov < o) continue;
            // S3: outward
            const bool outward = (e & 1) ? (strand == 0 || d + ly > lc) : (strand == 1 || d < 0);
            if (!outward) continue;
            // S2(c): mismatches over the whole contig overlap (N is a mismatch)
            const int64_t a0 = d > 0 ? d : 0, a1 = d + ly < lc ? d + ly : lc;
            int64_t M = 0;
            for (int64_t p = a0; p < a1; ++p) {
                const char a = y_at(X, ly, strand, (int)(p - d)), b = C[p];
                M += (a != b || code_of(a) > 3u) ? 1 : 0;
            }
            if (100 * M > (int64_t)mm * (a1 - a0)) continue;
            const unsigned long long idx = atomicAdd(n_rec, 1ull);
            if ((int64_t)idx < cap_rec) {
                rkey[idx] = ((uint64_t)e << 32) | (uint64_t)(r >> 1);
                rord[idx] = ((uint32_t)(r & 1) << 31) | ((uint32_t)strand << 30) | (uint32_t)(d + (1 << 29));
            }
        }
    }
}

// S4: first record of each (end, pair) (records sorted by key, then ord)
__global__ void k_sel_first(int64_t n, const uint64_t *__restrict__ key, int64_t *__restrict__ flag) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    flag[i] = (i == 0 || key[i] != key[i - 1]) ? 1 : 0;
}

__global__ void k_sel_compact(int64_t n, const uint64_t *__restrict__ key, const uint32_t *__restrict__ ord,
                              const int64_t *__restrict__ flag, const int64_t *__restrict__ pos,
                              int64_t *__restrict__ sel_end, int64_t *__restrict__ sel_pair, uint8_t *__restrict__ sel_flip) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= n || !flag[i]) return;
    const int64_t j = pos[i];
    sel_end[j] = (int64_t)(key[i] >> 32);
    sel_pair[j] = (int64_t)(key[i] & 0xffffffffull);
    const uint32_t mate = ord[i] >> 31, strand = (ord[i] >> 30) & 1u;
    sel_flip[j] = (uint8_t)((mate == 0u) == (strand == 1u));
}

// S6: end_read_off[e] = 2 x (selected pairs of ends < e); lens of the output reads
__global__ void k_sel_eoff(int64_t n_ends, int64_t n_sel, const int64_t *__restrict__ sel_end, int64_t *__restrict__ eoff) {
    const int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (e > n_ends) return;
    int64_t lo = 0, hi = n_sel;   // first j with sel_end[j] >= e
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (sel_end[mid] < e) lo = mid + 1; else hi = mid;
    }
    eoff[e] = 2 * lo;
}

__global__ void k_sel_lens(int64_t n_sel, const int64_t *__restrict__ sel_pair, const int64_t *__restrict__ roff,
                           int64_t *__restrict__ lens) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= 2 * n_sel) return;
    const int64_t src = 2 * sel_pair[i >> 1] + (i & 1);
    lens[i] = roff[src + 1] - roff[src];
}

// S5: one warp per output read; reverse complement (qualities reversed) for the mate on the - strand
__global__ void k_sel_copy(int64_t n_sel, const int64_t *__restrict__ sel_pair, const uint8_t *__restrict__ sel_flip,
                           const char *__restrict__ rseq, const char *__restrict__ rqual, const int64_t *__restrict__ roff,
                           const int64_t *__restrict__ ooff, char *__restrict__ oseq, char *__restrict__ oqual) {
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (warp >= 2 * n_sel) return;
    const int mate = (int)(warp & 1);
    const int64_t src = 2 * sel_pair[warp >> 1] + mate;
    const bool rc = (mate == 0) == (sel_flip[warp >> 1] != 0);
    const int64_t a = roff[src], L = roff[src + 1] - a, dst = ooff[warp];
    for (int64_t i = lane; i < L; i += 32) {
        if (rc) {
            oseq[dst + i] = comp_of(rseq[a + L - 1 - i]);
            oqual[dst + i] = rqual[a + L - 1 - i];
        } else {
            oseq[dst + i] = rseq[a + i];
            oqual[dst + i] = rqual[a + i];
        }
    }
}

}  // namespace sel
}  // namespace la
