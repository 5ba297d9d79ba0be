// la_smem.cuh — planner and the table kernels.
//
// Per attempt (one k) of one contig end, `build_link` runs on the CTA's builder warps:
//   [filter pass]  only when the unfiltered table may not fit: every voting k-mer occurrence sets a
//                  bit in B1 (atomicOr); a second sighting sets its bit in B2.  k-mers with fewer than
//                  two voting occurrences cannot reach min_votes >= 2, so they extend exactly like
//                  absent k-mers (DEADEND) and may be left out (reading #4); bitmap collisions only
//                  admit extra k-mers, never exclude one.
//   [build, Alg 1] every voting occurrence that passed the filter is inserted into an
//                  open-addressing table (shared memory; XL: L2-resident global scratch).  k <= 63: the
//                  slot holds the 2-bit k-mer itself (16 B), claimed with one 128-bit CAS; k >= 64: the
//                  slot holds tag|read|pos (pointer key), verified against the read.  The
//                  vote for the following base is one atomic on 8-bit counters (high-tier
//                  and low-only words; a carry re-routes the end to the global path).
//   [link]         per claimed slot (claim list): ext(lo, hi) (reading #1) and, for a base, the slot of
//                  the successor k-mer (next_kmer, Alg 2 line 15) -> a link word.
// All three passes are warp-convergent: lane per position (or per claimed slot), whole-warp probe
// rounds, claims counted once per warp.
// The walk (Alg 2) follows the link words from the start k-mer with a visited bit per
// slot (the loop-check table), then the k-shift rule picks the next k.
//   k_small (small tables): one end per CTA; every warp builds, thread 0 walks; reads staged once.
//   k_smem  (larger tables): one walker warp + builders, two ends in flight (mbarrier hand-off), so
//           the walk of one end overlaps the build of the other; XL streams reads from L2/HBM.
#pragma once
#include "la_device.cuh"
#include "la_inl32.cuh"
#include <type_traits>

namespace la {

enum : int { CLS_NOREADS = 0, CLS_SHORT = 1, CLS_S = 2, CLS_GLOBAL = 8 };   // CLS_S + class index (5 = XL)
// Phase clocks (tools/phase_profile.py builds with -DLA_PROFILE_CLOCKS=1): compiled out by default so
// the per-phase cycle accumulators take no registers in the production kernels.
#ifndef LA_PROFILE_CLOCKS
#define LA_PROFILE_CLOCKS 0
#endif
__device__ __forceinline__ long long la_clock() {
#if LA_PROFILE_CLOCKS
    return clock64();
#else
    return 0;
#endif
}

#ifndef LA_FQUEUE
#define LA_FQUEUE 0   // 1: filtered builds keep per-position filter indices and queue survivors (r02 experiment)
#endif
#ifndef LA_LDS_READS
#define LA_LDS_READS 1   // staged reads read through 32-bit shared addresses (LDS) in the dyn traversal
#endif
#ifndef LA_SMALL_FILTER_UNROLL
#define LA_SMALL_FILTER_UNROLL 2   // the same in k_small (less code per copy with 1: instruction-cache pressure)
#endif
#ifndef LA_FILTER_UNROLL
#define LA_FILTER_UNROLL 2   // positions per lane per iteration of the filter pass (la_inl32.cuh)
#endif
#ifndef LA_DYN
#define LA_DYN 1   // dynamic 32-position chunks in the filter / build passes of the shared-memory classes
                   // (warp_positions32_dyn; XL measured slower with them)
#endif
#ifndef LA_ANYN
#define LA_ANYN 1   // skip the per-position N test for ends without an N read (class list flag)
#endif
#ifndef LA_DEAD0
#define LA_DEAD0 1   // decide attempts whose start k-mer fails the filter without building (inl32_build_link)
#endif
#ifndef LA_WALK_PIPE
#define LA_WALK_PIPE 1   // software-pipelined walker loop (walk_links)
#endif
#ifndef LA_WALK_PIPE_SMALL
#define LA_WALK_PIPE_SMALL 0   // k_small: thread 0 walks with walk_links (pipelined) instead of its plain loop
#endif
#ifndef LA_NW_MERGE23
#define LA_NW_MERGE23 1   // k <= 32 on the 3-word inline path too (one code copy fewer: instruction-cache pressure)
#endif
#ifndef LA_UNIFORM_FLAG
#define LA_UNIFORM_FLAG 1   // planner marks ends whose reads all have the batch's longest length
#endif
#ifndef LA_STREAM_BIG
#define LA_STREAM_BIG 1   // largest shared-memory class also takes ends whose reads stay in global memory
#endif
#ifndef LA_MAX_LOAD
#define LA_MAX_LOAD 0.80f
#endif
constexpr float SMEM_MAX_LOAD = LA_MAX_LOAD;   // table load above which an end overflows (claims)

// ---- shared-memory layout ------------------------------------------------------------------------
// [info0: icap u32][info1: icap u32][walk strings: 4 x Wp][table region: B1 | B2 | keys | cnts]
// Two slot formats.  INLINE (k <= 63): 16 B key; REF (k >= 64): 8 B tag|read|pos.  + 8 B counters.
__host__ __device__ __forceinline__ bool inline_keys(int k) { return k <= 63; }
__host__ __device__ __forceinline__ uint32_t key_bytes(int k) { return inline_keys(k) ? 16u : 8u; }

struct SmemFixed {
    uint32_t icap;        // slots an info buffer can describe (max table capacity)
    uint32_t off_info1, off_walk, off_tab, tab_bytes;
    uint32_t off_filt, filt_bytes;   // XL only: the filter bitmaps stay in shared memory
    uint32_t off_queue;              // per builder warp: 64 x u32 survivor queue (build pass)
};
// survivor queue of the build pass (la_inl32.cuh): 64 positions per builder warp
__host__ __device__ __forceinline__ uint32_t queue_bytes(int nbw) { return LA_FQUEUE ? (uint32_t)nbw * 64u * 4u : 0u; }

constexpr uint32_t XL_ICAP = 16384u;   // XL: info buffers of 64 KB each; the rest of smem = filter

// gt_stride > 0: the table lives in a per-CTA global-memory scratch of gt_stride bytes (XL class);
// shared memory then holds the two info buffers, the walk strings and the filter bitmaps.
// single = true: one end in flight (k_small): one info buffer and two walk strings.
__host__ __device__ __forceinline__ SmemFixed smem_fixed(int W, uint32_t bytes, uint32_t gt_stride, bool single,
                                                         int nbw) {
    SmemFixed F;
    const uint32_t qb = queue_bytes(nbw);   // the queues sit at the end of the dynamic region
    bytes = bytes > qb + 256u ? ((bytes - qb) & ~15u) : 0u;
    F.off_queue = bytes;
    const uint32_t Wp = ((uint32_t)W + 15u) & ~15u;
    const uint32_t nwalk = single ? 2u : 4u;
    const uint32_t fixed = nwalk * Wp + 128u;
    const uint32_t rem = bytes > fixed ? bytes - fixed : 0u;
    if (gt_stride) {
        F.icap = rem / 16u;   // at most half of shared memory for the info buffers
        if (F.icap > XL_ICAP) F.icap = XL_ICAP;
        F.icap &= ~3u;
    } else {
        F.icap = (rem / (single ? 28u : 32u)) & ~3u;   // 24 B inline slot + 4 B info per end in flight
    }
    F.off_info1 = single ? 0u : F.icap * 4u;
    F.off_walk = (single ? 0u : F.off_info1) + F.icap * 4u;
    const uint32_t after = (F.off_walk + nwalk * Wp + 15u) & ~15u;
    if (gt_stride) {
        F.off_tab = 0u;   // relative to the CTA's global scratch
        F.tab_bytes = gt_stride;
        F.off_filt = after;
        F.filt_bytes = bytes > after + 32u ? ((bytes - after - 32u) & ~31u) : 0u;
    } else {
        F.off_tab = after;
        F.tab_bytes = bytes > F.off_tab + 32u ? bytes - F.off_tab - 32u : 0u;
        F.off_filt = 0u;
        F.filt_bytes = 0u;
    }
    return F;
}

struct SmemTab {
    uint32_t off_pref, off_b1, off_b2, off_keys, off_cnts, off_list, cap, mwords;
    uint32_t off_f;   // filtered tables: per position its filter bit index (u16 shared / u32 XL global)
};

__host__ __device__ __forceinline__ uint32_t pref_bytes(int r) { return (((uint32_t)r + 1u) * 4u + 15u) & ~15u; }
// shared-memory copy of the end's reads: packed bases + quality classes (SW words each), u16 length,
// u8 has-N flag
__host__ __device__ __forceinline__ uint32_t stage_bytes(int r, int SW) {
    return (((uint32_t)r * (uint32_t)SW * 16u + (uint32_t)r * 3u) + 15u) & ~15u;
}
// per-position filter indices of a filtered build (la_inl32.cuh): u16 in shared memory (bit indices
// < 65535, so at most MAX_SMEM_MBITS filter bits), u32 in the XL class's global scratch
constexpr uint32_t MAX_SMEM_MBITS = 65504u;
__host__ __device__ __forceinline__ uint32_t fpos_bytes(uint32_t U, bool gt) {
    return LA_FQUEUE ? (((gt ? 4u : 2u) * U + 15u) & ~15u) : 0u;
}

// U = voting-occurrence upper bound (sum over reads of max(0, len-k)); the table region starts with
// the per-read position prefix array (pref_bytes(r)).
// Counters: shared-memory tables pack lo[4] | hi[4] as 8-bit fields (8 B, carry detected); global
// (XL) tables use 8 x u32 (32 B) updated with fire-and-forget RED.ADD.
// counter bytes per slot: shared tables 8 (8-bit fields), XL 16 (16-bit fields) or 32 (wide, U >= 65536)
__host__ __device__ __forceinline__ uint32_t cnt_bytes(bool gt, bool wide = false) { return gt ? (wide ? 32u : 16u) : 8u; }
__host__ __device__ __forceinline__ bool xl_wide(uint32_t U) { return U >= 65536u; }

__host__ __device__ __forceinline__ SmemTab smem_tab(const SmemFixed &F, uint32_t U, bool allow_filter,
                                                     uint32_t kbytes, int r, bool gt, int SW, bool staged = true) {
    const bool wide = gt && xl_wide(U);
    SmemTab T;
    const uint32_t sb = (gt || !staged) ? 0u : stage_bytes(r, SW);   // shared-memory tables: reads staged first
    const uint32_t pb = pref_bytes(r) + sb;
    const uint32_t tab = F.tab_bytes > pb ? F.tab_bytes - pb : 0u;
    const uint32_t per_slot = kbytes + cnt_bytes(gt, wide) + 2u;   // key + counters + claim-list entry (u16)
    uint32_t cap_nf = tab / per_slot;
    if (cap_nf > F.icap) cap_nf = F.icap;
    cap_nf &= ~1u;
    uint32_t mwords = 0, cap = cap_nf;
    const bool filt = allow_filter && (float)U > SMEM_MAX_LOAD * (float)cap_nf;
    if (gt) {   // filter in shared memory, table (after the prefix array) in the global scratch
        if (filt) {
            mwords = (4u * U + 31u) / 32u;
            const uint32_t maxw = F.filt_bytes / 8u;
            if (mwords > maxw) mwords = maxw;
            mwords &= ~3u;
        }
        T.off_pref = 0u;
        T.off_b1 = F.off_filt;
        T.off_b2 = T.off_b1 + mwords * 4u;
        T.off_keys = pb;
    } else {
        if (filt) {
            // two bitmaps of ~4 bits per occurrence each (at most a quarter of the region each and
            // MAX_SMEM_MBITS bits), then the u16 filter index of every position
            mwords = (4u * U + 31u) / 32u;
            const uint32_t maxw = tab / 16u;
            if (mwords > maxw) mwords = maxw;
            if (LA_FQUEUE && mwords > MAX_SMEM_MBITS / 32u) mwords = MAX_SMEM_MBITS / 32u;
            mwords &= ~3u;
            const uint32_t used = 8u * mwords + fpos_bytes(U, false) + 16u;
            const uint32_t rem = tab > used ? tab - used : 0u;
            cap = rem / per_slot;
            if (cap > F.icap) cap = F.icap;
            cap &= ~1u;
        }
        T.off_pref = F.off_tab + sb;
        T.off_b1 = F.off_tab + pb;
        T.off_b2 = T.off_b1 + mwords * 4u;
        T.off_keys = (T.off_b2 + mwords * 4u + (mwords ? fpos_bytes(U, false) : 0u) + 15u) & ~15u;
    }
    T.cap = cap;
    T.mwords = mwords;
    T.off_cnts = T.off_keys + cap * kbytes;
    T.off_list = T.off_cnts + cap * cnt_bytes(gt, wide);
    // shared: right after B2; XL: in the global scratch after the claim list
    T.off_f = gt ? ((T.off_list + cap * 2u + 15u) & ~15u) : (T.off_b2 + mwords * 4u);
    return T;
}

// ---- XLC class (la_xlc.cuh): one end per 2-CTA cluster, table split over both SMs (DSMEM) ----
constexpr int XLC_THREADS = 1024;
constexpr uint32_t XLC_MAX_U = 65535u;   // 16-bit counter fields cannot carry below this
// Shared-memory layout of each CTA: [stage reads (if staged)][pref][B1 half | B2 half][keys half]
// [counters half][claim list][rank 0: info (cap x u32)] ... [2 walk strings at the end of the region,
// fixed across attempts].  Identical in both CTAs (info unused in rank 1), from (r, U, bytes, stage).
struct XlcLayout {
    uint32_t off_pref, off_b1, off_b2, off_keys, off_cnts, off_list, off_info, off_walk;
    uint32_t cap, half, hw, mwords;
    bool fits;
};
__host__ __device__ __forceinline__ float xlc_filtered_fraction(int r) {
    return r < 50 ? 0.30f : (r < 200 ? 0.16f : 0.10f);   // as the planner's filtered_fraction
}
__host__ __device__ __forceinline__ XlcLayout xlc_layout(uint32_t bytes, int r, int SW, uint32_t U, int W, bool stage) {
    XlcLayout L;
    const uint32_t Wp = ((uint32_t)(W > 0 ? W : 1) + 15u) & ~15u;
    const uint32_t sb = ((uint32_t)r * (uint32_t)SW * 16u + (uint32_t)r * 3u + 15u) & ~15u;
    const uint32_t pb = (((uint32_t)r + 1u) * 4u + 15u) & ~15u;
    const float est = (float)U * xlc_filtered_fraction(r) + 1024.f;   // filtered keys + margin, load <= 0.7
    // (no in-flight margin: warp_insert_c bounds every probe sequence, a full table overflows)
    uint32_t cap = ((uint32_t)(est / SMEM_MAX_LOAD) + 3u) & ~3u;
    if (cap < 4096u) cap = 4096u;
    L.cap = cap;
    L.half = cap / 2u;
    L.mwords = ((4u * U + 31u) / 32u + 7u) & ~7u;   // words of each bitmap (4 bits per occurrence)
    L.hw = L.mwords / 2u;
    L.off_walk = bytes > 2u * Wp ? ((bytes - 2u * Wp) & ~15u) : 0u;
    uint32_t o = stage ? sb : 0u;
    L.off_pref = o;
    o += pb;
    L.off_b1 = o;
    o += L.hw * 4u;
    L.off_b2 = o;
    o += L.hw * 4u;
    o = (o + 15u) & ~15u;
    L.off_keys = o;
    o += L.half * 16u;
    L.off_cnts = o;
    o += L.half * 16u;
    L.off_list = o;
    o += cap * 2u;   // one CTA may claim up to its limit (0.45 cap) of the whole table
    o = (o + 15u) & ~15u;
    L.off_info = o;
    o += cap * 4u;
    L.fits = o <= L.off_walk && U <= XLC_MAX_U && L.half <= 32768u && bytes > 2u * Wp;
    return L;
}


// ---- plan ------------------------------------------------------------------------------------
// Routing estimate of the filtered table: distinct k-mers with >= 2 voting occurrences plus filter
// false positives, as a fraction of the occurrences (measured on C2/C4 samples: 0.05-0.2, higher for
// ends with few reads).  A wrong guess only costs a redo in the global path.
// r02b (LA_FRAC_V2): finer buckets from the measured claims per occurrence (k-mers seen >= 2 times plus
// the expected filter false positives, 4 bits per occurrence per bitmap) on C4 ends at k = 21 and 33:
// maxima 0.34 / 0.33 / 0.22 / 0.14 / 0.11 / 0.06 / 0.085 for r < 10 / 25 / 50 / 100 / 200 / 400 / more
// (DESIGN.md §7); r01's three buckets (0.30 / 0.16 / 0.10) over-reserved the large ends ~1.7x.
#ifndef LA_FRAC_V2
#define LA_FRAC_V2 1
#endif
__host__ __device__ __forceinline__ float filtered_fraction(int64_t r) {
#if LA_FRAC_V2
    return r < 10 ? 0.36f : (r < 25 ? 0.34f : (r < 50 ? 0.24f : (r < 100 ? 0.16f : (r < 200 ? 0.12f : (r < 400 ? 0.075f : 0.095f)))));
#else
    return r < 50 ? 0.30f : (r < 200 ? 0.16f : 0.10f);
#endif
}

__host__ __device__ __forceinline__ uint32_t min_table_cap(uint32_t threads) { return 4u * threads; }

__device__ __forceinline__ bool fits(int64_t r, int64_t U, const DevParams &P, uint32_t bytes, uint32_t threads,
                                     int SW, bool single, bool stream = false) {
    const uint32_t min_cap = min_table_cap(threads);
    if (bytes == 0) return false;
    const SmemFixed F = smem_fixed(P.W, bytes, 0u, single, single ? (int)(threads / 32u) : (int)(threads / 32u) - 1);
    if (F.tab_bytes == 0) return false;
    if (r > 16384) return false;
    const SmemTab T = smem_tab(F, (uint32_t)U, P.V >= 2, key_bytes(P.k_min), (int)r, false, SW, !stream);
    if (T.cap < min_cap) return false;
    if (T.mwords == 0) return true;   // U <= 0.7 cap: cannot overflow
    return filtered_fraction(r) * (float)U + 64.f <= SMEM_MAX_LOAD * (float)T.cap;
}

// Shared-memory classes, smallest CTA first: (threads, CTAs/SM) = (64, 12), (128, 6), (256, 3),
// (512, 2), (1024, 1); one warp of each CTA walks, the others build.  The first class whose table is
// predicted to fit wins; G = global-memory rounds.
constexpr int N_SMEM_CLASSES = 5;
constexpr int C_XLC = N_SMEM_CLASSES + 1;   // class indices: 0-4 shared memory, 5 XL, 6 XLC
constexpr int N_TAB_CLASSES = N_SMEM_CLASSES + 2;
struct PlanBytes {
    uint32_t b[N_SMEM_CLASSES];   // dynamic shared memory per CTA
    uint32_t t[N_SMEM_CLASSES];   // threads per CTA
    uint32_t single;              // bit i: class i runs k_small (one end per CTA, no walker warp)
};


// XL class: 512-thread CTAs (1 per SM) whose tables live in a per-CTA global-memory scratch (L2-resident
// for the paper-shaped batch); shared memory keeps the info buffers (so the walk stays on-chip).
#ifndef LA_XL_THREADS
#define LA_XL_THREADS 1024   // 1024 vs 768 vs 512 threads: 154 / 156 / 162 ms on C4 (r01)
#endif
constexpr int XL_THREADS = LA_XL_THREADS;
constexpr int64_t XL_MAX_U = 1 << 21;
__host__ __device__ __forceinline__ uint32_t xl_needed_cap(int64_t r, int64_t U, bool filter) {
    const float need = filter ? (filtered_fraction(r) * (float)U + 1024.f) : (float)U;
    return (uint32_t)(need / SMEM_MAX_LOAD) + 16u;
}
// bytes of one CTA's global scratch for the largest XL end (U_max occurrences, r_max reads)
__host__ __device__ __forceinline__ uint32_t xl_stride(int64_t r_max, int64_t U_max, bool filter, uint32_t icap) {
    uint32_t cap = xl_needed_cap(r_max, U_max, filter);
    if (cap < min_table_cap(XL_THREADS)) cap = min_table_cap(XL_THREADS);   // claims + in-flight < cap
    if (cap > icap) cap = icap;
    return (pref_bytes((int)r_max) + 48u + cap * (16u + cnt_bytes(true, true) + 2u) + fpos_bytes((uint32_t)U_max, true) +
            255u) & ~255u;
}

// class-list entries: the end id, bit 30 set when a read of the end has an N (list_end / list_anyn)
constexpr int32_t LIST_ANYN = 1 << 30;
// bit 29: the end's reads are read from global memory (L1/L2) instead of being staged in shared memory
// (largest shared-memory class only, for ends whose staged reads would leave too little room for the
// table; r02b, LA_STREAM_BIG)
constexpr int32_t LIST_STREAM = 1 << 29;
// bit 28: every read of the end has the batch's longest length (P.maxlen): the first attempt's prefix
// pass is arithmetic (r02b: the planner already reads every length; the length scan was ~5% of the
// builders' time)
constexpr int32_t LIST_UNIFORM = 1 << 28;
__host__ __device__ __forceinline__ int list_end(int32_t v) { return v & (LIST_UNIFORM - 1); }
__host__ __device__ __forceinline__ bool list_uniform(int32_t v) { return (v & LIST_UNIFORM) != 0; }
__host__ __device__ __forceinline__ bool list_anyn(int32_t v) { return (v & LIST_ANYN) != 0; }
__host__ __device__ __forceinline__ bool list_stream(int32_t v) { return (v & LIST_STREAM) != 0; }

__global__ void k_plan(const int64_t *__restrict__ eoff, const int64_t *__restrict__ roff,
                       const uint8_t *__restrict__ rflag,
                       const int32_t *__restrict__ clen, int64_t n_ends, DevParams P, int SW, PlanBytes pb,
                       uint32_t xl_bytes, uint32_t xlc_bytes, int force_cls,
                       int32_t *__restrict__ cls, int32_t *__restrict__ out_len, uint8_t *__restrict__ out_term,
                       uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att, int32_t *__restrict__ lists,
                       uint32_t *__restrict__ keys, int32_t *__restrict__ list_G, int *__restrict__ ctr) {
    // ctr: [0..4] n per smem class, [5] n_G, [6] NOREADS, [7] SHORT, [8] n_XL, [9] max U_XL, [10] max r_XL,
    // [11] n_XLC
    const int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (e >= n_ends) return;
    const int64_t r = eoff[e + 1] - eoff[e];
    int c;
    if (r == 0) c = CLS_NOREADS;
    else if (clen[e] < P.k_start) c = CLS_SHORT;
    else {
        // exact voting-occurrence bounds U(k) = sum over reads of max(0, len - k) at the smallest k of
        // the schedule (table sizing) and at k_start (LPT key); reads shorter than k contribute 0
        int64_t U = 0, U0 = 0;
        int anyN = 0;   // some read of the end has an N: only then do the passes test k-mer windows for N
        bool uni = true;   // every read has length P.maxlen
        for (int64_t j = eoff[e]; j < eoff[e + 1]; ++j) {
            const int64_t l = roff[j + 1] - roff[j];
            U += l > P.k_min ? l - P.k_min : 0;
            U0 += l > P.k_start ? l - P.k_start : 0;
            anyN |= rflag[j];
            uni &= l == P.maxlen;
        }
        c = CLS_GLOBAL;
        int sc = -1;
        bool stream = false;
        if (U < (1ll << 30))
            for (int i = 0; i < N_SMEM_CLASSES && sc < 0; ++i)
                if (fits(r, U, P, pb.b[i], pb.t[i], SW, (pb.single >> i) & 1u)) sc = i;
        // the largest class with the reads left in global memory (L1/L2), before the L2-table XL class
        if (LA_STREAM_BIG && sc < 0 && U < (1ll << 30) && !((pb.single >> (N_SMEM_CLASSES - 1)) & 1u) &&
            fits(r, U, P, pb.b[N_SMEM_CLASSES - 1], pb.t[N_SMEM_CLASSES - 1], SW, false, true)) {
            sc = N_SMEM_CLASSES - 1;
            stream = true;
        }
        U0 = U0 > 0xffffffffll ? 0xffffffffll : U0;
        // XLC: the table split over a 2-CTA cluster's shared memory (no staging assumed; U < 65536)
        if (sc < 0 && xlc_bytes && P.V >= 2 && r <= 16384 && U <= XLC_MAX_U &&
            xlc_layout(xlc_bytes, (int)r, SW, (uint32_t)U, P.W, false).fits)
            sc = C_XLC;
        if (sc < 0 && xl_bytes && r <= 16384 && U <= XL_MAX_U &&
            xl_needed_cap(r, U, P.V >= 2) <= smem_fixed(P.W, xl_bytes, 1u, false, XL_THREADS / 32 - 1).icap)
            sc = N_SMEM_CLASSES;   // XL: table in global scratch
        // test hook (LA_FORCE_CLASS): every end with reads in one class; ends whose table does not
        // fit there overflow and are redone by the global path
        if (force_cls >= 0 && r <= 16384 && U <= XL_MAX_U) sc = force_cls;
        if (sc >= 0) {
            c = CLS_S + sc;
            const int i = atomicAdd(&ctr[sc == N_SMEM_CLASSES ? 8 : (sc == C_XLC ? 11 : sc)], 1);
            lists[sc * n_ends + i] =
                (int32_t)e | (anyN ? LIST_ANYN : 0) | (stream ? LIST_STREAM : 0) | (uni && LA_UNIFORM_FLAG ? LIST_UNIFORM : 0);
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
    // filtered: attempts built with the filter; inl / ref: attempts with inline / pointer (REF) keys;
    // dead0: attempts decided after the filter pass (start k-mer fails the filter: no build, no link)
    unsigned long long inserts, steps, attempts, filtered, inl, ref, dead0;
};
constexpr int GSTATS_WORDS = 7;
// out_dir[e]: direction of the end's k shifts (-1 down, +1 up, 0 none) recorded by the extension,
// so that la_replay_build can rerun exactly the same (end, k) attempts; OVF_DIR: the end left the
// class kernel (table overflow -> global path) and is not replayed.
constexpr int8_t OVF_DIR = 127;
__device__ __forceinline__ int8_t shift_dir(int shift) { return (int8_t)(shift > 0 ? 1 : (shift < 0 ? -1 : 0)); }

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

struct TabCtx {   // what a table operation needs
    uint64_t *keys;
    uint32_t *c32;   // per slot: word 0 = low-only votes[4] (8 bits each), word 1 = high votes[4]
    uint16_t *list;  // claimed slots in claim order (inline keys): the link pass visits only these
    uint32_t ks;     // shared-memory address of keys (shared tables): computed once, so the probe
                     // loops do not rematerialise the generic->shared conversion (S2R) every round
    uint32_t cap;
    const uint64_t *rseq;   // packed reads (global), for REF-format key verification
    int SW, k, KW;
    int wide;               // XL: 32-bit counter fields (U >= 65536), else 16-bit
};

// One vote for base b of slot s: a single atomic per vote.  Counter words hold the
// high-tier votes (q >= q_hi) and the low-only votes (q_lo <= q < q_hi) separately; the low tier of
// reading #1 is their sum (votes_of).  Shared memory: 8-bit fields of two u32 words (lo-only, hi),
// a field about to carry flags the end for the global path; global (XL): 8 x u32, RED.ADD.
template <bool GT>
__device__ __forceinline__ void vote_add(const TabCtx &T, uint32_t s, uint32_t b, bool hi, volatile int *ovf) {
    if (GT) {   // XL: fire-and-forget RED.ADD on 16-bit or (wide) 32-bit fields, as vote32 (la_inl32.cuh)
        if (T.wide) atomicAdd(&T.c32[8 * (size_t)s + (hi ? 4u : 0u) + b], 1u);
        else atomicAdd(&T.c32[4 * (size_t)s + (hi ? 2u : 0u) + (b >> 1)], 1u << (16 * (b & 1u)));
    } else {
        const uint32_t old = atomicAdd(&T.c32[2 * s + (hi ? 1u : 0u)], 1u << (8 * b));
        if (((old >> (8 * b)) & 0xffu) == 0xffu) *ovf = 1;   // an 8-bit counter would carry
    }
}

template <bool GT>
__device__ __forceinline__ void votes_of(const TabCtx &T, uint32_t s, uint32_t lo[4], uint32_t hi[4]) {
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

// Scalar lookup of a pointer-key (REF) table: the start k-mer
template <bool INL, int NW>
__device__ __forceinline__ uint32_t tab_lookup(const TabCtx &T, const KmerN<NW> &K, uint64_t h) {
    static_assert(!INL, "inline-key tables use lookup32 (la_inl32.cuh)");
    uint32_t s = slot_of(h, T.cap);
    const uint64_t tag = tag_of(h);
    for (uint32_t n = 0; n < T.cap; ++n) {
        const uint64_t w = T.keys[s];
        if (w == 0) return NONE;
        if ((w & TAG_MASK) == tag) {
            const KmerN<NW> K2 = extract_kmer<NW>(T.rseq + (size_t)slot_read(w) * T.SW, slot_pos(w), T.k, T.KW);
            if (kmer_eq(K, K2, T.KW)) return s;
        }
        s = (s + 1 == T.cap) ? 0 : s + 1;
    }
    return NONE;
}


// ---- warp-convergent passes for pointer keys (k >= 64) ----------------------------------------
__device__ __forceinline__ uint64_t nmask_word(uint64_t q) { return q & (q >> 1) & 0x5555555555555555ull; }

struct PosR {            // one lane's position, k-mer of up to 4 words
    KmerN<MAX_KW> K;
    uint32_t nb, rid;    // following base, read index (relative to the key rows)
    int p;
    bool vote, hi;
};

// f(act, v) per warp iteration, lane-per-position as warp_positions, for k <= 128.
template <typename F>
__device__ __forceinline__ void warp_positions_ref(const uint64_t *__restrict__ rseq, const uint64_t *__restrict__ rqc,
                                                   const uint8_t *__restrict__ rflag, const uint32_t *pref,
                                                   long long r0, int r, int SW, int k, int KW, int wid, int nwarps,
                                                   int lane, const volatile int *stop, F &&f) {
    const uint32_t total = pref[r];
    const uint32_t wb = (uint32_t)(((uint64_t)total * (uint32_t)wid) / (uint32_t)nwarps);
    const uint32_t we = (uint32_t)(((uint64_t)total * (uint32_t)(wid + 1)) / (uint32_t)nwarps);
    if (wb >= we) return;
    uint32_t g = wb + lane;
    int j;
    {
        const uint32_t gg = min(g, we - 1);
        int lo = 0, hi = r;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (pref[mid] <= gg) lo = mid; else hi = mid;
        }
        j = lo;
    }
    uint32_t pj0 = pref[j], pj1 = pref[j + 1];
    for (uint32_t base = wb; base < we; base += 32u, g += 32u) {
        if (((base - wb) & 127u) == 0 && __shfl_sync(0xffffffffu, *stop, 0)) return;
        const bool act = g < we;
        PosR v;
        v.vote = false;
        v.nb = 0;
        v.hi = false;
        v.p = 0;
        v.rid = 0;
#pragma unroll
        for (int w = 0; w < MAX_KW; ++w) v.K.w[w] = 0;
        if (act) {
            while (g >= pj1) {
                pj0 = pj1;
                pj1 = pref[++j + 1];
            }
            const long long rid = r0 + j;
            const uint64_t *R = rseq + rid * SW, *Q = rqc + rid * SW;
            const int p = (int)(g - pj0);
            v.K = extract_kmer<MAX_KW>(R, p, k, KW);
            v.p = p;
            v.rid = (uint32_t)rid;
            const int i = p + k, sh = 62 - ((i & 31) << 1);
            v.nb = (uint32_t)(R[i >> 5] >> sh) & 3u;
            const uint32_t nq = (uint32_t)(Q[i >> 5] >> sh) & 3u;
            v.vote = nq - 1u < 2u;
            v.hi = nq == 2u;
            if (v.vote && rflag[rid]) {   // reading #5: any N in [p, p+k) -> no entry
                const int q = p >> 5, s2 = (p & 31) << 1;
#pragma unroll
                for (int w = 0; w < MAX_KW; ++w) {
                    const int bits = 2 * k - 64 * w;
                    const uint64_t m = bits >= 64 ? ~0ull : (bits > 0 ? (~0ull << (64 - bits)) : 0ull);
                    const uint64_t n = funnel64(nmask_word(Q[q + w]), nmask_word(Q[q + w + 1]), s2) & m;
                    if (w < KW && n) v.vote = false;
                }
            }
        }
        f(act && v.vote, v);
    }
}

// Convergent insert with pointer keys: a round probes one slot; a tag match is verified against the
// k-mer at the slot's (read, pos) in the staged reads (exact equality).
template <bool GT>
__device__ __forceinline__ uint32_t ref_probe_find(const TabCtx &T, const KmerN<MAX_KW> &K, uint64_t tag, uint64_t w) {
    if ((w & TAG_MASK) != tag) return 0u;
    const KmerN<MAX_KW> K2 = extract_kmer<MAX_KW>(T.rseq + (size_t)slot_read(w) * T.SW, slot_pos(w), T.k, T.KW);
    return kmer_eq(K, K2, T.KW) ? 1u : 0u;
}

template <bool GT>
__device__ __forceinline__ void warp_insert_ref(const TabCtx &T, bool want, const PosR &v, uint64_t h, int lane,
                                                int *nclaim, int claim_limit, volatile int *ovf) {
    uint32_t s = slot_of(h, T.cap), hit = 0;
    const uint64_t tag = tag_of(h), mine = make_slot(tag, v.rid, (uint32_t)v.p);
    bool pend = want, found = false;
    volatile uint64_t *vk = T.keys;
    while (__any_sync(0xffffffffu, pend)) {
        bool claimed = false;
        if (pend) {
            uint64_t w = vk[s];
            if (w == 0) {
                if (*ovf) {
                    pend = false;
                } else {
                    w = atomicCAS((unsigned long long *)&T.keys[s], 0ull, (unsigned long long)mine);
                    if (w == 0) {
                        claimed = true;
                        pend = false;
                        found = true;
                        hit = s;
                    }
                }
            }
            if (pend && w != 0) {
                if (ref_probe_find<GT>(T, v.K, tag, w)) {
                    pend = false;
                    found = true;
                    hit = s;
                } else {
                    s = (s + 1 == T.cap) ? 0 : s + 1;
                }
            }
        }
        const unsigned cm = __ballot_sync(0xffffffffu, claimed);
        if (cm) {
            const int n = __popc(cm), leader = __ffs(cm) - 1;
            int first = 0;
            if (lane == leader) {
                first = atomicAdd(nclaim, n);
                if (first + n > claim_limit) *ovf = 1;
            }
            first = __shfl_sync(0xffffffffu, first, leader);
            if (claimed) T.list[first + __popc(cm & ((1u << lane) - 1u))] = (uint16_t)hit;
        }
    }
    if (found) vote_add<GT>(T, hit, v.nb, v.hi, ovf);
}

template <bool GT>
__device__ __forceinline__ uint32_t warp_lookup_ref(const TabCtx &T, bool want, const KmerN<MAX_KW> &K, uint64_t h) {
    uint32_t s = slot_of(h, T.cap), res = NONE, n = 0;
    const uint64_t tag = tag_of(h);
    bool pend = want;
    while (__any_sync(0xffffffffu, pend)) {
        if (pend) {
            const uint64_t w = T.keys[s];
            if (w == 0) {
                pend = false;
            } else if (ref_probe_find<GT>(T, K, tag, w)) {
                pend = false;
                res = s;
            } else {
                s = (s + 1 == T.cap) ? 0 : s + 1;
                if (++n >= T.cap) pend = false;
            }
        }
    }
    return res;
}

// ---- the kernel --------------------------------------------------------------------------------
struct EndSlot {            // one contig end in flight
    int e, r, ulen;         // ulen: common length of all the end's reads (0 if they differ)
    long long r0;
    int k, shift, kmax_eff, attempts;
    int best_len, best_term, best_k, best_buf;
    int done, dead, ovf;    // done: finished (refill); dead: no more ends; ovf: redo in the global path
    uint32_t start;         // the start k-mer's slot (NONE if absent) of the last build
    int rec_att;            // replay: attempts recorded by the extension
    int anyN;               // some read of the end has an N (from the class list entry)
    int stream;             // the end's reads stay in global memory (LIST_STREAM)
    unsigned long long ins, steps;
};

struct BuildCtl {           // builders' shared scratch
    int skip;               // 1: the current slot has no work (retired)
    int overflow, nclaim;
    uint32_t start;
    uint32_t start_h;       // hash of the start k-mer (inline keys); start_ok: it has no N
    int start_ok, dead0;    // dead0: the attempt is decided before the build (start k-mer < 2 votes)
    int ctr_f, ctr_b;       // position chunk counters of the filter / build pass (warp_positions32_dyn)
    SmemTab tb;             // this attempt's table layout, computed once by the leader (integer divisions)
    int lmin, lmax;
    uint32_t wsum[32];      // per builder warp: prefix-scan totals
};

__device__ __forceinline__ void builders_sync(int NB) { asm volatile("bar.sync 1, %0;" ::"r"(NB) : "memory"); }

// mbarrier handoff between the builders' leader and the walker (hardware-suspended waits).
__device__ __forceinline__ uint32_t smem_addr(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
// try_wait with a suspend-time hint: the waiting thread is suspended in hardware until the phase
// completes (or the hint, 1 ms, expires), so a long wait takes no issue slots from the builders on
// the same SM (ncu: a polling loop with __nanosleep was 44% of the kernel's executed instructions).
__device__ __forceinline__ bool mbar_try_wait(uint32_t addr, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared.b64 p, [%1], %2, %3;\n selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(addr), "r"(parity), "r"(1000000u)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    const uint32_t addr = smem_addr(bar);
    while (!mbar_try_wait(addr, parity)) {
    }
}

// Positions with a following base, per read: exclusive prefix pref[0..r] (pref[r] = U).  All NB
// builder threads call it; E.ulen records whether every read of the end has the same length (then the
// prefix is arithmetic from the next attempt on).
__device__ __forceinline__ void read_prefix(BuildCtl &B, EndSlot &E, uint32_t *pref, const uint16_t *gL, long long lr0,
                                            int r, int k, int ulen, int bt, int NB) {
    if (ulen >= 0) {   // all reads of the end have length ulen: arithmetic, no loads
        const uint32_t np = (uint32_t)max(0, ulen - k);
        for (int j = bt; j <= r; j += NB) pref[j] = (uint32_t)j * np;
        builders_sync(NB);
    } else {
        const int per = (r + NB - 1) / NB;
        const int j0 = min(r, bt * per), j1 = min(r, j0 + per);
        uint32_t loc = 0;
        int lmin = 1 << 30, lmax = -1;
        for (int j = j0; j < j1; ++j) {
            const int l = gL[lr0 + j];
            loc += (uint32_t)max(0, l - k);
            lmin = min(lmin, l);
            lmax = max(lmax, l);
        }
        const int lane = bt & 31, w = bt >> 5;
        uint32_t inc = loc;
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t v = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += v;
        }
        for (int o = 16; o; o >>= 1) {
            lmin = min(lmin, __shfl_xor_sync(0xffffffffu, lmin, o));
            lmax = max(lmax, __shfl_xor_sync(0xffffffffu, lmax, o));
        }
        if (bt == 0) {
            B.lmin = 1 << 30;
            B.lmax = -1;
        }
        if (lane == 31) B.wsum[w] = inc;
        builders_sync(NB);
        if (lane == 0) {
            atomicMin(&B.lmin, lmin);
            atomicMax(&B.lmax, lmax);
        }
        uint32_t off = inc - loc;
        for (int i = 0; i < w; ++i) off += B.wsum[i];
        for (int j = j0; j < j1; ++j) {
            pref[j] = off;
            off += (uint32_t)max(0, (int)gL[lr0 + j] - k);
        }
        if (bt == NB - 1) pref[r] = off;   // the last builder covers the last read (or none)
        builders_sync(NB);
        if (bt == 0) E.ulen = (r > 0 && B.lmin == B.lmax) ? B.lmax : -2;   // -2: lengths differ
    }
}

// The walk (Alg 2) over the link words of one attempt, by one thread: loop check before
// the lookup (reading #12, the visited bit), fork / dead end from the decided code (reading #1), at
// most W bases (reading #7).  Bases are packed four to a 32-bit store (wb 4-byte aligned).  Returns the
// walk length; term and the lookups made (a lookup per step, the LOOP step excluded) by reference.
__device__ __forceinline__ int walk_links(uint32_t *info, uint32_t node, int W, uint8_t *wb, int &term,
                                          unsigned long long &steps) {
    int i = 0;
    uint32_t pack = 0;
    term = T_MAXLEN;
#if LA_WALK_PIPE
    // software-pipelined: the successor's word is loaded before this step's checks resolve, so the
    // load latency overlaps the branch; the only word that can change in between is this node's own
    // (its visited bit), patched in when the successor is the node itself
    if (W > 0) {
        if (node == NEXT_NONE) {
            term = T_DEADEND;
        } else {
            uint32_t inf = info[node];
            for (;;) {
                const uint32_t nx = inf >> 4, code = inf & 7u;
                const uint32_t pre = info[nx == NEXT_NONE ? node : nx];   // speculative, always a valid slot
                if ((inf & 8u) | (code >= 4u)) {   // visited (loop check before the lookup) / fork / dead end
                    term = (inf & 8u) ? T_LOOP : (code == CODE_FORK ? T_FORK : T_DEADEND);
                    break;
                }
                info[node] = inf | 8u;
                pack |= ((0x54474341u >> (8 * code)) & 0xffu) << (8 * (i & 3));   // "ACGT"[code]
                if ((i & 3) == 3) {
                    *(uint32_t *)(wb + i - 3) = pack;
                    pack = 0;
                }
                ++i;
                if (i >= W) break;                                    // MAXLEN: no lookup after the W-th base
                if (nx == NEXT_NONE) {
                    term = T_DEADEND;
                    break;
                }
                inf = nx == node ? (pre | 8u) : pre;
                node = nx;
            }
        }
    }
    if (false)
#endif
    for (; i < W; ++i) {
        if (node == NEXT_NONE) {
            term = T_DEADEND;
            break;
        }
        const uint32_t inf = info[node], code = inf & 7u;
        if ((inf & 8u) | (code >= 4u)) {   // visited (loop check before the lookup) / fork / dead end
            term = (inf & 8u) ? T_LOOP : (code == CODE_FORK ? T_FORK : T_DEADEND);
            break;
        }
        info[node] = inf | 8u;
        pack |= ((0x54474341u >> (8 * code)) & 0xffu) << (8 * (i & 3));   // "ACGT"[code]
        if ((i & 3) == 3) {
            *(uint32_t *)(wb + i - 3) = pack;
            pack = 0;
        }
        node = inf >> 4;
    }
    for (int j = i & ~3; j < i; ++j) wb[j] = (uint8_t)(pack >> (8 * (j & 3)));
    steps = (term == T_LOOP || term == T_MAXLEN) ? (unsigned long long)i : (unsigned long long)i + 1ull;
    return i;
}

// Slot-parallel pass after the build: ext(lo, hi) (reading #1, a5) and, for a base, the successor
// k-mer's slot (next_kmer, Alg 2 line 15) -> info[s] = next << 4 | code.
__device__ __forceinline__ uint32_t link_info(int code, uint32_t nxt) {
    return (code < 4 ? (nxt == NONE ? NEXT_NONE : nxt) : NEXT_NONE) << 4 | (uint32_t)code;
}

// Inline keys (k <= 63) on 32-bit words (la_inl32.cuh): filter pass, build pass (Alg 1), link pass
// (a5) and the start k-mer's slot, for NW = ceil(2k/32) words.
template <int NW, bool GT, int UF = LA_FILTER_UNROLL>
__device__ __forceinline__ void inl32_build_link(BuildCtl &B, const TabCtx &TC, uint32_t *B1, uint32_t *B2,
                                                 uint32_t mbits, uint32_t *info, const uint64_t *__restrict__ rqc,
                                                 const uint8_t *__restrict__ rflag, const uint32_t *pref, long long r0,
                                                 int r, int ulen, const DevParams &P, const uint64_t *tail_e, int Tn,
                                                 uint64_t n0, uint64_t n1, int bt, int NB, long long &t_filter,
                                                 long long &t_build, bool replay, void *fpos, uint32_t *queue, bool anyN,
                                                 bool sreads) {
    const volatile int *stop = &B.overflow;
    const int k = TC.k;
    const int lane = bt & 31, wid = bt >> 5, nwarps = NB >> 5;
    const int claim_limit = (int)(SMEM_MAX_LOAD * (float)TC.cap);
    Tab32 T;
    T.keys = (unsigned char *)TC.keys;
    T.ks = TC.ks;
    T.c32 = TC.c32;
    T.list = TC.list;
    T.cap = TC.cap;
    T.wide = TC.wide;
    const uint32_t *R32 = (const uint32_t *)TC.rseq, *Q32 = (const uint32_t *)rqc;
    const int SW2 = 2 * TC.SW;
    // start k-mer: last k bases of the oriented contig (Alg 2 line 4; reading #6)
    K32<NW> Kst;
    if (bt == 0) {
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
    if (!mbits || !LA_FQUEUE) {
        if (mbits) {
            // ---- filter pass: B1 = seen once, B2 = seen at least twice (reading #4) ----
            auto filt = [&](bool, bool act, uint32_t, const K32<NW> &, uint32_t h, uint32_t, bool) {
#ifdef LA_PROBE_STATS
                                     {
                                         const unsigned am = __ballot_sync(0xffffffffu, act);
                                         if (lane == 0) { LA_PSTAT(8, 1); LA_PSTAT(9, __popc(am)); }
                                     }
#endif
                                     if (!act) return;
                                     const uint32_t fi = filt32(h, mbits);
                                     const uint32_t bit = 1u << (fi & 31);
                                     if (!(*(volatile uint32_t *)&B2[fi >> 5] & bit)) {
                                         if (LA_ABL_NOFILTATOM) {
                                             const uint32_t old = B1[fi >> 5];
                                             B1[fi >> 5] = old | bit;
                                             if (old & bit) B2[fi >> 5] |= bit;
                                         } else {
                                             const uint32_t old = atomicOr(&B1[fi >> 5], bit);
                                             if (old & bit) atomicOr(&B2[fi >> 5], bit);
                                         }
                                     }
                                 };
            if (LA_DYN && !GT && ulen > k && sreads && LA_LDS_READS)
                warp_positions32_dyn<NW, UF, true>(R32, Q32, ((LA_ANYN && !anyN) ? nullptr : rflag), pref[r], r0, SW2, k, ulen, lane,
                                                   stop, &B.ctr_f, filt);
            else if (LA_DYN && !GT && ulen > k)
                warp_positions32_dyn<NW, UF>(R32, Q32, ((LA_ANYN && !anyN) ? nullptr : rflag), pref[r], r0, SW2, k, ulen, lane, stop,
                                                           &B.ctr_f, filt);
            else if (sreads && LA_LDS_READS)
                warp_positions32<NW, UF, true>(R32, Q32, ((LA_ANYN && !anyN) ? nullptr : rflag), pref, r0, r, SW2, k, ulen, wid, nwarps, lane,
                                               stop, filt);
            else
                warp_positions32<NW, UF>(R32, Q32, ((LA_ANYN && !anyN) ? nullptr : rflag), pref, r0, r, SW2, k, ulen, wid, nwarps, lane,
                                                       stop, filt);
            builders_sync(NB);
            // The filter has no false negatives: a start k-mer whose B2 bit is clear has < 2 voting
            // occurrences, so with V >= 2 (filters are only used then) it extends to DEADEND at step 0
            // whatever the table holds (reading #1) — the walk of this attempt is decided: skip the
            // build and the link pass (the attempt still counts its U inserts, the method's work).
            if (LA_DEAD0) {
                const uint32_t fs = filt32(B.start_h, mbits);
                if (!B.start_ok || !((B2[fs >> 5] >> (fs & 31)) & 1u)) {
                    if (bt == 0) {
                        B.start = NONE;
                        B.dead0 = 1;
                    }
                    builders_sync(NB);
                    t_filter = t_build = la_clock();
                    return;
                }
            }
        }
        t_filter = la_clock();
        // ---- build (Alg 1): every voting occurrence that passed the filter ----
        uint32_t pend = 0;   // carry check of this lane's last vote (vote32d)
        auto build = [&](bool, bool act, uint32_t, const K32<NW> &K, uint32_t h, uint32_t nb, bool hi) {
            bool want = act;
            if (mbits) {
                const uint32_t fi = filt32(h, mbits);
                want = want && ((B2[fi >> 5] >> (fi & 31)) & 1u);
            }
            warp_insert32<GT>(T, want, key_form<NW>(K, h), h, nb, hi, lane, &B.nclaim, claim_limit, &B.overflow, pend);
        };
        if (LA_DYN && !GT && ulen > k && sreads && LA_LDS_READS)
            warp_positions32_dyn<NW, 1, true>(R32, Q32, ((LA_ANYN && !anyN) ? nullptr : rflag), pref[r], r0, SW2, k, ulen, lane, stop,
                                              &B.ctr_b, build);
        else if (LA_DYN && !GT && ulen > k)
            warp_positions32_dyn<NW, 1>(R32, Q32, ((LA_ANYN && !anyN) ? nullptr : rflag), pref[r], r0, SW2, k, ulen, lane, stop, &B.ctr_b, build);
        else if (sreads && LA_LDS_READS)
            warp_positions32<NW, 1, true>(R32, Q32, ((LA_ANYN && !anyN) ? nullptr : rflag), pref, r0, r, SW2, k, ulen, wid, nwarps, lane,
                                          stop, build);
        else
            warp_positions32<NW>(R32, Q32, ((LA_ANYN && !anyN) ? nullptr : rflag), pref, r0, r, SW2, k, ulen, wid, nwarps, lane, stop, build);
        flush_vote32(pend, &B.overflow);
    } else {
        // ---- filter pass: B1 = seen once, B2 = seen at least twice (reading #4); every position's
        // filter bit index (or FNONE: no vote) is kept for the build pass ----
        typedef typename std::conditional<GT, uint32_t, uint16_t>::type FT;
        FT *fp = (FT *)fpos;
        const uint32_t FNONE = GT ? 0xFFFFFFFFu : 0xFFFFu;
        warp_positions32<NW>(R32, Q32, rflag, pref, r0, r, SW2, k, ulen, wid, nwarps, lane, stop,
                             [&](bool inr, bool act, uint32_t g, const K32<NW> &, uint32_t h, uint32_t, bool) {
                                 const uint32_t fi = filt32(h, mbits);
                                 if (inr) fp[g] = (FT)(act ? fi : FNONE);
                                 if (!act) return;
                                 const uint32_t bit = 1u << (fi & 31);
                                 if (!(*(volatile uint32_t *)&B2[fi >> 5] & bit)) {
                                     const uint32_t old = atomicOr(&B1[fi >> 5], bit);
                                     if (old & bit) atomicOr(&B2[fi >> 5], bit);
                                 }
                             });
        builders_sync(NB);
        t_filter = la_clock();
        // ---- build (Alg 1): the positions whose filter bit is in B2 are queued per warp (64 slots
        // in shared memory) and inserted 32 at a time, so the probe rounds run with full warps ----
        const KMask m = kmask32<NW>(k);
        const uint32_t total = pref[r];
        const uint32_t wb = (uint32_t)(((uint64_t)total * (uint32_t)wid) / (uint32_t)nwarps);
        const uint32_t we = (uint32_t)(((uint64_t)total * (uint32_t)(wid + 1)) / (uint32_t)nwarps);
        uint32_t pend = 0;   // carry check of this lane's last vote (vote32d)
        auto insert_batch = [&](bool has, uint32_t g) {
            int j = 0, p = 0;
            if (has) pos_of(g, pref, r, ulen, k, j, p);
            const long long row = (r0 + j) * (long long)SW2;
            const uint32_t *Rr = R32 + row, *Qr = Q32 + row;
            const K32<NW> K = extract32<NW>(Rr, p, m);
            const uint32_t nb = base32(Rr, p + k), nq = base32(Qr, p + k);
            const uint32_t h = hash32<NW>(K);
            warp_insert32<GT>(T, has, key_form<NW>(K, h), h, nb, nq == 2u, lane, &B.nclaim, claim_limit, &B.overflow,
                              pend);
        };
        uint32_t qn = 0;   // queued positions (warp-uniform)
        const unsigned lt = (1u << lane) - 1u;
        for (uint32_t base = wb; base < we; base += 32u) {
            if (((base - wb) & 127u) == 0 && __shfl_sync(0xffffffffu, *stop, 0)) break;
            const uint32_t g = base + lane;
            bool want = false;
            if (g < we) {
                const uint32_t fi = fp[g];
                want = fi != FNONE && ((B2[fi >> 5] >> (fi & 31)) & 1u);
            }
            const unsigned wm = __ballot_sync(0xffffffffu, want);
            if (want) queue[qn + __popc(wm & lt)] = g;
            qn += __popc(wm);
            if (qn >= 32u) {
                __syncwarp();
                const uint32_t gq = queue[lane], gx = queue[32 + lane];
                __syncwarp();
                if (lane < qn - 32u) queue[lane] = gx;
                qn -= 32u;
                insert_batch(true, gq);
            }
        }
        __syncwarp();
        if (__shfl_sync(0xffffffffu, *stop, 0) == 0 && qn) insert_batch(lane < qn, lane < qn ? queue[lane] : 0u);
        flush_vote32(pend, &B.overflow);
    }
    builders_sync(NB);
    t_build = la_clock();
    if (B.overflow || replay) return;   // replay: the hash-build phase only (no link pass, no walk)
    // ---- ext rule + successor links (a5), over the claimed slots, all lanes busy ----
    const uint32_t nocc = min((uint32_t)B.nclaim, T.cap);
    for (uint32_t base = (uint32_t)wid * 32u; base < nocc; base += (uint32_t)NB) {
        const uint32_t i = base + lane;
        const bool has = i < nocc;
        const uint32_t s = has ? (uint32_t)T.list[i] : 0u;
        K32<NW> K;
#pragma unroll
        for (int w = 0; w < NW; ++w) K.w[w] = 0u;
        int code = CODE_DEADEND;
        if (has) {
            K = key_of<NW>(ld_slot<GT>(T, s));
            uint32_t lo[4], hi[4];
            votes32<GT>(T, s, lo, hi);
            code = ext_rule32(lo, hi, P.V, P.F);
            if (code < 4) roll32<NW>(K, k, (uint32_t)code);
        }
        const uint32_t h = hash32<NW>(K);
        const uint32_t t = warp_lookup32<GT>(T, has && code < 4, key_form<NW>(K, h), h);
        if (has) info[s] = link_info(code, t);
    }
    if (bt == 0) B.start = B.start_ok ? lookup32<GT>(T, key_form<NW>(Kst, B.start_h), B.start_h) : NONE;
}

// Each inline-key width NW is a full copy of the filter / build / link passes, and the table kernels
// are sensitive to instruction-cache pressure (r02b: C4 attempts run k = 33 then 25, which were two
// hot copies, NW = 3 and 2); LA_NW_MERGE23 runs both on the 3-word code.
template <bool INL, bool GT, int UF = LA_FILTER_UNROLL>
__device__ __forceinline__ void build_link(BuildCtl &B, const TabCtx &T, uint32_t *B1, uint32_t *B2, uint32_t mbits,
                                           uint32_t *info, const uint64_t *__restrict__ rqc,
                                           const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag,
                                           const uint32_t *pref, long long r0, int r, const DevParams &P,
                                           const uint64_t *tail_e, int Tn, uint64_t n0, uint64_t n1, int bt, int NB,
                                           long long &t_filter, long long &t_build, bool replay, int ulen, void *fpos,
                                           uint32_t *queue, bool anyN, bool sreads = false) {
    if (INL) {
        // LA_NW_MERGE23: 17 <= k <= 32 on the 3-word code (the masks of kmask32 cover the last two words,
        // so a 3-word k-mer needs k >= 17); k <= 16 keeps the 2-word code
        const int nw = kw32(T.k);
        if (nw <= 2 && !(LA_NW_MERGE23 && T.k >= 17))
            inl32_build_link<2, GT, UF>(B, T, B1, B2, mbits, info, rqc, rflag, pref, r0, r, ulen, P, tail_e, Tn, n0, n1,
                                    bt, NB, t_filter, t_build, replay, fpos, queue, anyN, sreads);
        else if (nw <= 3)
            inl32_build_link<3, GT, UF>(B, T, B1, B2, mbits, info, rqc, rflag, pref, r0, r, ulen, P, tail_e, Tn, n0, n1,
                                    bt, NB, t_filter, t_build, replay, fpos, queue, anyN, sreads);
        else
            inl32_build_link<4, GT, UF>(B, T, B1, B2, mbits, info, rqc, rflag, pref, r0, r, ulen, P, tail_e, Tn, n0, n1,
                                    bt, NB, t_filter, t_build, replay, fpos, queue, anyN, sreads);
        return;
    }
    // ---- pointer keys (k >= 64): the same passes with 4-word k-mers ----
    const volatile int *stop = &B.overflow;
    const int k = T.k, KW = T.KW;
    const int lane = bt & 31, wid = bt >> 5, nwarps = NB >> 5;
    const int claim_limit = (int)(SMEM_MAX_LOAD * (float)T.cap);
    if (mbits) {
        warp_positions_ref(T.rseq, rqc, rflag, pref, r0, r, T.SW, k, KW, wid, nwarps, lane, stop,
                           [&](bool act, const PosR &v) {
                               if (!act) return;
                               const uint32_t fi = filt_index(hash_kmer(v.K, KW), mbits);
                               const uint32_t bit = 1u << (fi & 31);
                               if (!(*(volatile uint32_t *)&B2[fi >> 5] & bit)) {
                                   const uint32_t old = atomicOr(&B1[fi >> 5], bit);
                                   if (old & bit) atomicOr(&B2[fi >> 5], bit);
                               }
                           });
        builders_sync(NB);
    }
    t_filter = la_clock();
    warp_positions_ref(T.rseq, rqc, rflag, pref, r0, r, T.SW, k, KW, wid, nwarps, lane, stop,
                       [&](bool act, const PosR &v) {
                           const uint64_t h = hash_kmer(v.K, KW);
                           bool want = act;
                           if (mbits) {
                               const uint32_t fi = filt_index(h, mbits);
                               want = want && ((B2[fi >> 5] >> (fi & 31)) & 1u);
                           }
                           warp_insert_ref<GT>(T, want, v, h, lane, &B.nclaim, claim_limit, &B.overflow);
                       });
    builders_sync(NB);
    t_build = la_clock();
    if (B.overflow || replay) return;   // replay: the hash-build phase only (no link pass, no walk)
    // ---- ext rule + successor links (a5) into the end's info buffer ----
    {
        const uint32_t nocc = min((uint32_t)B.nclaim, T.cap);
        for (uint32_t base = (uint32_t)wid * 32u; base < nocc; base += (uint32_t)NB) {
            const uint32_t i = base + lane;
            const bool has = i < nocc;
            const uint32_t s = has ? (uint32_t)T.list[i] : 0u;
            KmerN<MAX_KW> K;
#pragma unroll
            for (int w = 0; w < MAX_KW; ++w) K.w[w] = 0;
            int code = CODE_DEADEND;
            if (has) {
                const uint64_t w = T.keys[s];
                K = extract_kmer<MAX_KW>(T.rseq + (size_t)slot_read(w) * T.SW, slot_pos(w), k, KW);
                uint32_t lo[4], hi[4];
                votes_of<GT>(T, s, lo, hi);
                code = ext_rule32(lo, hi, P.V, P.F);
                if (code < 4) roll_kmer(K, k, KW, (uint32_t)code);
            }
            const uint32_t t = warp_lookup_ref<GT>(T, has && code < 4, K, hash_kmer(K, KW));
            if (has) info[s] = link_info(code, t);
        }
    }
    if (bt == 0) {
        // start k-mer: last k bases of the oriented contig (Alg 2 line 4; reading #6)
        const int p = Tn - k;
        bool hasN = false;
        hasN = any_n_range(n0, n1, p, Tn);
        uint32_t st = NONE;
        if (!hasN) {
            uint64_t Tw[TAIL_W];
#pragma unroll
            for (int i = 0; i < TAIL_W; ++i) Tw[i] = tail_e[i];
            const KmerN<MAX_KW> K = extract_kmer<MAX_KW>(Tw, p, k, KW);
            st = tab_lookup<false, MAX_KW>(T, K, hash_kmer(K, KW));
        }
        B.start = st;
    }
}

// MINB: resident CTAs per SM the class is launched with (register budget 65536 / (MINB * BLOCK))
template <int BLOCK, bool GT, int MINB = (768 / BLOCK > 0 ? 768 / BLOCK : 1)>
__global__ void __launch_bounds__(BLOCK, MINB) k_smem(
    const int32_t *__restrict__ list, int n_list, int *__restrict__ work_ctr,
    const uint64_t *__restrict__ rseq, const uint64_t *__restrict__ rqc,
    const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag,
    const int64_t *__restrict__ eoff, const uint64_t *__restrict__ tail,
    const uint64_t *__restrict__ tailN, const int32_t *__restrict__ clen, int SW, DevParams P,
    uint32_t smem_bytes, uint8_t *__restrict__ walk_buf, int32_t *__restrict__ out_len,
    uint8_t *__restrict__ out_term, uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att,
    int8_t *__restrict__ out_dir, int32_t *__restrict__ ovf_list, int *__restrict__ n_ovf, GlobalStats *__restrict__ gstats,
    unsigned char *__restrict__ gscratch, uint32_t gstride, unsigned long long *__restrict__ prof) {
    static_assert(BLOCK >= 64, "one walker warp + at least one builder warp");
    constexpr int NB = BLOCK - 32;   // builder threads
    extern __shared__ __align__(16) unsigned char sm[];
    __shared__ EndSlot S[2];
    __shared__ BuildCtl B;
    __shared__ __align__(8) uint64_t built[2], walked[2];   // mbarriers: slot s built / walked
    __shared__ unsigned long long s_acc[GSTATS_WORDS];   // work counters (GlobalStats order)
    const int tid = threadIdx.x;
    // the fixed layout lives in shared memory: computed once, read with LDS (kept in registers, the
    // 64-register classes rematerialised its divisions inside the loops: ~4% of their instructions)
    __shared__ SmemFixed sFX;
    if (threadIdx.x == 0) sFX = smem_fixed(P.W, smem_bytes, GT ? gstride : 0u, false, NB / 32);
    __syncthreads();
    const SmemFixed &FX = sFX;
    // table region: shared memory, or this CTA's slice of the global scratch (XL class)
    unsigned char *tbase = GT ? gscratch + (size_t)blockIdx.x * gstride : sm;
    const int Wp = (P.W + 15) & ~15;
    uint8_t *wstr = sm + FX.off_walk;   // end slot s: buffers 2s, 2s+1 (current / best)
    if (tid == 0) {
        for (int i = 0; i < 2; ++i) {
            mbar_init(&built[i], 1);
            mbar_init(&walked[i], 1);
            S[i].done = 1;   // empty: the builders fetch an end first
            S[i].dead = 0;
            S[i].ovf = 0;
        }
        for (int i = 0; i < GSTATS_WORDS; ++i) s_acc[i] = 0;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    // The two end slots strictly alternate: builders build slot 0, slot 1, then wait for slot 0's
    // walk, rebuild it (next k) or refill it (next end), and so on; the walker walks 0, 1, 0, ...
    if (tid < 32) {
        // ============================ walker warp ============================
        const int lane = tid;

        uint32_t phase = 0u, alive = 3u;   // bit s: mbarrier parity / slot still in use
        long long w_wait = 0, w_walk = 0;
        for (int s = 0; alive; s ^= 1) {
            if (!((alive >> s) & 1u)) continue;
            const long long tw0 = la_clock();
            if (lane == 0) mbar_wait(&built[s], (phase >> s) & 1u);
            w_wait += la_clock() - tw0;
            phase ^= 1u << s;
            EndSlot &E = S[s];
            // lane 0 alone reads the slot's state (it waited on the mbarrier) and broadcasts it
            int st_dead = 0, st_ovf = 0;
            if (lane == 0) {
                st_dead = E.dead;
                st_ovf = E.ovf;
            }
            st_dead = __shfl_sync(0xffffffffu, st_dead, 0);
            st_ovf = __shfl_sync(0xffffffffu, st_ovf, 0);
            if (st_dead) {
                alive &= ~(1u << s);
                continue;
            }
            if (st_ovf) {   // the build overflowed: the global path owns this end; pass the slot back
                if (lane == 0) mbar_arrive(&walked[s]);
                continue;
            }
            int done = 0, bl = 0, bb = 0;
            const long long tw1 = la_clock();
            if (lane == 0 && P.replay) {   // replay: the recorded k sequence instead of the walk
                E.attempts += 1;
                done = E.attempts >= E.rec_att;
                E.k += E.shift;
            } else if (lane == 0) {
                // ---- walk (Alg 2) over the successor links ----
                uint32_t *info = (uint32_t *)(sm + (s ? FX.off_info1 : 0u));
                uint8_t *wb = wstr + (2 * s + (E.best_buf ^ 1)) * Wp;
                int term;
                unsigned long long steps;
                const int len = walk_links(info, E.start == NONE ? NEXT_NONE : E.start, P.W, wb, term, steps);
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
            w_walk += la_clock() - tw1;
            if (done && P.replay) {
                if (lane == 0) {
                    s_acc[0] += E.ins;
                    s_acc[2] += E.attempts;
                    E.done = 1;
                }
            } else if (done) {
                // ---- the selected walk -> HBM ----
                __syncwarp();   // lane 0's walk string is complete
                const int e = __shfl_sync(0xffffffffu, lane == 0 ? E.e : 0, 0);
                const uint8_t *bw = wstr + (2 * s + bb) * Wp;
                uint8_t *dst = walk_buf + (size_t)e * P.W;
                for (int i = lane; i < bl; i += 32) dst[i] = bw[i];
                if (lane == 0) {
                    out_len[e] = bl;
                    out_term[e] = (uint8_t)E.best_term;
                    out_k[e] = (uint8_t)E.best_k;
                    out_att[e] = (uint8_t)E.attempts;
                    out_dir[e] = shift_dir(E.shift);
                    s_acc[0] += E.ins;   // per-CTA work counters in shared memory (no registers)
                    s_acc[1] += E.steps;
                    s_acc[2] += E.attempts;
                    E.done = 1;
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&walked[s]);   // release: the state above is visible to the builders
        }
        if (lane == 0) {
            atomicAdd(&gstats->inserts, s_acc[0]);
            atomicAdd(&gstats->steps, s_acc[1]);
            atomicAdd(&gstats->attempts, s_acc[2]);
            if (prof) {
                atomicAdd(&prof[6], (unsigned long long)w_wait);
                atomicAdd(&prof[7], (unsigned long long)w_walk);
            }
        }
        return;
    }

    // ============================ builders ============================
    const int bt = tid - 32;
    uint32_t wphase = 0u, first = 3u, alive = 3u;   // bit s; alive is identical in every builder
    long long b_t[6] = {0, 0, 0, 0, 0, 0};   // builder-leader cycles: wait, prefix, clear, filter, build, link
    for (int s = 0; alive; s ^= 1) {
        if (!((alive >> s) & 1u)) continue;
        EndSlot &E = S[s];
        const long long ta = la_clock();
        if (bt == 0) {
            if (!((first >> s) & 1u)) {
                mbar_wait(&walked[s], (wphase >> s) & 1u);   // acquire: the walker's update of slot s
                wphase ^= 1u << s;
            }
            first &= ~(1u << s);
            B.overflow = 0;
            B.nclaim = 0;
            B.dead0 = 0;
            B.ctr_f = B.ctr_b = 0;
            if (E.done) {   // refill the slot with the next end, or retire it
                int idx, e = 0, lv = 0;
                do {   // replay: ends that left this kernel (overflow) in the extension are not replayed
                    idx = atomicAdd(work_ctr, 1);
                    if (idx < n_list) {
                        lv = list[idx];
                        e = list_end(lv);
                    }
                } while (P.replay && idx < n_list && out_dir[e] == OVF_DIR);
                if (idx >= n_list) {
                    E.dead = 1;
                    mbar_arrive(&built[s]);   // the walker sees `dead` and retires the slot too
                } else {
                    E.e = e;
                    E.anyN = list_anyn(lv);
                    E.stream = !GT && list_stream(lv);
                    E.r0 = eoff[e];
                    E.r = (int)(eoff[e + 1] - E.r0);
                    E.ulen = list_uniform(lv) ? P.maxlen : -1;   // else unknown until the first prefix pass
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
            }
        }
        builders_sync(NB);
        const long long tb = la_clock();
        b_t[0] += tb - ta;
        // the slot's own, monotonic `dead` flag — not the shared B.skip, which the leader rewrites for
        // the other slot right away (a builder still reading B.skip could see the other slot's value)
        if (E.dead) {
            alive &= ~(1u << s);
            continue;
        }
        const int k = E.k;
        const int KW = kwords(k);
        const bool INL = inline_keys(k);
        const long long r0 = E.r0;
        const int r = E.r;
        const int ulen = E.ulen;
        // shared-memory tables: stage the end's reads (coalesced 16 B copies); the XL class streams
        // them from HBM/L2 instead
        // shared-memory tables: the end's reads are staged in shared memory (coalesced 16 B copies) and
        // every builder access is a plain LDS (the pointers below are shared-memory pointers whenever
        // !GT, so the compiler emits LDS, not generic loads); the XL class streams them from HBM/L2.
        unsigned char *stage = tbase + FX.off_tab;
        const bool stream = !GT && E.stream;   // reads from global memory, like the XL class
        const bool no_room = !GT && (stream ? 0u : stage_bytes(r, SW)) + pref_bytes(r) + 64u * 24u > FX.tab_bytes;
        uint64_t *sR = (uint64_t *)stage;
        uint64_t *sQ = sR + (size_t)r * SW;
        uint16_t *sL = (uint16_t *)(sQ + (size_t)r * SW);
        uint8_t *sF = (uint8_t *)(sL + r);
        const uint64_t *gR = (GT || stream) ? rseq : sR;
        const uint64_t *gQ = (GT || stream) ? rqc : sQ;
        const uint16_t *gL = (GT || stream) ? rlen : sL;
        const uint8_t *gF = (GT || stream) ? rflag : sF;
        long long lr0 = (GT || stream) ? r0 : 0;   // first read index in (gR, gQ, gL, gF)
        if (!GT && !stream && !no_room) {
            const uint4 *a4 = (const uint4 *)(rseq + r0 * SW);
            const uint4 *b4 = (const uint4 *)(rqc + r0 * SW);
            const int n4 = r * SW / 2;   // SW is even
            for (int i = bt; i < n4; i += NB) {
                ((uint4 *)sR)[i] = __ldg(&a4[i]);
                ((uint4 *)sQ)[i] = __ldg(&b4[i]);
            }
            for (int i = bt; i < r; i += NB) {
                sL[i] = __ldg(&rlen[r0 + i]);
                sF[i] = __ldg(&rflag[r0 + i]);
            }
            builders_sync(NB);
        }
        // positions with a following base, per read (exclusive prefix, pref[r] = U) -> table plan
        uint32_t *pref = (uint32_t *)(stage + ((GT || stream) ? 0u : stage_bytes(r, SW)));
        if (no_room) {   // the reads alone do not fit this CTA's shared memory: no table (overflow)
        } else {
            read_prefix(B, E, pref, gL, lr0, r, k, ulen, bt, NB);
        }
        const uint32_t U = no_room ? 0u : pref[r];
        const long long tc = la_clock();
        b_t[1] += tc - tb;
        long long td = tc, t_filter = tc, t_build = tc;
        // XL: stage this end's reads in shared memory when they fit beside the filter bitmaps (the
        // streamed reads were the XL kernel's top stall: long scoreboard on L2, ncu r01)
        SmemFixed FXt = FX;
        bool xl_staged = false;   // XL: this end's reads staged in shared memory
        if (GT && !no_room) {
            const uint32_t xs = (stage_bytes(r, SW) + 127u) & ~127u;
            const uint32_t mw = ((4u * U + 31u) / 32u + 3u) & ~3u;
            if (xs + 8u * mw + 256u <= FX.filt_bytes) {
                uint64_t *xR = (uint64_t *)(sm + FX.off_filt);
                uint64_t *xQ = xR + (size_t)r * SW;
                uint16_t *xL = (uint16_t *)(xQ + (size_t)r * SW);
                uint8_t *xF = (uint8_t *)(xL + r);
                const uint4 *a4 = (const uint4 *)(rseq + r0 * SW);
                const uint4 *b4 = (const uint4 *)(rqc + r0 * SW);
                const int n4 = r * SW / 2;   // SW is even
                for (int i = bt; i < n4; i += NB) {
                    ((uint4 *)xR)[i] = __ldg(&a4[i]);
                    ((uint4 *)xQ)[i] = __ldg(&b4[i]);
                }
                for (int i = bt; i < r; i += NB) {
                    xL[i] = __ldg(&rlen[r0 + i]);
                    xF[i] = __ldg(&rflag[r0 + i]);
                }
                builders_sync(NB);
                xl_staged = true;
                gR = xR;
                gQ = xQ;
                gL = xL;
                gF = xF;
                lr0 = 0;
                FXt.off_filt += xs;
                FXt.filt_bytes -= xs;
            }
        }
        if (bt == 0) {   // the attempt's table layout, once (broadcast through shared memory)
            SmemTab tb = smem_tab(FXt, U, P.V >= 2, key_bytes(k), r, GT, SW, !stream);
            if (GT) {   // XL: size the global table for this end (less to clear, scan and cache)
                const uint32_t need = max(xl_needed_cap(r, U, tb.mwords != 0), min_table_cap(BLOCK));
                if (tb.cap > need) {
                    tb.cap = (need + 1u) & ~1u;
                    tb.off_cnts = tb.off_keys + tb.cap * key_bytes(k);   // counters follow the keys
                    tb.off_list = tb.off_cnts + tb.cap * cnt_bytes(true, xl_wide(U));
                    tb.off_f = (tb.off_list + tb.cap * 2u + 15u) & ~15u;
                }
            }
            B.tb = tb;
        }
        builders_sync(NB);
        const SmemTab TB = B.tb;
        bool ovf = no_room || TB.cap < min_table_cap(BLOCK);   // no room at this k (claims + in-flight < cap)
        if (!ovf) {
            const uint32_t mbits = TB.mwords * 32u;
            if (bt == 0) {
                s_acc[3] += mbits ? 1 : 0;
                s_acc[INL ? 4 : 5] += 1;
            }
            uint32_t *B1 = (uint32_t *)(sm + TB.off_b1);   // filters: always shared memory
            uint32_t *B2 = (uint32_t *)(sm + TB.off_b2);
            TabCtx T;
            T.keys = (uint64_t *)(tbase + TB.off_keys);
            T.c32 = (uint32_t *)(tbase + TB.off_cnts);
            T.list = (uint16_t *)(tbase + TB.off_list);
            T.ks = GT ? 0u : (uint32_t)__cvta_generic_to_shared(T.keys);
            T.cap = TB.cap;
            T.rseq = gR;   // REF keys store read indices relative to gR
            T.SW = SW;
            T.k = k;
            T.KW = KW;
            T.wide = GT && xl_wide(U) ? 1 : 0;
            // clear keys + counters (contiguous) and the filters
            {
                const uint4 z = make_uint4(0, 0, 0, 0);
                uint4 *a = (uint4 *)T.keys;
                const uint32_t n16 = (TB.cap * (key_bytes(k) + cnt_bytes(GT, GT && xl_wide(U)))) / 16u;
                for (uint32_t i = bt; i < n16; i += NB) a[i] = z;
                for (uint32_t i = bt; i < 2u * TB.mwords; i += NB) B1[i] = 0;   // B1, B2 contiguous
            }
            builders_sync(NB);
            td = la_clock();
            t_filter = t_build = td;
            const int e = E.e;
            const int Tn = min((int)clen[e], 128);
            const uint64_t *tail_e = tail + (size_t)e * TAIL_W;
            const uint64_t n0 = tailN[2 * (size_t)e], n1 = tailN[2 * (size_t)e + 1];
            uint32_t *info = (uint32_t *)(sm + (s ? FX.off_info1 : 0u));
            const int ulen_now = E.ulen;   // set by read_prefix (published by the barrier above)
            void *fpos = GT ? (void *)(tbase + TB.off_f) : (void *)(sm + TB.off_f);
            uint32_t *queue = (uint32_t *)(sm + FX.off_queue) + (bt >> 5) * 64;
            if (INL)
                build_link<true, GT>(B, T, B1, B2, mbits, info, gQ, gL, gF, pref, lr0, r, P, tail_e, Tn, n0, n1, bt, NB,
                                     t_filter, t_build, P.replay != 0, ulen_now, fpos, queue, E.anyN != 0, GT ? xl_staged : !stream);
            else
                build_link<false, GT>(B, T, B1, B2, mbits, info, gQ, gL, gF, pref, lr0, r, P, tail_e, Tn, n0, n1, bt, NB,
                                      t_filter, t_build, P.replay != 0, ulen_now, fpos, queue, E.anyN != 0, GT ? xl_staged : !stream);
            ovf = B.overflow != 0;   // uniform: last written before build_link's last barrier
            if (bt == 0) s_acc[6] += B.dead0;
        }
        builders_sync(NB);   // info buffer complete; the table is free for the next build
        {
            const long long te = la_clock();
            b_t[2] += td - tc;
            b_t[3] += t_filter - td;
            b_t[4] += t_build - t_filter;
            b_t[5] += te - t_build;
        }
        if (bt == 0) {
            if (ovf) {
                // table or counter overflow: the global path redoes this end from scratch; the
                // slot is refilled on its next turn (the walker only passes it through)
                if (!P.replay) {
                    ovf_list[atomicAdd(n_ovf, 1)] = E.e;
                    out_dir[E.e] = OVF_DIR;
                }
                E.ovf = 1;
                E.done = 1;
            } else {
                E.start = B.start;
                E.ins += U;
            }
            mbar_arrive(&built[s]);   // release: info buffer + slot state visible to the walker
        }
    }
    if (bt == 0) {
        atomicAdd(&gstats->filtered, s_acc[3]);
        atomicAdd(&gstats->inl, s_acc[4]);
        atomicAdd(&gstats->ref, s_acc[5]);
        atomicAdd(&gstats->dead0, s_acc[6]);
        if (prof)
            for (int i = 0; i < 6; ++i) atomicAdd(&prof[i], (unsigned long long)b_t[i]);
    }
}


// ---- k_small: one end per CTA, every thread builds, thread 0 walks -------------------------------
// For the small-table classes the walk (a few thousand cycles) is short next to the build, so a
// dedicated walker warp only halves the warps that build (ncu: the builders are latency-bound at
// ~2 warps/SMSP).  Here all BLOCK threads build; after the link pass thread 0 walks while the others
// wait at the barrier (other CTAs on the SM keep the issue slots busy).  The reads are staged in
// shared memory once per end (not per attempt).
template <int BLOCK, int MINB = (768 / BLOCK > 0 ? 768 / BLOCK : 1)>
__global__ void __launch_bounds__(BLOCK, MINB) k_small(
    const int32_t *__restrict__ list, int n_list, int *__restrict__ work_ctr,
    const uint64_t *__restrict__ rseq, const uint64_t *__restrict__ rqc,
    const uint16_t *__restrict__ rlen, const uint8_t *__restrict__ rflag,
    const int64_t *__restrict__ eoff, const uint64_t *__restrict__ tail,
    const uint64_t *__restrict__ tailN, const int32_t *__restrict__ clen, int SW, DevParams P,
    uint32_t smem_bytes, uint8_t *__restrict__ walk_buf, int32_t *__restrict__ out_len,
    uint8_t *__restrict__ out_term, uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att,
    int8_t *__restrict__ out_dir, int32_t *__restrict__ ovf_list, int *__restrict__ n_ovf, GlobalStats *__restrict__ gstats,
    unsigned char *__restrict__ gscratch, uint32_t gstride, unsigned long long *__restrict__ prof) {
    (void)gscratch;
    (void)gstride;
    constexpr int NB = BLOCK;
    extern __shared__ __align__(16) unsigned char sm[];
    __shared__ EndSlot E;
    __shared__ BuildCtl B;
    __shared__ int s_done;
    __shared__ unsigned long long s_acc[GSTATS_WORDS];   // work counters (GlobalStats order)
    const int bt = threadIdx.x;
    __shared__ SmemFixed sFX;   // as in k_smem: computed once, read from shared memory
    if (threadIdx.x == 0) sFX = smem_fixed(P.W, smem_bytes, 0u, true, NB / 32);
    __syncthreads();
    const SmemFixed &FX = sFX;
    const int Wp = (P.W + 15) & ~15;
    uint8_t *wstr = sm + FX.off_walk;   // two walk strings: current / best
    uint32_t *info = (uint32_t *)sm;
    if (bt < GSTATS_WORDS) s_acc[bt] = 0;   // published by the first __syncthreads below
    long long b_t[8] = {0, 0, 0, 0, 0, 0, 0, 0};   // leader cycles: fetch, prefix, clear, filter, build, link, -, walk
    for (;;) {
        const long long ta = la_clock();
        if (bt == 0) {
            int idx, e = 0, lv = 0;
            do {   // replay: ends that left this kernel (overflow) in the extension are not replayed
                idx = atomicAdd(work_ctr, 1);
                if (idx < n_list) {
                        lv = list[idx];
                        e = list_end(lv);
                    }
            } while (P.replay && idx < n_list && out_dir[e] == OVF_DIR);
            B.skip = idx >= n_list;
            if (!B.skip) {
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
                if (P.replay) {
                    E.rec_att = out_att[e];
                    E.shift = out_dir[e] * P.k_shift;
                }
            }
        }
        __syncthreads();
        if (B.skip) break;
        const int e = E.e;
        const int r = E.r;
        const long long r0 = E.r0;
        // stage the end's reads once (coalesced 16 B copies)
        unsigned char *stage = sm + FX.off_tab;
        bool ovf = stage_bytes(r, SW) + pref_bytes(r) + 64u * 24u > FX.tab_bytes;
        uint64_t *sR = (uint64_t *)stage;
        uint64_t *sQ = sR + (size_t)r * SW;
        uint16_t *sL = (uint16_t *)(sQ + (size_t)r * SW);
        uint8_t *sF = (uint8_t *)(sL + r);
        if (!ovf) {
            const uint4 *a4 = (const uint4 *)(rseq + r0 * SW);
            const uint4 *b4 = (const uint4 *)(rqc + r0 * SW);
            const int n4 = r * SW / 2;   // SW is even
            for (int i = bt; i < n4; i += NB) {
                ((uint4 *)sR)[i] = __ldg(&a4[i]);
                ((uint4 *)sQ)[i] = __ldg(&b4[i]);
            }
            for (int i = bt; i < r; i += NB) {
                sL[i] = __ldg(&rlen[r0 + i]);
                sF[i] = __ldg(&rflag[r0 + i]);
            }
        }
        uint32_t *pref = (uint32_t *)(stage + stage_bytes(r, SW));
        const int Tn = min((int)clen[e], 128);
        const uint64_t *tail_e = tail + (size_t)e * TAIL_W;
        const uint64_t n0 = tailN[2 * (size_t)e], n1 = tailN[2 * (size_t)e + 1];
        __syncthreads();
        b_t[0] += la_clock() - ta;
        while (!ovf) {   // attempts (k schedule)
            const long long tb = la_clock();
            const int k = E.k;
            const int KW = kwords(k);
            read_prefix(B, E, pref, sL, 0, r, k, E.ulen, bt, NB);
            const uint32_t U = pref[r];
            if (bt == 0) B.tb = smem_tab(FX, U, P.V >= 2, key_bytes(k), r, false, SW);   // once per attempt
            __syncthreads();
            const SmemTab TB = B.tb;
            if (TB.cap < min_table_cap(BLOCK)) {
                ovf = true;
                break;
            }
            const uint32_t mbits = TB.mwords * 32u;
            if (bt == 0) {
                s_acc[3] += mbits ? 1 : 0;
                s_acc[inline_keys(k) ? 4 : 5] += 1;
            }
            uint32_t *B1 = (uint32_t *)(sm + TB.off_b1);
            uint32_t *B2 = (uint32_t *)(sm + TB.off_b2);
            TabCtx T;
            T.keys = (uint64_t *)(sm + TB.off_keys);
            T.c32 = (uint32_t *)(sm + TB.off_cnts);
            T.list = (uint16_t *)(sm + TB.off_list);
            T.ks = (uint32_t)__cvta_generic_to_shared(T.keys);
            T.cap = TB.cap;
            T.rseq = sR;
            T.SW = SW;
            T.k = k;
            T.KW = KW;
            T.wide = 0;
            if (bt == 0) {
                B.overflow = 0;
                B.nclaim = 0;
                B.dead0 = 0;
                B.ctr_f = B.ctr_b = 0;
            }
            const long long tc = la_clock();
            {
                const uint4 z = make_uint4(0, 0, 0, 0);
                uint4 *a = (uint4 *)T.keys;
                const uint32_t n16 = (TB.cap * (key_bytes(k) + cnt_bytes(false))) / 16u;
                for (uint32_t i = bt; i < n16; i += NB) a[i] = z;
                for (uint32_t i = bt; i < 2u * TB.mwords; i += NB) B1[i] = 0;
            }
            __syncthreads();
            const long long td = la_clock();
            long long t_filter = td, t_build = td;
            const int ulen_now = E.ulen;   // set by read_prefix (published by the barrier above)
            void *fpos = (void *)(sm + TB.off_f);
            uint32_t *queue = (uint32_t *)(sm + FX.off_queue) + (bt >> 5) * 64;
            if (inline_keys(k))
                build_link<true, false, LA_SMALL_FILTER_UNROLL>(B, T, B1, B2, mbits, info, sQ, sL, sF, pref, 0, r, P, tail_e, Tn, n0, n1, bt,
                                        NB, t_filter, t_build, P.replay != 0, ulen_now, fpos, queue, E.anyN != 0, true);
            else
                build_link<false, false>(B, T, B1, B2, mbits, info, sQ, sL, sF, pref, 0, r, P, tail_e, Tn, n0, n1, bt,
                                         NB, t_filter, t_build, P.replay != 0, ulen_now, fpos, queue, E.anyN != 0, true);
            __syncthreads();
            const long long te = la_clock();
            b_t[1] += tc - tb;
            b_t[2] += td - tc;
            b_t[3] += t_filter - td;
            b_t[4] += t_build - t_filter;
            b_t[5] += te - t_build;
            if (bt == 0) s_acc[6] += B.dead0;
            if (B.overflow) {
                ovf = true;
                break;
            }
            if (bt == 0 && P.replay) {   // replay: the recorded k sequence instead of the walk
                E.ins += U;
                E.attempts += 1;
                s_done = E.attempts >= E.rec_att;
                E.k += E.shift;
            } else if (bt == 0) {
                // ---- walk (Alg 2) over the successor links ----
                E.ins += U;
                uint8_t *wb = wstr + (E.best_buf ^ 1) * Wp;
                // (k_small keeps the plain per-step loop: walk_links measured 5% slower here, where the
                // walk's latency is exposed to the waiting CTA rather than its issue slots)
                uint32_t node = B.start == NONE ? NEXT_NONE : B.start;
                int len = 0, term = T_MAXLEN;
                unsigned long long steps = 0;
#if LA_WALK_PIPE_SMALL
                len = walk_links(info, node, P.W, wb, term, steps);
                if (false)
#endif
                for (int i = 0; i < P.W; ++i) {
                    ++steps;   // a lookup; the loop check of a present k-mer precedes it (below)
                    if (node == NEXT_NONE) { term = T_DEADEND; break; }
                    const uint32_t inf = info[node];
                    if (inf & 8u) { term = T_LOOP; --steps; break; }   // visited: loop check before lookup
                    info[node] = inf | 8u;
                    const uint32_t code = inf & 7u;
                    if (code == CODE_FORK) { term = T_FORK; break; }
                    if (code == CODE_DEADEND) { term = T_DEADEND; break; }
                    wb[len++] = (uint8_t)(0x54474341u >> (8 * code));   // "ACGT"[code] without a memory lookup
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
                s_done = next_k(term, kk, sh, E.kmax_eff, P) ? 1 : 0;
                E.k = kk;
                E.shift = sh;
            }
            __syncthreads();
            b_t[7] += la_clock() - te;
            if (s_done) break;
        }
        if (ovf) {   // table or counter overflow: the global path redoes this end from scratch
            if (bt == 0 && !P.replay) {
                ovf_list[atomicAdd(n_ovf, 1)] = e;
                out_dir[e] = OVF_DIR;
            }
        } else if (P.replay) {
            if (bt == 0) {
                s_acc[0] += E.ins;
                s_acc[2] += E.attempts;
            }
        } else {
            const int bl = E.best_len;
            const uint8_t *bw = wstr + E.best_buf * Wp;
            uint8_t *dst = walk_buf + (size_t)e * P.W;
            for (int i = bt; i < bl; i += NB) dst[i] = bw[i];
            if (bt == 0) {
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
        __syncthreads();   // E and the staged reads are reused by the next end
    }
    if (bt == 0) {
        unsigned long long *g = &gstats->inserts;
        for (int i = 0; i < GSTATS_WORDS; ++i) atomicAdd(&g[i], s_acc[i]);
        if (prof) {
            for (int i = 0; i < 6; ++i) atomicAdd(&prof[i], (unsigned long long)b_t[i]);
            atomicAdd(&prof[7], (unsigned long long)b_t[7]);
        }
    }
}

}  // namespace la

