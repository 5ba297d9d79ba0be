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

// Read encoder (a2): oriented 2-bit bases and quality classes; LEFT-end reads are reverse
// complemented with reversed qualities (reading #14).  A CTA takes ENC_R consecutive
// reads, copies their contiguous byte range of seq and qual into shared memory with coalesced 16 B
// loads, then one thread per (read, 32-base word) packs from shared memory (r01: a thread-per-word
// encoder doing per-thread global byte loads ran at ~0.45 TB/s on C4 and was removed).
constexpr int ENC_R = 64;
constexpr int ENC_BYTES = ENC_R * MAX_READ_LEN + 32;
__global__ void __launch_bounds__(256) k_encode_reads_staged(
    const char *__restrict__ seq, const char *__restrict__ qual, const int64_t *__restrict__ roff,
    const int32_t *__restrict__ read_end, int64_t n_reads, int SW, DevParams P, uint64_t *__restrict__ rseq,
    uint64_t *__restrict__ rqc, uint16_t *__restrict__ rlen, uint8_t *__restrict__ rflag, uint32_t *err) {
    __shared__ __align__(16) unsigned char sS[ENC_BYTES], sQ[ENC_BYTES];
    const int64_t j0 = (int64_t)blockIdx.x * ENC_R;
    const int64_t j1 = min(j0 + ENC_R, n_reads);
    const int64_t b0 = roff[j0], b1 = roff[j1];
    const int64_t a0 = b0 & ~15ll;                       // 16 B aligned start (base pointers permitting)
    const bool vec = ((((uintptr_t)seq) | ((uintptr_t)qual)) & 15u) == 0;
    const int64_t lo = vec ? a0 : b0;
    const int nbytes = (int)(b1 - lo);                   // <= ENC_R*300 + 15 (lengths validated)
    if (vec) {
        const int n16 = (nbytes + 15) >> 4;
        const uint4 *gs = (const uint4 *)(seq + lo), *gq = (const uint4 *)(qual + lo);
        for (int i = threadIdx.x; i < n16; i += blockDim.x) {
            ((uint4 *)sS)[i] = __ldg(gs + i);   // may read up to 15 B past b1: within the 16 B granule
            ((uint4 *)sQ)[i] = __ldg(gq + i);
        }
    } else {
        for (int i = threadIdx.x; i < nbytes; i += blockDim.x) {
            sS[i] = (unsigned char)seq[lo + i];
            sQ[i] = (unsigned char)qual[lo + i];
        }
    }
    __shared__ int s_o[ENC_R], s_len[ENC_R];
    __shared__ uint8_t s_left[ENC_R];
    for (int jj = threadIdx.x; jj < (int)(j1 - j0); jj += blockDim.x) {
        const int64_t a = roff[j0 + jj];
        s_o[jj] = (int)(a - lo);
        s_len[jj] = (int)(roff[j0 + jj + 1] - a);
        s_left[jj] = (read_end[j0 + jj] & 1) == 0;
    }
    __syncthreads();
    // thread per (read, 32-base word), branch-free per base (a data-dependent switch split the warp
    // four ways): ACGT -> 0123 by ((c >> 2) ^ (c >> 1)) & 3; validity from a bit mask over 'A'..'T';
    // N (or an invalid character, reported) -> code 0, class 3.  (Measured alternatives, r01: a warp
    // per word with ballots was 4x slower — one serial dependency chain per warp.)
    uint32_t e = 0;
    const int nw = (int)(j1 - j0) * SW;
    for (int t = threadIdx.x; t < nw; t += blockDim.x) {
        const int jj = t / SW, w = t - jj * SW;
        const int o = s_o[jj], len = s_len[jj];
        const bool left = s_left[jj];
        const int nb = min(32, len - w * 32);   // bases of this word (<= 0: padding word)
        uint32_t hi32 = 0, lo32 = 0, qhi = 0, qlo = 0;   // 32-bit halves of the packed words
        bool hasN = false;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
            const bool in = i < nb;
            const int ib = w * 32 + i;
            const int src = in ? (left ? o + len - 1 - ib : o + ib) : 0;
            const uint32_t c = sS[src];
            const int q = (int)sQ[src] - P.qual_offset;
            const uint32_t d = c - 65u;
            const bool valid = d < 20u && ((0x82045u >> d) & 1u);   // A C G N T
            const bool isn = !valid || c == 'N';
            uint32_t code = ((c >> 2) ^ (c >> 1)) & 3u;
            code = left ? 3u - code : code;
            uint32_t qc = q >= P.q_hi ? 2u : (q >= P.q_lo ? 1u : 0u);
            code = (in && !isn) ? code : 0u;
            qc = in ? (isn ? 3u : qc) : 0u;
            e |= (in && !valid) ? ERR_READ_CHAR : 0u;
            e |= (in && q < 0) ? ERR_QUAL_CHAR : 0u;
            hasN |= in && isn;
            if (i < 16) {
                hi32 |= code << (30 - 2 * i);
                qhi |= qc << (30 - 2 * i);
            } else {
                lo32 |= code << (62 - 2 * i);
                qlo |= qc << (62 - 2 * i);
            }
        }
        const int64_t j = j0 + jj;
        rseq[j * SW + w] = ((uint64_t)hi32 << 32) | lo32;
        rqc[j * SW + w] = ((uint64_t)qhi << 32) | qlo;
        if (w == 0) rlen[j] = (uint16_t)len;
        if (hasN) rflag[j] = 1;   // rflag zeroed before launch
    }
    for (int o = 16; o; o >>= 1) e |= __shfl_xor_sync(0xffffffffu, e, o);
    if (e && (threadIdx.x & 31) == 0) atomicOr(err, e);
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

}  // namespace la

#include "la_smem.cuh"
#include "la_xlc.cuh"
#include "la_global.cuh"

namespace la {

// ------------------------------------------------------------------------------------------------
// emit (a9)
// ------------------------------------------------------------------------------------------------
// ---- NEXT N3 co-execution: gather the host's ends, scatter its results ----
__global__ void k_cx_counts(const int32_t *__restrict__ list, int m, const int64_t *__restrict__ eoff,
                            int64_t *__restrict__ cnt) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < m) cnt[i] = eoff[list_end(list[i]) + 1] - eoff[list_end(list[i])];
    else if (i == m) cnt[i] = 0;
}
// one warp per end: its reads' packed rows, lengths, and the contig tail
__global__ void k_cx_gather(const int32_t *__restrict__ list, int m, const int64_t *__restrict__ eoff,
                            const int64_t *__restrict__ goff, int SW, const uint64_t *__restrict__ rseq,
                            const uint64_t *__restrict__ rqc, const uint16_t *__restrict__ rlen,
                            const uint64_t *__restrict__ tail, const uint64_t *__restrict__ tailN,
                            const int32_t *__restrict__ clen, uint64_t *__restrict__ g_rseq,
                            uint64_t *__restrict__ g_rqc, uint16_t *__restrict__ g_rlen, uint64_t *__restrict__ g_tail,
                            uint64_t *__restrict__ g_tailN, int32_t *__restrict__ g_clen) {
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int i = (int)(t >> 5), lane = (int)(t & 31);
    if (i >= m) return;
    const int e = list_end(list[i]);
    const int64_t r0 = eoff[e], n = eoff[e + 1] - r0, g0 = goff[i];
    for (int64_t w = lane; w < n * SW; w += 32) {
        g_rseq[g0 * SW + w] = rseq[r0 * SW + w];
        g_rqc[g0 * SW + w] = rqc[r0 * SW + w];
    }
    for (int64_t j = lane; j < n; j += 32) g_rlen[g0 + j] = rlen[r0 + j];
    if (lane < TAIL_W) g_tail[(int64_t)i * TAIL_W + lane] = tail[(int64_t)e * TAIL_W + lane];
    if (lane < 2) g_tailN[2 * (int64_t)i + lane] = tailN[2 * (int64_t)e + lane];
    if (lane == 0) g_clen[i] = clen[e];
}
__global__ void k_cx_scatter(const int32_t *__restrict__ list, int m, int W, const int32_t *__restrict__ len,
                             const uint8_t *__restrict__ term, const uint8_t *__restrict__ kk,
                             const uint8_t *__restrict__ att, const int8_t *__restrict__ dir,
                             const uint8_t *__restrict__ walk, int32_t *__restrict__ out_len,
                             uint8_t *__restrict__ out_term, uint8_t *__restrict__ out_k, uint8_t *__restrict__ out_att,
                             int8_t *__restrict__ out_dir, uint8_t *__restrict__ walk_buf) {
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int i = (int)(t >> 5), lane = (int)(t & 31);
    if (i >= m) return;
    const int e = list_end(list[i]);
    for (int j = lane; j < len[i]; j += 32) walk_buf[(int64_t)e * W + j] = walk[(int64_t)i * W + j];
    if (lane == 0) {
        out_len[e] = len[i];
        out_term[e] = term[i];
        out_k[e] = kk[i];
        out_att[e] = att[i];
        out_dir[e] = dir[i];
    }
}

// ends per attempt count (la_stats.attempts_hist; the last bin collects >= LA_HIST - 1)
__global__ void k_att_hist(const uint8_t *__restrict__ att, int64_t n, unsigned long long *__restrict__ hist) {
    __shared__ unsigned int h[LA_HIST];
    if (threadIdx.x < LA_HIST) h[threadIdx.x] = 0;
    __syncthreads();
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) atomicAdd(&h[min((int)att[i], LA_HIST - 1)], 1u);
    __syncthreads();
    if (threadIdx.x < LA_HIST && h[threadIdx.x]) atomicAdd(&hist[threadIdx.x], (unsigned long long)h[threadIdx.x]);
}

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
