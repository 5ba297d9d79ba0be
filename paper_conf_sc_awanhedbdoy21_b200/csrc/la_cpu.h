// la_cpu.h — the host (CPU) implementation of local assembly used by the CPU+GPU co-execution mode
// (the paper's CPU/GPU co-scheduling, §4.3, Fig 11).
//
// Product code of the library (not the test oracle, which it shares nothing with): it extends ends
// from the same oriented 2-bit encoding the device kernels read (la_device.cuh layout), gathered for
// the selected ends by the device (locassm.cu), so its results are written back into the same
// result arrays and emitted by the same device compaction as the GPU's.
#pragma once
#include <cstdint>

namespace la_cpu {

struct Params {   // the la_params knobs, as the device's DevParams
    int k_start, k_min, k_max, k_shift, W, V, F;
};

// Gathered input of n ends (host memory).  End i owns reads [roff[i], roff[i+1]) of rseq / rqc (SW
// 64-bit words per read, 2-bit codes, base j at bit 62 - 2*(j%32) of word j/32; quality class 0 = no
// vote, 1 = low tier, 2 = both tiers, 3 = N), rlen; tail[5*i..] = the last <= 128 bases of the
// oriented contig (same packing), tailN[2*i..] its N mask, clen[i] the contig length.
struct Input {
    int n, SW;
    const int64_t *roff;
    const uint64_t *rseq, *rqc;
    const uint16_t *rlen;
    const uint64_t *tail, *tailN;
    const int32_t *clen;
};

// Results of end i: walk[i*W .. +len[i]) in walk orientation (as the device's walk buffer), term,
// k of the returned walk, attempts, direction of the k shifts; work counters summed over the ends.
struct Output {
    int32_t *len;
    uint8_t *walk, *term, *k_used, *att;
    int8_t *dir;
    int64_t inserts, walk_steps, attempts;
};

// Extends the n ends on `threads` host threads (>= 1).
void extend(const Input &in, const Params &P, int threads, Output &out);

}  // namespace la_cpu
