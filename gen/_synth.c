/* _synth.c — fast, seeded synthesis of genomes and sequenced reads for gen/synth.py.
 *
 * Input synthesis only (no k-mers, votes or walks).  Every random draw is a counter-based hash of
 * (seed, object id, position), so the output does not depend on thread count or chunking.
 * Build: gcc -O3 -fopenmp -shared -fPIC (gen/synth.py builds it on first use).
 */
#include <stdint.h>

static inline uint64_t mix(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

static inline double u01(uint64_t h) { return (double)(h >> 11) * (1.0 / 9007199254740992.0); }

/* i.i.d. genome with G+C content gc: codes 0..3 = A,C,G,T */
void synth_genome(uint8_t *out, int64_t n, double gc, uint64_t seed) {
    const double pa = (1.0 - gc) / 2, pc = gc / 2;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        double u = u01(mix(seed ^ mix((uint64_t)i)));
        out[i] = u < pa ? 0 : (u < pa + pc ? 1 : (u < pa + 2 * pc ? 2 : 3));
    }
}

/* Reads of length L starting at genome_all[start[i]]: uniform substitutions at rate err, N calls at
 * rate nrate (Q2); correct bases Q30-40 with prob 0.9 else Q2-29, substituted bases Q2-25.
 * uid[i] identifies the physical read (the same read copied into two ends is identical).
 * seq_out: ASCII ACGTN, qual_out: Phred+33. */
void synth_reads(const uint8_t *genome_all, const int64_t *start, const int64_t *uid, int64_t n, int L,
                 uint64_t seed, double err, double nrate, uint8_t *seq_out, uint8_t *qual_out) {
    static const uint8_t ASC[5] = {'A', 'C', 'G', 'T', 'N'};
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        const uint8_t *g = genome_all + start[i];
        const uint64_t base = mix(seed ^ mix((uint64_t)uid[i] * 0x100000001B3ull));
        for (int p = 0; p < L; ++p) {
            uint64_t h1 = mix(base + (uint64_t)p * 0x632BE59BD9B4E019ull);
            uint64_t h2 = mix(h1);
            double u = u01(h1);
            uint8_t b = g[p];
            int q;
            if (u < err) {
                b = (uint8_t)((b + 1 + (h2 % 3)) & 3);
                q = 2 + (int)((h2 >> 8) % 24);
            } else if (u < err + nrate) {
                b = 4;
                q = 2;
            } else {
                double v = u01(h2);
                q = v < 0.9 ? 30 + (int)((h2 >> 8) % 11) : 2 + (int)((h2 >> 8) % 28);
            }
            seq_out[i * L + p] = ASC[b];
            qual_out[i * L + p] = (uint8_t)(q + 33);
        }
    }
}
