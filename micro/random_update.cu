// random_update.cu — microbenchmarks of the roofline denominators:
// the random-update rate of the memory that holds a k-mer table.
//   smem_atomic_inc32: random 32-bit atomicAdd(+1) into a per-CTA shared-memory table (ATOMS.POPC.INC)
//   smem_atomic_add32: random 32-bit atomicAdd of a variable increment, old value returned (ATOMS.ADD)
//                      = the vote update of the table
//   smem_cas64      : random 64-bit atomicCAS into shared memory (ATOMS.CAS.64)
//   smem_load64     : random 64-bit loads from shared memory (LDS.64, the probe)
//   global_red_l2   : random 32-bit atomicAdd (RED.ADD) into a 64 MB L2-resident global table
//   global_red_hbm  : same into a 4 GB table (HBM-bound)
//   smem_hash_insert: the table's insert primitive in isolation — hash a 2-word k-mer key, whole-warp
//                     probe rounds over slot pairs (16 B keys, 128-bit CAS claim), one 8-bit-field vote
//                     atomic with carry check — on a 110 KB table at load 0.3 (keys from a pool of
//                     0.3 x capacity distinct keys): the achievable insert rate of the table design,
//                     without position extraction, filter pass, link or walk
// Output: one JSON line, G updates/s per variant (best of 5, CUDA events).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro/random_update micro/random_update.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
    return x;
}

template <int MODE>
__global__ void k_smem(int iters, uint32_t words, unsigned long long *sink) {
    extern __shared__ uint32_t t[];
    for (uint32_t i = threadIdx.x; i < words; i += blockDim.x) t[i] = 0;
    __syncthreads();
    uint32_t x = hsh(blockIdx.x * 7919u + threadIdx.x);
    uint64_t acc = 0;
    for (int it = 0; it < iters; ++it) {
        x = hsh(x + it);
        if (MODE == 0) {
            atomicAdd(&t[x % words], 1u);
        } else if (MODE == 3) {   // the table's vote update: 32-bit add of a data-dependent increment
            acc += atomicAdd(&t[x % words], 1u << ((x >> 24) & 31));
        } else if (MODE == 1) {
            unsigned long long *t64 = (unsigned long long *)t;
            acc += atomicCAS(&t64[x % (words / 2)], 0ull, (unsigned long long)x);
        } else {
            const unsigned long long *t64 = (const unsigned long long *)t;
            acc += t64[x % (words / 2)];
        }
    }
    __syncthreads();
    if (acc == 0x12345678ull) sink[0] = acc + t[threadIdx.x % words];
}

__device__ __forceinline__ uint32_t key_hash(uint64_t w0, uint64_t w1) {   // as la::hash_kmer<2> (low word)
    uint32_t h = ((uint32_t)w0 ^ ((uint32_t)(w0 >> 32) * 0x85EBCA6Bu)) * 0xCC9E2D51u;
    h ^= ((uint32_t)w1 ^ ((uint32_t)(w1 >> 32) * 0x27D4EB2Fu)) * 0x1B873593u;
    h ^= h >> 15;
    h *= 0x2C1B3C6Du;
    h ^= h >> 12;
    return h;
}

__global__ void k_hash_insert(int iters, uint32_t cap, uint32_t pool, unsigned long long *sink) {
    extern __shared__ __align__(16) uint64_t tk[];   // cap x 16 B keys, then cap x 8 B counters
    uint32_t *cnt = (uint32_t *)(tk + 2 * cap);
    __shared__ int nclaim;
    for (uint32_t i = threadIdx.x; i < 3 * cap; i += blockDim.x) tk[i] = 0;
    if (threadIdx.x == 0) nclaim = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    uint32_t x = hsh(blockIdx.x * 7919u + threadIdx.x);
    uint32_t carry = 0;
    for (int it = 0; it < iters; ++it) {
        x = hsh(x + it);
        const uint32_t id = x % pool;                     // key id: ~pool distinct keys, mostly hits
        const uint64_t a = ((uint64_t)hsh(2 * id + 1) << 32) | hsh(2 * id + 7);
        const uint64_t bb = ~(((uint64_t)hsh(2 * id + 3) << 32) & ~3ull);   // never all-ones: y != 0
        const uint32_t h = key_hash(a, ~bb);
        uint32_t s = (uint32_t)(((uint64_t)h * cap) >> 32) & ~1u, hit = 0;
        bool pend = true, found = false;
        while (__any_sync(0xffffffffu, pend)) {
            bool claimed = false;
            if (pend) {
                uint64_t xs[2], ys[2];
                const unsigned ka = (unsigned)__cvta_generic_to_shared(&tk[2 * s]);
                asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];" : "=l"(xs[0]), "=l"(ys[0]) : "r"(ka) : "memory");
                asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];" : "=l"(xs[1]), "=l"(ys[1]) : "r"(ka + 16u) : "memory");
#pragma unroll
                for (int u = 0; u < 2 && pend; ++u) {
                    uint64_t xx = xs[u], yy = ys[u];
                    if (yy == 0) {
                        const unsigned addr = (unsigned)__cvta_generic_to_shared(&tk[2 * (s + u)]);
                        asm volatile("{\n .reg .b128 d, b, c;\n mov.b128 b, {%2, %3};\n mov.b128 c, {%4, %5};\n"
                                     " atom.shared.cas.b128 d, [%6], b, c;\n mov.b128 {%0, %1}, d;\n}"
                                     : "=l"(xx), "=l"(yy) : "l"(0ull), "l"(0ull), "l"(a), "l"(bb), "r"(addr) : "memory");
                        if (yy == 0) { claimed = true; xx = a; yy = bb; }
                    }
                    if (xx == a && yy == bb) { pend = false; found = true; hit = s + u; }
                }
                if (pend) s = s + 2 >= cap ? 0 : s + 2;
            }
            const unsigned cm = __ballot_sync(0xffffffffu, claimed);
            if (cm && lane == __ffs(cm) - 1) atomicAdd(&nclaim, __popc(cm));
        }
        if (found) {
            const uint32_t b = x >> 30;
            const uint32_t old = atomicAdd(&cnt[2 * hit + ((x >> 29) & 1u)], 1u << (8 * b));
            carry |= ((old >> (8 * b)) & 0xffu) == 0xffu;
        }
    }
    __syncthreads();
    if (carry == 0x12345678u) sink[0] = nclaim;
}

__global__ void k_global(uint32_t *tab, uint64_t words, int iters) {
    uint32_t x = hsh(blockIdx.x * 7919u + threadIdx.x);
    for (int it = 0; it < iters; ++it) {
        x = hsh(x + it);
        uint64_t i = ((uint64_t)x * 0x9E3779B1u + it) % words;
        atomicAdd(&tab[i], 1u);
    }
}

int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    const int sms = p.multiProcessorCount;
    unsigned long long *sink;
    cudaMalloc(&sink, 64);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int threads = 256, ctas_per_sm = 2;
    const uint32_t bytes = 110 * 1024;
    const uint32_t words = bytes / 4;
    const int iters = 4096;
    double res[7] = {0, 0, 0, 0, 0, 0, 0};
    cudaFuncSetAttribute(k_smem<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    cudaFuncSetAttribute(k_smem<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    cudaFuncSetAttribute(k_smem<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    cudaFuncSetAttribute(k_smem<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    for (int mode = 0; mode < 4; ++mode) {
        double best = 0;
        for (int rep = 0; rep < 6; ++rep) {
            cudaEventRecord(a);
            if (mode == 0) k_smem<0><<<sms * ctas_per_sm, threads, bytes>>>(iters, words, sink);
            if (mode == 1) k_smem<1><<<sms * ctas_per_sm, threads, bytes>>>(iters, words, sink);
            if (mode == 2) k_smem<2><<<sms * ctas_per_sm, threads, bytes>>>(iters, words, sink);
            if (mode == 3) k_smem<3><<<sms * ctas_per_sm, threads, bytes>>>(iters, words, sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            double ops = (double)sms * ctas_per_sm * threads * iters;
            if (rep) best = best > ops / ms / 1e6 ? best : ops / ms / 1e6;
        }
        res[mode] = best;
    }
    {   // table insert primitive: 110 KB = cap x 24 B, pool = 0.3 cap distinct keys
        const uint32_t cap = (bytes / 24) & ~1u, pool = (uint32_t)(0.3 * cap);
        const int hi_iters = 2048;
        cudaFuncSetAttribute(k_hash_insert, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
        double best = 0;
        for (int rep = 0; rep < 6; ++rep) {
            cudaEventRecord(a);
            k_hash_insert<<<sms * ctas_per_sm, threads, bytes>>>(hi_iters, cap, pool, sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            double ops = (double)sms * ctas_per_sm * threads * hi_iters;
            if (rep) best = best > ops / ms / 1e6 ? best : ops / ms / 1e6;
        }
        res[6] = best;
    }
    for (int g = 0; g < 2; ++g) {
        uint64_t words_g = g == 0 ? (64ull << 20) / 4 : (4ull << 30) / 4;
        uint32_t *tab;
        if (cudaMalloc(&tab, words_g * 4) != cudaSuccess) continue;
        cudaMemset(tab, 0, words_g * 4);
        double best = 0;
        const int gi = 256;
        const int grid = sms * 8;
        for (int rep = 0; rep < 6; ++rep) {
            cudaEventRecord(a);
            k_global<<<grid, 256>>>(tab, words_g, gi);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            double ops = (double)grid * 256 * gi;
            if (rep) best = best > ops / ms / 1e6 ? best : ops / ms / 1e6;
        }
        res[4 + g] = best;
        cudaFree(tab);
    }
    printf("{\"unit\": \"G updates/s\", \"smem_atomic_inc32\": %.2f, \"smem_cas64\": %.2f, \"smem_load64\": %.2f, "
           "\"smem_atomic_add32\": %.2f, \"global_red_l2\": %.2f, \"global_red_hbm\": %.2f, "
           "\"smem_hash_insert\": %.2f, \"sms\": %d, "
           "\"smem_ctas_per_sm\": %d, \"threads\": %d, \"smem_bytes_per_cta\": %u, \"err\": \"%s\"}\n",
           res[0], res[1], res[2], res[3], res[4], res[5], res[6], sms, ctas_per_sm, threads, bytes,
           cudaGetErrorString(cudaGetLastError()));
    return 0;
}
