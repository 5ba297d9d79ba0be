// locassm.cu — the C ABI (include/locassm.h) and the host-side runtime of the sm_100a local-assembly
// library: context, validation + encode on load, planning, launches, result compaction.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -shared -Xcompiler -fPIC
// (see paper_conf_sc_awanhedbdoy21_b200/build.py).  No torch types cross this boundary.
#include <cuda_runtime.h>
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "locassm.h"
#include "la_cpu.h"
#include "la_kernels.cuh"
#include "la_select.cuh"

using namespace la;

namespace {

struct DevBuf {
    void *p = nullptr;
    size_t n = 0;
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
    }
};

struct HostBuf {
    void *p = nullptr;
    size_t n = 0;
    void release() {
        if (p) cudaFreeHost(p);
        p = nullptr;
        n = 0;
    }
};

// NEXT N4 (la_select_reads): device copies of the pool and the selection's scratch and results.
struct SelBufs {
    DevBuf cseq, coff, rseq, rqual, roff, wcnt, woff, key, val, key2, val2, flag, uidx, ustart, hkey, hval, nrec,
        rkey, rord, rkey2, rord2, send, spair, sflip, eoff, lens, ooff, oseq, oqual;
    void release() {
        for (DevBuf *b : {&cseq, &coff, &rseq, &rqual, &roff, &wcnt, &woff, &key, &val, &key2, &val2, &flag, &uidx,
                          &ustart, &hkey, &hval, &nrec, &rkey, &rord, &rkey2, &rord2, &send, &spair, &sflip, &eoff,
                          &lens, &ooff, &oseq, &oqual})
            b->release();
    }
};

// Encoded batch (device), produced by la_load_batch.
struct Encoded {
    int64_t n_contigs = 0, n_ends = 0, n_reads = 0;
    int SW = 2, maxlen = 0;
    DevBuf eoff, roff, rseq, rqc, rlen, rflag, tail, tailN, clen;
    void release() {
        for (DevBuf *b : {&eoff, &roff, &rseq, &rqc, &rlen, &rflag, &tail, &tailN, &clen}) b->release();
    }
};

}  // namespace

namespace {
// Table-class kernels by (threads, resident CTAs per SM, k_small?): the launch bound gives each
// instantiation the register budget 65536 / (threads x CTAs).  LA_CLASSES picks among these.
using ClassKernel = void (*)(const int32_t *, int, int *, const uint64_t *, const uint64_t *, const uint16_t *,
                             const uint8_t *, const int64_t *, const uint64_t *, const uint64_t *, const int32_t *,
                             int, DevParams, uint32_t, uint8_t *, int32_t *, uint8_t *, uint8_t *, uint8_t *,
                             int8_t *, int32_t *, int *, GlobalStats *, unsigned char *, uint32_t,
                             unsigned long long *);
struct ClassEntry {
    int threads, ctas;
    bool small;
    ClassKernel fn;
};
const ClassEntry kClassKernels[] = {   // the five classes la_create configures (see cls_threads / cls_ctas)
    {64, 12, true, k_small<64, 12>},
    {128, 6, true, k_small<128, 6>},
    {256, 3, false, k_smem<256, false, 3>},
    {512, 2, false, k_smem<512, false, 2>},
    {1024, 1, false, k_smem<1024, false, 1>},
#ifdef LA_EXTRA_CLASSES   // tuning builds only (tools/ab_build.sh): other (threads x CTAs/SM) shapes
    {64, 16, true, k_small<64, 16>},   {128, 8, true, k_small<128, 8>},  {96, 8, true, k_small<96, 8>},
    {256, 4, false, k_smem<256, false, 4>}, {256, 3, true, k_small<256, 3>}, {32, 24, true, k_small<32, 24>},
    {32, 16, true, k_small<32, 16>},   {64, 10, true, k_small<64, 10>},
#endif
};
const ClassEntry *find_class_kernel(int threads, int ctas, bool small) {
    for (const ClassEntry &k : kClassKernels)
        if (k.threads == threads && k.ctas == ctas && k.small == small) return &k;
    return nullptr;
}
}  // namespace

struct la_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    bool sticky = false;
    bool loaded = false;
    std::string err;
    int n_sm = 148;
    int cls_threads[N_SMEM_CLASSES] = {64, 128, 256, 512, 1024};   // r01: 256x2 -> 512x2 155 -> 146 ms, 512x1 -> 1024x1 166 -> 162 ms
    int cls_ctas[N_SMEM_CLASSES] = {12, 6, 3, 2, 1};   // resident CTAs per SM of each shared-memory class
    uint32_t cls_bytes[N_SMEM_CLASSES] = {0, 0, 0, 0, 0};   // dynamic shared memory per CTA
    uint32_t xl_bytes = 0;        // dynamic shared memory of the XL class (the rest of the SM's 228 KB is L1)
    uint32_t small_mask = 0x3u;   // classes run by k_small (one end per CTA, no walker warp)
    la_params params{};
    DevParams dp{};
    Encoded enc, spare;   // current encoding; la_load_batch fills `spare` and swaps on success
    // scratch (grow-only)
    DevBuf raw_seq, raw_qual, raw_coff, raw_cseq, read_end, errw;
    DevBuf cls, out_len, out_term, out_k, out_att, walk_buf, smem_list, smem_key, smem_list2,
        smem_key2, glob_list, ctrs, ext_off, ext_seq, gstats, cub_tmp;
    DevBuf g_state, g_act, g_act2, g_still, g_cap, g_nrd, g_capoff, g_rdoff, g_slots, g_cnt, g_vis,
        g_cur;
    DevBuf lens64, xl_scratch, prof, out_dir, hist;
    // NEXT N3 co-execution (la_set_coexec): host threads, share of the smallest class's ends, buffers
    int coexec_threads = 0;
    double coexec_share = 0.0;
    DevBuf cx_cnt, cx_roff, cx_rseq, cx_rqc, cx_rlen, cx_tail, cx_tailN, cx_clen, cx_len, cx_term, cx_k, cx_att,
        cx_dir, cx_walk;
    HostBuf hx_roff, hx_rseq, hx_rqc, hx_rlen, hx_tail, hx_tailN, hx_clen, hx_len, hx_term, hx_k, hx_att, hx_dir,
        hx_walk;
    // plan of the last la_extend (la_replay_build reruns its class lists)
    bool extended = false;
    int plan_ncls[N_SMEM_CLASSES] = {0, 0, 0, 0, 0};
    int plan_nxl = 0, plan_xl_umax = 0, plan_xl_rmax = 0, plan_nxlc = 0;
    uint32_t xlc_bytes = 0;   // dynamic shared memory per CTA of the XLC cluster class (0: not planned)
    uint32_t xlc_force_bytes = 0;   // the same for LA_FORCE_CLASS=6
    HostBuf h_ext_off, h_ext_seq, h_term, h_k, h_att, h_small;
    // la_extend_streamed: copy stream, double-buffered raw staging (A/B), chunk-ordering events
    cudaStream_t copy_stream = nullptr;
    DevBuf st_seq[2], st_qual[2], st_cseq[2], st_coff[2], st_roff[2], st_eoff[2];
    cudaEvent_t ev_copied[2] = {}, ev_loaded[2] = {};
    int64_t g_attempts = 0;
    cudaEvent_t ev[6] = {};
    cudaEvent_t ev_rep[2] = {};   // la_replay_build start / end
    cudaEvent_t ev_cls[N_TAB_CLASSES + 1] = {};   // end of class c (5 XL, 6 XLC); [N_TAB_CLASSES] classes may start
    cudaEvent_t ev_cls0[N_TAB_CLASSES] = {};      // start of class c
    // one stream per table class (LA_CONCURRENT_CLASSES=1): the persistent class kernels launched together (largest tables
    // first) so that the tail of one class overlaps the start of the next; LA_SERIAL_CLASSES=1: one stream
    cudaStream_t cls_stream[N_TAB_CLASSES] = {};
    // r02: the class kernels run one after another on the context stream by default.  Measured on C4S,
    // launching them on six streams at once gave the same step time (each persistent class kernel
    // fills the GPU, so only their tails can overlap) while making the per-class times overlapping
    // spans; LA_CONCURRENT_CLASSES=1 restores the concurrent launch.
    bool concurrent_classes = false;
    SelBufs sel;   // NEXT N4
    la_stats stats{};
};

namespace {

la_status fail(la_ctx *c, la_status s, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) {
        c->err = buf;
        if (s == LA_ERR_CUDA) c->sticky = true;
    }
    return s;
}

#define CK(call)                                                                              \
    do {                                                                                      \
        cudaError_t _e = (call);                                                              \
        if (_e != cudaSuccess)                                                                \
            return fail(ctx, _e == cudaErrorMemoryAllocation ? LA_ERR_OOM : LA_ERR_CUDA,      \
                        "%s failed: %s (%s:%d)", #call, cudaGetErrorString(_e), __FILE__,     \
                        __LINE__);                                                            \
    } while (0)

#define CKL()                                                                                 \
    do {                                                                                      \
        ctx->stats.kernel_launches++;                                                         \
        cudaError_t _e = cudaGetLastError();                                                  \
        if (_e != cudaSuccess)                                                                \
            return fail(ctx, LA_ERR_CUDA, "kernel launch failed: %s (%s:%d)",                 \
                        cudaGetErrorString(_e), __FILE__, __LINE__);                          \
    } while (0)

cudaError_t grow(DevBuf &b, size_t bytes) {
    if (bytes <= b.n && b.p) return cudaSuccess;
    b.release();
    size_t n = std::max<size_t>(bytes, 256);
    cudaError_t e = cudaMalloc(&b.p, n);
    if (e == cudaSuccess) b.n = n;
    else b.p = nullptr;
    return e;
}

cudaError_t grow_host(HostBuf &b, size_t bytes) {
    if (bytes <= b.n && b.p) return cudaSuccess;
    b.release();
    size_t n = std::max<size_t>(bytes, 256);
    cudaError_t e = cudaMallocHost(&b.p, n);
    if (e == cudaSuccess) b.n = n;
    else b.p = nullptr;
    return e;
}

template <typename T>
T *P(DevBuf &b) { return (T *)b.p; }

bool valid_params(const la_params &p, std::string &why) {
    char buf[256];
    if (!(p.k_min >= 1 && p.k_min <= p.k_start && p.k_start <= p.k_max && p.k_max <= 128)) {
        snprintf(buf, sizeof buf, "k schedule must satisfy 1 <= k_min <= k_start <= k_max <= 128 (got %d %d %d)",
                 p.k_min, p.k_start, p.k_max);
        why = buf;
        return false;
    }
    if (p.k_shift < 1) { why = "k_shift must be >= 1"; return false; }
    if (p.max_walk_len < 0 || p.max_walk_len > 1024) { why = "max_walk_len must be in 0..1024"; return false; }
    if (p.qual_offset < 0 || p.qual_offset > 127) { why = "qual_offset must be in 0..127"; return false; }
    if (!(p.q_lo >= 0 && p.q_lo <= p.q_hi && p.q_hi <= 93)) { why = "need 0 <= q_lo <= q_hi <= 93"; return false; }
    if (p.min_votes < 1) { why = "min_votes must be >= 1"; return false; }
    if (p.min_frac_pct < 0 || p.min_frac_pct > 100) { why = "min_frac_pct must be in 0..100"; return false; }
    return true;
}

inline unsigned blocks(int64_t n, int b) { return (unsigned)((n + b - 1) / b); }

}  // namespace

// ================================================================================================
extern "C" la_status la_create(la_ctx **out, int device, void *cuda_stream) {
    if (!out) return LA_ERR_INVALID_ARG;
    *out = nullptr;
    la_ctx *ctx = new la_ctx();
    ctx->device = device;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        delete ctx;
        return LA_ERR_CUDA;
    }
    if (device < 0 || device >= ndev) { delete ctx; return LA_ERR_INVALID_ARG; }
    if (cudaSetDevice(device) != cudaSuccess) { delete ctx; return LA_ERR_CUDA; }
    cudaDeviceProp prop;
    cudaGetDeviceProperties(&prop, device);
    ctx->n_sm = prop.multiProcessorCount;
    // tuning hook: LA_CLASSES="64x12,128x6,256x3,512x2,1024x1" (threads x CTAs/SM per class) and
    // LA_SMALL_MASK (bit i: class i runs k_small); a combination without a kernel instantiation
    // (kClassKernels) leaves the defaults in place
    {
        int th[N_SMEM_CLASSES], ct[N_SMEM_CLASSES];
        uint32_t mask = ctx->small_mask;
        for (int i = 0; i < N_SMEM_CLASSES; ++i) {
            th[i] = ctx->cls_threads[i];
            ct[i] = ctx->cls_ctas[i];
        }
        if (const char *cfg = getenv("LA_CLASSES")) {
            int t, c, n = 0;
            const char *q = cfg;
            while (n < N_SMEM_CLASSES && sscanf(q, "%dx%d", &t, &c) == 2) {
                th[n] = t;
                ct[n] = std::max(1, c);
                ++n;
                q = strchr(q, ',');
                if (!q) break;
                ++q;
            }
        }
        if (const char *m = getenv("LA_SMALL_MASK")) mask = (uint32_t)strtoul(m, nullptr, 0);
        bool ok = true;
        for (int i = 0; i < N_SMEM_CLASSES; ++i) ok &= find_class_kernel(th[i], ct[i], (mask >> i) & 1u) != nullptr;
        if (ok) {
            for (int i = 0; i < N_SMEM_CLASSES; ++i) {
                ctx->cls_threads[i] = th[i];
                ctx->cls_ctas[i] = ct[i];
            }
            ctx->small_mask = mask;
        } else {
            fprintf(stderr, "locassm: LA_CLASSES / LA_SMALL_MASK names a class without a kernel; using defaults\n");
        }
    }
    // dynamic smem per CTA: the SM's shared memory split between resident CTAs (1 KB reserved each),
    // minus the largest static shared memory of the class kernels (queried, not assumed)
    size_t stat = 512;
    {
        cudaFuncAttributes fa;
        for (const ClassEntry &k : kClassKernels)
            if (cudaFuncGetAttributes(&fa, k.fn) == cudaSuccess) stat = std::max(stat, fa.sharedSizeBytes);
        if (cudaFuncGetAttributes(&fa, k_smem<XL_THREADS, true>) == cudaSuccess) stat = std::max(stat, fa.sharedSizeBytes);
        if (cudaFuncGetAttributes(&fa, k_xlc) == cudaSuccess) stat = std::max(stat, fa.sharedSizeBytes);
        cudaGetLastError();
        stat = (stat + 127) & ~(size_t)127;
    }
    for (int i = 0; i < N_SMEM_CLASSES; ++i) {
        size_t per = prop.sharedMemPerMultiprocessor / ctx->cls_ctas[i] - 1024 - stat;
        per = std::min(per, (size_t)prop.sharedMemPerBlockOptin - stat);
        ctx->cls_bytes[i] = (uint32_t)(per & ~(size_t)127);
    }
    // XL: tables live in L2; shared memory holds the link words and filter bitmaps, and whatever the
    // class leaves unused becomes L1 for the end's streamed reads (tuning hook LA_XL_SMEM_KB)
    ctx->xl_bytes = ctx->cls_bytes[N_SMEM_CLASSES - 1];
    if (const char *x = getenv("LA_XL_SMEM_KB")) {
        const uint32_t b = (uint32_t)atoi(x) * 1024u;
        if (b >= 96u * 1024u && b < ctx->xl_bytes) ctx->xl_bytes = b;
    }
    if (cuda_stream) ctx->stream = (cudaStream_t)cuda_stream;
    else {
        if (cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking) != cudaSuccess) {
            delete ctx;
            return LA_ERR_CUDA;
        }
        ctx->own_stream = true;
    }
    for (auto &e : ctx->ev) cudaEventCreate(&e);
    for (auto &e : ctx->ev_rep) cudaEventCreate(&e);
    for (auto &e : ctx->ev_cls) cudaEventCreate(&e);
    for (auto &e : ctx->ev_cls0) cudaEventCreate(&e);
    for (auto &q : ctx->cls_stream)
        if (cudaStreamCreateWithFlags(&q, cudaStreamNonBlocking) != cudaSuccess) q = nullptr;
    if (getenv("LA_CONCURRENT_CLASSES") && atoi(getenv("LA_CONCURRENT_CLASSES"))) ctx->concurrent_classes = true;
    if (getenv("LA_SERIAL_CLASSES") && atoi(getenv("LA_SERIAL_CLASSES"))) ctx->concurrent_classes = false;
    bool attr_ok = cudaFuncSetAttribute(k_smem<XL_THREADS, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        ctx->cls_bytes[N_SMEM_CLASSES - 1]) == cudaSuccess;
    {   // XL: ask for the smallest shared-memory carveout that holds xl_bytes (the rest is L1)
        const int pct = (int)std::min<size_t>(100, ((size_t)ctx->xl_bytes + 2048) * 100 / prop.sharedMemPerMultiprocessor + 1);
        attr_ok &= cudaFuncSetAttribute(k_smem<XL_THREADS, true>, cudaFuncAttributePreferredSharedMemoryCarveout,
                                        pct) == cudaSuccess;
    }
    {
        uint32_t mx = 0;
        for (int i = 0; i < N_SMEM_CLASSES; ++i) mx = std::max(mx, ctx->cls_bytes[i]);
        for (const ClassEntry &k : kClassKernels)
            attr_ok &= cudaFuncSetAttribute(k.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, mx) == cudaSuccess;
    }
    // XLC (2-CTA clusters, la_xlc.cuh): opt-in (LA_XLC=1).  Measured on C4S it ran its ends at 21 G
    // inserts/s against the XL class's 36 (step 140.2 vs 130.6 ms), so the planner does not route ends to
    // it by default; LA_FORCE_CLASS=6 (tests) forces it.
    ctx->xlc_bytes = (getenv("LA_XLC") && atoi(getenv("LA_XLC"))) ? ctx->cls_bytes[N_SMEM_CLASSES - 1] : 0u;
    ctx->xlc_force_bytes = ctx->cls_bytes[N_SMEM_CLASSES - 1];
    attr_ok &= cudaFuncSetAttribute(k_xlc, cudaFuncAttributeMaxDynamicSharedMemorySize, ctx->cls_bytes[N_SMEM_CLASSES - 1]) ==
               cudaSuccess;
    if (!attr_ok) {
        cudaGetLastError();
        la_destroy(ctx);
        return LA_ERR_CUDA;
    }
    *out = ctx;
    return LA_OK;
}

extern "C" la_status la_destroy(la_ctx *ctx) {
    if (!ctx) return LA_OK;
    cudaSetDevice(ctx->device);
    if (ctx->stream) cudaStreamSynchronize(ctx->stream);
    ctx->enc.release();
    ctx->spare.release();
    ctx->sel.release();
    for (int i = 0; i < 2; ++i) {
        for (DevBuf *b : {&ctx->st_seq[i], &ctx->st_qual[i], &ctx->st_cseq[i], &ctx->st_coff[i], &ctx->st_roff[i],
                          &ctx->st_eoff[i]})
            b->release();
        if (ctx->ev_copied[i]) cudaEventDestroy(ctx->ev_copied[i]);
        if (ctx->ev_loaded[i]) cudaEventDestroy(ctx->ev_loaded[i]);
    }
    if (ctx->copy_stream) cudaStreamDestroy(ctx->copy_stream);
    for (DevBuf *b : {&ctx->raw_seq, &ctx->raw_qual, &ctx->raw_coff, &ctx->raw_cseq, &ctx->read_end,
                      &ctx->errw, &ctx->cls, &ctx->out_len, &ctx->out_term, &ctx->out_k, &ctx->out_att,
                      &ctx->walk_buf, &ctx->smem_list, &ctx->smem_key, &ctx->smem_list2, &ctx->smem_key2,
                      &ctx->glob_list, &ctx->ctrs, &ctx->ext_off, &ctx->ext_seq, &ctx->gstats,
                      &ctx->cub_tmp, &ctx->g_state, &ctx->g_act, &ctx->g_act2, &ctx->g_still, &ctx->g_cap,
                      &ctx->g_nrd, &ctx->g_capoff, &ctx->g_rdoff, &ctx->g_slots, &ctx->g_cnt, &ctx->g_vis,
                      &ctx->g_cur, &ctx->lens64, &ctx->xl_scratch, &ctx->prof, &ctx->out_dir, &ctx->hist,
                      &ctx->cx_cnt, &ctx->cx_roff, &ctx->cx_rseq, &ctx->cx_rqc, &ctx->cx_rlen, &ctx->cx_tail,
                      &ctx->cx_tailN, &ctx->cx_clen, &ctx->cx_len, &ctx->cx_term, &ctx->cx_k, &ctx->cx_att,
                      &ctx->cx_dir, &ctx->cx_walk})
        b->release();
    for (HostBuf *b : {&ctx->hx_roff, &ctx->hx_rseq, &ctx->hx_rqc, &ctx->hx_rlen, &ctx->hx_tail, &ctx->hx_tailN,
                       &ctx->hx_clen, &ctx->hx_len, &ctx->hx_term, &ctx->hx_k, &ctx->hx_att, &ctx->hx_dir,
                       &ctx->hx_walk})
        b->release();
    for (HostBuf *b : {&ctx->h_ext_off, &ctx->h_ext_seq, &ctx->h_term, &ctx->h_k, &ctx->h_att, &ctx->h_small})
        b->release();
    for (auto &e : ctx->ev)
        if (e) cudaEventDestroy(e);
    for (auto &e : ctx->ev_rep)
        if (e) cudaEventDestroy(e);
    for (auto &q : ctx->cls_stream)
        if (q) {
            cudaStreamSynchronize(q);
            cudaStreamDestroy(q);
        }
    for (auto &e : ctx->ev_cls)
        if (e) cudaEventDestroy(e);
    for (auto &e : ctx->ev_cls0)
        if (e) cudaEventDestroy(e);
    if (ctx->own_stream && ctx->stream) cudaStreamDestroy(ctx->stream);
    delete ctx;
    return LA_OK;
}

extern "C" const char *la_last_error(const la_ctx *ctx) { return ctx ? ctx->err.c_str() : "null context"; }

extern "C" la_status la_get_stats(const la_ctx *ctx, la_stats *out) {
    if (!ctx || !out) return LA_ERR_INVALID_ARG;
    *out = ctx->stats;
    return LA_OK;
}

extern "C" int64_t la_plan_global_capacity(int64_t inserts) { return global_capacity(inserts); }
#ifdef LA_PROBE_STATS
extern "C" int la_debug_probe_stats(unsigned long long *out, int reset) {
    if (cudaMemcpyFromSymbol(out, g_probe_stats, sizeof(unsigned long long) * 12) != cudaSuccess) return -1;
    if (reset) {
        unsigned long long z[12] = {};
        cudaMemcpyToSymbol(g_probe_stats, z, sizeof(z));
    }
    return 0;
}
#endif
extern "C" double la_paper_load_factor(int32_t l, int32_t k) { return (double)(l - k + 1) / (double)l; }

// ================================================================================================
// la_load_batch: copy (if host), validate and encode on the device
// ================================================================================================
namespace {

la_status copy_in(la_ctx *ctx, DevBuf &dst, const void *src, size_t bytes, bool host) {
    CK(grow(dst, bytes + 16));
    if (bytes) CK(cudaMemcpyAsync(dst.p, src, bytes, host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice,
                                  ctx->stream));
    return LA_OK;
}

la_status read_i64(la_ctx *ctx, const int64_t *p, bool host, int64_t *v) {
    if (host) { *v = *p; return LA_OK; }
    CK(cudaMemcpyAsync(v, p, 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return LA_OK;
}

}  // namespace

extern "C" la_status la_load_batch(la_ctx *ctx, const la_batch *b, const la_params *params) {
    if (!ctx) return LA_ERR_INVALID_ARG;
    if (ctx->sticky) return fail(ctx, LA_ERR_CUDA, "context has a sticky CUDA error: %s", ctx->err.c_str());
    if (!b || !params) return fail(ctx, LA_ERR_INVALID_ARG, "null batch or params");
    std::string why;
    if (!valid_params(*params, why)) return fail(ctx, LA_ERR_INVALID_ARG, "%s", why.c_str());
    if (b->mem != LA_MEM_HOST && b->mem != LA_MEM_DEVICE) return fail(ctx, LA_ERR_INVALID_ARG, "bad mem kind");
    if (b->n_contigs < 0 || b->n_reads < 0) return fail(ctx, LA_ERR_INVALID_ARG, "negative sizes");
    if (b->n_reads >= (1ll << 32)) return fail(ctx, LA_ERR_INVALID_ARG, "more than 2^32 reads");
    if (!b->contig_off || !b->read_off || !b->end_read_off)
        return fail(ctx, LA_ERR_INVALID_ARG, "null offsets array");
    cudaSetDevice(ctx->device);
    const bool host = b->mem == LA_MEM_HOST;
    const int64_t nC = b->n_contigs, nE = 2 * nC, nR = b->n_reads;
    int64_t c0, cN, r0, rN, e0, eN;
    la_status s;
    if ((s = read_i64(ctx, b->contig_off, host, &c0)) || (s = read_i64(ctx, b->contig_off + nC, host, &cN)) ||
        (s = read_i64(ctx, b->read_off, host, &r0)) || (s = read_i64(ctx, b->read_off + nR, host, &rN)) ||
        (s = read_i64(ctx, b->end_read_off, host, &e0)) || (s = read_i64(ctx, b->end_read_off + nE, host, &eN)))
        return s;
    if (c0 != 0 || r0 != 0 || e0 != 0) return fail(ctx, LA_ERR_INVALID_ARG, "offsets must start at 0");
    if (cN < 0 || rN < 0) return fail(ctx, LA_ERR_INVALID_ARG, "negative total length");
    if (eN != nR) return fail(ctx, LA_ERR_INVALID_ARG, "end_read_off[2*n_contigs] (%lld) != n_reads (%lld)",
                              (long long)eN, (long long)nR);
    if (rN > (int64_t)nR * MAX_READ_LEN) return fail(ctx, LA_ERR_INVALID_ARG, "reads longer than 300 bases");
    if ((cN && !b->contig_seq) || (rN && (!b->read_seq || !b->read_qual)))
        return fail(ctx, LA_ERR_INVALID_ARG, "null sequence pointer");

    Encoded &E = ctx->spare;   // swapped into ctx->enc only if valid (context unchanged on error)
    E.n_contigs = nC;
    E.n_ends = nE;
    E.n_reads = nR;
    const la_status ok = [&]() -> la_status {
        cudaStream_t st = ctx->stream;
        la_status s2;
        // raw inputs on the device
        const char *d_seq, *d_qual, *d_cseq;
        const int64_t *d_coff;
        CK(grow(E.eoff, (nE + 1) * 8));
        CK(grow(E.roff, (nR + 1) * 8));
        CK(cudaMemcpyAsync(E.eoff.p, b->end_read_off, (nE + 1) * 8,
                           host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(E.roff.p, b->read_off, (nR + 1) * 8,
                           host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice, st));
        if (host) {
            if ((s2 = copy_in(ctx, ctx->raw_seq, b->read_seq, rN, true))) return s2;
            if ((s2 = copy_in(ctx, ctx->raw_qual, b->read_qual, rN, true))) return s2;
            if ((s2 = copy_in(ctx, ctx->raw_cseq, b->contig_seq, cN, true))) return s2;
            if ((s2 = copy_in(ctx, ctx->raw_coff, b->contig_off, (nC + 1) * 8, true))) return s2;
            d_seq = P<char>(ctx->raw_seq);
            d_qual = P<char>(ctx->raw_qual);
            d_cseq = P<char>(ctx->raw_cseq);
            d_coff = P<int64_t>(ctx->raw_coff);
        } else {
            d_seq = b->read_seq;
            d_qual = b->read_qual;
            d_cseq = b->contig_seq;
            d_coff = b->contig_off;
        }
        // offsets + max read length
        CK(grow(ctx->errw, 64));
        uint32_t *d_err = P<uint32_t>(ctx->errw);
        int *d_maxlen = (int *)(d_err + 1);
        CK(cudaMemsetAsync(d_err, 0, 8, st));
        if (nC) { k_check_offsets<<<blocks(nC, 256), 256, 0, st>>>(d_coff, nC, 0, d_err, nullptr); CKL(); }
        if (nE) { k_check_offsets<<<blocks(nE, 256), 256, 0, st>>>(P<int64_t>(E.eoff), nE, 0, d_err, nullptr); CKL(); }
        if (nR) { k_check_offsets<<<blocks(nR, 256), 256, 0, st>>>(P<int64_t>(E.roff), nR, 1, d_err, d_maxlen); CKL(); }
        uint32_t hv[2] = {0, 0};
        CK(cudaMemcpyAsync(hv, d_err, 8, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        if (hv[0] & ERR_OFFSETS) return fail(ctx, LA_ERR_INVALID_ARG, "offsets are not non-decreasing");
        if (hv[0] & ERR_READ_LEN) return fail(ctx, LA_ERR_INVALID_ARG, "a read is longer than 300 bases");
        const int maxlen = (int)hv[1];
        int SW = (maxlen + 31) / 32 + 2;
        SW = (SW + 1) & ~1;   // even: 16 B aligned rows
        E.SW = SW;
        E.maxlen = maxlen;
        // encode reads
        CK(grow(ctx->read_end, std::max<int64_t>(nR, 1) * 4));
        CK(grow(E.rseq, std::max<int64_t>(nR, 1) * SW * 8));
        CK(grow(E.rqc, std::max<int64_t>(nR, 1) * SW * 8));
        CK(grow(E.rlen, std::max<int64_t>(nR, 1) * 2 + 16));
        CK(grow(E.rflag, std::max<int64_t>(nR, 1) + 16));
        CK(grow(E.tail, std::max<int64_t>(nE, 1) * TAIL_W * 8));
        CK(grow(E.tailN, std::max<int64_t>(nE, 1) * 16));
        CK(grow(E.clen, std::max<int64_t>(nE, 1) * 4));
        DevParams dp{params->k_start, params->k_min, params->k_max, params->k_shift, params->max_walk_len,
                     params->qual_offset, params->q_lo, params->q_hi, params->min_votes, params->min_frac_pct, 0,
                     maxlen};
        if (nR) {
            CK(cudaMemsetAsync(E.rflag.p, 0, nR, st));
            k_read_end<<<blocks(nR, 256), 256, 0, st>>>(P<int64_t>(E.eoff), nE, nR, P<int32_t>(ctx->read_end));
            CKL();
            k_encode_reads_staged<<<blocks(nR, ENC_R), 256, 0, st>>>(
                d_seq, d_qual, P<int64_t>(E.roff), P<int32_t>(ctx->read_end), nR, SW, dp, P<uint64_t>(E.rseq),
                P<uint64_t>(E.rqc), P<uint16_t>(E.rlen), P<uint8_t>(E.rflag), d_err);
            CKL();
        }
        if (cN) { k_check_contigs<<<blocks(cN, 256), 256, 0, st>>>(d_cseq, cN, d_err); CKL(); }
        if (nE) {
            k_encode_tails<<<blocks(nE, 128), 128, 0, st>>>(d_cseq, d_coff, nE, P<uint64_t>(E.tail),
                                                            P<uint64_t>(E.tailN), P<int32_t>(E.clen));
            CKL();
        }
        CK(cudaMemcpyAsync(hv, d_err, 4, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        if (hv[0] & ERR_READ_CHAR) return fail(ctx, LA_ERR_INVALID_ARG, "read base outside ACGTN");
        if (hv[0] & ERR_QUAL_CHAR) return fail(ctx, LA_ERR_INVALID_ARG, "quality character below qual_offset");
        if (hv[0] & ERR_CONTIG_CHAR) return fail(ctx, LA_ERR_INVALID_ARG, "contig base outside ACGTN");
        ctx->dp = dp;
        return LA_OK;
    }();
    if (ok != LA_OK) return ok;
    std::swap(ctx->enc, ctx->spare);
    ctx->params = *params;
    ctx->loaded = true;
    ctx->extended = false;
    return LA_OK;
}

// ================================================================================================
// la_extend
// ================================================================================================
namespace {

la_status run_global(la_ctx *ctx, const int32_t *d_list, int n_list, double *ms_unused) {
    (void)ms_unused;
    cudaStream_t st = ctx->stream;
    Encoded &E = ctx->enc;
    const DevParams &dp = ctx->dp;
    if (n_list == 0) return LA_OK;
    CK(grow(ctx->g_state, (size_t)n_list * sizeof(GState)));
    CK(grow(ctx->g_act, (size_t)n_list * 4));
    CK(grow(ctx->g_act2, (size_t)n_list * 4));
    CK(grow(ctx->g_still, (size_t)n_list * 4));
    CK(grow(ctx->g_cap, (size_t)(n_list + 1) * 8));
    CK(grow(ctx->g_nrd, (size_t)(n_list + 1) * 8));
    CK(grow(ctx->g_capoff, (size_t)(n_list + 1) * 8));
    CK(grow(ctx->g_rdoff, (size_t)(n_list + 1) * 8));
    CK(grow(ctx->g_cur, (size_t)n_list * std::max(dp.W, 1)));
    GState *gs = P<GState>(ctx->g_state);
    k_g_init<<<blocks(n_list, 256), 256, 0, st>>>(d_list, n_list, P<int32_t>(E.clen), dp, gs, P<int32_t>(ctx->g_act));
    CKL();
    int *d_ctr = P<int>(ctx->ctrs) + 8;
    unsigned long long *d_gst = P<unsigned long long>(ctx->gstats);
    int n_act = n_list;
    const int nseg = std::max(1, (E.maxlen - dp.k_min + GSEG - 1) / GSEG);   // positions per read
    int64_t *h = (int64_t *)ctx->h_small.p;
    // memory budget of one wave of global tables (slots: 8 B key + 32 B counters + 1 visited bit)
    const int64_t budget = (getenv("LA_GLOBAL_BUDGET_MB") ? atoll(getenv("LA_GLOBAL_BUDGET_MB")) : 8192) << 20;
    std::vector<int64_t> hcap, hnrd, capoff, rdoff;
    while (n_act > 0) {
        ctx->stats.global_rounds++;
        int32_t *act = P<int32_t>(ctx->g_act);
        k_g_caps<<<n_act, 256, 0, st>>>(act, n_act, d_list, gs, P<int64_t>(E.eoff), P<uint16_t>(E.rlen),
                                        P<int64_t>(ctx->g_cap), P<int64_t>(ctx->g_nrd));
        CKL();
        hcap.resize(n_act);
        hnrd.resize(n_act);
        CK(cudaMemcpyAsync(hcap.data(), ctx->g_cap.p, (size_t)n_act * 8, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(hnrd.data(), ctx->g_nrd.p, (size_t)n_act * 8, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        // waves of consecutive active ends whose tables fit the budget
        for (int a = 0; a < n_act;) {
            int b = a;
            int64_t tot = 0, nrd = 0;
            capoff.assign(1, 0);
            rdoff.assign(1, 0);
            while (b < n_act && (b == a || (tot + hcap[b]) * 41 <= budget)) {
                if (hcap[b] >= (int64_t)NONE)
                    return fail(ctx, LA_ERR_CAPACITY, "global table of one end too large (%lld slots)", (long long)hcap[b]);
                tot += hcap[b];
                nrd += hnrd[b];
                capoff.push_back(tot);
                rdoff.push_back(nrd);
                ++b;
            }
            const int n = b - a;
            CK(cudaMemcpyAsync(ctx->g_capoff.p, capoff.data(), (size_t)(n + 1) * 8, cudaMemcpyHostToDevice, st));
            CK(cudaMemcpyAsync(ctx->g_rdoff.p, rdoff.data(), (size_t)(n + 1) * 8, cudaMemcpyHostToDevice, st));
            CK(grow(ctx->g_slots, (size_t)tot * 8));
            CK(grow(ctx->g_cnt, (size_t)tot * 32));
            const size_t visw = (size_t)(tot >> 5) + n + 2;
            CK(grow(ctx->g_vis, visw * 4));
            CK(cudaMemsetAsync(ctx->g_slots.p, 0, (size_t)tot * 8, st));
            CK(cudaMemsetAsync(ctx->g_cnt.p, 0, (size_t)tot * 32, st));
            CK(cudaMemsetAsync(ctx->g_vis.p, 0, visw * 4, st));
            if (nrd > 0) {
                k_g_build<<<blocks(nrd * nseg, 256), 256, 0, st>>>(
                    act + a, n, d_list, gs, P<int64_t>(E.eoff), P<int64_t>(ctx->g_rdoff), P<int64_t>(ctx->g_capoff),
                    nseg, P<uint64_t>(E.rseq), P<uint64_t>(E.rqc), P<uint16_t>(E.rlen), P<uint8_t>(E.rflag), E.SW,
                    P<uint64_t>(ctx->g_slots), P<uint32_t>(ctx->g_cnt), d_gst + 3);
                CKL();
            }
            if (tot > 0) {
                k_g_graph<<<blocks(tot, 256), 256, 0, st>>>(act + a, n, d_list, gs, P<int64_t>(ctx->g_capoff),
                                                            P<uint64_t>(E.rseq), E.SW, dp, P<uint64_t>(ctx->g_slots),
                                                            P<uint32_t>(ctx->g_cnt));
                CKL();
            }
            k_g_walk<<<blocks(n, 64), 64, 0, st>>>(
                act + a, n, d_list, gs, P<int64_t>(ctx->g_capoff), P<uint64_t>(E.rseq), E.SW, P<uint64_t>(E.tail),
                P<uint64_t>(E.tailN), P<int32_t>(E.clen), dp, P<uint64_t>(ctx->g_slots), P<uint32_t>(ctx->g_cnt),
                P<uint32_t>(ctx->g_vis), P<uint8_t>(ctx->g_cur), P<uint8_t>(ctx->walk_buf), P<int32_t>(ctx->out_len),
                P<uint8_t>(ctx->out_term), P<uint8_t>(ctx->out_k), P<uint8_t>(ctx->out_att),
                P<int32_t>(ctx->g_still) + a, d_gst + 4);
            CKL();
            a = b;
        }
        CK(cudaMemsetAsync(d_ctr, 0, 4, st));
        k_g_compact<<<blocks(n_act, 256), 256, 0, st>>>(act, n_act, P<int32_t>(ctx->g_still), P<int32_t>(ctx->g_act2), d_ctr);
        CKL();
        CK(cudaMemcpyAsync(h, d_ctr, 4, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        ctx->g_attempts += n_act;
        n_act = *(int *)h;
        std::swap(ctx->g_act, ctx->g_act2);
    }
    return LA_OK;
}

// The table-class kernels over the plan's class lists (XL + the five shared-memory classes), on
// one stream per class (LA_SERIAL_CLASSES=1: all on the context stream), joined back into the
// context stream.  replay = true: la_replay_build's build-only pass over the same lists.
la_status launch_classes(la_ctx *ctx, bool replay) {
    cudaStream_t st = ctx->stream;
    Encoded &E = ctx->enc;
    DevParams dp = ctx->dp;
    dp.replay = replay ? 1 : 0;
    const int64_t nE = E.n_ends;
    int *d_ctr = P<int>(ctx->ctrs);
    unsigned long long *d_gst = P<unsigned long long>(ctx->gstats);
    int32_t *lists = P<int32_t>(ctx->smem_list);
    int32_t *ovf_list = P<int32_t>(ctx->glob_list) + nE;
    const int n_xl = ctx->plan_nxl;
    // LA_PROFILE=1: per-class phase cycle counters (clock64) of the shared-memory kernels
    unsigned long long *prof = nullptr;
    if (!replay && getenv("LA_PROFILE") && atoi(getenv("LA_PROFILE"))) {
        CK(grow(ctx->prof, 8 * 8 * N_TAB_CLASSES));
        prof = P<unsigned long long>(ctx->prof);
        CK(cudaMemsetAsync(prof, 0, 8 * 8 * N_TAB_CLASSES, st));
    }
    CK(cudaEventRecord(ctx->ev_cls[N_TAB_CLASSES], st));
    auto cls_st = [&](int c) -> cudaStream_t {
        return (ctx->concurrent_classes && ctx->cls_stream[c]) ? ctx->cls_stream[c] : st;
    };
    for (int c = 0; c < N_TAB_CLASSES; ++c)
        if (cls_st(c) != st) CK(cudaStreamWaitEvent(cls_st(c), ctx->ev_cls[N_TAB_CLASSES], 0));
    // XLC (2-CTA clusters, tables in the pair's shared memory) first
    CK(cudaEventRecord(ctx->ev_cls0[C_XLC], cls_st(C_XLC)));
    if (ctx->plan_nxlc > 0) {
        const int clusters = (int)std::min<int64_t>((int64_t)ctx->n_sm / 2, ctx->plan_nxlc);
        k_xlc<<<2 * clusters, XLC_THREADS, ctx->xlc_force_bytes, cls_st(C_XLC)>>>(
            lists + (size_t)C_XLC * nE, ctx->plan_nxlc, d_ctr + 22, P<uint64_t>(E.rseq), P<uint64_t>(E.rqc),
            P<uint16_t>(E.rlen), P<uint8_t>(E.rflag), P<int64_t>(E.eoff), P<uint64_t>(E.tail), P<uint64_t>(E.tailN),
            P<int32_t>(E.clen), E.SW, dp, ctx->xlc_force_bytes, P<uint8_t>(ctx->walk_buf), P<int32_t>(ctx->out_len),
            P<uint8_t>(ctx->out_term), P<uint8_t>(ctx->out_k), P<uint8_t>(ctx->out_att), P<int8_t>(ctx->out_dir),
            ovf_list, d_ctr + 15, (GlobalStats *)(d_gst + 8 + GSTATS_WORDS * C_XLC));
        CKL();
    }
    CK(cudaEventRecord(ctx->ev_cls[C_XLC], cls_st(C_XLC)));
    // XL (global-scratch tables) first, then the shared-memory classes from the largest tables
    // (1 CTA/SM, all shared memory) to the smallest (12 CTAs/SM)
    CK(cudaEventRecord(ctx->ev_cls0[N_SMEM_CLASSES], cls_st(N_SMEM_CLASSES)));
    if (n_xl > 0) {
        cudaStream_t sx = cls_st(N_SMEM_CLASSES);
        const uint32_t bytes = ctx->xl_bytes;
        const uint32_t icap = smem_fixed(dp.W, bytes, 1u, false, XL_THREADS / 32 - 1).icap;
        const uint32_t stride = xl_stride(ctx->plan_xl_rmax, ctx->plan_xl_umax, dp.V >= 2, icap);
        const int grid = (int)std::min<int64_t>((int64_t)ctx->n_sm, n_xl);
        CK(grow(ctx->xl_scratch, (size_t)grid * stride));
        int32_t *lst = lists + (size_t)N_SMEM_CLASSES * nE;
        k_smem<XL_THREADS, true><<<grid, XL_THREADS, bytes, sx>>>(
            lst, n_xl, d_ctr + 21, P<uint64_t>(E.rseq), P<uint64_t>(E.rqc), P<uint16_t>(E.rlen), P<uint8_t>(E.rflag),
            P<int64_t>(E.eoff), P<uint64_t>(E.tail), P<uint64_t>(E.tailN), P<int32_t>(E.clen), E.SW, dp, bytes,
            P<uint8_t>(ctx->walk_buf), P<int32_t>(ctx->out_len), P<uint8_t>(ctx->out_term), P<uint8_t>(ctx->out_k),
            P<uint8_t>(ctx->out_att), P<int8_t>(ctx->out_dir), ovf_list, d_ctr + 15,
            (GlobalStats *)(d_gst + 8 + GSTATS_WORDS * N_SMEM_CLASSES), P<unsigned char>(ctx->xl_scratch), stride,
            prof ? prof + 8 * N_SMEM_CLASSES : nullptr);
        CKL();
        ctx->stats.ends_xl = n_xl;
        ctx->stats.xl_scratch_bytes = (int64_t)grid * stride;
    }
    CK(cudaEventRecord(ctx->ev_cls[N_SMEM_CLASSES], cls_st(N_SMEM_CLASSES)));   // end of XL
    for (int c = N_SMEM_CLASSES - 1; c >= 0; --c) {
        const int n = ctx->plan_ncls[c];
        CK(cudaEventRecord(ctx->ev_cls0[c], cls_st(c)));
        if (n > 0) {
            cudaStream_t sc = cls_st(c);
            const int grid = (int)std::min<int64_t>((int64_t)ctx->n_sm * ctx->cls_ctas[c], n);
            const uint32_t bytes = ctx->cls_bytes[c];
            int32_t *lst = lists + (size_t)c * nE;
            int *wc = d_ctr + 16 + c;
            const ClassEntry *ke = find_class_kernel(ctx->cls_threads[c], ctx->cls_ctas[c], (ctx->small_mask >> c) & 1u);
            if (!ke) return fail(ctx, LA_ERR_STATE, "no kernel instantiation for table class %d", c);
            ke->fn<<<grid, ke->threads, bytes, sc>>>(lst, n, wc, P<uint64_t>(E.rseq), P<uint64_t>(E.rqc),
                P<uint16_t>(E.rlen), P<uint8_t>(E.rflag), P<int64_t>(E.eoff), P<uint64_t>(E.tail), P<uint64_t>(E.tailN),
                P<int32_t>(E.clen), E.SW, dp, bytes, P<uint8_t>(ctx->walk_buf), P<int32_t>(ctx->out_len),
                P<uint8_t>(ctx->out_term), P<uint8_t>(ctx->out_k), P<uint8_t>(ctx->out_att), P<int8_t>(ctx->out_dir),
                ovf_list, d_ctr + 15, (GlobalStats *)(d_gst + 8 + GSTATS_WORDS * c), nullptr, 0u,
                prof ? prof + 8 * c : nullptr);
            CKL();
        }
        CK(cudaEventRecord(ctx->ev_cls[c], cls_st(c)));   // end of class c
    }
    for (int c = 0; c < N_TAB_CLASSES; ++c)   // join
        if (cls_st(c) != st) CK(cudaStreamWaitEvent(st, ctx->ev_cls[c], 0));
    return LA_OK;
}

// ---- NEXT N3: CPU+GPU co-execution (la_set_coexec) ---------------------------------------------
// The lightest ends of the smallest table class (the tail of its LPT-sorted list) are gathered on the
// device into compact arrays, copied to pinned host memory and extended by la_cpu::extend on host
// threads while the GPU's class kernels run; their results are copied back and scattered into the
// device result arrays, so the device compaction emits every end the same way.
struct Coexec {
    int m = 0;                 // ends given to the host
    const int32_t *list = nullptr;   // their ids (device, the class list's tail)
    int64_t reads = 0;
};

la_status coexec_gather(la_ctx *ctx, int32_t *d_list, int m, Coexec &cx) {
    cudaStream_t st = ctx->stream;
    Encoded &E = ctx->enc;
    const int SW = E.SW;
    cx.m = m;
    cx.list = d_list;
    CK(grow(ctx->cx_cnt, (size_t)(m + 1) * 8));
    CK(grow(ctx->cx_roff, (size_t)(m + 1) * 8));
    k_cx_counts<<<blocks(m + 1, 256), 256, 0, st>>>(d_list, m, P<int64_t>(E.eoff), P<int64_t>(ctx->cx_cnt));
    CKL();
    size_t tb = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, tb, P<int64_t>(ctx->cx_cnt), P<int64_t>(ctx->cx_roff), m + 1, st);
    CK(grow(ctx->cub_tmp, tb));
    cub::DeviceScan::ExclusiveSum(ctx->cub_tmp.p, tb, P<int64_t>(ctx->cx_cnt), P<int64_t>(ctx->cx_roff), m + 1, st);
    CKL();
    CK(grow_host(ctx->hx_roff, (size_t)(m + 1) * 8));
    CK(cudaMemcpyAsync(ctx->hx_roff.p, ctx->cx_roff.p, (size_t)(m + 1) * 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const int64_t R = ((int64_t *)ctx->hx_roff.p)[m];
    cx.reads = R;
    CK(grow(ctx->cx_rseq, (size_t)std::max<int64_t>(R, 1) * SW * 8));
    CK(grow(ctx->cx_rqc, (size_t)std::max<int64_t>(R, 1) * SW * 8));
    CK(grow(ctx->cx_rlen, (size_t)std::max<int64_t>(R, 1) * 2));
    CK(grow(ctx->cx_tail, (size_t)m * TAIL_W * 8));
    CK(grow(ctx->cx_tailN, (size_t)m * 16));
    CK(grow(ctx->cx_clen, (size_t)m * 4));
    k_cx_gather<<<blocks((int64_t)m * 32, 256), 256, 0, st>>>(
        d_list, m, P<int64_t>(E.eoff), P<int64_t>(ctx->cx_roff), SW, P<uint64_t>(E.rseq), P<uint64_t>(E.rqc),
        P<uint16_t>(E.rlen), P<uint64_t>(E.tail), P<uint64_t>(E.tailN), P<int32_t>(E.clen), P<uint64_t>(ctx->cx_rseq),
        P<uint64_t>(ctx->cx_rqc), P<uint16_t>(ctx->cx_rlen), P<uint64_t>(ctx->cx_tail), P<uint64_t>(ctx->cx_tailN),
        P<int32_t>(ctx->cx_clen));
    CKL();
    CK(grow_host(ctx->hx_rseq, (size_t)std::max<int64_t>(R, 1) * SW * 8));
    CK(grow_host(ctx->hx_rqc, (size_t)std::max<int64_t>(R, 1) * SW * 8));
    CK(grow_host(ctx->hx_rlen, (size_t)std::max<int64_t>(R, 1) * 2));
    CK(grow_host(ctx->hx_tail, (size_t)m * TAIL_W * 8));
    CK(grow_host(ctx->hx_tailN, (size_t)m * 16));
    CK(grow_host(ctx->hx_clen, (size_t)m * 4));
    if (R) {
        CK(cudaMemcpyAsync(ctx->hx_rseq.p, ctx->cx_rseq.p, (size_t)R * SW * 8, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(ctx->hx_rqc.p, ctx->cx_rqc.p, (size_t)R * SW * 8, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(ctx->hx_rlen.p, ctx->cx_rlen.p, (size_t)R * 2, cudaMemcpyDeviceToHost, st));
    }
    CK(cudaMemcpyAsync(ctx->hx_tail.p, ctx->cx_tail.p, (size_t)m * TAIL_W * 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(ctx->hx_tailN.p, ctx->cx_tailN.p, (size_t)m * 16, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(ctx->hx_clen.p, ctx->cx_clen.p, (size_t)m * 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    return LA_OK;
}

// host extension of the gathered ends (runs while the class kernels execute), then results -> device
la_status coexec_finish(la_ctx *ctx, const Coexec &cx) {
    cudaStream_t st = ctx->stream;
    const DevParams &dp = ctx->dp;
    const int m = cx.m, W = std::max(dp.W, 1);
    CK(grow_host(ctx->hx_len, (size_t)m * 4));
    CK(grow_host(ctx->hx_term, (size_t)m));
    CK(grow_host(ctx->hx_k, (size_t)m));
    CK(grow_host(ctx->hx_att, (size_t)m));
    CK(grow_host(ctx->hx_dir, (size_t)m));
    CK(grow_host(ctx->hx_walk, (size_t)m * W));
    la_cpu::Input in{m, ctx->enc.SW, (const int64_t *)ctx->hx_roff.p, (const uint64_t *)ctx->hx_rseq.p,
                     (const uint64_t *)ctx->hx_rqc.p, (const uint16_t *)ctx->hx_rlen.p,
                     (const uint64_t *)ctx->hx_tail.p, (const uint64_t *)ctx->hx_tailN.p,
                     (const int32_t *)ctx->hx_clen.p};
    la_cpu::Output out{(int32_t *)ctx->hx_len.p, (uint8_t *)ctx->hx_walk.p, (uint8_t *)ctx->hx_term.p,
                       (uint8_t *)ctx->hx_k.p, (uint8_t *)ctx->hx_att.p, (int8_t *)ctx->hx_dir.p, 0, 0, 0};
    la_cpu::Params cp{dp.k_start, dp.k_min, dp.k_max, dp.k_shift, dp.W, dp.V, dp.F};
    la_cpu::extend(in, cp, ctx->coexec_threads, out);
    ctx->stats.cpu_ends = m;
    ctx->stats.cpu_inserts = out.inserts;
    ctx->stats.cpu_walk_steps = out.walk_steps;
    ctx->stats.cpu_attempts = out.attempts;
    CK(grow(ctx->cx_len, (size_t)m * 4));
    CK(grow(ctx->cx_term, (size_t)m));
    CK(grow(ctx->cx_k, (size_t)m));
    CK(grow(ctx->cx_att, (size_t)m));
    CK(grow(ctx->cx_dir, (size_t)m));
    CK(grow(ctx->cx_walk, (size_t)m * W));
    CK(cudaMemcpyAsync(ctx->cx_len.p, ctx->hx_len.p, (size_t)m * 4, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(ctx->cx_term.p, ctx->hx_term.p, (size_t)m, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(ctx->cx_k.p, ctx->hx_k.p, (size_t)m, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(ctx->cx_att.p, ctx->hx_att.p, (size_t)m, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(ctx->cx_dir.p, ctx->hx_dir.p, (size_t)m, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(ctx->cx_walk.p, ctx->hx_walk.p, (size_t)m * W, cudaMemcpyHostToDevice, st));
    k_cx_scatter<<<blocks((int64_t)m * 32, 256), 256, 0, st>>>(
        cx.list, m, W, P<int32_t>(ctx->cx_len), P<uint8_t>(ctx->cx_term), P<uint8_t>(ctx->cx_k),
        P<uint8_t>(ctx->cx_att), P<int8_t>(ctx->cx_dir), P<uint8_t>(ctx->cx_walk), P<int32_t>(ctx->out_len),
        P<uint8_t>(ctx->out_term), P<uint8_t>(ctx->out_k), P<uint8_t>(ctx->out_att), P<int8_t>(ctx->out_dir),
        P<uint8_t>(ctx->walk_buf));
    CKL();
    return LA_OK;
}

la_status extend_impl(la_ctx *ctx, la_result *out, bool to_host) {
    if (!ctx || !out) return LA_ERR_INVALID_ARG;
    if (ctx->sticky) return fail(ctx, LA_ERR_CUDA, "context has a sticky CUDA error: %s", ctx->err.c_str());
    if (!ctx->loaded) return fail(ctx, LA_ERR_STATE, "la_extend before a successful la_load_batch");
    cudaSetDevice(ctx->device);
    cudaStream_t st = ctx->stream;
    Encoded &E = ctx->enc;
    const DevParams &dp = ctx->dp;
    const int64_t nE = E.n_ends;
    const int W = std::max(dp.W, 1);
    ctx->stats = la_stats{};
    ctx->g_attempts = 0;
    ctx->stats.smem_bytes_per_cta = ctx->cls_bytes[0];
    ctx->stats.smem_ctas_per_sm = ctx->cls_ctas[0];

    CK(grow(ctx->cls, std::max<int64_t>(nE, 1) * 4));
    CK(grow(ctx->out_len, std::max<int64_t>(nE, 1) * 4));
    CK(grow(ctx->out_term, std::max<int64_t>(nE, 1)));
    CK(grow(ctx->out_k, std::max<int64_t>(nE, 1)));
    CK(grow(ctx->out_att, std::max<int64_t>(nE, 1)));
    CK(grow(ctx->walk_buf, std::max<int64_t>(nE, 1) * W));
    CK(grow(ctx->smem_list, std::max<int64_t>(nE, 1) * 4 * N_TAB_CLASSES));
    CK(grow(ctx->smem_key, std::max<int64_t>(nE, 1) * 4 * N_TAB_CLASSES));
    CK(grow(ctx->smem_list2, std::max<int64_t>(nE, 1) * 4));
    CK(grow(ctx->smem_key2, std::max<int64_t>(nE, 1) * 4));
    CK(grow(ctx->glob_list, std::max<int64_t>(nE, 1) * 4 * 2));
    CK(grow(ctx->ctrs, 256));
    CK(grow(ctx->gstats, 512));
    CK(grow(ctx->out_dir, std::max<int64_t>(nE, 1)));
    CK(grow(ctx->hist, 8 * LA_HIST));
    CK(grow(ctx->ext_off, (nE + 1) * 8));
    CK(grow_host(ctx->h_small, 1024));
    int *d_ctr = P<int>(ctx->ctrs);   // [0..4] n per class [5] n_G [6] NOREADS [7] SHORT [15] n_ovf [16..20] work
    unsigned long long *d_gst = P<unsigned long long>(ctx->gstats);

    CK(cudaEventRecord(ctx->ev[0], st));
    CK(cudaMemsetAsync(d_ctr, 0, 128, st));
    CK(cudaMemsetAsync(d_gst, 0, 512, st));
    int *h = (int *)ctx->h_small.p;
    int ncls[N_SMEM_CLASSES] = {0, 0, 0, 0, 0};
    int n_glob = 0, n_xl = 0, xl_umax = 0, xl_rmax = 0, n_xlc = 0;
    int32_t *lists = P<int32_t>(ctx->smem_list);
    uint32_t *keys = P<uint32_t>(ctx->smem_key);
    if (nE) {
        // test hook: force every end with reads onto the global path
        const bool force_global = getenv("LA_FORCE_GLOBAL") && atoi(getenv("LA_FORCE_GLOBAL")) != 0;
        // test hook: pretend every end fits the small-table kernel (exercises the overflow redo)
        const bool force_smem = getenv("LA_FORCE_SMEM") && atoi(getenv("LA_FORCE_SMEM")) != 0;
        PlanBytes pb;
        for (int i = 0; i < N_SMEM_CLASSES; ++i) {
            pb.b[i] = force_global ? 0u : ctx->cls_bytes[i];
            pb.t[i] = (uint32_t)ctx->cls_threads[i];
        }
        pb.single = ctx->small_mask;
        if (force_smem) pb.b[0] = 0xffffffffu;
        // test hook: every end with reads into table class LA_FORCE_CLASS (0..4 shared memory, 5 = XL)
        const int force_cls = getenv("LA_FORCE_CLASS") ? std::min(std::max(atoi(getenv("LA_FORCE_CLASS")), 0), 6) : -1;
        const uint32_t xlc_b = force_cls == C_XLC ? ctx->xlc_force_bytes : ctx->xlc_bytes;
        k_plan<<<blocks(nE, 256), 256, 0, st>>>(
            P<int64_t>(E.eoff), P<int64_t>(E.roff), P<uint8_t>(E.rflag), P<int32_t>(E.clen), nE, dp, E.SW, pb,
            (force_global || force_smem) ? 0u : ctx->xl_bytes, (force_global || force_smem) ? 0u : xlc_b,
            force_global ? -1 : force_cls, P<int32_t>(ctx->cls),
            P<int32_t>(ctx->out_len), P<uint8_t>(ctx->out_term), P<uint8_t>(ctx->out_k), P<uint8_t>(ctx->out_att),
            lists, keys, P<int32_t>(ctx->glob_list), d_ctr);
        CKL();
        CK(cudaMemcpyAsync(h, d_ctr, 4 * 12, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        for (int i = 0; i < N_SMEM_CLASSES; ++i) ncls[i] = h[i];
        n_glob = h[N_SMEM_CLASSES];
        ctx->stats.ends_by_class[0] = h[N_SMEM_CLASSES + 1];
        ctx->stats.ends_by_class[1] = h[N_SMEM_CLASSES + 2];
        n_xl = h[8];
        xl_umax = h[9];
        xl_rmax = h[10];
        n_xlc = h[11];
    }
    // LPT order for the persistent kernels: largest expected work first
    for (int c = 0; c < N_TAB_CLASSES; ++c) {
        const int n = c == N_SMEM_CLASSES ? n_xl : (c == C_XLC ? n_xlc : ncls[c]);
        if (n < 2) continue;
        int32_t *lst = lists + (size_t)c * nE;
        uint32_t *key = keys + (size_t)c * nE;
        size_t tb = 0;
        cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, key, P<uint32_t>(ctx->smem_key2), lst,
                                                  P<int32_t>(ctx->smem_list2), n, 0, 32, st);
        CK(grow(ctx->cub_tmp, tb));
        cub::DeviceRadixSort::SortPairsDescending(ctx->cub_tmp.p, tb, key, P<uint32_t>(ctx->smem_key2), lst,
                                                  P<int32_t>(ctx->smem_list2), n, 0, 32, st);
        CKL();
        CK(cudaMemcpyAsync(lst, ctx->smem_list2.p, (size_t)n * 4, cudaMemcpyDeviceToDevice, st));
    }
    // NEXT N3: the lightest ends of the smallest class (its list's tail) go to the host threads
    Coexec cx;
    if (ctx->coexec_threads > 0 && ctx->coexec_share > 0.0 && ncls[0] > 0) {
        const int m = (int)std::min<double>(ncls[0], std::floor(ctx->coexec_share * ncls[0] + 0.5));
        if (m > 0) {
            ncls[0] -= m;
            const la_status s0 = coexec_gather(ctx, lists + ncls[0], m, cx);
            if (s0 != LA_OK) return s0;
        }
    }
    CK(cudaEventRecord(ctx->ev[1], st));
    ctx->plan_nxl = n_xl;
    ctx->plan_xl_umax = xl_umax;
    ctx->plan_xl_rmax = xl_rmax;
    ctx->plan_nxlc = n_xlc;
    for (int c = 0; c < N_SMEM_CLASSES; ++c) ctx->plan_ncls[c] = ncls[c];
    int32_t *ovf_list = P<int32_t>(ctx->glob_list) + nE;
    {
        const la_status s0 = launch_classes(ctx, false);
        if (s0 != LA_OK) return s0;
    }
    if (cx.m) {   // the host's share, while the class kernels run
        const la_status s0 = coexec_finish(ctx, cx);
        if (s0 != LA_OK) return s0;
    }
    int n_ovf = 0;
    int n_smem = n_xl + n_xlc;
    for (int c = 0; c < N_SMEM_CLASSES; ++c) n_smem += ncls[c];
    if (n_smem > 0) {
        CK(cudaMemcpyAsync(h, d_ctr + 15, 4, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        n_ovf = h[0];
        if (n_ovf)   // append the overflowed ends to the global list
            CK(cudaMemcpyAsync(P<int32_t>(ctx->glob_list) + n_glob, ovf_list, (size_t)n_ovf * 4,
                               cudaMemcpyDeviceToDevice, st));
    }
    CK(cudaEventRecord(ctx->ev[2], st));
    la_status s = run_global(ctx, P<int32_t>(ctx->glob_list), n_glob + n_ovf, nullptr);
    if (s != LA_OK) return s;
    CK(cudaEventRecord(ctx->ev[3], st));
    // emit: exclusive scan of lengths -> ext_off; compact + reverse-complement LEFT ends
    {
        CK(grow(ctx->lens64, (nE + 1) * 8));
        k_len64<<<blocks(nE + 1, 256), 256, 0, st>>>(P<int32_t>(ctx->out_len), nE, P<int64_t>(ctx->lens64));
        CKL();
        CK(cudaMemsetAsync(ctx->hist.p, 0, 8 * LA_HIST, st));
        if (nE) {
            k_att_hist<<<blocks(nE, 256), 256, 0, st>>>(P<uint8_t>(ctx->out_att), nE, P<unsigned long long>(ctx->hist));
            CKL();
        }
        size_t tb = 0;
        cub::DeviceScan::ExclusiveSum(nullptr, tb, P<int64_t>(ctx->lens64), P<int64_t>(ctx->ext_off), nE + 1, st);
        CK(grow(ctx->cub_tmp, tb));
        cub::DeviceScan::ExclusiveSum(ctx->cub_tmp.p, tb, P<int64_t>(ctx->lens64), P<int64_t>(ctx->ext_off), nE + 1, st);
        CKL();
    }
    int64_t *h64 = (int64_t *)ctx->h_small.p;
    CK(cudaMemcpyAsync(h64, P<int64_t>(ctx->ext_off) + nE, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(h64 + 1, d_gst, 8 * (8 + GSTATS_WORDS * N_TAB_CLASSES), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(h64 + 64, ctx->hist.p, 8 * LA_HIST, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (getenv("LA_PROFILE") && atoi(getenv("LA_PROFILE")) && ctx->prof.p) {
        CK(cudaMemcpy(ctx->stats.prof_cycles, ctx->prof.p, sizeof(ctx->stats.prof_cycles), cudaMemcpyDeviceToHost));
    }
    // per-class stats (classes 0..4 shared memory, 5 = XL); fold them into the smem totals
    for (int i = 0; i < LA_HIST; ++i) ctx->stats.attempts_hist[i] = h64[64 + i];
    for (int c = 0; c < N_TAB_CLASSES; ++c) {
        const int64_t *g = h64 + 1 + 8 + GSTATS_WORDS * c;
        ctx->stats.cls_ends[c] = c < N_SMEM_CLASSES ? ncls[c] : (c == C_XLC ? n_xlc : n_xl);
        ctx->stats.cls_inserts[c] = g[0];
        ctx->stats.cls_attempts[c] = g[2];
        ctx->stats.cls_filtered[c] = g[3];
        ctx->stats.cls_inl_attempts[c] = g[4];
        ctx->stats.cls_ref_attempts[c] = g[5];
        ctx->stats.cls_dead0[c] = g[6];
        h64[1] += g[0];
        h64[2] += g[1];
        h64[3] += g[2];
    }
    const int64_t total = h64[0];
    // d_gst: [0] smem inserts [1] smem walk steps [2] smem attempts [3] global inserts [4] global steps
    ctx->stats.inserts = h64[1] + h64[4] + ctx->stats.cpu_inserts;
    ctx->stats.inserts_smem = h64[1];
    ctx->stats.walk_steps = h64[2] + h64[5] + ctx->stats.cpu_walk_steps;
    ctx->stats.attempts = h64[3] + ctx->g_attempts + ctx->stats.cpu_attempts;
    ctx->stats.ext_bases = total;
    CK(grow(ctx->ext_seq, total + 16));
    if (nE) {
        k_emit<<<blocks(nE * 32, 256), 256, 0, st>>>(P<uint8_t>(ctx->walk_buf), W, P<int64_t>(ctx->ext_off), nE,
                                                     P<char>(ctx->ext_seq));
        CKL();
    }
    CK(cudaEventRecord(ctx->ev[4], st));
    if (to_host) {
        CK(grow_host(ctx->h_ext_off, (nE + 1) * 8));
        CK(grow_host(ctx->h_ext_seq, total + 16));
        CK(grow_host(ctx->h_term, nE + 16));
        CK(grow_host(ctx->h_k, nE + 16));
        CK(grow_host(ctx->h_att, nE + 16));
        CK(cudaMemcpyAsync(ctx->h_ext_off.p, ctx->ext_off.p, (nE + 1) * 8, cudaMemcpyDeviceToHost, st));
        if (total) CK(cudaMemcpyAsync(ctx->h_ext_seq.p, ctx->ext_seq.p, total, cudaMemcpyDeviceToHost, st));
        if (nE) {
            CK(cudaMemcpyAsync(ctx->h_term.p, ctx->out_term.p, nE, cudaMemcpyDeviceToHost, st));
            CK(cudaMemcpyAsync(ctx->h_k.p, ctx->out_k.p, nE, cudaMemcpyDeviceToHost, st));
            CK(cudaMemcpyAsync(ctx->h_att.p, ctx->out_att.p, nE, cudaMemcpyDeviceToHost, st));
        }
        out->ext_off = (const int64_t *)ctx->h_ext_off.p;
        out->ext_seq = (const char *)ctx->h_ext_seq.p;
        out->term = (const uint8_t *)ctx->h_term.p;
        out->k_used = (const uint8_t *)ctx->h_k.p;
        out->n_attempts = (const uint8_t *)ctx->h_att.p;
    } else {
        out->ext_off = P<int64_t>(ctx->ext_off);
        out->ext_seq = P<char>(ctx->ext_seq);
        out->term = P<uint8_t>(ctx->out_term);
        out->k_used = P<uint8_t>(ctx->out_k);
        out->n_attempts = P<uint8_t>(ctx->out_att);
    }
    out->n_ends = nE;
    CK(cudaStreamSynchronize(st));
    float ms = 0;
    cudaEventElapsedTime(&ms, ctx->ev[0], ctx->ev[4]);
    ctx->stats.ms_total = ms;
    cudaEventElapsedTime(&ms, ctx->ev[1], ctx->ev[2]);
    ctx->stats.ms_smem = ms;
    cudaEventElapsedTime(&ms, ctx->ev[2], ctx->ev[3]);
    ctx->stats.ms_global = ms;
    cudaEventElapsedTime(&ms, ctx->ev[3], ctx->ev[4]);
    ctx->stats.ms_emit = ms;
    for (int c = 0; c < N_TAB_CLASSES; ++c) {   // start -> end of each class kernel
        float m = 0;
        cudaEventElapsedTime(&m, ctx->ev_cls0[c], ctx->ev_cls[c]);
        ctx->stats.cls_ms[c] = m;
    }
    // class counts (host-side tally from the plan counters)
    ctx->stats.ends_by_class[2] = n_smem - n_ovf + cx.m;   // the host's ends are counted with class 0
    ctx->stats.ends_by_class[3] = n_glob;
    ctx->stats.ends_by_class[4] = n_ovf;
    ctx->stats.ends_medium = ncls[3] + ncls[4];
    ctx->stats.ms_smem_medium = ctx->stats.cls_ms[N_SMEM_CLASSES] + ctx->stats.cls_ms[3] + ctx->stats.cls_ms[4];
    ctx->stats.ms_build = -1.0;   // set by la_replay_build
    ctx->stats.ms_walk = -1.0;
    ctx->extended = true;
    return LA_OK;
}

}  // namespace

extern "C" la_status la_extend(la_ctx *ctx, la_result *out) { return extend_impl(ctx, out, true); }

// ---- NEXT N1: streamed load + extend of a host batch (Fig 4) ----------------
namespace la {
// in-place rebase of a copied offsets slice: a[i] -= base (the slice's first element)
__global__ void k_rebase(int64_t *__restrict__ a, int64_t n, int64_t base) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) a[i] -= base;
}
__global__ void k_add_i64(const int64_t *__restrict__ a, int64_t n, int64_t add, int64_t *__restrict__ out) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < n) out[i] = a[i] + add;
}
}  // namespace la

extern "C" la_status la_extend_streamed(la_ctx *ctx, const la_batch *b, const la_params *params, int32_t n_chunks,
                                        la_result *out) {
    if (!ctx || !out) return LA_ERR_INVALID_ARG;
    if (ctx->sticky) return fail(ctx, LA_ERR_CUDA, "context has a sticky CUDA error: %s", ctx->err.c_str());
    if (!b || !params) return fail(ctx, LA_ERR_INVALID_ARG, "null batch or params");
    if (b->mem != LA_MEM_HOST) return fail(ctx, LA_ERR_INVALID_ARG, "la_extend_streamed takes a host batch");
    if (n_chunks < 1 || n_chunks > 4096) return fail(ctx, LA_ERR_INVALID_ARG, "n_chunks must be in 1..4096");
    if (b->n_contigs < 0 || b->n_reads < 0) return fail(ctx, LA_ERR_INVALID_ARG, "negative sizes");
    if (!b->contig_off || !b->read_off || !b->end_read_off)
        return fail(ctx, LA_ERR_INVALID_ARG, "null offsets array");
    cudaSetDevice(ctx->device);
    const int64_t nC = b->n_contigs, nE = 2 * nC, nR = b->n_reads;
    const int64_t *coff = b->contig_off, *roff = b->read_off, *eoff = b->end_read_off;
    // the chunking reads offsets at the cut points: check the global invariants it relies on first
    if (coff[0] != 0 || roff[0] != 0 || eoff[0] != 0) return fail(ctx, LA_ERR_INVALID_ARG, "offsets must start at 0");
    if (eoff[nE] != nR)
        return fail(ctx, LA_ERR_INVALID_ARG, "end_read_off[2*n_contigs] (%lld) != n_reads (%lld)",
                    (long long)eoff[nE], (long long)nR);
    const int64_t total_bytes = roff[nR];
    if (total_bytes < 0 || coff[nC] < 0) return fail(ctx, LA_ERR_INVALID_ARG, "negative total length");
    // contig cuts with ~equal read bytes per chunk (binary search over the monotone prefix); a
    // non-monotone offsets array is rejected by la_load_batch of the chunk that contains it
    std::vector<int64_t> cut(1, 0);
    for (int i = 1; i < n_chunks; ++i) {
        const int64_t target = total_bytes * i / n_chunks;
        int64_t lo = cut.back(), hi = nC;
        while (lo < hi) {
            const int64_t mid = (lo + hi) / 2;
            const int64_t e = eoff[2 * mid];
            const int64_t r = (e >= 0 && e <= nR) ? roff[e] : total_bytes;
            if (r < target) lo = mid + 1; else hi = mid;
        }
        if (lo > cut.back() && lo < nC) cut.push_back(lo);
    }
    cut.push_back(nC);
    const int nchunk = (int)cut.size() - 1;
    if (!ctx->copy_stream) {
        CK(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking));
        for (int i = 0; i < 2; ++i) {
            CK(cudaEventCreateWithFlags(&ctx->ev_copied[i], cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&ctx->ev_loaded[i], cudaEventDisableTiming));
        }
    }
    cudaStream_t cs = ctx->copy_stream, st = ctx->stream;
    const int W = std::max(params->max_walk_len, 1);
    // combined host results (pinned, grow-only): the extension bytes are bounded by W per end
    CK(grow_host(ctx->h_ext_off, (nE + 1) * 8));
    CK(grow_host(ctx->h_ext_seq, nE * (int64_t)W + 16));
    CK(grow_host(ctx->h_term, nE + 16));
    CK(grow_host(ctx->h_k, nE + 16));
    CK(grow_host(ctx->h_att, nE + 16));
    int64_t *h_off = (int64_t *)ctx->h_ext_off.p;
    h_off[0] = 0;
    // chunk c: contigs [cut[c], cut[c+1]) -> ends, reads, bytes (all contiguous ranges)
    struct Chunk { int64_t c0, c1, r0, r1, b0, b1, s0, s1; };
    std::vector<Chunk> chunks(nchunk);
    for (int c = 0; c < nchunk; ++c) {   // cut points must be ordered (the chunks check the rest)
        Chunk &k = chunks[c];
        k.c0 = cut[c]; k.c1 = cut[c + 1];
        k.r0 = eoff[2 * k.c0]; k.r1 = eoff[2 * k.c1];
        if (k.r0 < 0 || k.r1 < k.r0 || k.r1 > nR)
            return fail(ctx, LA_ERR_INVALID_ARG, "offsets are not non-decreasing");
        k.b0 = roff[k.r0]; k.b1 = roff[k.r1];
        k.s0 = coff[k.c0]; k.s1 = coff[k.c1];
        if (k.b0 < 0 || k.b1 < k.b0 || k.s0 < 0 || k.s1 < k.s0)
            return fail(ctx, LA_ERR_INVALID_ARG, "offsets are not non-decreasing");
    }
    auto chunk = [&](int c) { return chunks[c]; };
    auto enqueue_copy = [&](int c) -> la_status {
        const int i = c & 1;
        const Chunk k = chunk(c);
        const int64_t nc = k.c1 - k.c0, nr = k.r1 - k.r0;
        CK(grow(ctx->st_seq[i], k.b1 - k.b0 + 16));
        CK(grow(ctx->st_qual[i], k.b1 - k.b0 + 16));
        CK(grow(ctx->st_cseq[i], k.s1 - k.s0 + 16));
        CK(grow(ctx->st_coff[i], (nc + 1) * 8));
        CK(grow(ctx->st_roff[i], (nr + 1) * 8));
        CK(grow(ctx->st_eoff[i], (2 * nc + 1) * 8));
        if (c >= 2) CK(cudaStreamWaitEvent(cs, ctx->ev_loaded[i], 0));   // chunk c-2 is encoded: buffer free
        if (k.b1 > k.b0) {
            if (!b->read_seq || !b->read_qual) return fail(ctx, LA_ERR_INVALID_ARG, "null sequence pointer");
            CK(cudaMemcpyAsync(ctx->st_seq[i].p, b->read_seq + k.b0, k.b1 - k.b0, cudaMemcpyHostToDevice, cs));
            CK(cudaMemcpyAsync(ctx->st_qual[i].p, b->read_qual + k.b0, k.b1 - k.b0, cudaMemcpyHostToDevice, cs));
        }
        if (k.s1 > k.s0) {
            if (!b->contig_seq) return fail(ctx, LA_ERR_INVALID_ARG, "null sequence pointer");
            CK(cudaMemcpyAsync(ctx->st_cseq[i].p, b->contig_seq + k.s0, k.s1 - k.s0, cudaMemcpyHostToDevice, cs));
        }
        CK(cudaMemcpyAsync(ctx->st_coff[i].p, coff + k.c0, (nc + 1) * 8, cudaMemcpyHostToDevice, cs));
        CK(cudaMemcpyAsync(ctx->st_roff[i].p, roff + k.r0, (nr + 1) * 8, cudaMemcpyHostToDevice, cs));
        CK(cudaMemcpyAsync(ctx->st_eoff[i].p, eoff + 2 * k.c0, (2 * nc + 1) * 8, cudaMemcpyHostToDevice, cs));
        CK(cudaEventRecord(ctx->ev_copied[i], cs));
        return LA_OK;
    };
    la_stats acc{};
    // every error return after the first enqueue_copy first drains the copy stream, so the caller's
    // (pinned) host buffers are no longer read by queued DMA when la_extend_streamed returns
    const la_status run = [&]() -> la_status {
        la_status s;
        if ((s = enqueue_copy(0))) return s;
        if (nchunk > 1 && (s = enqueue_copy(1))) return s;
        int64_t bases = 0;
        for (int c = 0; c < nchunk; ++c) {
            const int i = c & 1;
            const Chunk k = chunk(c);
            const int64_t nc = k.c1 - k.c0, nr = k.r1 - k.r0;
            CK(cudaStreamWaitEvent(st, ctx->ev_copied[i], 0));
            k_rebase<<<blocks(nc + 1, 256), 256, 0, st>>>(P<int64_t>(ctx->st_coff[i]), nc + 1, k.s0);
            k_rebase<<<blocks(nr + 1, 256), 256, 0, st>>>(P<int64_t>(ctx->st_roff[i]), nr + 1, k.b0);
            k_rebase<<<blocks(2 * nc + 1, 256), 256, 0, st>>>(P<int64_t>(ctx->st_eoff[i]), 2 * nc + 1, k.r0);
            CK(cudaGetLastError());
            la_batch sub{};
            sub.mem = LA_MEM_DEVICE;
            sub.n_contigs = (int32_t)nc;
            sub.contig_seq = P<char>(ctx->st_cseq[i]);
            sub.contig_off = P<int64_t>(ctx->st_coff[i]);
            sub.n_reads = nr;
            sub.read_seq = P<char>(ctx->st_seq[i]);
            sub.read_qual = P<char>(ctx->st_qual[i]);
            sub.read_off = P<int64_t>(ctx->st_roff[i]);
            sub.end_read_off = P<int64_t>(ctx->st_eoff[i]);
            if ((s = la_load_batch(ctx, &sub, params))) return s;
            CK(cudaEventRecord(ctx->ev_loaded[i], st));   // staging buffer i may be refilled
            if (c + 2 < nchunk && (s = enqueue_copy(c + 2))) return s;
            la_result r{};
            if ((s = extend_impl(ctx, &r, false))) return s;
            const int64_t ne = 2 * nc, nb = ctx->stats.ext_bases;
            // results of this chunk -> the combined host buffers (device-side rebase of ext_off)
            CK(grow(ctx->lens64, (ne + 1) * 8));
            k_add_i64<<<blocks(ne + 1, 256), 256, 0, st>>>(P<int64_t>(ctx->ext_off), ne + 1, bases, P<int64_t>(ctx->lens64));
            CK(cudaGetLastError());
            const int64_t e0 = 2 * k.c0;
            CK(cudaMemcpyAsync(h_off + e0 + 1, P<int64_t>(ctx->lens64) + 1, ne * 8, cudaMemcpyDeviceToHost, st));
            if (nb) CK(cudaMemcpyAsync((char *)ctx->h_ext_seq.p + bases, ctx->ext_seq.p, nb, cudaMemcpyDeviceToHost, st));
            if (ne) {
                CK(cudaMemcpyAsync((uint8_t *)ctx->h_term.p + e0, ctx->out_term.p, ne, cudaMemcpyDeviceToHost, st));
                CK(cudaMemcpyAsync((uint8_t *)ctx->h_k.p + e0, ctx->out_k.p, ne, cudaMemcpyDeviceToHost, st));
                CK(cudaMemcpyAsync((uint8_t *)ctx->h_att.p + e0, ctx->out_att.p, ne, cudaMemcpyDeviceToHost, st));
            }
            bases += nb;
            // accumulate the work and device-time counters over chunks
            const la_stats &x = ctx->stats;
            acc.ms_total += x.ms_total;
            acc.ms_smem += x.ms_smem;
            acc.ms_global += x.ms_global;
            acc.ms_emit += x.ms_emit;
            acc.inserts += x.inserts;
            acc.inserts_smem += x.inserts_smem;
            acc.walk_steps += x.walk_steps;
            acc.attempts += x.attempts;
            acc.ext_bases += x.ext_bases;
            for (int q = 0; q < 5; ++q) acc.ends_by_class[q] += x.ends_by_class[q];
            acc.kernel_launches += x.kernel_launches + 4;   // + the rebase / offset kernels
            acc.global_rounds += x.global_rounds;
            acc.ends_medium += x.ends_medium;
            acc.ms_smem_medium += x.ms_smem_medium;
            acc.ends_xl += x.ends_xl;
            acc.cpu_ends += x.cpu_ends;
            acc.cpu_inserts += x.cpu_inserts;
            acc.cpu_walk_steps += x.cpu_walk_steps;
            acc.cpu_attempts += x.cpu_attempts;
            acc.xl_scratch_bytes = std::max(acc.xl_scratch_bytes, x.xl_scratch_bytes);
            for (int q = 0; q < N_TAB_CLASSES; ++q) {
                acc.cls_ends[q] += x.cls_ends[q];
                acc.cls_inserts[q] += x.cls_inserts[q];
                acc.cls_attempts[q] += x.cls_attempts[q];
                acc.cls_filtered[q] += x.cls_filtered[q];
                acc.cls_inl_attempts[q] += x.cls_inl_attempts[q];
                acc.cls_ref_attempts[q] += x.cls_ref_attempts[q];
                acc.cls_dead0[q] += x.cls_dead0[q];
                acc.cls_ms[q] += x.cls_ms[q];
            }
            for (int q = 0; q < LA_HIST; ++q) acc.attempts_hist[q] += x.attempts_hist[q];
            acc.smem_bytes_per_cta = x.smem_bytes_per_cta;
            acc.smem_ctas_per_sm = x.smem_ctas_per_sm;
        }
        CK(cudaStreamSynchronize(st));
        return LA_OK;
    }();
    if (run != LA_OK) {
        cudaStreamSynchronize(cs);
        return run;
    }
    acc.ms_build = acc.ms_walk = -1.0;
    ctx->stats = acc;
    ctx->extended = false;   // the device holds only the last chunk: nothing to replay
    out->n_ends = nE;
    out->ext_off = h_off;
    out->ext_seq = (const char *)ctx->h_ext_seq.p;
    out->term = (const uint8_t *)ctx->h_term.p;
    out->k_used = (const uint8_t *)ctx->h_k.p;
    out->n_attempts = (const uint8_t *)ctx->h_att.p;
    return LA_OK;
}
extern "C" la_status la_extend_device(la_ctx *ctx, la_result *out) { return extend_impl(ctx, out, false); }

extern "C" la_status la_set_coexec(la_ctx *ctx, int32_t n_threads, double cpu_share) {
    if (!ctx) return LA_ERR_INVALID_ARG;
    if (n_threads < 0 || n_threads > 1024 || !(cpu_share >= 0.0 && cpu_share <= 1.0))
        return fail(ctx, LA_ERR_INVALID_ARG, "la_set_coexec: need 0 <= n_threads <= 1024 and 0 <= cpu_share <= 1");
    ctx->coexec_threads = n_threads;
    ctx->coexec_share = cpu_share;
    return LA_OK;
}

// Build-only replay (SURVEY §8(d) timing protocol step 5): the table-class kernels rerun, over the
// class lists of the last la_extend, exactly the (end, k) attempts it made (k_start + i * shift for
// i < n_attempts, the direction recorded per end in out_dir) with the link pass and the walk
// disabled: staging, per-read prefix, table clear, filter and build passes (Alg 1) only.
extern "C" la_status la_replay_build(la_ctx *ctx) {
    if (!ctx) return LA_ERR_INVALID_ARG;
    if (ctx->sticky) return fail(ctx, LA_ERR_CUDA, "context has a sticky CUDA error: %s", ctx->err.c_str());
    if (!ctx->extended) return fail(ctx, LA_ERR_STATE, "la_replay_build needs a completed la_extend of the loaded batch");
    CK(cudaSetDevice(ctx->device));
    cudaStream_t st = ctx->stream;
    int *d_ctr = P<int>(ctx->ctrs);
    unsigned long long *d_gst = P<unsigned long long>(ctx->gstats);
    CK(cudaMemsetAsync(d_ctr + 15, 0, 4 * 8, st));   // overflow count + the class work counters (16..22)
    CK(cudaMemsetAsync(d_gst + 8, 0, 8 * GSTATS_WORDS * N_TAB_CLASSES, st));
    CK(cudaEventRecord(ctx->ev_rep[0], st));
    const la_status s = launch_classes(ctx, true);
    if (s != LA_OK) return s;
    CK(cudaEventRecord(ctx->ev_rep[1], st));
    int64_t *h64 = (int64_t *)ctx->h_small.p;
    CK(cudaMemcpyAsync(h64, d_gst + 8, 8 * GSTATS_WORDS * N_TAB_CLASSES, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    float ms = 0;
    cudaEventElapsedTime(&ms, ctx->ev_rep[0], ctx->ev_rep[1]);
    ctx->stats.ms_build = ms;
    ctx->stats.ms_walk = ctx->stats.ms_smem - ms;   // the rest of the table phase: link + walk + hand-offs
    for (int c = 0; c < N_TAB_CLASSES; ++c) {
        float m = 0;
        cudaEventElapsedTime(&m, ctx->ev_cls0[c], ctx->ev_cls[c]);
        ctx->stats.cls_build_ms[c] = m;
        ctx->stats.cls_build_inserts[c] = h64[GSTATS_WORDS * c];
    }
    return LA_OK;
}

// ---- NEXT N1: on-device append of extensions to contigs (Fig 4 "Append extensions to contigs",
// P:L464 "appended to the end of contig") -------------------------------------------------------
namespace la {
// Warp-cooperative copy of n bytes src -> dst for any alignment of either: byte copies up to the
// first 16-byte-aligned destination address and after the last one, 16-byte stores in between.  Each
// 16-byte destination chunk takes its source bytes from the two aligned 16-byte words that hold
// them (both contain at least one byte of the source range, so they lie inside its allocation) and
// realigns them with funnel shifts.  Every destination byte is written by exactly one lane.
__device__ __forceinline__ void warp_copy(char *__restrict__ dst, const char *__restrict__ src, int64_t n, int lane) {
    if (n <= 0) return;
    const int64_t mis = (int64_t)((16 - ((uintptr_t)dst & 15)) & 15);
    const int64_t head = n < mis ? n : mis;
    if (lane < head) dst[lane] = src[lane];
    const int64_t nbody = (n - head) >> 4;
    const int64_t tail0 = head + (nbody << 4);
    if (lane < n - tail0) dst[tail0 + lane] = src[tail0 + lane];
    if (nbody == 0) return;
    uint4 *__restrict__ d4 = reinterpret_cast<uint4 *>(dst + head);
    const char *s = src + head;
    const int sh = (int)((uintptr_t)s & 15);
    const uint4 *__restrict__ s4 = reinterpret_cast<const uint4 *>(s - sh);
    if (sh == 0) {
        for (int64_t i = lane; i < nbody; i += 32) d4[i] = __ldg(s4 + i);
        return;
    }
    const int q = sh >> 2, r = (sh & 3) * 8;
    for (int64_t i = lane; i < nbody; i += 32) {
        const uint4 lo = __ldg(s4 + i), hi = __ldg(s4 + i + 1);
        const uint32_t w[8] = {lo.x, lo.y, lo.z, lo.w, hi.x, hi.y, hi.z, hi.w};
        uint32_t o[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const uint32_t a0 = q == 0 ? w[k] : q == 1 ? w[k + 1] : q == 2 ? w[k + 2] : w[k + 3];
            const uint32_t a1 = q == 0 ? w[k + 1] : q == 1 ? w[k + 2] : q == 2 ? w[k + 3] : w[k + 4];
            o[k] = __funnelshift_r(a0, a1, r);
        }
        d4[i] = make_uint4(o[0], o[1], o[2], o[3]);
    }
}

// One warp per contig (grid-stride): out[c] = ext(2c) + contig c + ext(2c+1).  The output offset is
// closed-form (no scan): out_off[c] = (contig_off[c] - contig_off[0]) + (ext_off[2c] - ext_off[0]),
// because each contig's output is its two ends' extensions around it, in end order.  HBM-bound copy
// (algorithmic bytes: the sequence bytes read once and written once, plus the offsets).
__global__ void __launch_bounds__(256) k_append_ext(int64_t n_contigs, const char *__restrict__ cseq,
                                                    const int64_t *__restrict__ coff, const int64_t *__restrict__ eoff,
                                                    const char *__restrict__ eseq, char *__restrict__ out,
                                                    int64_t *__restrict__ out_off) {
    const int lane = threadIdx.x & 31;
    const int64_t warp0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t c0 = coff[0], e0 = eoff[0];
    for (int64_t c = warp0; c < n_contigs; c += nwarps) {
        const int64_t cb = coff[c], ce = coff[c + 1];
        const int64_t lb = eoff[2 * c], le = eoff[2 * c + 1], re = eoff[2 * c + 2];
        const int64_t o = (cb - c0) + (lb - e0);
        if (lane == 0) {
            out_off[c] = o;
            if (c == n_contigs - 1) out_off[n_contigs] = o + (ce - cb) + (re - lb);
        }
        char *dst = out + o;
        warp_copy(dst, eseq + lb, le - lb, lane);
        dst += le - lb;
        warp_copy(dst, cseq + cb, ce - cb, lane);
        dst += ce - cb;
        warp_copy(dst, eseq + le, re - le, lane);
    }
}
}  // namespace la

extern "C" la_status la_append_extensions(la_ctx *ctx, int32_t n_contigs, const char *contig_seq,
                                          const int64_t *contig_off, const int64_t *ext_off, const char *ext_seq,
                                          char *out_seq, int64_t *out_off) {
    if (!ctx) return LA_ERR_INVALID_ARG;
    if (ctx->sticky) return fail(ctx, LA_ERR_CUDA, "context is in a sticky CUDA error state");
    if (n_contigs < 0 || !contig_off || !ext_off || !out_off)
        return fail(ctx, LA_ERR_INVALID_ARG, "la_append_extensions: n_contigs < 0 or a NULL offsets pointer");
    CK(cudaSetDevice(ctx->device));
    if (n_contigs == 0) {
        CK(cudaMemsetAsync(out_off, 0, sizeof(int64_t), ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        return LA_OK;
    }
    const int threads = 256;
    const int64_t want = ((int64_t)n_contigs * 32 + threads - 1) / threads;
    const int blocks = (int)std::min<int64_t>(want, (int64_t)ctx->n_sm * 8);
    k_append_ext<<<blocks, threads, 0, ctx->stream>>>(n_contigs, contig_seq, contig_off, ext_off, ext_seq, out_seq,
                                                       out_off);
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(ctx->stream));
    return LA_OK;
}

// ================================================================================================
// NEXT N4: la_select_reads — candidate-read selection on the device (la_select.cuh)
// ================================================================================================
namespace {

template <typename T>
la_status cub_scan(la_ctx *ctx, const T *in, T *out, int64_t n) {
    size_t tb = 0;
    CK(cub::DeviceScan::ExclusiveSum(nullptr, tb, in, out, n, ctx->stream));
    CK(grow(ctx->cub_tmp, tb));
    CK(cub::DeviceScan::ExclusiveSum(ctx->cub_tmp.p, tb, in, out, n, ctx->stream));
    return LA_OK;
}

template <typename K, typename V>
la_status cub_sort_pairs(la_ctx *ctx, const K *kin, K *kout, const V *vin, V *vout, int64_t n) {
    size_t tb = 0;
    CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, kin, kout, vin, vout, n, 0, (int)(8 * sizeof(K)), ctx->stream));
    CK(grow(ctx->cub_tmp, tb));
    CK(cub::DeviceRadixSort::SortPairs(ctx->cub_tmp.p, tb, kin, kout, vin, vout, n, 0, (int)(8 * sizeof(K)),
                                       ctx->stream));
    return LA_OK;
}

la_status d2h_i64(la_ctx *ctx, const int64_t *d, int64_t *h) {
    CK(cudaMemcpyAsync(h, d, 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return LA_OK;
}

}  // namespace

extern "C" la_status la_select_reads(la_ctx *ctx, const la_pool *pool, const la_sel_params *sp, la_selection *out) {
    if (!ctx) return LA_ERR_INVALID_ARG;
    if (ctx->sticky) return fail(ctx, LA_ERR_CUDA, "context has a sticky CUDA error: %s", ctx->err.c_str());
    if (!pool || !sp || !out) return fail(ctx, LA_ERR_INVALID_ARG, "la_select_reads: null argument");
    if (pool->n_contigs < 0 || pool->n_pairs < 0 || pool->n_pairs > 0xFFFFFFFFll)
        return fail(ctx, LA_ERR_INVALID_ARG, "la_select_reads: n_contigs or n_pairs out of range");
    if (!pool->contig_off || !pool->read_off || (pool->n_pairs && (!pool->read_seq || !pool->read_qual)) ||
        (pool->n_contigs && !pool->contig_seq))
        return fail(ctx, LA_ERR_INVALID_ARG, "la_select_reads: null pool array");
    if (pool->mem != LA_MEM_HOST && pool->mem != LA_MEM_DEVICE)
        return fail(ctx, LA_ERR_INVALID_ARG, "la_select_reads: mem must be LA_MEM_HOST or LA_MEM_DEVICE");
    if (!(sp->seed_len >= 1 && sp->seed_len <= 31 && sp->seed_stride >= 1 && sp->window >= sp->seed_len &&
          sp->window <= 65535 && sp->min_overlap >= 0 && sp->max_mism_pct >= 0 && sp->max_mism_pct <= 100))
        return fail(ctx, LA_ERR_INVALID_ARG, "la_select_reads: parameters out of range");
    CK(cudaSetDevice(ctx->device));
    cudaStream_t st = ctx->stream;
    SelBufs &S = ctx->sel;
    const bool host = pool->mem == LA_MEM_HOST;
    const int64_t nC = pool->n_contigs, nE = 2 * nC, nR = 2 * pool->n_pairs;
    // ---- input: offsets validated (monotone, starting at 0), arrays copied to the device ----
    int64_t c0, cN, r0, rN;
    la_status rc;
    if ((rc = read_i64(ctx, pool->contig_off, host, &c0)) != LA_OK) return rc;
    if ((rc = read_i64(ctx, pool->contig_off + nC, host, &cN)) != LA_OK) return rc;
    if ((rc = read_i64(ctx, pool->read_off, host, &r0)) != LA_OK) return rc;
    if ((rc = read_i64(ctx, pool->read_off + nR, host, &rN)) != LA_OK) return rc;
    if (c0 != 0 || r0 != 0 || cN < 0 || rN < 0)
        return fail(ctx, LA_ERR_INVALID_ARG, "la_select_reads: offsets must start at 0 and be non-decreasing");
    if ((rc = copy_in(ctx, S.coff, pool->contig_off, 8 * (size_t)(nC + 1), host)) != LA_OK) return rc;
    if ((rc = copy_in(ctx, S.roff, pool->read_off, 8 * (size_t)(nR + 1), host)) != LA_OK) return rc;
    if ((rc = copy_in(ctx, S.cseq, pool->contig_seq, (size_t)cN, host)) != LA_OK) return rc;
    if ((rc = copy_in(ctx, S.rseq, pool->read_seq, (size_t)rN, host)) != LA_OK) return rc;
    if ((rc = copy_in(ctx, S.rqual, pool->read_qual, (size_t)rN, host)) != LA_OK) return rc;
    CK(grow(ctx->errw, 16));
    uint32_t *d_err = P<uint32_t>(ctx->errw);
    CK(cudaMemsetAsync(d_err, 0, 4, st));
    if (nC) { k_check_offsets<<<blocks(nC, 256), 256, 0, st>>>(P<int64_t>(S.coff), nC, 0, d_err, nullptr); CKL(); }
    if (nR) { k_check_offsets<<<blocks(nR, 256), 256, 0, st>>>(P<int64_t>(S.roff), nR, 0, d_err, nullptr); CKL(); }
    uint32_t h_err = 0;
    CK(cudaMemcpyAsync(&h_err, d_err, 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (h_err) return fail(ctx, LA_ERR_INVALID_ARG, "la_select_reads: offsets are not non-decreasing");
    const int w = sp->window, s = sp->seed_len, t = sp->seed_stride;
    // ---- index of the end windows' seeds (S1, S2a) ----
    CK(grow(S.wcnt, 8 * (size_t)(nE + 1)));
    CK(grow(S.woff, 8 * (size_t)(nE + 1)));
    CK(cudaMemsetAsync(S.wcnt.p, 0, 8 * (size_t)(nE + 1), st));
    if (nE) { sel::k_sel_wcount<<<blocks(nE, 256), 256, 0, st>>>(nE, P<int64_t>(S.coff), w, s, P<int64_t>(S.wcnt)); CKL(); }
    if ((rc = cub_scan(ctx, P<int64_t>(S.wcnt), P<int64_t>(S.woff), nE + 1)) != LA_OK) return rc;
    int64_t nI = 0;
    if ((rc = d2h_i64(ctx, P<int64_t>(S.woff) + nE, &nI)) != LA_OK) return rc;
    int64_t nU = 0;
    uint64_t cap_mask = 0;
    if (nI) {
        for (DevBuf *b : {&S.key, &S.val, &S.key2, &S.val2}) CK(grow(*b, 8 * (size_t)nI));
        CK(grow(S.flag, 8 * (size_t)(nI + 1)));
        CK(grow(S.uidx, 8 * (size_t)(nI + 1)));
        sel::k_sel_index<<<blocks(32 * nE, 256), 256, 0, st>>>(nE, P<char>(S.cseq), P<int64_t>(S.coff), P<int64_t>(S.woff),
                                                                w, s, P<uint64_t>(S.key), P<uint64_t>(S.val));
        CKL();
        if ((rc = cub_sort_pairs(ctx, P<uint64_t>(S.key), P<uint64_t>(S.key2), P<uint64_t>(S.val), P<uint64_t>(S.val2),
                                 nI)) != LA_OK)
            return rc;
        CK(cudaMemsetAsync(P<int64_t>(S.flag) + nI, 0, 8, st));
        sel::k_sel_runs<<<blocks(nI, 256), 256, 0, st>>>(nI, P<uint64_t>(S.key2), P<int64_t>(S.flag));
        CKL();
        if ((rc = cub_scan(ctx, P<int64_t>(S.flag), P<int64_t>(S.uidx), nI + 1)) != LA_OK) return rc;
        if ((rc = d2h_i64(ctx, P<int64_t>(S.uidx) + nI, &nU)) != LA_OK) return rc;
    }
    {
        uint64_t cap = 1024;
        while (cap < 2 * (uint64_t)nU) cap <<= 1;
        cap_mask = cap - 1;
        CK(grow(S.hkey, 8 * cap));
        CK(grow(S.hval, 8 * cap));
        CK(grow(S.ustart, 8 * (size_t)(nU + 1)));
        CK(cudaMemsetAsync(S.hkey.p, 0, 8 * cap, st));
        CK(cudaMemsetAsync(S.ustart.p, 0, 8 * (size_t)(nU + 1), st));
        if (nU) {
            sel::k_sel_hash<<<blocks(nI, 256), 256, 0, st>>>(nI, P<uint64_t>(S.key2), P<int64_t>(S.flag), P<int64_t>(S.uidx),
                                                              P<int64_t>(S.ustart), cap_mask,
                                                              P<unsigned long long>(S.hkey), P<int64_t>(S.hval));
            CKL();
            // ustart[nU] = number of valid entries (KEY_NONE sorts last): the last run ends there
            sel::k_sel_nvalid<<<blocks(nI, 256), 256, 0, st>>>(nI, P<uint64_t>(S.key2), P<int64_t>(S.ustart) + nU);
            CKL();
        }
    }
    // ---- queries (S2, S3): records of qualifying alignments; regrown and rerun if they overflow ----
    CK(grow(S.nrec, 8));
    int64_t cap_rec = std::max<int64_t>(1024, 2 * nR);
    int64_t n_rec = 0;
    for (int pass = 0; pass < 8; ++pass) {
        for (DevBuf *b : {&S.rkey, &S.rkey2}) CK(grow(*b, 8 * (size_t)cap_rec));
        for (DevBuf *b : {&S.rord, &S.rord2}) CK(grow(*b, 4 * (size_t)cap_rec));
        CK(cudaMemsetAsync(S.nrec.p, 0, 8, st));
        if (nR && nU) {
            sel::k_sel_query<<<blocks(2 * nR, 128), 128, 0, st>>>(
                nR / 2 * 2, P<char>(S.rseq), P<int64_t>(S.roff), P<char>(S.cseq), P<int64_t>(S.coff), w, s, t,
                sp->min_overlap, sp->max_mism_pct, P<unsigned long long>(S.hkey), P<int64_t>(S.hval), cap_mask,
                P<int64_t>(S.ustart), P<uint64_t>(S.val2), P<unsigned long long>(S.nrec), cap_rec, P<uint64_t>(S.rkey),
                P<uint32_t>(S.rord));
            CKL();
        }
        if ((rc = d2h_i64(ctx, P<int64_t>(S.nrec), &n_rec)) != LA_OK) return rc;
        if (n_rec <= cap_rec) break;
        cap_rec = n_rec + n_rec / 4 + 1024;
        if (pass == 7) return fail(ctx, LA_ERR_CAPACITY, "la_select_reads: record buffer did not converge");
    }
    // ---- S4: sort records by (end, pair), then (mate, strand, d); keep the first of each (end, pair) ----
    int64_t n_sel = 0;
    if (n_rec) {
        // stable radix sorts: by ord first (carrying the key), then by key (carrying the ord)
        if ((rc = cub_sort_pairs(ctx, P<uint32_t>(S.rord), P<uint32_t>(S.rord2), P<uint64_t>(S.rkey), P<uint64_t>(S.rkey2),
                                 n_rec)) != LA_OK)
            return rc;
        if ((rc = cub_sort_pairs(ctx, P<uint64_t>(S.rkey2), P<uint64_t>(S.rkey), P<uint32_t>(S.rord2), P<uint32_t>(S.rord),
                                 n_rec)) != LA_OK)
            return rc;
        CK(grow(S.flag, 8 * (size_t)(n_rec + 1)));
        CK(grow(S.uidx, 8 * (size_t)(n_rec + 1)));
        CK(cudaMemsetAsync(P<int64_t>(S.flag) + n_rec, 0, 8, st));
        sel::k_sel_first<<<blocks(n_rec, 256), 256, 0, st>>>(n_rec, P<uint64_t>(S.rkey), P<int64_t>(S.flag));
        CKL();
        if ((rc = cub_scan(ctx, P<int64_t>(S.flag), P<int64_t>(S.uidx), n_rec + 1)) != LA_OK) return rc;
        if ((rc = d2h_i64(ctx, P<int64_t>(S.uidx) + n_rec, &n_sel)) != LA_OK) return rc;
    }
    CK(grow(S.send, 8 * (size_t)(n_sel + 1)));
    CK(grow(S.spair, 8 * (size_t)(n_sel + 1)));
    CK(grow(S.sflip, (size_t)(n_sel + 1)));
    if (n_sel) {
        sel::k_sel_compact<<<blocks(n_rec, 256), 256, 0, st>>>(n_rec, P<uint64_t>(S.rkey), P<uint32_t>(S.rord),
                                                                P<int64_t>(S.flag), P<int64_t>(S.uidx), P<int64_t>(S.send),
                                                                P<int64_t>(S.spair), P<uint8_t>(S.sflip));
        CKL();
    }
    // ---- S5-S6: the batch ----
    const int64_t nOut = 2 * n_sel;
    CK(grow(S.eoff, 8 * (size_t)(nE + 1)));
    CK(grow(S.lens, 8 * (size_t)(nOut + 1)));
    CK(grow(S.ooff, 8 * (size_t)(nOut + 1)));
    sel::k_sel_eoff<<<blocks(nE + 1, 256), 256, 0, st>>>(nE, n_sel, P<int64_t>(S.send), P<int64_t>(S.eoff));
    CKL();
    CK(cudaMemsetAsync(P<int64_t>(S.lens) + nOut, 0, 8, st));
    if (nOut) {
        sel::k_sel_lens<<<blocks(nOut, 256), 256, 0, st>>>(n_sel, P<int64_t>(S.spair), P<int64_t>(S.roff), P<int64_t>(S.lens));
        CKL();
    }
    if ((rc = cub_scan(ctx, P<int64_t>(S.lens), P<int64_t>(S.ooff), nOut + 1)) != LA_OK) return rc;
    int64_t out_bytes = 0;
    if ((rc = d2h_i64(ctx, P<int64_t>(S.ooff) + nOut, &out_bytes)) != LA_OK) return rc;
    CK(grow(S.oseq, (size_t)out_bytes + 16));
    CK(grow(S.oqual, (size_t)out_bytes + 16));
    if (nOut) {
        sel::k_sel_copy<<<blocks(32 * nOut, 256), 256, 0, st>>>(n_sel, P<int64_t>(S.spair), P<uint8_t>(S.sflip), P<char>(S.rseq),
                                                                 P<char>(S.rqual), P<int64_t>(S.roff), P<int64_t>(S.ooff),
                                                                 P<char>(S.oseq), P<char>(S.oqual));
        CKL();
    }
    CK(cudaStreamSynchronize(st));
    out->n_sel = n_sel;
    out->sel_end = P<int64_t>(S.send);
    out->sel_pair = P<int64_t>(S.spair);
    out->sel_flip = P<uint8_t>(S.sflip);
    la_batch &B = out->batch;
    B.mem = LA_MEM_DEVICE;
    B.n_contigs = (int32_t)nC;
    B.contig_seq = P<char>(S.cseq);
    B.contig_off = P<int64_t>(S.coff);
    B.n_reads = nOut;
    B.read_seq = P<char>(S.oseq);
    B.read_qual = P<char>(S.oqual);
    B.read_off = P<int64_t>(S.ooff);
    B.end_read_off = P<int64_t>(S.eoff);
    return LA_OK;
}
