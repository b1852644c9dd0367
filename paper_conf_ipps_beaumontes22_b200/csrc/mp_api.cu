// mp_api.cu -- C ABI of libmadpipe (include/madpipe.h): validation, device
// memory, the batched candidate sweep engine, winner re-solve and traceback.
//
// Every step of the DP path runs in the kernels of mp_kernels.cu; this file
// only validates arguments, moves the O(L) profile to the device, lays out the
// DP tables in HBM and issues the launches (DESIGN.md sections 6-7).
#include <algorithm>
#include <numeric>
#include <chrono>
#include <climits>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include "../../include/madpipe.h"
#include "mp_internal.cuh"

using namespace mp;

struct DevBuf {
    void *p = nullptr;
    size_t n = 0;
    cudaError_t ensure(size_t bytes) {
        if (bytes <= n) return cudaSuccess;
        if (p) cudaFree(p);
        p = nullptr; n = 0;
        size_t want = std::max(bytes, (size_t)256);
        cudaError_t e = cudaMalloc(&p, want);
        if (e == cudaSuccess) n = want;
        return e;
    }
    void release() { if (p) cudaFree(p); p = nullptr; n = 0; }
};

struct madpipe_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    int64_t mem_budget = 0;
    std::string err;
    DevBuf tdesc;
    DevBuf tables, jobs, tiles, chains, chain_data, jl, counts, roots, trace, stages, scratch, codes, flags,
        tlist;
    cudaEvent_t ev_a = nullptr, ev_b = nullptr;
    cudaStream_t aux = nullptr;        // second stream: trans_kernel(l+1) overlaps step(l)
    cudaEvent_t ev_tr[4] = {}, ev_st[4] = {}, ev_w = nullptr;
    double sweep_ms = 0.0, step_ms = 0.0;
    int64_t launches = 0;
    int64_t h2d_bytes = 0, d2h_bytes = 0;
    int64_t last_cell_updates = 0, last_effective = 0, last_useful = 0, last_segs = 0;
    int64_t last_load_bytes = 0, last_store_bytes = 0;   // step kernel: source segments in, rows out
    int per_launch_timing = 0;
    int kernel = -1;          // MADPIPE_KERNEL: v1 = plain loads, persist, pair (1 = retired per-tile TMA);
                              // -1 (default): pair for P > 33 (n_mem <= 8), else persist
                              // when a row segment is >= 1 KB, else v1
    int prof = 0;             // MADPIPE_PROF=1: cycle counters of the persistent step kernel to stderr
    int n_prod = 4;           // MADPIPE_NPROD: producer warps of the persistent step kernel (1..4)
    int tile_block = 1;       // MADPIPE_TILE_BLOCK: consecutive tiles per interleaved block (1 = round-robin)
    // MADPIPE_AUX_GRID=t,f: persistent grids of t and f blocks per SM for the pair path's list
    // builder and fixup kernels (they run side by side on two streams; 0 = one block per item)
    int aux_grid_trans = 0, aux_grid_fix = 0;
    int replay_pass = -1, replay_reps = 0, replay_diag = 0;
    int pass_timing = 0;
    int pair_min_p = 16;      // MADPIPE_PAIR_MIN_P: smallest P dispatched to the two-layer kernel      // MADPIPE_PASS_TIMING=1: per-pass step / fixup / list-builder / gap times to stderr   // MADPIPE_REPLAY=pass,reps,diag (diagnostic)
    int trans_overlap = 0;    // MADPIPE_TRANS_OVERLAP=1: pair path builds pass i+1's lists beside step(i) (measured
                              // slower at GPT: 909 vs 886 ms, 5% more entries kept unverified + contention)
    DevBuf profbuf;
    int num_sms = 148;
    int n_rec = 0;            // step-kernel launches bracketed by per-launch events in the last batch
    int last_kernel = -1;     // step kernel of the largest batch of the last timed sweep
    int last_kernel_jobs = 0;
    std::vector<cudaEvent_t> ev_pool;
    // multi-GPU: this process's rank of `world`, and the NCCL communicator
    // over which a7 (the min-reduction) and the batch's result all-gather run
    int32_t rank = 0, world = 1;
    void *comm = nullptr;
    DevBuf gather;
};

static thread_local std::string g_err;

// NVTX ranges per phase of the path (a1 prep, a2-a6 sweep batches, a7 all-reduce, a8 resolve
// + traceback, batch plan / all-gather): header-only NVTX v3, a no-op unless a tool
// (nsys, ncu --nvtx) attaches.
struct Nvtx {
    explicit Nvtx(const char *name) { nvtxRangePushA(name); }
    ~Nvtx() { nvtxRangePop(); }
};

static int fail(madpipe_ctx *ctx, int code, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (ctx) ctx->err = buf;
    g_err = buf;
    return code;
}

#define CUDA_TRY(ctx, expr)                                                                   \
    do {                                                                                      \
        cudaError_t _e = (expr);                                                              \
        if (_e != cudaSuccess)                                                                \
            return fail(ctx, _e == cudaErrorMemoryAllocation ? MADPIPE_ENOMEM : MADPIPE_ECUDA, \
                        "%s: %s (%s:%d)", #expr, cudaGetErrorString(_e), __FILE__, __LINE__); \
    } while (0)

// All host<->device traffic of the library goes through these two counters
// (reported by madpipe_last_io for the bench's e2e record).
static cudaError_t h2d(madpipe_ctx *ctx, void *dst, const void *src, size_t bytes) {
    ctx->h2d_bytes += (int64_t)bytes;
    return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, ctx->stream);
}
static cudaError_t d2h(madpipe_ctx *ctx, void *dst, const void *src, size_t bytes) {
    ctx->d2h_bytes += (int64_t)bytes;
    return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, ctx->stream);
}

static int fill_int_max(madpipe_ctx *ctx, int32_t *dev, size_t n) {
    std::vector<int32_t> h(n, INT32_MAX);
    CUDA_TRY(ctx, h2d(ctx, dev, h.data(), sizeof(int32_t) * n));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return MADPIPE_OK;
}

static int nmp_of(int n_m) {
    int n = 2;
    while (n < n_m) n <<= 1;
    return n;
}

// ---------------------------------------------------------------------------
// host-only helpers
// ---------------------------------------------------------------------------
static int validate_impl(const madpipe_chain *ch, int32_t P, int64_t M, double beta,
                         const madpipe_disc *disc, bool host_arrays, std::string *why) {
    auto bad = [&](const char *msg) { if (why) *why = msg; return MADPIPE_EINVAL; };
    if (!ch || !disc) return bad("null chain or disc");
    if (ch->L < 1) return bad("L < 1");
    if (P < 1) return bad("P < 1");
    if (M <= 0) return bad("M <= 0");
    if (!(beta > 0.0)) return bad("beta must be > 0 (and not NaN)");
    if (disc->n_mem < 2 || disc->n_mem > 64) return bad("n_mem outside [2, 64]");
    if (disc->n_delay < 2 || disc->n_delay > 65535) return bad("n_delay outside [2, 65535]");
    if (disc->n_periods < 1) return bad("n_periods < 1");
    if (disc->v_range != 0 && disc->v_range != 1) return bad("v_range not in {0,1}");
    if (!ch->uF || !ch->uB || !ch->W || !ch->a) return bad("null chain array");
    if (!host_arrays) return MADPIPE_OK;   // device arrays are checked by the caller
    const int L = ch->L;
    double U = 0.0, SC = 0.0;
    long double sumW = 0, sumA = 0;
    for (int i = 0; i < L; i++) {
        const double f = ch->uF[i], b = ch->uB[i];
        if (!std::isfinite(f) || !std::isfinite(b) || f < 0.0 || b < 0.0 || !(f + b > 0.0))
            return bad("uF/uB must be finite, >= 0, with uF+uB > 0");
        if (ch->W[i] < 0) return bad("W < 0");
        U += f + b;
        sumW += (long double)ch->W[i];
    }
    for (int i = 0; i <= L; i++) {
        if (ch->a[i] < 0) return bad("a < 0");
        if (i < L) sumA += (long double)ch->a[i];
        if (i >= 1 && i <= L - 1) SC += 2.0 * (double)ch->a[i] / beta;
    }
    // overflow guards of the int64 memory model: g <= gmax
    const double lb = U / P;
    const double vmax = 2.0 * (U + SC) + (U + SC);      // SAFE range at tau = ub (largest)
    const long double gmax = std::ceil((vmax + U) / lb) + 2.0;
    const long double worst = 3.0L * sumW + gmax * sumA +
                              4.0L * (long double)*std::max_element(ch->a, ch->a + L + 1);
    const long double lim = 9.0e18L;   // < 2^63
    if (!(worst < lim)) return bad("int64 overflow guard: 3*sum W + g_max*sum a too large");
    if (!((long double)(M - 1) + (long double)(disc->n_mem - 1) * worst < lim))
        return bad("int64 overflow guard: (M-1) + (n_mem-1)*memory too large");
    return MADPIPE_OK;
}

extern "C" int madpipe_validate(const madpipe_chain *chain, int32_t P, int64_t M, double beta,
                                const madpipe_disc *disc) {
    std::string why;
    int rc = validate_impl(chain, P, M, beta, disc, true, &why);
    if (rc) g_err = why;
    return rc;
}

extern "C" int madpipe_shard(int32_t n_periods, int32_t rank, int32_t world, int32_t *out,
                             int32_t *count) {
    if (n_periods < 1 || world < 1 || rank < 0 || rank >= world || !count)
        return fail(nullptr, MADPIPE_EINVAL, "bad shard arguments");
    int32_t c = 0;
    for (int32_t j = rank; j < n_periods; j += world) {
        if (out) out[c] = j;
        c++;
    }
    *count = c;
    return MADPIPE_OK;
}

extern "C" int64_t madpipe_cell_updates(const madpipe_chain *ch, int32_t P,
                                        const madpipe_disc *disc, double tau) {
    if (!ch || !disc || ch->L < 1 || P < 1) return -1;
    if (P < 2) return 0;
    const int L = ch->L;
    std::vector<double> Up(L + 1, 0.0);
    for (int i = 1; i <= L; i++) Up[i] = Up[i - 1] + (ch->uF[i - 1] + ch->uB[i - 1]);
    int64_t total = 0;
    int k = 1;
    for (int l = 1; l <= L; l++) {          // two-pointer scan: kmin(l) is non-decreasing in l
        if (k > l) k = l;
        while (k <= l && Up[l] - Up[k - 1] > tau) k++;
        if (k <= l) total += (int64_t)(l - k + 1);
    }
    return total * (int64_t)(P - 1) * disc->n_delay * disc->n_mem;
}

extern "C" const char *madpipe_last_error(const madpipe_ctx *ctx) {
    return ctx ? ctx->err.c_str() : g_err.c_str();
}

// ---------------------------------------------------------------------------
// context
// ---------------------------------------------------------------------------
extern "C" int madpipe_get_unique_id(uint8_t id[128]) {
    if (!id) return fail(nullptr, MADPIPE_EINVAL, "null id");
    std::string why;
    if (comm_unique_id(id, &why)) return fail(nullptr, MADPIPE_ENCCL, "%s", why.c_str());
    return MADPIPE_OK;
}

extern "C" int madpipe_ctx_create(madpipe_ctx **out, int device, int32_t rank, int32_t world,
                                  const uint8_t *nccl_id, void *cuda_stream, int64_t mem_budget) {
    if (!out) return fail(nullptr, MADPIPE_EINVAL, "null out");
    *out = nullptr;
    if (world < 1 || rank < 0 || rank >= world) return fail(nullptr, MADPIPE_EINVAL, "bad rank %d / world %d", rank, world);
    if (world > 1 && !nccl_id) return fail(nullptr, MADPIPE_EINVAL, "world > 1 needs an NCCL id");
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n == 0)
        return fail(nullptr, MADPIPE_ECUDA, "no CUDA device: %s", cudaGetErrorString(e));
    if (device < 0 || device >= n) return fail(nullptr, MADPIPE_EINVAL, "bad device %d", device);
    e = cudaSetDevice(device);
    if (e != cudaSuccess) return fail(nullptr, MADPIPE_ECUDA, "cudaSetDevice: %s", cudaGetErrorString(e));
    madpipe_ctx *c = new madpipe_ctx();
    c->device = device;
    c->rank = rank;
    c->world = world;
    if (nccl_id) {
        std::string why;
        if (comm_init(&c->comm, world, rank, nccl_id, &why)) {
            delete c;
            return fail(nullptr, MADPIPE_ENCCL, "%s", why.c_str());
        }
    }
    if (cuda_stream) {
        c->stream = (cudaStream_t)cuda_stream;
    } else {
        if (cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking) != cudaSuccess) {
            comm_destroy(c->comm);
            delete c;
            return fail(nullptr, MADPIPE_ECUDA, "cudaStreamCreate failed");
        }
        c->own_stream = true;
    }
    size_t fr = 0, tot = 0;
    cudaMemGetInfo(&fr, &tot);
    c->mem_budget = mem_budget > 0 ? mem_budget : (int64_t)(0.6 * (double)fr);
    const char *kern = getenv("MADPIPE_KERNEL");
    if (kern && strcmp(kern, "v1") == 0) c->kernel = 0;
    if (kern && strcmp(kern, "persist") == 0) c->kernel = 2;
    if (kern && strcmp(kern, "pair") == 0) c->kernel = 3;
    cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device);
    const char *pf = getenv("MADPIPE_PROF");
    c->prof = pf && pf[0] == '1';
    if (const char *e = getenv("MADPIPE_NPROD")) c->n_prod = std::max(1, std::min(4, atoi(e)));
    if (const char *e = getenv("MADPIPE_TILE_BLOCK")) c->tile_block = std::max(1, atoi(e));
    if (const char *e = getenv("MADPIPE_TRANS_OVERLAP")) c->trans_overlap = std::max(0, std::min(2, atoi(e)));
    if (const char *e = getenv("MADPIPE_PASS_TIMING")) c->pass_timing = atoi(e) != 0;
    if (const char *e = getenv("MADPIPE_PAIR_MIN_P")) c->pair_min_p = std::max(2, atoi(e));
    if (const char *e = getenv("MADPIPE_REPLAY")) sscanf(e, "%d,%d,%d", &c->replay_pass, &c->replay_reps, &c->replay_diag);
    if (const char *e = getenv("MADPIPE_AUX_GRID")) {
        int t = 0, f = 0;
        if (sscanf(e, "%d,%d", &t, &f) == 2) { c->aux_grid_trans = t * c->num_sms; c->aux_grid_fix = f * c->num_sms; }
    }
    cudaEventCreate(&c->ev_a);
    cudaEventCreate(&c->ev_b);
    cudaStreamCreateWithFlags(&c->aux, cudaStreamNonBlocking);
    for (int i = 0; i < 4; i++) {
        cudaEventCreateWithFlags(&c->ev_tr[i], cudaEventDisableTiming);
        cudaEventCreateWithFlags(&c->ev_st[i], cudaEventDisableTiming);
    }
    cudaEventCreateWithFlags(&c->ev_w, cudaEventDisableTiming);
    *out = c;
    return MADPIPE_OK;
}

extern "C" void madpipe_ctx_destroy(madpipe_ctx *c) {
    if (!c) return;
    cudaSetDevice(c->device);
    cudaStreamSynchronize(c->stream);
    c->profbuf.release();
    c->tdesc.release();
    DevBuf *bufs[] = {&c->tables, &c->jobs, &c->tiles, &c->chains, &c->chain_data, &c->jl,
                      &c->counts, &c->roots, &c->trace, &c->stages, &c->scratch, &c->codes, &c->flags, &c->tlist};
    for (DevBuf *b : bufs) b->release();
    for (cudaEvent_t ev : c->ev_pool) cudaEventDestroy(ev);
    if (c->aux) { cudaStreamSynchronize(c->aux); cudaStreamDestroy(c->aux); }
    for (int i = 0; i < 4; i++) {
        if (c->ev_tr[i]) cudaEventDestroy(c->ev_tr[i]);
        if (c->ev_st[i]) cudaEventDestroy(c->ev_st[i]);
    }
    if (c->ev_w) cudaEventDestroy(c->ev_w);
    if (c->ev_a) cudaEventDestroy(c->ev_a);
    if (c->ev_b) cudaEventDestroy(c->ev_b);
    if (c->own_stream) cudaStreamDestroy(c->stream);
    c->gather.release();
    comm_destroy(c->comm);
    delete c;
}

extern "C" int madpipe_ctx_info(const madpipe_ctx *c, int32_t *rank, int32_t *world, int32_t *nccl_version) {
    if (!c) return MADPIPE_EINVAL;
    if (rank) *rank = c->rank;
    if (world) *world = c->world;
    if (nccl_version) *nccl_version = c->comm ? comm_version() : 0;
    return MADPIPE_OK;
}

extern "C" int madpipe_last_timing(const madpipe_ctx *c, double *sweep_ms, double *step_ms,
                                   int64_t *launches) {
    if (!c) return MADPIPE_EINVAL;
    if (sweep_ms) *sweep_ms = c->sweep_ms;
    if (step_ms) *step_ms = c->step_ms;
    if (launches) *launches = c->launches;
    return MADPIPE_OK;
}

extern "C" int madpipe_last_counts(const madpipe_ctx *c, int64_t *cell_updates,
                                   int64_t *effective_updates, int64_t *useful_updates) {
    if (!c) return MADPIPE_EINVAL;
    if (cell_updates) *cell_updates = c->last_cell_updates;
    if (effective_updates) *effective_updates = c->last_effective;
    if (useful_updates) *useful_updates = c->last_useful;
    return MADPIPE_OK;
}

extern "C" int madpipe_last_step_bytes(const madpipe_ctx *c, int64_t *load_bytes, int64_t *store_bytes,
                                       int64_t *segments) {
    if (!c) return MADPIPE_EINVAL;
    if (load_bytes) *load_bytes = c->last_load_bytes;
    if (store_bytes) *store_bytes = c->last_store_bytes;
    if (segments) *segments = c->last_segs;
    return MADPIPE_OK;
}

extern "C" int madpipe_last_kernel(const madpipe_ctx *c, int32_t *kernel) {
    if (!c || !kernel) return MADPIPE_EINVAL;
    *kernel = c->last_kernel;
    return MADPIPE_OK;
}

extern "C" int madpipe_last_io(const madpipe_ctx *c, int64_t *h2d_bytes, int64_t *d2h_bytes) {
    if (!c) return MADPIPE_EINVAL;
    if (h2d_bytes) *h2d_bytes = c->h2d_bytes;
    if (d2h_bytes) *d2h_bytes = c->d2h_bytes;
    return MADPIPE_OK;
}

extern "C" int madpipe_set_timing(madpipe_ctx *c, int per_launch) {
    if (!c) return MADPIPE_EINVAL;
    c->per_launch_timing = per_launch;
    return MADPIPE_OK;
}

// ---------------------------------------------------------------------------
// Engine
// ---------------------------------------------------------------------------
namespace {

struct ChainSpec {
    madpipe_chain c;    // host or device pointers
    bool on_device;
    int32_t P;
    int64_t M;
    double beta;
};

struct JobSpec {
    int chain;
    int j;
};

// Upload chains (if on host), allocate derived arrays, run prep_kernel.
int upload_chains(madpipe_ctx *ctx, const std::vector<ChainSpec> &cs, std::vector<ChainDev> &cd) {
    Nvtx nv("madpipe a1 prep");
    const int n = (int)cs.size();
    size_t bytes = 0;
    auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
    for (const auto &c : cs) {
        const size_t L = (size_t)c.c.L;
        if (!c.on_device) bytes += al(L * 8) * 3 + al((L + 1) * 8);   // uF, uB, W, a
        bytes += al((L + 1) * 8) * 4 + al(4 * 8);                     // Up, Wp, Ap, C, scal
    }
    CUDA_TRY(ctx, ctx->chain_data.ensure(bytes));
    CUDA_TRY(ctx, ctx->chains.ensure(sizeof(ChainDev) * n));
    char *base = (char *)ctx->chain_data.p;
    size_t off = 0;
    auto take = [&](size_t b) { char *p = base + off; off += al(b); return (void *)p; };
    cd.resize(n);
    // host staging of the inputs: one pinned-free contiguous copy per chain
    for (int i = 0; i < n; i++) {
        const auto &c = cs[i];
        const size_t L = (size_t)c.c.L;
        ChainDev &d = cd[i];
        if (c.on_device) {
            d.uF = c.c.uF; d.uB = c.c.uB; d.W = c.c.W; d.a = c.c.a;
        } else {
            double *uF = (double *)take(L * 8), *uB = (double *)take(L * 8);
            int64_t *W = (int64_t *)take(L * 8), *a = (int64_t *)take((L + 1) * 8);
            CUDA_TRY(ctx, h2d(ctx, uF, c.c.uF, L * 8));
            CUDA_TRY(ctx, h2d(ctx, uB, c.c.uB, L * 8));
            CUDA_TRY(ctx, h2d(ctx, W, c.c.W, L * 8));
            CUDA_TRY(ctx, h2d(ctx, a, c.c.a, (L + 1) * 8));
            d.uF = uF; d.uB = uB; d.W = W; d.a = a;
        }
        d.Up = (double *)take((L + 1) * 8);
        d.Wp = (int64_t *)take((L + 1) * 8);
        d.Ap = (int64_t *)take((L + 1) * 8);
        d.C = (double *)take((L + 1) * 8);
        d.scal = (double *)take(4 * 8);
        d.L = c.c.L; d.P = c.P; d.M = c.M; d.beta = c.beta;
    }
    CUDA_TRY(ctx, h2d(ctx, ctx->chains.p, cd.data(), sizeof(ChainDev) * n));
    launch_prep((ChainDev *)ctx->chains.p, n, ctx->stream);
    ctx->launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    return MADPIPE_OK;
}

size_t table_doubles(const ChainSpec &c, const madpipe_disc *disc) {
    return (size_t)(c.c.L + 1) * (size_t)disc->n_delay * (size_t)c.P * (size_t)nmp_of(disc->n_mem);
}

// Tile geometry of one job on the plain-load kernel: np processor rows x vb delay rows,
// one thread each, for CTAs of `threads` threads (128 when every chain of the batch has
// P <= 16, so that small tiles do not leave most of a 256-thread CTA idle).
void tile_geom(int P, int n_v, int threads, int *vb, int *np, int *n_ptiles, int *n_tiles) {
    const int rows = std::max(1, P - 1);
    *np = std::min(rows, threads);
    *n_ptiles = (rows + *np - 1) / *np;
    *vb = std::max(1, std::min(n_v, threads / *np));
    *n_tiles = ((n_v + *vb - 1) / *vb) * *n_ptiles;
}

// Step kernel of a job (measured): the persistent TMA kernel moves one row
// segment per stage, which pays off from ~1 KB segments; below, plain loads win; the
// two-layer kernel where it measured faster: P > 33 at GPT shape (profiles/r01_pair_dispatch.md),
// with its one-row-per-thread mode for tiles of <= 32 processors from P = 17 on the config-5
// batch (profiles/r02_batch.md), and from P = 16 in round 2b (Inception/VGG shapes 214 / 33 ms
// vs 224 / 35 ms with the single-layer kernel, config 5 13.3 vs 13.7 s; MADPIPE_PAIR_MIN_P),
// n_mem <= 8.  MADPIPE_KERNEL forces one (falling back where it does not apply).
int step_kernel_for(const madpipe_ctx *ctx, int P, int nmp, int n_v, int all_maxL) {
    int k = ctx->kernel;
    if (k == 3 && !pair_supported(P, nmp, n_v, all_maxL)) k = -1;
    if (k < 0) {
        int vb_, np_, npt_, nt_;
        persist_geom(P, n_v, nmp, &vb_, &np_, &npt_, &nt_);
        k = (np_ + 1) * nmp * 8 >= 1024 ? 2 : 0;
        if (P >= ctx->pair_min_p && pair_supported(P, nmp, n_v, all_maxL)) k = 3;
    }
    return k;
}

struct BatchHook {
    // called after each batch's tables are complete (before they are reused)
    virtual int after_batch(madpipe_ctx *ctx, const std::vector<int> &job_ids, Job *jobs_dev) {
        (void)ctx; (void)job_ids; (void)jobs_dev;
        return MADPIPE_OK;
    }
    virtual ~BatchHook() {}
};

// Run the DP for a list of jobs in memory-bounded batches.  jl_dev[chain] gets
// atomicMin'ed with feasible candidate indices; roots_dev (optional) receives
// each job's root value at its index in `jobs`.  counts_host receives each
// job's relaxation count.  With early_exit, jobs whose chain already has a
// smaller feasible candidate are skipped (decided between batches).
int run_jobs(madpipe_ctx *ctx, const std::vector<ChainSpec> &cs, const std::vector<ChainDev> &cd,
             const madpipe_disc *disc, const std::vector<JobSpec> &js, int32_t *jl_dev,
             double *roots_dev, double *taus_dev, std::vector<uint64_t> *counts_host, bool early_exit,
             BatchHook *hook, bool timed) {
    const int nmp = nmp_of(disc->n_mem);
    const int n_chains = (int)cs.size();
    if (counts_host) counts_host->assign(js.size(), 0);
    std::vector<int32_t> jl_host(n_chains, INT32_MAX);
    size_t next = 0;
    if (timed) {
        ctx->sweep_ms = 0.0; ctx->step_ms = 0.0;
        ctx->last_cell_updates = 0; ctx->last_effective = 0; ctx->last_useful = 0; ctx->last_segs = 0;
        ctx->last_kernel = -1; ctx->last_kernel_jobs = 0;
        ctx->last_load_bytes = 0; ctx->last_store_bytes = 0;
    }
    std::vector<Job> hjobs;
    std::vector<int32_t> htiles;
    std::vector<int> ids;
    std::vector<unsigned long long> hcounts;
    const size_t budget = (size_t)ctx->mem_budget;
    // early exit: small first batches that double (time-to-placement); otherwise as
    // many jobs as the table budget holds
    size_t cap_jobs = early_exit ? (size_t)std::max(8, 2 * n_chains) : SIZE_MAX;
    int all_maxL = 1;
    for (const auto &c : cs) all_maxL = std::max(all_maxL, (int)c.c.L);
    while (next < js.size()) {
        // ---- form a batch
        hjobs.clear(); htiles.clear(); ids.clear();
        auto kernel_for = [&](int P) { return step_kernel_for(ctx, P, nmp, disc->n_delay, all_maxL); };
        // CTA size of the plain-load kernel: 128 threads if every chain on it has P <= 17
        int v1_threads = 128;
        for (const auto &c : cs)
            if (c.P > 17 && kernel_for(c.P) == 0) v1_threads = kThreads;
        while (next < js.size() && early_exit && jl_host[js[next].chain] < js[next].j) next++;
        const int kern = next < js.size() ? kernel_for(cs[js[next].chain].P) : 0;
        size_t used = 0;
        int maxL = 0;
        size_t max_slab = 0;
        for (; next < js.size(); next++) {
            const JobSpec &s = js[next];
            if (early_exit && jl_host[s.chain] < s.j) continue;
            const ChainSpec &c = cs[s.chain];
            const size_t bytes = table_doubles(c, disc) * 8;
            if (!hjobs.empty() && (used + bytes > budget || hjobs.size() >= cap_jobs)) break;
            // one step kernel per launch; chains of different P share it (each job carries
            // its own tile geometry) except on the single-layer persistent kernel, whose
            // ring and tile shape are set per launch
            if (!hjobs.empty() && (kernel_for(c.P) != kern || (kern == 2 && c.P != hjobs[0].P))) break;
            if (hjobs.empty() && bytes > budget && bytes > ctx->tables.n) {
                // a single job larger than the budget: try anyway (may fail with ENOMEM)
            }
            Job J{};
            const ChainDev &d = cd[s.chain];
            J.Up = d.Up; J.Wp = d.Wp; J.Ap = d.Ap; J.a = d.a; J.C = d.C; J.scal = d.scal;
            J.table = (double *)(uintptr_t)used;   // offset, patched below
            J.M = c.M; J.L = c.c.L; J.P = c.P; J.n_v = disc->n_delay; J.n_m = disc->n_mem;
            J.vsafe = disc->v_range == MADPIPE_VRANGE_SAFE; J.j = s.j; J.n_c = disc->n_periods;
            J.chain = s.chain;
            J.gid = (int32_t)next;
            int n_tiles;
            if (kern == 3) {
                int nvt;
                pair_geom(c.P, disc->n_delay, &J.np, &J.n_ptiles, &nvt, &n_tiles);
                J.vb = 0;
            } else if (kern == 2) {
                persist_geom(c.P, disc->n_delay, nmp, &J.vb, &J.np, &J.n_ptiles, &n_tiles);
            } else {
                tile_geom(c.P, disc->n_delay, v1_threads, &J.vb, &J.np, &J.n_ptiles, &n_tiles);
            }
            J.tile0 = (int32_t)htiles.size();
            for (int t = 0; t < n_tiles; t++) htiles.push_back((int32_t)hjobs.size());
            used += (bytes + 255) & ~(size_t)255;
            maxL = std::max(maxL, J.L);
            max_slab = std::max(max_slab, (size_t)disc->n_delay * c.P * nmp);
            hjobs.push_back(J);
            ids.push_back((int)next);
        }
        if (hjobs.empty()) break;
        char nv_name[96];
        snprintf(nv_name, sizeof nv_name, "madpipe a2-a6 batch: %d jobs, P=%d, kernel %d", (int)hjobs.size(),
                 hjobs[0].P, kern);
        Nvtx nv(nv_name);
        if (cap_jobs != SIZE_MAX) cap_jobs *= 2;
        CUDA_TRY(ctx, ctx->tables.ensure(used));
        for (auto &J : hjobs) J.table = (double *)((char *)ctx->tables.p + (uintptr_t)J.table);
        const int nj = (int)hjobs.size();
        CUDA_TRY(ctx, ctx->jobs.ensure(sizeof(Job) * nj));
        CUDA_TRY(ctx, ctx->tiles.ensure(sizeof(int32_t) * htiles.size()));
        CUDA_TRY(ctx, ctx->counts.ensure(sizeof(unsigned long long) * 4 * nj + sizeof(int32_t) * nj));
        for (int i = 0; i < nj; i++) {
            hjobs[i].eff = (unsigned long long *)ctx->counts.p + nj + i;
            hjobs[i].useful = (unsigned long long *)ctx->counts.p + 2 * nj + i;
            hjobs[i].segs = (unsigned long long *)ctx->counts.p + 3 * nj + i;
            hjobs[i].kmin_l = (int32_t *)((unsigned long long *)ctx->counts.p + 4 * nj) + i;
        }
        int n_v_max = 0;
        size_t list_buf_entries = 0, cnt_buf_entries = 0;
        if (kern == 3) {
            // merged two-layer lists: [job][v-tile][cap] PairEntry + [job][v-tile] counts, two buffers
            const int cap = pair_list_cap(maxL);
            size_t total = 0, vtotal = 0;
            for (auto &J : hjobs) {
                int np_, npt_, nvt_, nt_;
                pair_geom(J.P, J.n_v, &np_, &npt_, &nvt_, &nt_);
                total += (size_t)nvt_ * (size_t)cap;
                vtotal += (size_t)nvt_;
                n_v_max = std::max(n_v_max, J.n_v);
            }
            CUDA_TRY(ctx, ctx->tlist.ensure(2 * total * pair_entry_bytes()));
            // option k = l+1 transitions of the layer-(l+1) rows: [job][2][n_v]
            size_t voff_fx = 0;
            CUDA_TRY(ctx, ctx->codes.ensure(2 * (size_t)nj * (size_t)disc->n_delay * sizeof(int32_t)));
            list_buf_entries = total;
            cnt_buf_entries = vtotal;
            size_t off = 0, voff = 0, ftotal = 0, wtotal = 0;
            // tile descriptors: (list offset of the tile's v-tile, processor tile)
            std::vector<int32_t> hdesc(2 * htiles.size());
            for (auto &J : hjobs) {
                int np_, npt_, nvt_, nt_;
                pair_geom(J.P, J.n_v, &np_, &npt_, &nvt_, &nt_);
                J.tlist = (TransEntry *)((char *)ctx->tlist.p + off * pair_entry_bytes());
                J.tcount = nullptr;
                J.code_cap = cap;
                J.codes = (int32_t *)ctx->codes.p + 2 * (size_t)voff_fx;
                voff_fx += (size_t)J.n_v;
                for (int vt = 0; vt < nvt_; vt++)
                    for (int pt = 0; pt < npt_; pt++) {
                        const size_t t = (size_t)J.tile0 + (size_t)vt * npt_ + pt;
                        hdesc[2 * t] = (int32_t)(off + (size_t)vt * cap);
                        hdesc[2 * t + 1] = pt;
                    }
                off += (size_t)nvt_ * (size_t)cap;
                voff += (size_t)nvt_;
                ftotal += (size_t)(J.L + 1) * (size_t)J.n_v;
                wtotal += (size_t)(J.L + 1);
            }
            CUDA_TRY(ctx, ctx->flags.ensure(ftotal * sizeof(uint32_t) + wtotal * sizeof(int32_t)));
            size_t foff = 0, woff = 0;
            int32_t *wbase = (int32_t *)((uint32_t *)ctx->flags.p + ftotal);
            for (auto &J : hjobs) {
                J.rowflag = (uint32_t *)ctx->flags.p + foff;
                foff += (size_t)(J.L + 1) * (size_t)J.n_v;
                J.kwin = wbase + woff;
                woff += (size_t)(J.L + 1);
            }
            if (off > (size_t)INT32_MAX) return fail(ctx, MADPIPE_ENOMEM, "pair lists exceed 2^31 entries");
            CUDA_TRY(ctx, ctx->tdesc.ensure(sizeof(int32_t) * hdesc.size()));
            CUDA_TRY(ctx, h2d(ctx, ctx->tdesc.p, hdesc.data(), sizeof(int32_t) * hdesc.size()));
        }
        if (kern == 2) {
            // useful-transition lists of one layer: [job][v][maxL] entries + [job][v] counts
            size_t total = 0, vtotal = 0;
            for (auto &J : hjobs) {
                total += (size_t)J.n_v * (size_t)maxL;
                vtotal += (size_t)J.n_v;
                n_v_max = std::max(n_v_max, J.n_v);
            }
            // two buffers (layers l and l+1 are live at once when trans(l+1) overlaps step(l))
            CUDA_TRY(ctx, ctx->tlist.ensure(2 * total * sizeof(TransEntry)));
            CUDA_TRY(ctx, ctx->codes.ensure(2 * vtotal * sizeof(int32_t)));
            list_buf_entries = total;
            size_t off = 0, voff = 0, ftotal = 0;
            for (auto &J : hjobs) {
                J.tlist = (TransEntry *)ctx->tlist.p + off;
                J.tcount = (int32_t *)ctx->codes.p + voff;
                J.code_cap = maxL;
                off += (size_t)J.n_v * (size_t)maxL;
                voff += (size_t)J.n_v;
                ftotal += (size_t)(J.L + 1) * (size_t)J.n_v;
            }
            size_t wtotal = 0;
            for (auto &J : hjobs) wtotal += (size_t)(J.L + 1);
            CUDA_TRY(ctx, ctx->flags.ensure(ftotal * sizeof(uint32_t) + wtotal * sizeof(int32_t)));
            size_t foff = 0, woff = 0;
            int32_t *wbase = (int32_t *)((uint32_t *)ctx->flags.p + ftotal);
            for (auto &J : hjobs) {
                J.rowflag = (uint32_t *)ctx->flags.p + foff;
                foff += (size_t)(J.L + 1) * (size_t)J.n_v;
                J.kwin = wbase + woff;
                woff += (size_t)(J.L + 1);
            }
        }
        Job *djobs = (Job *)ctx->jobs.p;
        CUDA_TRY(ctx, h2d(ctx, djobs, hjobs.data(), sizeof(Job) * nj));
        CUDA_TRY(ctx, h2d(ctx, ctx->tiles.p, htiles.data(), sizeof(int32_t) * htiles.size()));
        CUDA_TRY(ctx, cudaMemsetAsync(ctx->counts.p, 0, sizeof(unsigned long long) * 4 * nj, ctx->stream));
        if (timed) CUDA_TRY(ctx, cudaEventRecord(ctx->ev_a, ctx->stream));
        launch_jobs_init(djobs, nj, ctx->stream);
        launch_init_slab0(djobs, nj, nmp, (int)std::min(max_slab, (size_t)INT32_MAX), ctx->stream);
        ctx->launches += 2;
        const int n_tiles = (int)htiles.size();
        int persist_grid = 0, nsg = 0, p_np = 0, p_vb = 0;
        if (kern == 3) {
            for (const auto &J : hjobs) p_np = std::max(p_np, J.np);   // processor rows per tile
            nsg = pair_nsl(p_np, nmp);
            if (nsg < 4) return fail(ctx, MADPIPE_EINVAL, "row segment too large for the pair step kernel ring");
            persist_grid = std::min(n_tiles, ctx->num_sms * pair_blocks_per_sm(nmp, p_np, nsg));
        }
        if (kern == 2) {
            p_np = hjobs[0].np;
            p_vb = hjobs[0].vb;
            nsg = persist_nsg(p_np, p_vb, nmp);
            if (nsg < 2) return fail(ctx, MADPIPE_EINVAL, "row segment too large for the step kernel ring");
            persist_grid = std::min(n_tiles, ctx->num_sms * persist_blocks_per_sm(nmp, p_np, p_vb, nsg, ctx->n_prod));
        }
        const bool per_launch = timed && ctx->per_launch_timing;
        if (ctx->prof) {
            CUDA_TRY(ctx, ctx->profbuf.ensure(16 * sizeof(unsigned long long)));
            CUDA_TRY(ctx, cudaMemsetAsync(ctx->profbuf.p, 0, 16 * sizeof(unsigned long long), ctx->stream));
        }
        if (per_launch && ctx->ev_pool.size() < (size_t)(2 * maxL)) {
            while (ctx->ev_pool.size() < (size_t)(2 * maxL)) {
                cudaEvent_t ev;
                CUDA_TRY(ctx, cudaEventCreate(&ev));
                ctx->ev_pool.push_back(ev);
            }
        }
        if (kern == 3) {
            launch_window(djobs, nj, maxL, ctx->stream);
            ctx->launches++;
            int n_rec = 0;
            const int cap = pair_list_cap(maxL);
            // pass i covers layers l = 2i+1, l+1 with list buffer i % 2.
            // trans_overlap = 1 (MADPIPE_TRANS_OVERLAP=1; measured slower):
            //   stream: [wait trans(i)] (mark) step(i) -> fixup(i)
            //   aux:    [wait mark]     trans(i+1)     -- runs beside step(i)
            //   trans(i+1) needs the final slabs <= l-1 (fixup(i-1) precedes the mark) and keeps
            //   every live entry reading slabs l, l+1 unverified (unv_from = l); it writes list
            //   buffer (i+1) % 2, last read by step(i-1).
            // trans_overlap = 0 (default, round 1):
            //   aux:    [wait step(i)]  trans(i+1)     -- beside fixup(i); it reads the final flags of
            //   slabs <= l and, for slab l+1, a superset of what fixup(i) will flag (fix_slab).
            launch_pair_trans(djobs, nj, n_v_max, 1, nmp, 0, -1, INT_MAX, 0, ctx->stream);
            ctx->launches++;
            // MADPIPE_PASS_TIMING (diagnostic): events before/after each step, after each fixup (main
            // stream) and after each list build (aux stream)
            std::vector<cudaEvent_t> pt;
            const int n_pass = (maxL + 1) / 2;
            if (ctx->pass_timing) {
                pt.resize(4 * (size_t)n_pass);
                for (auto &e : pt) cudaEventCreate(&e);
            }
            for (int l = 1; l <= maxL; l += 2) {
                const int i = l >> 1, b = i & 1;
                if (i >= 1 && ctx->trans_overlap != 2) CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->stream, ctx->ev_tr[b], 0));
                if (ctx->trans_overlap == 1 && l + 2 <= maxL) {
                    CUDA_TRY(ctx, cudaEventRecord(ctx->ev_st[b], ctx->stream));
                    CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->aux, ctx->ev_st[b], 0));
                    launch_pair_trans(djobs, nj, n_v_max, l + 2, nmp, (size_t)(b ^ 1) * list_buf_entries, -1, l,
                                      0, ctx->aux);
                    CUDA_TRY(ctx, cudaEventRecord(ctx->ev_tr[b ^ 1], ctx->aux));
                    ctx->launches++;
                }
                if (i == ctx->replay_pass && ctx->replay_reps > 0) {
                    // diagnostic (MADPIPE_REPLAY=pass,reps,diag): this pass's step kernel
                    // re-launched on the same lists (it reads slabs <= l-1 and writes l, l+1: idempotent)
                    // and timed alone; with an MP_DIAG=1 build, diag bit 0 drops the relaxation and bit 1
                    // the copies in the re-launches only
                    cudaEvent_t e0, e1;
                    cudaEventCreate(&e0);
                    cudaEventCreate(&e1);
                    cudaEventRecord(e0, ctx->stream);
                    for (int rp = 0; rp < ctx->replay_reps; rp++)
                        launch_pair_step((const int2 *)ctx->tdesc.p, n_tiles, ctx->tlist.p, b * list_buf_entries, cap,
                                         nmp, p_np, nsg, persist_grid, nullptr, ctx->stream, ctx->replay_diag);
                    cudaEventRecord(e1, ctx->stream);
                    cudaEventSynchronize(e1);
                    float ms = 0.f;
                    cudaEventElapsedTime(&ms, e0, e1);
                    fprintf(stderr, "[madpipe replay] pass %d, diag %d, %d jobs, %d tiles: %.4f ms per step launch\n", i,
                            ctx->replay_diag, nj, n_tiles, ms / ctx->replay_reps);
                    cudaEventDestroy(e0);
                    cudaEventDestroy(e1);
                }
                if (per_launch) cudaEventRecord(ctx->ev_pool[2 * n_rec], ctx->stream);
                if (ctx->pass_timing) cudaEventRecord(pt[4 * i], ctx->stream);
                launch_pair_step((const int2 *)ctx->tdesc.p, n_tiles, ctx->tlist.p, b * list_buf_entries, cap, nmp,
                                 p_np, nsg, persist_grid,
                                 (unsigned long long *)(ctx->prof ? ctx->profbuf.p : nullptr),
                                 ctx->stream);
                if (per_launch) cudaEventRecord(ctx->ev_pool[2 * n_rec + 1], ctx->stream);
                if (ctx->pass_timing) cudaEventRecord(pt[4 * i + 1], ctx->stream);
                n_rec++;
                ctx->launches++;
                if (ctx->trans_overlap == 0 && l + 2 <= maxL) {
                    CUDA_TRY(ctx, cudaEventRecord(ctx->ev_st[b], ctx->stream));
                    CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->aux, ctx->ev_st[b], 0));
                    launch_pair_trans(djobs, nj, n_v_max, l + 2, nmp, (size_t)(b ^ 1) * list_buf_entries, l + 1,
                                      INT_MAX, ctx->aux_grid_trans, ctx->aux);
                    CUDA_TRY(ctx, cudaEventRecord(ctx->ev_tr[b ^ 1], ctx->aux));
                    if (ctx->pass_timing) cudaEventRecord(pt[4 * i + 3], ctx->aux);
                    ctx->launches++;
                }
                if (l + 1 <= maxL) {
                    launch_pair_fixup(djobs, nj, n_v_max, l + 1, nmp, ctx->aux_grid_fix, ctx->stream);
                    ctx->launches++;
                }
                if (ctx->pass_timing) cudaEventRecord(pt[4 * i + 2], ctx->stream);
                if (ctx->trans_overlap == 2 && l + 2 <= maxL) {
                    // serial: the lists of pass i+1 after fixup(i) on the same stream (every flag final)
                    launch_pair_trans(djobs, nj, n_v_max, l + 2, nmp, (size_t)(b ^ 1) * list_buf_entries, -1, INT_MAX,
                                      ctx->aux_grid_trans, ctx->stream);
                    if (ctx->pass_timing) cudaEventRecord(pt[4 * i + 3], ctx->stream);
                    ctx->launches++;
                }
            }
            ctx->n_rec = n_rec;
            if (ctx->pass_timing) {
                cudaStreamSynchronize(ctx->stream);
                cudaStreamSynchronize(ctx->aux);
                double st = 0, fx = 0, tr = 0, gap = 0, crit = 0;
                for (int q = 0; q < n_pass; q++) {
                    float a = 0.f;
                    cudaEventElapsedTime(&a, pt[4 * q], pt[4 * q + 1]);
                    st += a;
                    cudaEventElapsedTime(&a, pt[4 * q + 1], pt[4 * q + 2]);
                    fx += a;
                    if (2 * q + 3 <= maxL) {
                        cudaEventElapsedTime(&a, pt[4 * q + 1], pt[4 * q + 3]);
                        tr += a;
                    }
                    if (q + 1 < n_pass) {
                        cudaEventElapsedTime(&a, pt[4 * q + 1], pt[4 * (q + 1)]);
                        crit += a;
                        cudaEventElapsedTime(&a, pt[4 * q + 2], pt[4 * (q + 1)]);
                        gap += a;
                    }
                }
                fprintf(stderr, "[madpipe pass timing] %d jobs, %d passes: step %.3f ms, step end -> fixup end %.3f ms, "
                        "step end -> next lists built %.3f ms, step end -> next step start %.3f ms, fixup end -> next step "
                        "start %.3f ms\n", nj, n_pass, st, fx, tr, crit, gap);
                for (auto &e : pt) cudaEventDestroy(e);
            }
        } else {
        if (kern == 2) {
            launch_window(djobs, nj, maxL, ctx->stream);
            ctx->launches++;
            CUDA_TRY(ctx, cudaEventRecord(ctx->ev_w, ctx->stream));
            CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->aux, ctx->ev_w, 0));
        }
        for (int l = 1; l <= maxL; l++) {
            const size_t buf_off = (size_t)(l & 1) * list_buf_entries;
            if (kern == 2) {
                // trans(l) on the aux stream, overlapping step(l-1): it needs step(l-2) done
                // (the flags of slabs <= l-2 and the list buffer l%2 it overwrites)
                if (l >= 3) CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->aux, ctx->ev_st[(l - 2) & 3], 0));
                launch_trans(djobs, nj, n_v_max, l, nmp, buf_off, /*verify_last=*/0, ctx->aux);
                ctx->launches++;
                CUDA_TRY(ctx, cudaEventRecord(ctx->ev_tr[l & 3], ctx->aux));
                CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->stream, ctx->ev_tr[l & 3], 0));
            }
            // per-launch events bracket the step kernel alone (bench roofline)
            if (per_launch) cudaEventRecord(ctx->ev_pool[2 * (l - 1)], ctx->stream);
            if (kern == 2)
                launch_step_persist(djobs, (const int32_t *)ctx->tiles.p, n_tiles, l, nmp, p_np, p_vb, nsg,
                                    persist_grid, (unsigned long long *)(ctx->prof ? ctx->profbuf.p : nullptr),
                                    ctx->n_prod, ctx->tile_block, buf_off, ctx->stream);
            else
                launch_step(djobs, (const int32_t *)ctx->tiles.p, n_tiles, l, nmp, v1_threads, ctx->stream);
            if (per_launch) cudaEventRecord(ctx->ev_pool[2 * (l - 1) + 1], ctx->stream);
            if (kern == 2) CUDA_TRY(ctx, cudaEventRecord(ctx->ev_st[l & 3], ctx->stream));
        }
        ctx->launches += maxL;
        ctx->n_rec = maxL;
        }
        launch_root(djobs, nj, nmp, jl_dev, roots_dev, taus_dev, ctx->stream);
        launch_count(djobs, nj, (unsigned long long *)ctx->counts.p, ctx->stream);
        ctx->launches += 2;
        CUDA_TRY(ctx, cudaGetLastError());
        if (timed) CUDA_TRY(ctx, cudaEventRecord(ctx->ev_b, ctx->stream));
        if (ctx->prof && timed && kern == 3) {
            unsigned long long pc[9];
            CUDA_TRY(ctx, cudaMemcpyAsync(pc, ctx->profbuf.p, sizeof pc, cudaMemcpyDeviceToHost, ctx->stream));
            CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
            const double g = (double)std::max(1, persist_grid);
            fprintf(stderr,
                    "[madpipe prof pair] batch of %d jobs, %d CTAs: producer %.3g cyc/CTA (empty waits %.1f%%, "
                    "tile setup %.1f%%, push %.1f%%), %.3g tiles/CTA; consumer %.3g cyc/warp (queue waits %.1f%%, full waits "
                    "%.1f%%), %.3g slot visits/warp\n",
                    nj, persist_grid, pc[0] / g, 100.0 * pc[1] / std::max(1ull, pc[0]),
                    100.0 * pc[2] / std::max(1ull, pc[0]), 100.0 * pc[8] / std::max(1ull, pc[0]), pc[7] / g, pc[3] / (g * 8),
                    100.0 * pc[4] / std::max(1ull, pc[3]), 100.0 * pc[5] / std::max(1ull, pc[3]), pc[6] / (g * 8));
        } else
        if (ctx->prof && timed) {
            unsigned long long pc[8];
            CUDA_TRY(ctx, cudaMemcpyAsync(pc, ctx->profbuf.p, sizeof pc, cudaMemcpyDeviceToHost, ctx->stream));
            CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
            fprintf(stderr,
                    "[madpipe prof] batch of %d jobs, %d CTAs: producer total %.3g cyc/CTA: setup %.1f%% "
                    "lists %.1f%% issue %.1f%% (empty waits %.1f%%); consumer warp0 waits on full %.1f%%; "
                    "tiles %llu\n",
                    nj, persist_grid, (double)pc[0] / std::max(1, persist_grid), 100.0 * pc[1] / std::max(1ull, pc[0]),
                    100.0 * pc[2] / std::max(1ull, pc[0]), 100.0 * pc[3] / std::max(1ull, pc[0]),
                    100.0 * pc[4] / std::max(1ull, pc[0]), 100.0 * pc[6] / std::max(1ull, pc[5]), pc[7]);
        }
        if (hook) {
            int rc = hook->after_batch(ctx, ids, djobs);
            if (rc) return rc;
        }
        hcounts.resize(4 * nj);
        CUDA_TRY(ctx, d2h(ctx, hcounts.data(), ctx->counts.p, sizeof(unsigned long long) * 4 * nj));
        if (early_exit)
            CUDA_TRY(ctx, d2h(ctx, jl_host.data(), jl_dev, sizeof(int32_t) * n_chains));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
        if (counts_host)
            for (int i = 0; i < nj; i++) (*counts_host)[ids[i]] = hcounts[i];
        if (timed) {
            for (int i = 0; i < nj; i++) {
                ctx->last_cell_updates += (int64_t)hcounts[i];
                ctx->last_effective += (int64_t)hcounts[nj + i];
                ctx->last_useful += (int64_t)hcounts[2 * nj + i];
                ctx->last_segs += (int64_t)hcounts[3 * nj + i];
                // algorithmic bytes of the step kernel: every source
                // segment it brings on chip -- (np+1) rows of nmp doubles per p-tile --
                // and every output row p >= 1 it stores
                const Job &J = hjobs[i];
                const int64_t rowb = (int64_t)nmp * 8;
                const int64_t seg = (int64_t)(J.P - 1 + J.n_ptiles) * rowb;
                if (kern == 3) ctx->last_load_bytes += (int64_t)hcounts[3 * nj + i] * seg;
                else if (kern == 2 && J.P > 1)
                    ctx->last_load_bytes += (int64_t)(hcounts[2 * nj + i] / ((uint64_t)(J.P - 1) * J.n_m)) * seg;
                ctx->last_store_bytes += (int64_t)J.L * J.n_v * (J.P - 1) * rowb;
            }
        }
        if (timed && nj > ctx->last_kernel_jobs) { ctx->last_kernel = kern; ctx->last_kernel_jobs = nj; }
        if (timed) {
            float ms = 0.f;
            cudaEventElapsedTime(&ms, ctx->ev_a, ctx->ev_b);
            ctx->sweep_ms += ms;
            double kms = 0.0;
            if (per_launch) {
                for (int l = 1; l <= ctx->n_rec; l++) {
                    float m2 = 0.f;
                    cudaEventElapsedTime(&m2, ctx->ev_pool[2 * (l - 1)], ctx->ev_pool[2 * (l - 1) + 1]);
                    kms += m2;
                }
                ctx->step_ms += kms;
            }
            if (ctx->prof) {
                uint64_t u = 0, e = 0;
                for (int i = 0; i < nj; i++) { u += hcounts[2 * nj + i]; e += hcounts[nj + i]; }
                fprintf(stderr, "[madpipe batch] P=%d jobs=%d maxL=%d kernel=%d tiles=%d: %.3f ms (step %.3f ms), "
                                "effective %.3g, useful %.3g\n",
                        hjobs[0].P, nj, maxL, kern, n_tiles, ms, kms, (double)e, (double)u);
            }
        }
    }
    return MADPIPE_OK;
}

// Traceback hook: after the winners' tables are built, trace them back.
struct TraceHook : BatchHook {
    int nmp, stride;
    std::vector<TraceOut> outs;
    std::vector<int32_t> stages;          // [job][3][stride]
    std::vector<double> taus;
    int after_batch(madpipe_ctx *ctx, const std::vector<int> &ids, Job *jobs_dev) override {
        const int nj = (int)ids.size();
        CUDA_TRY(ctx, ctx->trace.ensure(sizeof(TraceOut) * nj));
        CUDA_TRY(ctx, ctx->stages.ensure(sizeof(int32_t) * 3 * (size_t)stride * nj));
        launch_traceback(jobs_dev, nj, nmp, (TraceOut *)ctx->trace.p, (int32_t *)ctx->stages.p,
                         stride, ctx->stream);
        ctx->launches++;
        CUDA_TRY(ctx, cudaGetLastError());
        std::vector<TraceOut> o(nj);
        std::vector<int32_t> st(3 * (size_t)stride * nj);
        std::vector<Job> jb(nj);
        CUDA_TRY(ctx, d2h(ctx, o.data(), ctx->trace.p, sizeof(TraceOut) * nj));
        CUDA_TRY(ctx, d2h(ctx, st.data(), ctx->stages.p, sizeof(int32_t) * st.size()));
        CUDA_TRY(ctx, d2h(ctx, jb.data(), jobs_dev, sizeof(Job) * nj));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
        for (int i = 0; i < nj; i++) {
            outs[ids[i]] = o[i];
            taus[ids[i]] = jb[i].tau;
            std::copy(st.begin() + (size_t)i * 3 * stride, st.begin() + (size_t)(i + 1) * 3 * stride,
                      stages.begin() + (size_t)ids[i] * 3 * stride);
        }
        return MADPIPE_OK;
    }
};

// madpipe_alloc of candidate j from its traceback (period = tau_j, Q16)
void fill_from_trace(madpipe_alloc *o, int32_t j, double tau, const TraceOut &t, const int32_t *st, int stride) {
    o->period = tau;
    o->load_period = t.load_period;
    o->special_load = t.special_load;
    o->cand_index = j;
    o->n_stages = t.n_stages;
    for (int s = 0; s < t.n_stages; s++) {
        if (o->stage_first) o->stage_first[s] = st[s];
        if (o->stage_last) o->stage_last[s] = st[stride + s];
        if (o->stage_proc) o->stage_proc[s] = st[2 * stride + s];
    }
}

// One-rank sweeps (a8 without the re-solve): after each batch, every chain's smallest
// feasible candidate found so far is traced back straight from the batch's tables, before
// they are reused.  A chain's candidates run in ascending order (batch_sweep keeps them
// candidate-major), so the batch holding its final winner traces it.  jl_dev: the sweep's
// device int32[n_chains].
struct SweepTraceHook : BatchHook {
    int nmp = 0, stride = 1, n_chains = 0;
    const std::vector<JobSpec> *js = nullptr;   // the job list of the current run_jobs call
    const int32_t *jl_dev = nullptr;
    std::vector<int32_t> best;                  // per chain: the candidate traced so far
    std::vector<TraceOut> outs;
    std::vector<int32_t> stages;                // [chain][3][stride]
    std::vector<double> taus;
    void init(int n, int nmp_, int stride_, const int32_t *jl) {
        n_chains = n; nmp = nmp_; stride = std::max(1, stride_); jl_dev = jl;
        best.assign(n, INT32_MAX);
        outs.assign(n, TraceOut{});
        stages.assign(3 * (size_t)stride * n, 0);
        taus.assign(n, 0.0);
    }
    int after_batch(madpipe_ctx *ctx, const std::vector<int> &ids, Job *jobs_dev) override {
        std::vector<int32_t> jl(n_chains);
        CUDA_TRY(ctx, d2h(ctx, jl.data(), jl_dev, sizeof(int32_t) * n_chains));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
        std::vector<int> sel;                   // batch positions of newly found winners
        for (size_t i = 0; i < ids.size(); i++) {
            const JobSpec &s = (*js)[ids[i]];
            if (s.j == jl[s.chain] && jl[s.chain] < best[s.chain]) sel.push_back((int)i);
        }
        if (sel.empty()) return MADPIPE_OK;
        const int K = (int)sel.size(), nj = (int)ids.size();
        CUDA_TRY(ctx, ctx->trace.ensure(sizeof(TraceOut) * K));
        CUDA_TRY(ctx, ctx->stages.ensure(sizeof(int32_t) * 3 * (size_t)stride * K));
        for (int k = 0; k < K; k++) {
            launch_traceback(jobs_dev + sel[k], 1, nmp, (TraceOut *)ctx->trace.p + k,
                             (int32_t *)ctx->stages.p + 3 * (size_t)stride * k, stride, ctx->stream);
            ctx->launches++;
        }
        CUDA_TRY(ctx, cudaGetLastError());
        std::vector<TraceOut> o(K);
        std::vector<int32_t> st(3 * (size_t)stride * K);
        std::vector<Job> jb(nj);
        CUDA_TRY(ctx, d2h(ctx, o.data(), ctx->trace.p, sizeof(TraceOut) * K));
        CUDA_TRY(ctx, d2h(ctx, st.data(), ctx->stages.p, sizeof(int32_t) * st.size()));
        CUDA_TRY(ctx, d2h(ctx, jb.data(), jobs_dev, sizeof(Job) * nj));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
        for (int k = 0; k < K; k++) {
            const int c = (*js)[ids[sel[k]]].chain;
            outs[c] = o[k];
            taus[c] = jb[sel[k]].tau;
            best[c] = jl[c];
            std::copy(st.begin() + 3 * (size_t)stride * k, st.begin() + 3 * (size_t)stride * (k + 1),
                      stages.begin() + 3 * (size_t)stride * c);
        }
        return MADPIPE_OK;
    }
};

void fill_infeasible(madpipe_alloc *out, int64_t cu) {
    out->period = INFINITY;
    out->load_period = INFINITY;
    out->special_load = INFINITY;
    out->cand_index = -1;
    out->n_stages = 0;
    out->cell_updates = cu;
}

// Resolve the winners (one job per chain with jstar[c] != INT32_MAX).
int resolve_impl(madpipe_ctx *ctx, const std::vector<ChainSpec> &cs, const std::vector<ChainDev> &cd,
                 const madpipe_disc *disc, const std::vector<int32_t> &jstar, madpipe_alloc *outs) {
    Nvtx nv("madpipe a8 resolve + traceback");
    std::vector<JobSpec> js;
    int maxL = 1;
    for (int c = 0; c < (int)cs.size(); c++) {
        maxL = std::max(maxL, (int)cs[c].c.L);
        if (jstar[c] != INT32_MAX && jstar[c] >= 0) js.push_back({c, jstar[c]});
    }
    // group the winners by step kernel (and P on the single-layer persistent kernel), as
    // batch_sweep does, so that they run as a few batches and not one per kernel change
    {
        const int nmp = nmp_of(disc->n_mem);
        std::stable_sort(js.begin(), js.end(), [&](const JobSpec &a, const JobSpec &b) {
            const int ka = step_kernel_for(ctx, cs[a.chain].P, nmp, disc->n_delay, maxL);
            const int kb = step_kernel_for(ctx, cs[b.chain].P, nmp, disc->n_delay, maxL);
            const int ga = ka * 65536 + (ka == 2 ? cs[a.chain].P : 0), gb = kb * 65536 + (kb == 2 ? cs[b.chain].P : 0);
            return ga < gb;
        });
    }
    TraceHook hook;
    hook.nmp = nmp_of(disc->n_mem);
    hook.stride = maxL;
    hook.outs.assign(js.size(), TraceOut{});
    hook.stages.assign(js.size() * 3 * (size_t)maxL, 0);
    hook.taus.assign(js.size(), 0.0);
    CUDA_TRY(ctx, ctx->jl.ensure(sizeof(int32_t) * std::max<size_t>(1, cs.size())));
    { int _r = fill_int_max(ctx, (int32_t *)ctx->jl.p, cs.size()); if (_r) return _r; }
    if (!js.empty()) {
        int rc = run_jobs(ctx, cs, cd, disc, js, (int32_t *)ctx->jl.p, nullptr, nullptr, nullptr, false,
                          &hook, false);
        if (rc) return rc;
    }
    for (size_t i = 0; i < js.size(); i++) {
        madpipe_alloc *o = outs + js[i].chain;
        const TraceOut &t = hook.outs[i];
        if (t.status != 0)
            return fail(ctx, MADPIPE_ESTATE, "resolve of candidate %d: %s", js[i].j,
                        t.status == 1 ? "root is infeasible" : "traceback found no decision");
        fill_from_trace(o, js[i].j, hook.taus[i], t, hook.stages.data() + i * 3 * (size_t)maxL, maxL);
    }
    return MADPIPE_OK;
}

// true if p is device (or managed) memory of the current device
bool is_device_ptr(const void *p) {
    cudaPointerAttributes at{};
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

int begin(madpipe_ctx *ctx) {
    if (!ctx) return fail(nullptr, MADPIPE_EINVAL, "null ctx");
    ctx->err.clear();
    ctx->launches = 0;
    ctx->h2d_bytes = 0;
    ctx->d2h_bytes = 0;
    cudaError_t e = cudaSetDevice(ctx->device);
    if (e != cudaSuccess) return fail(ctx, MADPIPE_ECUDA, "cudaSetDevice: %s", cudaGetErrorString(e));
    return MADPIPE_OK;
}

int check_one(madpipe_ctx *ctx, const madpipe_chain *ch, int32_t P, int64_t M, double beta,
              const madpipe_disc *disc, bool host) {
    std::string why;
    int rc = validate_impl(ch, P, M, beta, disc, host, &why);
    if (rc) return fail(ctx, rc, "invalid argument: %s", why.c_str());
    return MADPIPE_OK;
}

std::vector<JobSpec> shard_jobs(int chain, int n_c, int rank, int world) {
    std::vector<JobSpec> js;
    for (int j = rank; j < n_c; j += world) js.push_back({chain, j});
    return js;
}

// a7: min-reduce n int32 candidate indices (device) over the ctx's communicator, on
// the ctx's stream.  Without a communicator (world 1) this is the identity.
int allreduce_min(madpipe_ctx *ctx, int32_t *dev, size_t n) {
    if (!ctx->comm) return MADPIPE_OK;
    Nvtx nv("madpipe a7 allreduce(MIN)");
    std::string why;
    if (comm_allreduce_min_i32(ctx->comm, dev, n, ctx->stream, &why))
        return fail(ctx, MADPIPE_ENCCL, "%s", why.c_str());
    return MADPIPE_OK;
}

int solve_common(madpipe_ctx *ctx, const madpipe_chain *chain, bool on_device, int32_t P, int64_t M,
                 double beta, const madpipe_disc *disc, madpipe_alloc *out) {
    int rc = begin(ctx);
    if (rc) return rc;
    if (!out) return fail(ctx, MADPIPE_EINVAL, "null out");
    rc = check_one(ctx, chain, P, M, beta, disc, !on_device);
    if (rc) return rc;
    std::vector<ChainSpec> cs{{*chain, on_device, P, M, beta}};
    std::vector<ChainDev> cd;
    rc = upload_chains(ctx, cs, cd);
    if (rc) return rc;
    CUDA_TRY(ctx, ctx->jl.ensure(sizeof(int32_t)));
    int64_t cu = 0;
    int32_t jstar = INT32_MAX;
    const int R = ctx->rank, W = ctx->world;
    // one rank: the winner is traced back from its sweep batch (no re-solve)
    SweepTraceHook th;
    th.init(1, nmp_of(disc->n_mem), (int)chain->L, (const int32_t *)ctx->jl.p);
    // One round: this rank evaluates its share of `js` (ascending; with `early`, it stops
    // at its first feasible candidate -- exact, a smaller feasible index always wins),
    // then the ranks min-reduce their smallest feasible index (a7, one all-reduce).
    auto sweep = [&](const std::vector<JobSpec> &js, bool early, double *ms_acc, double *kern_acc,
                     int64_t *eff_acc, int64_t *useful_acc) -> int {
        int r = fill_int_max(ctx, (int32_t *)ctx->jl.p, 1);
        if (r) return r;
        std::vector<JobSpec> mine;
        for (size_t i = (size_t)R; i < js.size(); i += (size_t)W) mine.push_back(js[i]);
        std::vector<uint64_t> counts;
        if (!mine.empty()) {
            th.js = &mine;
            r = run_jobs(ctx, cs, cd, disc, mine, (int32_t *)ctx->jl.p, nullptr, nullptr, &counts, early,
                         W == 1 ? &th : nullptr, true);
            if (r) return r;
            for (auto x : counts) cu += (int64_t)x;
            *ms_acc += ctx->sweep_ms; *kern_acc += ctx->step_ms;
            *eff_acc += ctx->last_effective; *useful_acc += ctx->last_useful;
        }
        r = allreduce_min(ctx, (int32_t *)ctx->jl.p, 1);
        if (r) return r;
        int32_t j = INT32_MAX;
        CUDA_TRY(ctx, d2h(ctx, &j, ctx->jl.p, sizeof(int32_t)));
        CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
        jstar = j;
        return MADPIPE_OK;
    };
    double ms = 0.0, kern = 0.0;
    int64_t eff = 0, useful = 0;
    const int n_c = disc->n_periods;
    if (disc->early_exit == 2 && n_c > 4) {
        // NEXT row f3, coarse-to-fine: every s-th candidate in ascending order until one is
        // feasible (J1), then the candidates of the gap (J1-s, J1); each round is split over
        // the ranks and ends in one all-reduce.  Exact when feasibility is monotone in the
        // period; early_exit = 1 is exact without that assumption.
        const int step = std::max(2, (int)std::lround(std::sqrt((double)n_c)));
        std::vector<JobSpec> coarse;
        for (int j = 0; j < n_c; j += step) coarse.push_back({0, j});
        if (coarse.back().j != n_c - 1) coarse.push_back({0, n_c - 1});
        rc = sweep(coarse, true, &ms, &kern, &eff, &useful);
        if (rc) return rc;
        if (jstar != INT32_MAX && jstar > 0) {
            const int J1 = jstar;
            std::vector<JobSpec> fine;
            for (int j = std::max(0, J1 - step + 1); j < J1; j++) fine.push_back({0, j});
            if (!fine.empty()) {
                rc = sweep(fine, true, &ms, &kern, &eff, &useful);
                if (rc) return rc;
                if (jstar == INT32_MAX) jstar = J1;
            }
        }
    } else {
        rc = sweep(shard_jobs(0, n_c, 0, 1), disc->early_exit != 0, &ms, &kern, &eff, &useful);
        if (rc) return rc;
    }
    ctx->sweep_ms = ms; ctx->step_ms = kern;
    ctx->last_cell_updates = cu; ctx->last_effective = eff; ctx->last_useful = useful;
    if (jstar == INT32_MAX) {
        fill_infeasible(out, cu);
        return MADPIPE_INFEASIBLE;
    }
    // a8: one rank traced the winner in its sweep batch; at N ranks every rank re-solves the
    // winner and traces it back (deterministic: no broadcast)
    if (W == 1 && th.best[0] == jstar) {
        if (th.outs[0].status != 0)
            return fail(ctx, MADPIPE_ESTATE, "traceback of candidate %d: %s", jstar,
                        th.outs[0].status == 1 ? "root is infeasible" : "traceback found no decision");
        fill_from_trace(out, jstar, th.taus[0], th.outs[0], th.stages.data(), th.stride);
        out->cell_updates = cu;
        return MADPIPE_OK;
    }
    std::vector<int32_t> js{jstar};
    rc = resolve_impl(ctx, cs, cd, disc, js, out);
    out->cell_updates = cu;
    return rc;
}

// ---------------------------------------------------------------------------
// batch work plan: LPT over the (chain, candidate) work list
// ---------------------------------------------------------------------------
// Host estimate of the cost of job (chain, j): its cell-updates at tau_j,
// sum_l (l - kmin(l) + 1) (P-1) n_v n_m, with the same prefix sums and grid formula as
// prep_kernel / jobs_init_kernel.  Only used to balance ranks; identical on every rank.
void batch_costs(const std::vector<ChainSpec> &cs, const madpipe_disc *disc, std::vector<int64_t> &cost) {
    const int n_c = disc->n_periods;
    cost.assign(cs.size() * (size_t)n_c, 0);
    std::vector<double> Up;
    for (size_t c = 0; c < cs.size(); c++) {
        const madpipe_chain &ch = cs[c].c;
        const int L = ch.L, P = cs[c].P;
        Up.assign(L + 1, 0.0);
        for (int i = 1; i <= L; i++) Up[i] = Up[i - 1] + (ch.uF[i - 1] + ch.uB[i - 1]);
        double SC = 0.0;
        for (int i = 1; i <= L - 1; i++) SC = SC + (2.0 * (double)ch.a[i]) / cs[c].beta;
        const double lb = Up[L] / (double)P, ub = Up[L] + SC;
        const int64_t per = (int64_t)std::max(0, P - 1) * disc->n_delay * disc->n_mem;
        for (int j = 0; j < n_c; j++) {
            const double tau = n_c == 1 ? ub : lb + (double)j * ((ub - lb) / (double)(n_c - 1));
            int64_t t = 0;
            int k = 1;
            for (int l = 1; l <= L; l++) {
                while (k <= l && Up[l] - Up[k - 1] > tau) k++;
                if (k <= l) t += (int64_t)(l - k + 1);
            }
            // + one (L+1) x n_v x P row sweep of fixed work per job (init, trans, roots)
            cost[c * (size_t)n_c + j] = t * per + (int64_t)(L + 1) * disc->n_delay * P;
        }
    }
}

// Longest-processing-time-first: items by decreasing cost (ties: lower index first),
// each to the rank with the smallest load so far (ties: lower rank).  Deterministic.
void lpt(const std::vector<int64_t> &cost, const std::vector<int32_t> &items, int world, std::vector<int32_t> &owner,
         std::vector<int64_t> *load_out) {
    std::vector<int32_t> order(items);
    std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return cost[a] > cost[b]; });
    std::vector<int64_t> load(world, 0);
    for (int32_t it : order) {
        int best = 0;
        for (int r = 1; r < world; r++) if (load[r] < load[best]) best = r;
        owner[it] = best;
        load[best] += cost[it];
    }
    if (load_out) *load_out = load;
}

// owner[c * n_c + j] = rank that evaluates candidate j of chain c
void batch_plan(const std::vector<ChainSpec> &cs, const madpipe_disc *disc, int world, std::vector<int32_t> &owner,
                std::vector<int64_t> *load, std::vector<int64_t> *cost_out) {
    Nvtx nv("madpipe batch plan (LPT)");
    std::vector<int64_t> cost;
    batch_costs(cs, disc, cost);
    owner.assign(cost.size(), 0);
    std::vector<int32_t> items(cost.size());
    for (size_t i = 0; i < items.size(); i++) items[i] = (int32_t)i;
    if (world > 1) lpt(cost, items, world, owner, load);
    else if (load) load->assign(1, std::accumulate(cost.begin(), cost.end(), (int64_t)0));
    if (cost_out) *cost_out = std::move(cost);
}

// rowner[c] = rank that re-solves chain c's winner j*[c] (LPT on the winners' costs); -1 if none
void resolve_plan(const std::vector<int64_t> &cost, int n_c, const std::vector<int32_t> &jstar, int world,
                  std::vector<int32_t> &rowner) {
    const int n = (int)jstar.size();
    rowner.assign(n, -1);
    std::vector<int64_t> wc(n, 0);
    std::vector<int32_t> items;
    for (int c = 0; c < n; c++)
        if (jstar[c] != INT32_MAX && jstar[c] >= 0) { items.push_back(c); wc[c] = cost[(size_t)c * n_c + jstar[c]]; }
    std::vector<int32_t> own(n, -1);
    if (world > 1) lpt(wc, items, world, own, nullptr);
    else for (int c : items) own[c] = 0;
    for (int c : items) rowner[c] = own[c];
}

int prepare_batch(madpipe_ctx *ctx, int32_t n, const madpipe_chain *chains, const int32_t *P, const int64_t *M,
                  const double *beta, const madpipe_disc *disc, std::vector<ChainSpec> &cs) {
    if (n < 1 || !chains || !P || !M || !beta || !disc)
        return fail(ctx, MADPIPE_EINVAL, "bad batch arguments");
    for (int i = 0; i < n; i++) {
        int rc = check_one(ctx, &chains[i], P[i], M[i], beta[i], disc, true);
        if (rc) return fail(ctx, rc, "chain %d: %s", i, ctx->err.c_str());
        cs.push_back({chains[i], false, P[i], M[i], beta[i]});
    }
    return MADPIPE_OK;
}

// This rank's share of the batch sweep: jl_dev[c] <- smallest feasible candidate of chain
// c among the jobs this rank owns (INT32_MAX if none); cu[c] <- this rank's cell-updates.
int batch_sweep(madpipe_ctx *ctx, const std::vector<ChainSpec> &cs, const std::vector<ChainDev> &cd,
                const madpipe_disc *disc, int rank, int world, const std::vector<int32_t> &owner,
                std::vector<int64_t> &cu, SweepTraceHook *th = nullptr) {
    const int n = (int)cs.size(), n_c = disc->n_periods;
    CUDA_TRY(ctx, ctx->jl.ensure(sizeof(int32_t) * n));
    { int _r = fill_int_max(ctx, (int32_t *)ctx->jl.p, n); if (_r) return _r; }
    // candidate-major order keeps small (cheap) periods of every chain first, so early
    // exit prunes the expensive large periods
    std::vector<JobSpec> js;
    for (int j = 0; j < n_c; j++)
        for (int c = 0; c < n; c++)
            if (world == 1 || owner[(size_t)c * n_c + j] == rank) js.push_back({c, j});
    // group by step kernel (one kernel per launch; the single-layer persistent kernel also
    // needs one P per launch); within a group candidate-major, so that with early exit the
    // first batches hold every chain's cheapest candidates
    const int nmp = nmp_of(disc->n_mem);
    int all_maxL = 1;
    for (const auto &c : cs) all_maxL = std::max(all_maxL, (int)c.c.L);
    std::vector<int> grp(n);
    for (int c = 0; c < n; c++) {
        const int k = step_kernel_for(ctx, cs[c].P, nmp, disc->n_delay, all_maxL);
        grp[c] = k * 65536 + (k == 2 ? cs[c].P : 0);
    }
    std::stable_sort(js.begin(), js.end(), [&](const JobSpec &a, const JobSpec &b) { return grp[a.chain] < grp[b.chain]; });
    cu.assign(n, 0);
    if (js.empty()) return MADPIPE_OK;
    std::vector<uint64_t> counts;
    if (th) {
        int maxL = 1;
        for (const auto &c : cs) maxL = std::max(maxL, (int)c.c.L);
        th->init(n, nmp, maxL, (const int32_t *)ctx->jl.p);
        th->js = &js;
    }
    int rc = run_jobs(ctx, cs, cd, disc, js, (int32_t *)ctx->jl.p, nullptr, nullptr, &counts,
                      disc->early_exit != 0, th, true);
    if (rc) return rc;
    for (size_t i = 0; i < js.size(); i++) cu[js[i].chain] += (int64_t)counts[i];
    return MADPIPE_OK;
}

// Re-solve and trace back the winners this rank owns (rowner[c] == rank); out[c] of the
// other chains is left untouched.
int batch_resolve(madpipe_ctx *ctx, const std::vector<ChainSpec> &cs, const std::vector<ChainDev> &cd,
                  const madpipe_disc *disc, const std::vector<int32_t> &jstar, const std::vector<int32_t> &rowner,
                  int rank, madpipe_alloc *out) {
    std::vector<int32_t> mine(jstar.size(), INT32_MAX);
    bool any = false;
    for (size_t c = 0; c < jstar.size(); c++)
        if (rowner[c] == rank) { mine[c] = jstar[c]; any = true; }
    if (!any) return MADPIPE_OK;
    return resolve_impl(ctx, cs, cd, disc, mine, out);
}

// Fixed-size int32 record of one chain's result for the all-gather:
// [period, load_period, special_load as 2 words each][cand_index][n_stages][first|last|proc x Lmax]
constexpr int kRecHead = 8;
void pack_rec(const madpipe_alloc &o, int Lmax, int32_t *r) {
    memcpy(r, &o.period, 8);
    memcpy(r + 2, &o.load_period, 8);
    memcpy(r + 4, &o.special_load, 8);
    r[6] = o.cand_index;
    r[7] = o.n_stages;
    for (int s = 0; s < o.n_stages; s++) {
        r[kRecHead + s] = o.stage_first[s];
        r[kRecHead + Lmax + s] = o.stage_last[s];
        r[kRecHead + 2 * Lmax + s] = o.stage_proc[s];
    }
}
void unpack_rec(const int32_t *r, int Lmax, madpipe_alloc &o) {
    memcpy(&o.period, r, 8);
    memcpy(&o.load_period, r + 2, 8);
    memcpy(&o.special_load, r + 4, 8);
    o.cand_index = r[6];
    o.n_stages = r[7];
    for (int s = 0; s < o.n_stages; s++) {
        if (o.stage_first) o.stage_first[s] = r[kRecHead + s];
        if (o.stage_last) o.stage_last[s] = r[kRecHead + Lmax + s];
        if (o.stage_proc) o.stage_proc[s] = r[kRecHead + 2 * Lmax + s];
    }
}

}  // namespace

// ---------------------------------------------------------------------------
// public entry points
// ---------------------------------------------------------------------------
extern "C" int madpipe_solve(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                             double beta, const madpipe_disc *disc, madpipe_alloc *out) {
    return solve_common(ctx, chain, false, P, M, beta, disc, out);
}

extern "C" int madpipe_solve_dev(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                                 double beta, const madpipe_disc *disc, madpipe_alloc *out) {
    return solve_common(ctx, chain, true, P, M, beta, disc, out);
}

extern "C" int madpipe_sweep(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                             double beta, const madpipe_disc *disc, int32_t rank, int32_t world,
                             int32_t *j_local, int64_t *cell_updates_out) {
    int rc = begin(ctx);
    if (rc) return rc;
    if (world < 1 || rank < 0 || rank >= world || !j_local)
        return fail(ctx, MADPIPE_EINVAL, "bad rank/world/j_local");
    const bool dev = chain && is_device_ptr(chain->uF);
    rc = check_one(ctx, chain, P, M, beta, disc, !dev);
    if (rc) return rc;
    std::vector<ChainSpec> cs{{*chain, dev, P, M, beta}};
    std::vector<ChainDev> cd;
    rc = upload_chains(ctx, cs, cd);
    if (rc) return rc;
    { int _r = fill_int_max(ctx, (int32_t *)j_local, 1); if (_r) return _r; }
    std::vector<uint64_t> counts;
    rc = run_jobs(ctx, cs, cd, disc, shard_jobs(0, disc->n_periods, rank, world), j_local, nullptr,
                  nullptr, &counts, disc->early_exit != 0, nullptr, true);
    if (rc) return rc;
    int64_t cu = 0;
    for (auto x : counts) cu += (int64_t)x;
    if (cell_updates_out) *cell_updates_out = cu;
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return MADPIPE_OK;
}

extern "C" int madpipe_resolve(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                               double beta, const madpipe_disc *disc, const int32_t *j_star,
                               madpipe_alloc *out) {
    int rc = begin(ctx);
    if (rc) return rc;
    if (!j_star || !out) return fail(ctx, MADPIPE_EINVAL, "null j_star/out");
    const bool dev = chain && is_device_ptr(chain->uF);
    rc = check_one(ctx, chain, P, M, beta, disc, !dev);
    if (rc) return rc;
    int32_t js = INT32_MAX;
    CUDA_TRY(ctx, d2h(ctx, &js, j_star, sizeof(int32_t)));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    if (js == INT32_MAX) {
        fill_infeasible(out, 0);
        return MADPIPE_INFEASIBLE;
    }
    if (js < 0 || js >= disc->n_periods) return fail(ctx, MADPIPE_EINVAL, "j_star out of range");
    std::vector<ChainSpec> cs{{*chain, dev, P, M, beta}};
    std::vector<ChainDev> cd;
    rc = upload_chains(ctx, cs, cd);
    if (rc) return rc;
    std::vector<int32_t> jv{js};
    int64_t keep = out->cell_updates;
    rc = resolve_impl(ctx, cs, cd, disc, jv, out);
    out->cell_updates = keep;
    return rc;
}

extern "C" int madpipe_solve_batch(madpipe_ctx *ctx, int32_t n, const madpipe_chain *chains,
                                   const int32_t *P, const int64_t *M, const double *beta,
                                   const madpipe_disc *disc, madpipe_alloc *out) {
    int rc = begin(ctx);
    if (rc) return rc;
    if (!out) return fail(ctx, MADPIPE_EINVAL, "null out");
    std::vector<ChainSpec> cs;
    rc = prepare_batch(ctx, n, chains, P, M, beta, disc, cs);
    if (rc) return rc;
    const int R = ctx->rank, W = ctx->world, n_c = disc->n_periods;
    // the same deterministic plan on every rank (identical inputs, SPMD)
    std::vector<int32_t> owner;
    std::vector<int64_t> cost;
    if (W > 1 || ctx->comm) batch_plan(cs, disc, W, owner, nullptr, &cost);
    std::vector<ChainDev> cd;
    rc = upload_chains(ctx, cs, cd);
    if (rc) return rc;
    std::vector<int64_t> cu;
    SweepTraceHook th;                            // one rank: winners traced in their sweep batches
    const bool one = W == 1 && !ctx->comm;
    rc = batch_sweep(ctx, cs, cd, disc, R, W, owner, cu, one ? &th : nullptr);
    if (rc) return rc;
    rc = allreduce_min(ctx, (int32_t *)ctx->jl.p, (size_t)n);     // a7 over int32[n]
    if (rc) return rc;
    std::vector<int32_t> jstar(n);
    CUDA_TRY(ctx, d2h(ctx, jstar.data(), ctx->jl.p, sizeof(int32_t) * n));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    for (int i = 0; i < n; i++) fill_infeasible(&out[i], cu[i]);
    if (one) {
        // winners traced during the sweep; anything else (none expected) is re-solved
        std::vector<int32_t> rest(n, INT32_MAX);
        bool any = false;
        for (int c = 0; c < n; c++) {
            if (jstar[c] == INT32_MAX) continue;
            if (th.best.size() == (size_t)n && th.best[c] == jstar[c]) {
                if (th.outs[c].status != 0)
                    return fail(ctx, MADPIPE_ESTATE, "traceback of chain %d candidate %d: %s", c, jstar[c],
                                th.outs[c].status == 1 ? "root is infeasible" : "traceback found no decision");
                fill_from_trace(&out[c], jstar[c], th.taus[c], th.outs[c],
                                th.stages.data() + 3 * (size_t)th.stride * c, th.stride);
            } else {
                rest[c] = jstar[c];
                any = true;
            }
        }
        if (any) {
            std::vector<int32_t> all(n, 0);
            rc = batch_resolve(ctx, cs, cd, disc, rest, all, 0, out);
            if (rc) return rc;
        }
        for (int i = 0; i < n; i++) out[i].cell_updates = cu[i];
        return MADPIPE_OK;
    }
    // each winner is re-solved by its owner, then one all-gather of fixed-size records
    std::vector<int32_t> rowner;
    resolve_plan(cost, n_c, jstar, W, rowner);
    int Lmax = 1;
    for (const auto &c : cs) Lmax = std::max(Lmax, (int)c.c.L);
    std::vector<int32_t> mine_idx;
    std::vector<int> per_rank(W, 0);
    for (int c = 0; c < n; c++) if (rowner[c] >= 0) per_rank[rowner[c]]++;
    const int slots = std::max(1, *std::max_element(per_rank.begin(), per_rank.end()));
    const size_t rec = (size_t)kRecHead + 3 * (size_t)Lmax;
    std::vector<int32_t> st(3 * (size_t)Lmax * n, 0);
    std::vector<madpipe_alloc> tmp(n);
    for (int c = 0; c < n; c++) {
        tmp[c] = out[c];
        tmp[c].stage_first = st.data() + 3 * (size_t)Lmax * c;
        tmp[c].stage_last = tmp[c].stage_first + Lmax;
        tmp[c].stage_proc = tmp[c].stage_last + Lmax;
    }
    rc = batch_resolve(ctx, cs, cd, disc, jstar, rowner, R, tmp.data());
    if (rc) return rc;
    std::vector<int32_t> sendh((size_t)slots * rec, 0);
    int k = 0;
    for (int c = 0; c < n; c++)
        if (rowner[c] == R) pack_rec(tmp[c], Lmax, sendh.data() + (size_t)(k++) * rec);
    CUDA_TRY(ctx, ctx->gather.ensure(sizeof(int32_t) * (size_t)slots * rec * (size_t)(W + 1)));
    int32_t *sendd = (int32_t *)ctx->gather.p, *recvd = sendd + (size_t)slots * rec;
    CUDA_TRY(ctx, h2d(ctx, sendd, sendh.data(), sizeof(int32_t) * sendh.size()));
    {
        Nvtx nv("madpipe batch allgather");
        std::string why;
        if (comm_allgather_i32(ctx->comm, sendd, recvd, (size_t)slots * rec, ctx->stream, &why))
            return fail(ctx, MADPIPE_ENCCL, "%s", why.c_str());
    }
    std::vector<int32_t> recvh((size_t)W * slots * rec);
    CUDA_TRY(ctx, d2h(ctx, recvh.data(), recvd, sizeof(int32_t) * recvh.size()));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    std::vector<int> next(W, 0);
    for (int c = 0; c < n; c++) {
        const int r = rowner[c];
        if (r < 0) continue;
        unpack_rec(recvh.data() + ((size_t)r * slots + (size_t)(next[r]++)) * rec, Lmax, out[c]);
    }
    for (int i = 0; i < n; i++) out[i].cell_updates = cu[i];
    return MADPIPE_OK;
}

extern "C" int madpipe_batch_plan(int32_t n, const madpipe_chain *chains, const int32_t *P, const double *beta,
                                  const madpipe_disc *disc, int32_t world, int32_t *owner, int64_t *load,
                                  int64_t *cost) {
    if (n < 1 || !chains || !P || !beta || !disc || world < 1 || disc->n_periods < 1)
        return fail(nullptr, MADPIPE_EINVAL, "bad batch plan arguments");
    std::vector<ChainSpec> cs;
    for (int i = 0; i < n; i++) {
        if (chains[i].L < 1 || P[i] < 1 || !chains[i].uF || !chains[i].uB || !chains[i].a)
            return fail(nullptr, MADPIPE_EINVAL, "chain %d invalid", i);
        cs.push_back({chains[i], false, P[i], 1, beta[i]});
    }
    std::vector<int32_t> own;
    std::vector<int64_t> ld, cst;
    batch_plan(cs, disc, world, own, &ld, &cst);
    if (owner) std::copy(own.begin(), own.end(), owner);
    if (load) std::copy(ld.begin(), ld.end(), load);
    if (cost) std::copy(cst.begin(), cst.end(), cost);
    return MADPIPE_OK;
}

extern "C" int madpipe_resolve_plan(int32_t n, const madpipe_chain *chains, const int32_t *P, const double *beta,
                                    const madpipe_disc *disc, const int32_t *j_star, int32_t world,
                                    int32_t *owner) {
    if (n < 1 || !chains || !P || !beta || !disc || !j_star || !owner || world < 1)
        return fail(nullptr, MADPIPE_EINVAL, "bad resolve plan arguments");
    std::vector<ChainSpec> cs;
    for (int i = 0; i < n; i++) cs.push_back({chains[i], false, P[i], 1, beta[i]});
    std::vector<int64_t> cost;
    batch_costs(cs, disc, cost);
    std::vector<int32_t> js(j_star, j_star + n), ro;
    resolve_plan(cost, disc->n_periods, js, world, ro);
    std::copy(ro.begin(), ro.end(), owner);
    return MADPIPE_OK;
}

extern "C" int madpipe_sweep_batch(madpipe_ctx *ctx, int32_t n, const madpipe_chain *chains, const int32_t *P,
                                   const int64_t *M, const double *beta, const madpipe_disc *disc, int32_t rank,
                                   int32_t world, int32_t *j_local, int64_t *cell_updates_out) {
    int rc = begin(ctx);
    if (rc) return rc;
    if (world < 1 || rank < 0 || rank >= world || !j_local)
        return fail(ctx, MADPIPE_EINVAL, "bad rank/world/j_local");
    std::vector<ChainSpec> cs;
    rc = prepare_batch(ctx, n, chains, P, M, beta, disc, cs);
    if (rc) return rc;
    std::vector<int32_t> owner;
    if (world > 1) batch_plan(cs, disc, world, owner, nullptr, nullptr);
    std::vector<ChainDev> cd;
    rc = upload_chains(ctx, cs, cd);
    if (rc) return rc;
    std::vector<int64_t> cu;
    rc = batch_sweep(ctx, cs, cd, disc, rank, world, owner, cu);
    if (rc) return rc;
    CUDA_TRY(ctx, d2h(ctx, j_local, ctx->jl.p, sizeof(int32_t) * n));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    if (cell_updates_out) std::copy(cu.begin(), cu.end(), cell_updates_out);
    return MADPIPE_OK;
}

extern "C" int madpipe_resolve_batch(madpipe_ctx *ctx, int32_t n, const madpipe_chain *chains, const int32_t *P,
                                     const int64_t *M, const double *beta, const madpipe_disc *disc,
                                     const int32_t *j_star, int32_t rank, int32_t world, madpipe_alloc *out) {
    int rc = begin(ctx);
    if (rc) return rc;
    if (world < 1 || rank < 0 || rank >= world || !j_star || !out)
        return fail(ctx, MADPIPE_EINVAL, "bad rank/world/j_star/out");
    std::vector<ChainSpec> cs;
    rc = prepare_batch(ctx, n, chains, P, M, beta, disc, cs);
    if (rc) return rc;
    std::vector<int32_t> js(j_star, j_star + n), rowner;
    for (int c = 0; c < n; c++)
        if (js[c] != INT32_MAX && (js[c] < 0 || js[c] >= disc->n_periods))
            return fail(ctx, MADPIPE_EINVAL, "j_star[%d] out of range", c);
    std::vector<int64_t> cost;
    batch_costs(cs, disc, cost);
    resolve_plan(cost, disc->n_periods, js, world, rowner);
    std::vector<ChainDev> cd;
    rc = upload_chains(ctx, cs, cd);
    if (rc) return rc;
    for (int c = 0; c < n; c++) {
        if (rowner[c] != rank) continue;
        const int64_t keep = out[c].cell_updates;
        fill_infeasible(&out[c], keep);
    }
    rc = batch_resolve(ctx, cs, cd, disc, js, rowner, rank, out);
    return rc;
}

extern "C" int madpipe_candidates(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                                  double beta, const madpipe_disc *disc, double *tau_out,
                                  double *root_out) {
    int rc = begin(ctx);
    if (rc) return rc;
    rc = check_one(ctx, chain, P, M, beta, disc, true);
    if (rc) return rc;
    std::vector<ChainSpec> cs{{*chain, false, P, M, beta}};
    std::vector<ChainDev> cd;
    rc = upload_chains(ctx, cs, cd);
    if (rc) return rc;
    const int n_c = disc->n_periods;
    CUDA_TRY(ctx, ctx->jl.ensure(sizeof(int32_t)));
    { int _r = fill_int_max(ctx, (int32_t *)ctx->jl.p, 1); if (_r) return _r; }
    CUDA_TRY(ctx, ctx->scratch.ensure(sizeof(double) * 2 * n_c));
    double *roots_dev = (double *)ctx->scratch.p, *taus_dev = roots_dev + n_c;
    madpipe_disc d2 = *disc;
    d2.early_exit = 0;
    std::vector<JobSpec> js = shard_jobs(0, n_c, 0, 1);
    rc = run_jobs(ctx, cs, cd, &d2, js, (int32_t *)ctx->jl.p, roots_dev, taus_dev, nullptr, false,
                  nullptr, true);
    if (rc) return rc;
    if (root_out)
        CUDA_TRY(ctx, d2h(ctx, root_out, roots_dev, sizeof(double) * n_c));
    if (tau_out)
        CUDA_TRY(ctx, d2h(ctx, tau_out, taus_dev, sizeof(double) * n_c));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return MADPIPE_OK;
}

namespace {
struct ExportHook : BatchHook {
    int nmp, L, P, n_v, n_m;
    double *A_dev = nullptr;
    int32_t *arg_dev = nullptr;
    int after_batch(madpipe_ctx *ctx, const std::vector<int> &, Job *jobs_dev) override {
        launch_export(jobs_dev, nmp, A_dev, L, P, n_v, n_m, ctx->stream);
        ctx->launches++;
        if (arg_dev) { launch_argmin(jobs_dev, nmp, arg_dev, L, P, n_v, n_m, ctx->stream); ctx->launches++; }
        CUDA_TRY(ctx, cudaGetLastError());
        return MADPIPE_OK;
    }
};
}  // namespace

extern "C" int madpipe_dp_table(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                                double beta, const madpipe_disc *disc, int32_t j, double *A_out,
                                int32_t *arg_out) {
    int rc = begin(ctx);
    if (rc) return rc;
    rc = check_one(ctx, chain, P, M, beta, disc, true);
    if (rc) return rc;
    if (j < 0 || j >= disc->n_periods || !A_out) return fail(ctx, MADPIPE_EINVAL, "bad j / A_out");
    std::vector<ChainSpec> cs{{*chain, false, P, M, beta}};
    std::vector<ChainDev> cd;
    rc = upload_chains(ctx, cs, cd);
    if (rc) return rc;
    const size_t cells = (size_t)(chain->L + 1) * P * disc->n_delay * disc->n_mem;
    CUDA_TRY(ctx, ctx->scratch.ensure(cells * (sizeof(double) + sizeof(int32_t))));
    ExportHook hook;
    hook.nmp = nmp_of(disc->n_mem); hook.L = chain->L; hook.P = P; hook.n_v = disc->n_delay;
    hook.n_m = disc->n_mem;
    hook.A_dev = (double *)ctx->scratch.p;
    hook.arg_dev = arg_out ? (int32_t *)((char *)ctx->scratch.p + cells * sizeof(double)) : nullptr;
    CUDA_TRY(ctx, ctx->jl.ensure(sizeof(int32_t)));
    { int _r = fill_int_max(ctx, (int32_t *)ctx->jl.p, 1); if (_r) return _r; }
    std::vector<JobSpec> js{{0, j}};
    rc = run_jobs(ctx, cs, cd, disc, js, (int32_t *)ctx->jl.p, nullptr, nullptr, nullptr, false, &hook,
                  false);
    if (rc) return rc;
    CUDA_TRY(ctx, d2h(ctx, A_out, hook.A_dev, cells * sizeof(double)));
    if (arg_out)
        CUDA_TRY(ctx, d2h(ctx, arg_out, hook.arg_dev, cells * sizeof(int32_t)));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return MADPIPE_OK;
}

// ---------------------------------------------------------------------------
// NEXT row f1: paper-literal MadPipe-DP + Algorithm 1 (mp_literal.cu)
// ---------------------------------------------------------------------------
namespace {

struct LitRun {
    std::vector<ChainSpec> cs;
    std::vector<ChainDev> cd;
    Job hj{};
    Job *dj = nullptr;
    int nmp = 2, n_t = 2;
    double dt = 0.0, U = 0.0, SC = 0.0, lb = 0.0, ub = 0.0;
    size_t cells = 0;
};

int lit_setup(madpipe_ctx *ctx, LitRun &R, const madpipe_chain *chain, int32_t P, int64_t M, double beta,
              int n_mem, int n_delay, int n_t) {
    madpipe_disc d{n_mem, n_delay, 1, MADPIPE_VRANGE_PAPER, 0};
    int rc = check_one(ctx, chain, P, M, beta, &d, true);
    if (rc) return rc;
    if (n_t < 2 || n_t > 1 << 20) return fail(ctx, MADPIPE_EINVAL, "n_tp must be in [2, 2^20]");
    R.cs = {{*chain, false, P, M, beta}};
    rc = upload_chains(ctx, R.cs, R.cd);
    if (rc) return rc;
    double scal[4];
    CUDA_TRY(ctx, d2h(ctx, scal, R.cd[0].scal, sizeof scal));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    R.SC = scal[0]; R.lb = scal[1]; R.ub = scal[2]; R.U = scal[3];
    R.n_t = n_t;
    R.dt = R.U / (double)(n_t - 1);              // n_t values in [0, U(1,L)]
    R.nmp = nmp_of(n_mem);
    R.cells = (size_t)(chain->L + 1) * n_delay * (size_t)n_t * P * R.nmp;
    CUDA_TRY(ctx, ctx->tables.ensure(R.cells * sizeof(double)));
    CUDA_TRY(ctx, ctx->jobs.ensure(sizeof(Job)));
    Job &J = R.hj;
    const ChainDev &c = R.cd[0];
    J.Up = c.Up; J.Wp = c.Wp; J.Ap = c.Ap; J.a = c.a; J.C = c.C; J.scal = c.scal;
    J.table = (double *)ctx->tables.p;
    J.M = M; J.L = chain->L; J.P = P; J.n_v = n_delay; J.n_m = n_mem; J.vsafe = 0;
    J.dV = (R.U + R.SC) / (double)(n_delay - 1);  // PAPER V range (Q8)
    R.dj = (Job *)ctx->jobs.p;
    return MADPIPE_OK;
}

// one literal DP at target That; returns its root T(L, P-1, 0, 0, 0)
int lit_run(madpipe_ctx *ctx, LitRun &R, double That, double *root) {
    R.hj.tau = That;
    CUDA_TRY(ctx, h2d(ctx, R.dj, &R.hj, sizeof(Job)));
    launch_lit_init(R.dj, R.n_t, R.dt, R.nmp, (int64_t)R.hj.n_v * R.n_t * R.hj.P * R.nmp, ctx->stream);
    for (int l = 1; l <= R.hj.L; l++)
        launch_lit_step(R.dj, R.n_t, R.dt, R.nmp, R.hj.n_v, R.hj.P, l, ctx->stream);
    ctx->launches += 1 + R.hj.L;
    CUDA_TRY(ctx, cudaGetLastError());
    const size_t ridx = (((size_t)R.hj.L * R.hj.n_v) * R.n_t * (size_t)R.hj.P + (size_t)(R.hj.P - 1)) * R.nmp;
    CUDA_TRY(ctx, d2h(ctx, root, (double *)ctx->tables.p + ridx, sizeof(double)));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return MADPIPE_OK;
}

}  // namespace

extern "C" int madpipe_literal_table(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                                     double beta, int32_t n_mem, int32_t n_delay, int32_t n_tp, double That,
                                     double *A_out, int32_t *arg_out) {
    int rc = begin(ctx);
    if (rc) return rc;
    if (!A_out || !(That > 0.0)) return fail(ctx, MADPIPE_EINVAL, "bad A_out / That");
    LitRun R;
    rc = lit_setup(ctx, R, chain, P, M, beta, n_mem, n_delay, n_tp);
    if (rc) return rc;
    double root;
    rc = lit_run(ctx, R, That, &root);
    if (rc) return rc;
    const size_t out_cells = (size_t)(chain->L + 1) * P * n_tp * n_delay * n_mem;
    CUDA_TRY(ctx, ctx->scratch.ensure(out_cells * (sizeof(double) + sizeof(int32_t))));
    double *A_dev = (double *)ctx->scratch.p;
    int32_t *arg_dev = (int32_t *)(A_dev + out_cells);
    launch_lit_export(R.dj, R.n_t, R.dt, R.nmp, A_dev, arg_out ? arg_dev : nullptr, ctx->stream);
    CUDA_TRY(ctx, cudaGetLastError());
    CUDA_TRY(ctx, d2h(ctx, A_out, A_dev, out_cells * sizeof(double)));
    if (arg_out) CUDA_TRY(ctx, d2h(ctx, arg_out, arg_dev, out_cells * sizeof(int32_t)));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    return MADPIPE_OK;
}

extern "C" int madpipe_solve_paper(madpipe_ctx *ctx, const madpipe_chain *chain, int32_t P, int64_t M,
                                   double beta, int32_t n_mem, int32_t n_delay, int32_t n_tp, int32_t K,
                                   madpipe_alloc *out, double *T_hist, double *That_hist) {
    int rc = begin(ctx);
    if (rc) return rc;
    if (!out || K < 1) return fail(ctx, MADPIPE_EINVAL, "bad out / K");
    LitRun R;
    rc = lit_setup(ctx, R, chain, P, M, beta, n_mem, n_delay, n_tp);
    if (rc) return rc;
    double lb = R.lb, ub = R.ub, That = lb;   // Algorithm 1 lines 1-3 (Q4)
    double best = INFINITY, best_That = 0.0;
    int bi = -1;
    for (int i = 0; i < K; i++) {
        double T;
        rc = lit_run(ctx, R, That, &T);           // line 4: T_i = MadPipe-DP(That_i)
        if (rc) return rc;
        if (T_hist) T_hist[i] = T;
        if (That_hist) That_hist[i] = That;
        const double Tm = T > That ? T : That;    // max(T_i, That_i)
        if (Tm < best) { best = Tm; bi = i; best_That = That; }
        const double lo = T < That ? T : That;
        if (lo > lb) lb = lo;                     // lb <- max(lb, min(T_i, That_i))  (Q15)
        if (Tm < ub) ub = Tm;                     // ub <- min(ub, max(T_i, That_i))
        That = (lb + ub) / 2.0;
    }
    fill_infeasible(out, 0);
    if (bi < 0 || !std::isfinite(best)) return MADPIPE_INFEASIBLE;
    double root;
    rc = lit_run(ctx, R, best_That, &root);       // re-solve the winner and trace it back
    if (rc) return rc;
    const int L = chain->L;
    CUDA_TRY(ctx, ctx->stages.ensure(sizeof(int32_t) * (3 * (size_t)L + 1)));
    int32_t *st = (int32_t *)ctx->stages.p;
    launch_lit_traceback(R.dj, R.n_t, R.dt, R.nmp, st, st + 3 * L, ctx->stream);
    ctx->launches++;
    CUDA_TRY(ctx, cudaGetLastError());
    std::vector<int32_t> h(3 * (size_t)L + 1);
    CUDA_TRY(ctx, d2h(ctx, h.data(), st, h.size() * sizeof(int32_t)));
    CUDA_TRY(ctx, cudaStreamSynchronize(ctx->stream));
    const int ns = h[3 * L];
    if (ns < 0) return fail(ctx, MADPIPE_ESTATE, "literal traceback found no decision");
    // reverse into chain order, number the normal GPUs, allocation period
    std::vector<double> Up(L + 1, 0.0);
    for (int i = 1; i <= L; i++) Up[i] = Up[i - 1] + (chain->uF[i - 1] + chain->uB[i - 1]);
    int next_normal = 0;
    double lp = 0.0, special = 0.0;
    for (int q = 0; q < ns; q++) {
        const int src = ns - 1 - q;
        const int f = h[src], l = h[L + src], kind = h[2 * L + src];
        const double u = Up[l] - Up[f - 1];
        if (out->stage_first) out->stage_first[q] = f;
        if (out->stage_last) out->stage_last[q] = l;
        if (out->stage_proc) out->stage_proc[q] = kind ? P - 1 : next_normal;
        if (!kind) { next_normal++; lp = std::max(lp, u); } else special += u;
        if (f > 1) lp = std::max(lp, 2.0 * (double)chain->a[f - 1] / beta);
    }
    out->n_stages = ns;
    out->period = best;
    out->special_load = special;
    out->load_period = std::max(lp, special);
    out->cand_index = bi;
    out->cell_updates = 0;
    return MADPIPE_OK;
}
