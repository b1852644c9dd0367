// mp_internal.cuh -- internal structures of libmadpipe (B200 / sm_100a).
//
// Product code: shares nothing with oracle/ (the CPU oracle used by tests).
// Paper references: "P:n" = line n of the MadPipe paper text; "Qn" = the
// readings listed in DESIGN.md section 3.
#pragma once
#include <cstdint>
#include <string>
#include <cuda_runtime.h>

namespace mp {

// Per-chain device arrays (section 8(a) step a1, P:155 / P:159 / P:147).
struct ChainDev {
    const double  *uF, *uB;     // [L]
    const int64_t *W, *a;       // [L], [L+1]
    double  *Up;                // [L+1] prefix sums of uF+uB
    int64_t *Wp, *Ap;           // [L+1] prefix sums of W_i and a_{i-1}
    double  *C;                 // [L+1] C[i] = 2 a_i / beta (i=1..L-1), C[0]=C[L]=0
    double  *scal;              // [4]  SC, lb, ub, U(1,L)
    int32_t L, P;
    int64_t M;
    double  beta;
};

// One unit of the sweep: a (chain, candidate period) pair.
struct Job {
    const double  *Up;
    const int64_t *Wp, *Ap, *a;
    const double  *C;
    double  *table;     // [(L+1)][n_v][P][NMP] fp64, m innermost
    double   tau, dV;   // filled on device by jobs_init_kernel
    int64_t  M;
    int32_t  L, P, n_v, n_m;
    int32_t  vsafe;     // 1 = SAFE v_range (saturate), 0 = PAPER (overflow infeasible)
    int32_t  j;         // candidate index
    int32_t  n_c;       // number of candidates of the chain
    int32_t  chain;     // chain index (batch API)
    int32_t  tile0;     // first tile of this job in the step grid
    int32_t  vb;        // delay rows per tile
    int32_t  np;        // p rows (>=1) per tile
    int32_t  n_ptiles;  // tiles along p
    int32_t  gid;       // index of the job in the caller's job list (root/tau export)
    const double *scal; // chain scalars (SC, lb, ub, U(1,L))
    unsigned long long *eff;  // effective (non-skipped) relaxations of this job
    int32_t *codes;     // [n_v][code_cap] transition codes of layer l, k = kmin_l + kk (persist path)
    int32_t *kmin_l;    // window start of layer l for this job (written by trans_kernel)
    int32_t code_cap;   // row capacity of codes (>= longest window of the batch)
    int32_t pad_;
    uint32_t *rowflag;  // [(L+1)][n_v]: 1 if row (l, v) holds a finite value (persist path)
    unsigned long long *useful;  // live relaxations whose source row is not all +inf
    struct TransEntry *tlist;    // [n_v][code_cap] useful transitions of layer l (persist path)
    int32_t *tcount;             // [n_v] their number
    int32_t *kwin;               // [L+1] window start max(kmin_tau(l), kmin_W(l)) (window_kernel)
    unsigned long long *segs;    // source segments loaded (pair path: merged list entries)
};

// One useful transition of layer l for delay row v, in ascending k (trans_kernel).
struct TransEntry {
    double U;        // U(k,l)
    int32_t code;    // pack_trans(v', d, nf)
    int32_t k;
};

// Result of a traceback, written by traceback_kernel.
struct TraceOut {
    double  load_period;
    double  special_load;
    int32_t n_stages;
    int32_t status;     // 0 ok, 1 infeasible root, 2 broken path
    // followed in memory by stage arrays (first,last,proc) of capacity L each
};

constexpr int kThreads = 256;        // threads per step CTA
constexpr int kTransSmem = 2048;     // transition entries staged per chunk
constexpr int kMaxKChunk = 512;

// Transition packing (int32): bit 31 set = skip this k;
//   bits 0..15 vn, bits 16..23 d (clamped to 255), bit 24 nf.
__host__ __device__ inline int32_t pack_trans(int vn, int64_t d, bool nf) {
    int dd = d > 255 ? 255 : (int)d;
    return (int32_t)((unsigned)vn | ((unsigned)dd << 16) | ((nf ? 1u : 0u) << 24));
}

// kernel launchers (mp_kernels.cu)
void launch_prep(ChainDev *chains_dev, int n_chains, cudaStream_t s);
void launch_jobs_init(Job *jobs, int n_jobs, cudaStream_t s);
void launch_init_slab0(const Job *jobs, int n_jobs, int nmp, int max_cells, cudaStream_t s);
void launch_step(const Job *jobs, const int32_t *tile_job, int n_tiles, int l, int nmp, int threads,
                 cudaStream_t s);
void launch_step_persist(const Job *jobs, const int32_t *tile_job, int n_tiles, int l, int nmp, int np,
                         int vb, int nsg, int grid, unsigned long long *prof, int n_prod, int tile_block,
                         size_t buf_off, cudaStream_t s);
void pair_geom(int P, int n_v, int *np, int *n_ptiles, int *n_vtiles, int *n_tiles);
int pair_list_cap(int max_L);
size_t pair_entry_bytes();
int pair_nsl(int np, int nmp);
bool pair_supported(int P, int nmp, int n_v, int max_L);
void launch_pair_trans(const Job *jobs, int n_jobs, int n_v_max, int l, int nmp, size_t buf_off, int fix_slab,
                       int unv_from, int max_grid, cudaStream_t s);
void launch_pair_fixup(const Job *jobs, int n_jobs, int n_v_max, int l1, int nmp, int max_grid, cudaStream_t s);
void launch_pair_step(const int2 *tdesc, int n_tiles, const void *lists, size_t buf_off, int cap, int nmp, int np,
                      int nsl, int grid, unsigned long long *prof, cudaStream_t s, int diag = 0);
int pair_blocks_per_sm(int nmp, int np, int nsl);
int persist_blocks_per_sm(int nmp, int np, int vb, int nsg, int n_prod);
void persist_geom(int P, int n_v, int nmp, int *vb, int *np, int *n_ptiles, int *n_tiles);
int persist_nsg(int np, int vb, int nmp);
void launch_trans(const Job *jobs, int n_jobs, int n_v_max, int l, int nmp, size_t buf_off, int verify_last,
                  cudaStream_t s);
void launch_window(const Job *jobs, int n_jobs, int max_L, cudaStream_t s);
void launch_lit_init(const Job *job, int n_t, double dt, int nmp, int64_t cells, cudaStream_t s);
void launch_lit_step(const Job *job, int n_t, double dt, int nmp, int n_v, int P, int l, cudaStream_t s);
void launch_lit_export(const Job *job, int n_t, double dt, int nmp, double *A_out, int32_t *arg_out,
                       cudaStream_t s);
void launch_lit_traceback(const Job *job, int n_t, double dt, int nmp, int32_t *stages, int32_t *n_out,
                          cudaStream_t s);
void launch_root(const Job *jobs, int n_jobs, int nmp, int32_t *jl_per_chain, double *root_out,
                 double *tau_out, cudaStream_t s);
void launch_count(const Job *jobs, int n_jobs, unsigned long long *counts, cudaStream_t s);
void launch_traceback(const Job *jobs, int n_jobs, int nmp, TraceOut *outs, int32_t *stages,
                      int stage_stride, cudaStream_t s);
void launch_argmin(const Job *job, int nmp, int32_t *arg_out, int L, int P, int n_v, int n_m,
                   cudaStream_t s);
void launch_export(const Job *job, int nmp, double *A_out, int L, int P, int n_v, int n_m,
                   cudaStream_t s);

// ctx-owned NCCL communicator (mp_comm.cu; NCCL is dlopen'ed on first use).
// Each returns 0 or -1 with *why set.
int comm_unique_id(uint8_t id[128], std::string *why);
int comm_init(void **comm, int world, int rank, const uint8_t id[128], std::string *why);
void comm_destroy(void *comm);
int comm_allreduce_min_i32(void *comm, int32_t *buf, size_t n, cudaStream_t s, std::string *why);
int comm_allgather_i32(void *comm, const int32_t *send, int32_t *recv, size_t n_per_rank, cudaStream_t s,
                       std::string *why);
int comm_version();

}  // namespace mp
