// mp_comm.cu -- the ctx-owned NCCL communicator of libmadpipe.
//
// The hot path's only exchange step is a7, the global minimum of the ranks'
// smallest feasible candidate indices (one int32 per chain), plus, for the
// batch, the all-gather of the winners' allocations re-solved by their owners.
// NCCL is loaded at run time (dlopen of libnccl.so.2; MADPIPE_NCCL_LIB
// overrides the name), so the library loads and its host-only helpers work on
// machines without NCCL; only a ctx created with a communicator needs it.  In
// a process that already loaded torch, dlopen by soname returns torch's own
// NCCL, so one NCCL build serves both.
#include <dlfcn.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>

#include <nccl.h>

#include "mp_internal.cuh"

namespace mp {
namespace {

struct NcclApi {
    void *h = nullptr;
    ncclResult_t (*getUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*commInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*allReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*allGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    const char *(*errStr)(ncclResult_t) = nullptr;
    ncclResult_t (*getVersion)(int *) = nullptr;
    std::string err;
    bool ok = false;
};

NcclApi g_nccl;
std::once_flag g_once;

void load() {
    const char *names[] = {getenv("MADPIPE_NCCL_LIB"), "libnccl.so.2", "libnccl.so"};
    for (const char *n : names) {
        if (!n || !*n) continue;
        g_nccl.h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
        if (g_nccl.h) break;
    }
    if (!g_nccl.h) {
        const char *e = dlerror();
        g_nccl.err = std::string("cannot load libnccl.so.2: ") + (e ? e : "?");
        return;
    }
    auto sym = [](const char *s) { return dlsym(g_nccl.h, s); };
    g_nccl.getUniqueId = (decltype(g_nccl.getUniqueId))sym("ncclGetUniqueId");
    g_nccl.commInitRank = (decltype(g_nccl.commInitRank))sym("ncclCommInitRank");
    g_nccl.commDestroy = (decltype(g_nccl.commDestroy))sym("ncclCommDestroy");
    g_nccl.allReduce = (decltype(g_nccl.allReduce))sym("ncclAllReduce");
    g_nccl.allGather = (decltype(g_nccl.allGather))sym("ncclAllGather");
    g_nccl.errStr = (decltype(g_nccl.errStr))sym("ncclGetErrorString");
    g_nccl.getVersion = (decltype(g_nccl.getVersion))sym("ncclGetVersion");
    if (!g_nccl.getUniqueId || !g_nccl.commInitRank || !g_nccl.commDestroy || !g_nccl.allReduce ||
        !g_nccl.allGather || !g_nccl.errStr) {
        g_nccl.err = "libnccl.so.2 lacks a required symbol";
        return;
    }
    g_nccl.ok = true;
}

bool ready(std::string *why) {
    std::call_once(g_once, load);
    if (!g_nccl.ok && why) *why = g_nccl.err;
    return g_nccl.ok;
}

std::string rstr(ncclResult_t r) {
    return g_nccl.errStr ? g_nccl.errStr(r) : ("nccl error " + std::to_string((int)r));
}

}  // namespace

int comm_unique_id(uint8_t id[128], std::string *why) {
    if (!ready(why)) return -1;
    ncclUniqueId u;
    ncclResult_t r = g_nccl.getUniqueId(&u);
    if (r != ncclSuccess) { if (why) *why = "ncclGetUniqueId: " + rstr(r); return -1; }
    static_assert(sizeof(u) == 128, "ncclUniqueId is 128 bytes");
    memcpy(id, &u, 128);
    return 0;
}

int comm_init(void **comm, int world, int rank, const uint8_t id[128], std::string *why) {
    if (!ready(why)) return -1;
    ncclUniqueId u;
    memcpy(&u, id, 128);
    ncclComm_t c = nullptr;
    ncclResult_t r = g_nccl.commInitRank(&c, world, u, rank);
    if (r != ncclSuccess) { if (why) *why = "ncclCommInitRank: " + rstr(r); return -1; }
    *comm = (void *)c;
    return 0;
}

void comm_destroy(void *comm) {
    if (comm && g_nccl.ok) g_nccl.commDestroy((ncclComm_t)comm);
}

int comm_allreduce_min_i32(void *comm, int32_t *buf, size_t n, cudaStream_t s, std::string *why) {
    ncclResult_t r = g_nccl.allReduce(buf, buf, n, ncclInt32, ncclMin, (ncclComm_t)comm, s);
    if (r != ncclSuccess) { if (why) *why = "ncclAllReduce: " + rstr(r); return -1; }
    return 0;
}

int comm_allgather_i32(void *comm, const int32_t *send, int32_t *recv, size_t n_per_rank, cudaStream_t s,
                       std::string *why) {
    ncclResult_t r = g_nccl.allGather(send, recv, n_per_rank, ncclInt32, (ncclComm_t)comm, s);
    if (r != ncclSuccess) { if (why) *why = "ncclAllGather: " + rstr(r); return -1; }
    return 0;
}

int comm_version() {
    int v = 0;
    if (ready(nullptr) && g_nccl.getVersion) g_nccl.getVersion(&v);
    return v;
}

}  // namespace mp
