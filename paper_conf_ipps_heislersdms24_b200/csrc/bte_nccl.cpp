// bte_nccl.cpp -- dlopen wrapper over the NCCL C API (see bte_nccl.h).
#include "bte_nccl.h"

#include <dlfcn.h>
#include <nccl.h>

#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

namespace bte {
namespace nccl {
namespace {

struct Api {
    void *h = nullptr;
    ncclResult_t (*getUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*commInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*allReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*reduceScatter)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                                  cudaStream_t) = nullptr;
    ncclResult_t (*allGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*commSplit)(ncclComm_t, int, int, ncclComm_t *, ncclConfig_t *) = nullptr;
    ncclResult_t (*send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*groupStart)() = nullptr;
    ncclResult_t (*groupEnd)() = nullptr;
    const char *(*getErrorString)(ncclResult_t) = nullptr;
    std::string why;
};

Api *api() {
    static Api a;
    static std::once_flag once;
    std::call_once(once, [] {
        // BTE_NCCL_LIB (the Python binding points it at the torch-bundled NCCL), else the loader path
        const char *cands[] = {getenv("BTE_NCCL_LIB"), "libnccl.so.2", "libnccl.so"};
        for (const char *p : cands) {
            if (!p || !*p) continue;
            a.h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
            if (a.h) break;
        }
        if (!a.h) {
            a.why = "cannot dlopen libnccl.so.2 (set BTE_NCCL_LIB)";
            return;
        }
        a.getUniqueId = (decltype(a.getUniqueId))dlsym(a.h, "ncclGetUniqueId");
        a.commInitRank = (decltype(a.commInitRank))dlsym(a.h, "ncclCommInitRank");
        a.allReduce = (decltype(a.allReduce))dlsym(a.h, "ncclAllReduce");
        a.reduceScatter = (decltype(a.reduceScatter))dlsym(a.h, "ncclReduceScatter");
        a.allGather = (decltype(a.allGather))dlsym(a.h, "ncclAllGather");
        a.commDestroy = (decltype(a.commDestroy))dlsym(a.h, "ncclCommDestroy");
        a.getErrorString = (decltype(a.getErrorString))dlsym(a.h, "ncclGetErrorString");
        // (cell partitioning only: checked where used)
        a.commSplit = (decltype(a.commSplit))dlsym(a.h, "ncclCommSplit");
        a.send = (decltype(a.send))dlsym(a.h, "ncclSend");
        a.recv = (decltype(a.recv))dlsym(a.h, "ncclRecv");
        a.groupStart = (decltype(a.groupStart))dlsym(a.h, "ncclGroupStart");
        a.groupEnd = (decltype(a.groupEnd))dlsym(a.h, "ncclGroupEnd");
        if (!a.getUniqueId || !a.commInitRank || !a.allReduce || !a.reduceScatter || !a.allGather || !a.commDestroy ||
            !a.getErrorString) {
            a.why = "libnccl is missing a required symbol";
            a.h = nullptr;
        }
    });
    return a.h ? &a : nullptr;
}

const char *why() { return "NCCL unavailable: cannot load libnccl.so.2 with the required symbols (set BTE_NCCL_LIB)"; }

}  // namespace

bool unique_id(void *id128, std::string *err) {
    Api *a = api();
    if (!a) return *err = why(), false;
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId must be 128 bytes");
    ncclUniqueId id;
    ncclResult_t r = a->getUniqueId(&id);
    if (r != ncclSuccess) return *err = a->getErrorString(r), false;
    std::memcpy(id128, &id, sizeof id);
    return true;
}

bool init(Comm *c, const void *id128, int rank, int world, std::string *err) {
    Api *a = api();
    if (!a) return *err = why(), false;
    ncclUniqueId id;
    std::memcpy(&id, id128, sizeof id);
    ncclComm_t comm = nullptr;
    ncclResult_t r = a->commInitRank(&comm, world, id, rank);
    if (r != ncclSuccess) return *err = a->getErrorString(r), false;
    c->comm = comm;
    return true;
}

bool init_local(Comm *c, bte::group::Group *g, int rank, std::string *err) {
    return bte::group::attach(g, rank, &c->local, err);
}

bool allreduce_sum_f64(const Comm &c, double *buf, int64_t n, cudaStream_t s, std::string *err) {
    if (c.local) return bte::group::allreduce_f64(c.local, buf, n, false, s, err);
    Api *a = api();
    if (!a || !c.comm) return *err = why(), false;
    ncclResult_t r = a->allReduce(buf, buf, (size_t)n, ncclFloat64, ncclSum, (ncclComm_t)c.comm, s);
    if (r != ncclSuccess) return *err = a->getErrorString(r), false;
    return true;
}

bool reduce_scatter_sum_f64(const Comm &c, const double *send, double *recv, int64_t recvcount, cudaStream_t s,
                            std::string *err) {
    if (c.local) return bte::group::reduce_scatter_sum_f64(c.local, send, recv, recvcount, s, err);
    Api *a = api();
    if (!a || !c.comm) return *err = why(), false;
    ncclResult_t r = a->reduceScatter(send, recv, (size_t)recvcount, ncclFloat64, ncclSum, (ncclComm_t)c.comm, s);
    if (r != ncclSuccess) return *err = a->getErrorString(r), false;
    return true;
}

bool allgather_f64(const Comm &c, const double *send, double *recv, int64_t sendcount, cudaStream_t s,
                   std::string *err) {
    if (c.local) return bte::group::allgather_f64(c.local, send, recv, sendcount, s, err);
    Api *a = api();
    if (!a || !c.comm) return *err = why(), false;
    ncclResult_t r = a->allGather(send, recv, (size_t)sendcount, ncclFloat64, (ncclComm_t)c.comm, s);
    if (r != ncclSuccess) return *err = a->getErrorString(r), false;
    return true;
}

bool allreduce_max_f64(const Comm &c, double *buf, int64_t n, cudaStream_t s, std::string *err) {
    if (c.local) return bte::group::allreduce_f64(c.local, buf, n, true, s, err);
    Api *a = api();
    if (!a || !c.comm) return *err = why(), false;
    ncclResult_t r = a->allReduce(buf, buf, (size_t)n, ncclFloat64, ncclMax, (ncclComm_t)c.comm, s);
    if (r != ncclSuccess) return *err = a->getErrorString(r), false;
    return true;
}

bool split(const Comm &c, int color, int key, Comm *out, std::string *err) {
    if (c.local) return bte::group::split(c.local, color, key, &out->local, err);
    Api *a = api();
    if (!a || !c.comm) return *err = why(), false;
    if (!a->commSplit) return *err = "libnccl has no ncclCommSplit (NCCL >= 2.18 needed)", false;
    ncclComm_t nc = nullptr;
    ncclResult_t r = a->commSplit((ncclComm_t)c.comm, color, key, &nc, nullptr);
    if (r != ncclSuccess) return *err = a->getErrorString(r), false;
    out->comm = nc;
    return true;
}

bool exchange_f64(const Comm &c, const P2P *ops, int n_ops, cudaStream_t s, std::string *err) {
    if (c.local) {
        std::vector<bte::group::P2P> lo(n_ops);
        for (int i = 0; i < n_ops; ++i) lo[i] = {ops[i].peer, ops[i].send, ops[i].n_send, ops[i].recv, ops[i].n_recv};
        return bte::group::exchange_f64(c.local, lo.data(), n_ops, s, err);
    }
    Api *a = api();
    if (!a || !c.comm) return *err = why(), false;
    if (!a->send || !a->recv || !a->groupStart || !a->groupEnd)
        return *err = "libnccl has no ncclSend / ncclRecv / ncclGroupStart / ncclGroupEnd", false;
    ncclResult_t r = a->groupStart();
    for (int i = 0; i < n_ops && r == ncclSuccess; ++i) {
        if (ops[i].n_send > 0)
            r = a->send(ops[i].send, (size_t)ops[i].n_send, ncclFloat64, ops[i].peer, (ncclComm_t)c.comm, s);
        if (r == ncclSuccess && ops[i].n_recv > 0)
            r = a->recv(ops[i].recv, (size_t)ops[i].n_recv, ncclFloat64, ops[i].peer, (ncclComm_t)c.comm, s);
    }
    const ncclResult_t r2 = a->groupEnd();
    if (r == ncclSuccess) r = r2;
    if (r != ncclSuccess) return *err = a->getErrorString(r), false;
    return true;
}

void destroy(Comm &c) {
    if (c.local) {
        bte::group::release(c.local);
        c.local = nullptr;
        return;
    }
    Api *a = api();
    if (a && c.comm) a->commDestroy((ncclComm_t)c.comm);
    c.comm = nullptr;
}

}  // namespace nccl
}  // namespace bte
