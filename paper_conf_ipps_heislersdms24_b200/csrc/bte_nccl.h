// bte_nccl.h -- NCCL, loaded at run time with dlopen so that single-GPU use
// needs no NCCL and the library links against nothing but the CUDA runtime.
// Used for the per-step exchange of the band-sharded step (L760-763, SURVEY
// 8(e)): reduce-scatter of the per-cell energy partials, the temperature solve
// on this rank's cell chunk, all-gather of T (or one all-reduce of E and a
// replicated solve), and the halo exchange of the cell-partitioned step.
//
// Every call also takes an in-process communicator (bte_group.h: the ranks are
// host threads of one process): Comm.local set -> the same collective runs as
// device copies between the ranks' buffers instead of through NCCL.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include <string>

#include "bte_group.h"

namespace bte {
namespace nccl {

struct Comm {
    void *comm = nullptr;              // ncclComm_t
    bte::group::Rank *local = nullptr;  // in-process group endpoint (instead of NCCL)
};

// Endpoint `rank` of an in-process group (bte_group_create).
bool init_local(Comm *c, bte::group::Group *g, int rank, std::string *err);

// 128-byte ncclUniqueId into id128.
bool unique_id(void *id128, std::string *err);
bool init(Comm *c, const void *id128, int rank, int world, std::string *err);
// in-place sum of n doubles on stream
bool allreduce_sum_f64(const Comm &c, double *buf, int64_t n, cudaStream_t s, std::string *err);
// recv[recvcount] = this rank's chunk of the sum of every rank's send[world * recvcount]
bool reduce_scatter_sum_f64(const Comm &c, const double *send, double *recv, int64_t recvcount, cudaStream_t s,
                            std::string *err);
// recv[world * sendcount] = every rank's send[sendcount] in rank order (in place: send = recv + rank * sendcount)
bool allgather_f64(const Comm &c, const double *send, double *recv, int64_t sendcount, cudaStream_t s,
                   std::string *err);
// in-place max of n doubles (the positivity bound of a cell-partitioned run)
bool allreduce_max_f64(const Comm &c, double *buf, int64_t n, cudaStream_t s, std::string *err);
// sub-communicator of the ranks with the same colour, ordered by key (ncclCommSplit)
bool split(const Comm &c, int color, int key, Comm *out, std::string *err);
// halo exchange of a cell-partitioned run: one NCCL group of
// point-to-point sends and receives of doubles, peer[i] = world rank
struct P2P {
    int peer;
    const double *send;
    int64_t n_send;
    double *recv;
    int64_t n_recv;
};
bool exchange_f64(const Comm &c, const P2P *ops, int n_ops, cudaStream_t s, std::string *err);
void destroy(Comm &c);

}  // namespace nccl
}  // namespace bte
