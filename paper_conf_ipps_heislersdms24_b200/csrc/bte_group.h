// bte_group.h -- in-process communicator: the ranks of a band-sharded /
// cell-partitioned run are host threads of ONE process, each driving its own
// context (on any device, several may share one), and the step's exchanges
// (reduce-scatter of the per-cell energy, all-gather of T, the
// all-reduce variants; N3: the halo send/receive group and the split
// communicator of a band group) run as device copies between the ranks'
// buffers, ordered by CUDA events, with host barriers between the phases.
//
// Same semantics as the NCCL calls in bte_nccl.h (the library calls either
// through bte::nccl::*), so the multi-rank code path of bte_create / bte_step
// runs unchanged on one GPU.  Sums are taken in rank order, identically on
// every rank (every rank gets the same bits).  Not graph-capturable: contexts
// on a group step launch by launch.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <string>

namespace bte {
namespace group {

struct Group;  // shared by the ranks (opaque)
struct Rank;   // one rank's endpoint: its group, index and stream-ordering events

Group *create(int world);
void destroy(Group *g);  // after every endpoint is released
int world_of(const Group *g);

// Endpoint of `rank` (collective over the group's ranks: every rank calls it once).
bool attach(Group *g, int rank, Rank **out, std::string *err);
void release(Rank *r);

bool allreduce_f64(Rank *r, double *buf, int64_t n, bool max, cudaStream_t s, std::string *err);
bool reduce_scatter_sum_f64(Rank *r, const double *send, double *recv, int64_t recvcount, cudaStream_t s,
                            std::string *err);
bool allgather_f64(Rank *r, const double *send, double *recv, int64_t sendcount, cudaStream_t s, std::string *err);
struct P2P {
    int peer;
    const double *send;
    int64_t n_send;
    double *recv;
    int64_t n_recv;
};
bool exchange_f64(Rank *r, const P2P *ops, int n_ops, cudaStream_t s, std::string *err);
// Sub-group of the ranks with the same colour, ordered by (key, rank).
bool split(Rank *r, int color, int key, Rank **out, std::string *err);

}  // namespace group
}  // namespace bte
