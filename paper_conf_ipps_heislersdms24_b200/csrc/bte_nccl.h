// bte_nccl.h -- NCCL, loaded at run time with dlopen so that single-GPU use
// needs no NCCL and the library links against nothing but the CUDA runtime.
// Used for the one per-step collective of the band-sharded step: the
// all-reduce of the per-cell energy partials (L760-763).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include <string>

namespace bte {
namespace nccl {

struct Comm {
    void *comm = nullptr;  // ncclComm_t
};

// 128-byte ncclUniqueId into id128.
bool unique_id(void *id128, std::string *err);
bool init(Comm *c, const void *id128, int rank, int world, std::string *err);
// in-place sum of n doubles on stream
bool allreduce_sum_f64(const Comm &c, double *buf, int64_t n, cudaStream_t s, std::string *err);
void destroy(Comm &c);

}  // namespace nccl
}  // namespace bte
