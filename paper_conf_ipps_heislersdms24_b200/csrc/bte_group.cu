// bte_group.cu -- in-process communicator (see bte_group.h).
//
// Protocol of every collective, per rank (host thread), on its stream s:
//   1. record `ready` on s (the rank's inputs are produced), publish the
//      buffers in this collective's post slot, barrier;
//   2. make s wait for every rank's `ready`, enqueue the copies (cudaMemcpyAsync,
//      cudaMemcpyDefault: same device or peer) of what this rank receives and
//      the rank-order reduction kernel, record `done`, barrier;
//   3. make s wait for every rank's `done` (nobody overwrites a buffer a peer
//      still reads), then the in-place results (all-reduce) are written.
// Post slots and events alternate between two sets, so a rank that runs ahead
// into the next collective never touches what a slower rank still reads.
#include "bte_group.h"

#include <algorithm>
#include <chrono>
#include <condition_variable>
#include <map>
#include <mutex>
#include <vector>

namespace bte {
namespace group {

namespace {

constexpr int kBarrierTimeoutS = 120;

struct Post {
    const double *send = nullptr;
    double *recv = nullptr;
    int64_t n = 0;
    cudaEvent_t ready = nullptr, done = nullptr;
    std::vector<P2P> ops;
    int color = 0, key = 0;
};

__global__ void reduce_rows_kernel(const double *__restrict__ stage, int world, int64_t n, double *__restrict__ out,
                                   int take_max) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        double v = stage[i];
        for (int p = 1; p < world; ++p) {  // rank order, the same on every rank
            const double x = stage[(int64_t)p * n + i];
            v = take_max ? fmax(v, x) : v + x;
        }
        out[i] = v;
    }
}

}  // namespace

struct Group {
    int world = 1;
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    uint64_t gen = 0;
    std::vector<Post> post[2];
    std::map<std::pair<uint64_t, int>, Group *> kids;  // split sub-groups: (split number, colour)
    std::vector<Group *> owned;
};

struct Rank {
    Group *g = nullptr;
    int rank = 0;
    uint64_t seq = 0;     // collectives entered (selects the post / event set)
    uint64_t nsplit = 0;  // splits entered
    cudaEvent_t ready[2] = {nullptr, nullptr}, done[2] = {nullptr, nullptr};
    double *stage = nullptr;
    size_t stage_n = 0;
    int stage_dev = -1;
};

namespace {

bool barrier(Group *g, std::string *err) {
    std::unique_lock<std::mutex> lk(g->mu);
    const uint64_t my = g->gen;
    if (++g->arrived == g->world) {
        g->arrived = 0;
        ++g->gen;
        g->cv.notify_all();
        return true;
    }
    if (!g->cv.wait_for(lk, std::chrono::seconds(kBarrierTimeoutS), [&] { return g->gen != my; })) {
        *err = "in-process group: a rank did not enter the collective (barrier timed out)";
        return false;
    }
    return true;
}

bool cuda_ok(cudaError_t e, std::string *err) {
    if (e == cudaSuccess) return true;
    *err = std::string("in-process group: ") + cudaGetErrorString(e);
    return false;
}

double *stage_of(Rank *r, size_t n, std::string *err) {
    int dev = 0;
    if (!cuda_ok(cudaGetDevice(&dev), err)) return nullptr;
    if (r->stage && r->stage_n >= n && r->stage_dev == dev) return r->stage;
    if (r->stage) cudaFree(r->stage);
    r->stage = nullptr;
    if (!cuda_ok(cudaMalloc(&r->stage, std::max<size_t>(n, 1) * sizeof(double)), err)) return nullptr;
    r->stage_n = n;
    r->stage_dev = dev;
    return r->stage;
}

// Phase 1: publish and wait for every rank's inputs.  Returns this collective's post set.
std::vector<Post> *enter(Rank *r, Post p, cudaStream_t s, std::string *err) {
    const int k = (int)(r->seq & 1);
    if (!cuda_ok(cudaEventRecord(r->ready[k], s), err)) return nullptr;
    p.ready = r->ready[k];
    p.done = r->done[k];
    {
        std::lock_guard<std::mutex> lk(r->g->mu);
        r->g->post[k][r->rank] = std::move(p);
    }
    if (!barrier(r->g, err)) return nullptr;
    std::vector<Post> *ps = &r->g->post[k];
    for (int q = 0; q < r->g->world; ++q)
        if (q != r->rank && !cuda_ok(cudaStreamWaitEvent(s, (*ps)[q].ready, 0), err)) return nullptr;
    return ps;
}

// Phases 2-3: this rank's reads are enqueued; wait until every rank's are.
bool leave(Rank *r, std::vector<Post> *ps, cudaStream_t s, std::string *err) {
    const int k = (int)(r->seq & 1);
    if (!cuda_ok(cudaEventRecord(r->done[k], s), err)) return false;
    if (!barrier(r->g, err)) return false;
    for (int q = 0; q < r->g->world; ++q)
        if (q != r->rank && !cuda_ok(cudaStreamWaitEvent(s, (*ps)[q].done, 0), err)) return false;
    ++r->seq;
    return true;
}

bool reduce(const double *stage, int world, int64_t n, double *out, bool take_max, cudaStream_t s,
            std::string *err) {
    if (n <= 0) return true;
    const int tb = 256;
    const int64_t gb = std::min<int64_t>(4096, (n + tb - 1) / tb);
    reduce_rows_kernel<<<(unsigned)gb, tb, 0, s>>>(stage, world, n, out, take_max ? 1 : 0);
    return cuda_ok(cudaGetLastError(), err);
}

}  // namespace

Group *create(int world) {
    if (world < 1) return nullptr;
    Group *g = new Group();
    g->world = world;
    g->post[0].resize(world);
    g->post[1].resize(world);
    return g;
}

void destroy(Group *g) {
    if (!g) return;
    for (Group *k : g->owned) destroy(k);
    delete g;
}

int world_of(const Group *g) { return g ? g->world : 0; }

bool attach(Group *g, int rank, Rank **out, std::string *err) {
    if (!g || rank < 0 || rank >= g->world) return *err = "in-process group: rank out of range", false;
    Rank *r = new Rank();
    r->g = g;
    r->rank = rank;
    for (int k = 0; k < 2; ++k)
        if (!cuda_ok(cudaEventCreateWithFlags(&r->ready[k], cudaEventDisableTiming), err) ||
            !cuda_ok(cudaEventCreateWithFlags(&r->done[k], cudaEventDisableTiming), err)) {
            release(r);
            return false;
        }
    *out = r;
    return true;
}

void release(Rank *r) {
    if (!r) return;
    for (int k = 0; k < 2; ++k) {
        if (r->ready[k]) cudaEventDestroy(r->ready[k]);
        if (r->done[k]) cudaEventDestroy(r->done[k]);
    }
    if (r->stage) cudaFree(r->stage);
    delete r;
}

bool allreduce_f64(Rank *r, double *buf, int64_t n, bool take_max, cudaStream_t s, std::string *err) {
    const int P = r->g->world;
    double *st = stage_of(r, (size_t)P * n, err);
    if (!st) return false;
    Post p;
    p.send = buf;
    p.n = n;
    std::vector<Post> *ps = enter(r, p, s, err);
    if (!ps) return false;
    for (int q = 0; q < P; ++q)
        if (n > 0 && !cuda_ok(cudaMemcpyAsync(st + (int64_t)q * n, (*ps)[q].send, n * sizeof(double),
                                              cudaMemcpyDefault, s), err))
            return false;
    if (!leave(r, ps, s, err)) return false;  // (every rank has read every buffer before any is overwritten)
    return reduce(st, P, n, buf, take_max, s, err);
}

bool reduce_scatter_sum_f64(Rank *r, const double *send, double *recv, int64_t recvcount, cudaStream_t s,
                            std::string *err) {
    const int P = r->g->world;
    double *st = stage_of(r, (size_t)P * recvcount, err);
    if (!st) return false;
    Post p;
    p.send = send;
    p.n = recvcount;
    std::vector<Post> *ps = enter(r, p, s, err);
    if (!ps) return false;
    for (int q = 0; q < P; ++q)
        if (recvcount > 0 &&
            !cuda_ok(cudaMemcpyAsync(st + (int64_t)q * recvcount, (*ps)[q].send + (int64_t)r->rank * recvcount,
                                     recvcount * sizeof(double), cudaMemcpyDefault, s), err))
            return false;
    if (!reduce(st, P, recvcount, recv, false, s, err)) return false;
    return leave(r, ps, s, err);
}

bool allgather_f64(Rank *r, const double *send, double *recv, int64_t sendcount, cudaStream_t s, std::string *err) {
    const int P = r->g->world;
    Post p;
    p.send = send;
    p.n = sendcount;
    std::vector<Post> *ps = enter(r, p, s, err);
    if (!ps) return false;
    for (int q = 0; q < P; ++q) {
        double *dst = recv + (int64_t)q * sendcount;
        if (sendcount > 0 && (*ps)[q].send != dst &&
            !cuda_ok(cudaMemcpyAsync(dst, (*ps)[q].send, sendcount * sizeof(double), cudaMemcpyDefault, s), err))
            return false;
    }
    return leave(r, ps, s, err);
}

bool exchange_f64(Rank *r, const P2P *ops, int n_ops, cudaStream_t s, std::string *err) {
    Post p;
    p.ops.assign(ops, ops + n_ops);
    std::vector<Post> *ps = enter(r, p, s, err);
    if (!ps) return false;
    for (int i = 0; i < n_ops; ++i) {
        if (ops[i].n_recv <= 0) continue;
        const int q = ops[i].peer;
        if (q < 0 || q >= r->g->world) return *err = "in-process group: peer out of range", false;
        const P2P *match = nullptr;
        for (const P2P &o : (*ps)[q].ops)
            if (o.peer == r->rank) match = &o;
        if (!match || match->n_send != ops[i].n_recv)
            return *err = "in-process group: send / receive sizes of a peer pair differ", false;
        if (!cuda_ok(cudaMemcpyAsync(ops[i].recv, match->send, ops[i].n_recv * sizeof(double), cudaMemcpyDefault, s),
                     err))
            return false;
    }
    return leave(r, ps, s, err);
}

bool split(Rank *r, int color, int key, Rank **out, std::string *err) {
    Group *g = r->g;
    Post p;
    p.color = color;
    p.key = key;
    const int k = (int)(r->seq & 1);
    {
        std::lock_guard<std::mutex> lk(g->mu);
        g->post[k][r->rank] = p;
    }
    if (!barrier(g, err)) return false;
    std::vector<std::pair<int, int>> members;  // (key, old rank) of this colour
    for (int q = 0; q < g->world; ++q)
        if (g->post[k][q].color == color) members.push_back({g->post[k][q].key, q});
    std::sort(members.begin(), members.end());
    int me = 0;
    for (int i = 0; i < (int)members.size(); ++i)
        if (members[i].second == r->rank) me = i;
    Group *kid = nullptr;
    {
        std::lock_guard<std::mutex> lk(g->mu);
        Group *&slot = g->kids[{r->nsplit, color}];
        if (!slot) {
            slot = create((int)members.size());
            g->owned.push_back(slot);
        }
        kid = slot;
    }
    ++r->nsplit;
    if (!barrier(g, err)) return false;
    ++r->seq;
    return attach(kid, me, out, err);
}

}  // namespace group
}  // namespace bte
