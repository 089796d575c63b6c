// The n_wk / n_k exchange of a multi-GPU sweep (Eq. 4: the global
// ϕ is the sum of the per-GPU partial counts; Alg. 1 lines 14-15, L825-827)
// behind one interface with two backends:
//
//   NcclComm  one process per GPU (torchrun): ncclAllReduce / ncclAllGather
//             over NVLink / NVSwitch, enqueued on the caller's stream.
//   PeerComm  one process, one host thread per rank, each rank a context on
//             its own GPU (or several ranks on one GPU): the ranks exchange
//             device pointers through a host-side group and reduce by
//             reading each other's buffers directly -- a reduce-scatter
//             kernel (rank r sums slice r over all ranks, in place), then an
//             all-gather kernel (rank r copies every other slice from its
//             owner), over NVLink P2P when the devices differ.  Host barriers
//             order the phases.  It is what runs the library's world > 1 path
//             on a single B200 (tests), and a P2P data plane on a node.
//
// Both produce bit-identical integer sums (Eq. 4), so z on G ranks equals z
// on one GPU (SURVEY §8(c) "Multi-GPU" pin).
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/lda.h"
#include "lda_internal.h"

namespace lda {

// ---------------------------------------------------------------------------
// NCCL, opened at run time (only multi-process contexts need it), so that
// loading liblda.so never pins an NCCL build into the process before torch
// loads its own.  dlopen("libnccl.so.2") returns the copy already loaded by
// torch when there is one; LDA_NCCL_LIBRARY overrides the path.
// ---------------------------------------------------------------------------
struct NcclApi {
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
    std::string err;
    bool ok = false;
};

static NcclApi load_nccl() {
    NcclApi a;
    const char *env = std::getenv("LDA_NCCL_LIBRARY");
    const char *cands[] = {env, "libnccl.so.2", "libnccl.so"};
    void *h = nullptr;
    for (const char *c : cands) {
        if (!c) continue;
        h = dlopen(c, RTLD_NOW | RTLD_GLOBAL);
        if (h) break;
    }
    if (!h) {
        a.err = std::string("cannot dlopen NCCL: ") + dlerror();
        return a;
    }
#define LDA_SYM(field, name)                                              \
    a.field = reinterpret_cast<decltype(a.field)>(dlsym(h, name));        \
    if (!a.field) {                                                       \
        a.err = std::string("NCCL symbol missing: ") + name;              \
        return a;                                                         \
    }
    LDA_SYM(GetUniqueId, "ncclGetUniqueId")
    LDA_SYM(CommInitRank, "ncclCommInitRank")
    LDA_SYM(AllReduce, "ncclAllReduce")
    LDA_SYM(AllGather, "ncclAllGather")
    LDA_SYM(CommDestroy, "ncclCommDestroy")
    LDA_SYM(GetErrorString, "ncclGetErrorString")
#undef LDA_SYM
    a.ok = true;
    return a;
}

static const NcclApi &nccl() {
    static NcclApi api = load_nccl();
    return api;
}

int nccl_unique_id(void *out128, std::string &err) {
    if (!nccl().ok) {
        err = nccl().err;
        return LDA_ENCCL;
    }
    ncclUniqueId id;
    ncclResult_t r = nccl().GetUniqueId(&id);
    if (r != ncclSuccess) {
        err = std::string("ncclGetUniqueId: ") + nccl().GetErrorString(r);
        return LDA_ENCCL;
    }
    std::memcpy(out128, &id, sizeof(id));
    return LDA_OK;
}

namespace {

class NcclComm final : public Comm {
  public:
    NcclComm(ncclComm_t c, int rank, int world) : c_(c) {
        rank_ = rank;
        world_ = world;
    }
    ~NcclComm() override {
        if (c_ && nccl().ok) nccl().CommDestroy(c_);
    }
    const char *name() const override { return "nccl"; }
    int allreduce_i32(int32_t *buf, size_t n, void *stream, std::string &err) override {
        return check(nccl().AllReduce(buf, buf, n, ncclInt32, ncclSum, c_, static_cast<cudaStream_t>(stream)),
                     "ncclAllReduce(int32)", err);
    }
    int allreduce_f64(double *buf, size_t n, void *stream, std::string &err) override {
        return check(nccl().AllReduce(buf, buf, n, ncclFloat64, ncclSum, c_, static_cast<cudaStream_t>(stream)),
                     "ncclAllReduce(f64)", err);
    }
    int allgather_i64(const int64_t *send, int64_t *recv, size_t n, void *stream, std::string &err) override {
        return check(nccl().AllGather(send, recv, n, ncclInt64, c_, static_cast<cudaStream_t>(stream)),
                     "ncclAllGather(int64)", err);
    }

  private:
    static int check(ncclResult_t r, const char *what, std::string &err) {
        if (r == ncclSuccess) return LDA_OK;
        err = std::string(what) + ": " + nccl().GetErrorString(r);
        return LDA_ENCCL;
    }
    ncclComm_t c_ = nullptr;
};

}  // namespace

int make_nccl_comm(int rank, int world, const void *uid, int device, std::unique_ptr<Comm> &out,
                   std::string &err) {
    if (!nccl().ok) {
        err = nccl().err;
        return LDA_ENCCL;
    }
    cudaError_t ce = cudaSetDevice(device);
    if (ce != cudaSuccess) {
        err = std::string("cudaSetDevice: ") + cudaGetErrorString(ce);
        return LDA_ECUDA;
    }
    ncclUniqueId id;
    std::memcpy(&id, uid, sizeof(id));
    ncclComm_t c = nullptr;
    ncclResult_t r = nccl().CommInitRank(&c, world, id, rank);
    if (r != ncclSuccess) {
        err = std::string("ncclCommInitRank: ") + nccl().GetErrorString(r);
        return LDA_ENCCL;
    }
    out.reset(new NcclComm(c, rank, world));
    return LDA_OK;
}

// ---------------------------------------------------------------------------
// In-process peer group
// ---------------------------------------------------------------------------
PeerGroup::PeerGroup(int world) : world_(world), ptr_(world, nullptr), dev_(world, -1), joined_(world, 0) {}

int PeerGroup::join(int rank, int device, std::string &err) {
    std::lock_guard<std::mutex> lk(mu_);
    if (rank < 0 || rank >= world_) {
        err = "peer rank outside [0, world)";
        return LDA_EINVAL;
    }
    if (joined_[rank]) {
        err = "peer rank already joined";
        return LDA_EINVAL;
    }
    joined_[rank] = 1;
    dev_[rank] = device;
    return LDA_OK;
}

// Generation barrier over the ranks' host threads.  A rank that does not
// arrive within the timeout (it failed, or its thread is not running) breaks
// the group: every waiting and later call fails instead of hanging.
int PeerGroup::barrier(std::string &err) {
    std::unique_lock<std::mutex> lk(mu_);
    if (broken_) {
        err = "peer group is broken (a rank failed or timed out)";
        return LDA_ECUDA;
    }
    const uint64_t gen = gen_;
    if (++arrived_ == world_) {
        arrived_ = 0;
        ++gen_;
        cv_.notify_all();
        return LDA_OK;
    }
    const auto deadline = std::chrono::steady_clock::now() + std::chrono::seconds(timeout_s_);
    while (gen_ == gen && !broken_) {
        if (cv_.wait_until(lk, deadline) == std::cv_status::timeout && gen_ == gen) {
            broken_ = true;
            cv_.notify_all();
        }
    }
    if (gen_ == gen) {
        err = "peer group barrier: a rank did not arrive (failed or not driven by its own thread)";
        return LDA_ECUDA;
    }
    return LDA_OK;
}

void PeerGroup::set_ptr(int rank, void *p) {
    std::lock_guard<std::mutex> lk(mu_);
    ptr_[rank] = p;
}

void PeerGroup::ptrs(void **out) {
    std::lock_guard<std::mutex> lk(mu_);
    for (int g = 0; g < world_; ++g) out[g] = ptr_[g];
}

int PeerGroup::device(int rank) {
    std::lock_guard<std::mutex> lk(mu_);
    return dev_[rank];
}

void PeerGroup::mark_broken() {
    std::lock_guard<std::mutex> lk(mu_);
    broken_ = true;
    cv_.notify_all();
}

namespace {

class PeerComm final : public Comm {
  public:
    PeerComm(std::shared_ptr<PeerGroup> g, int rank, int device) : g_(std::move(g)), dev_(device) {
        rank_ = rank;
        world_ = g_->world();
    }
    const char *name() const override { return "peer"; }

    int allreduce_i32(int32_t *buf, size_t n, void *stream, std::string &err) override {
        return allreduce(buf, n, sizeof(int32_t), 0, stream, err);
    }
    int allreduce_f64(double *buf, size_t n, void *stream, std::string &err) override {
        return allreduce(buf, n, sizeof(double), 1, stream, err);
    }
    int allgather_i64(const int64_t *send, int64_t *recv, size_t n, void *stream, std::string &err) override {
        cudaStream_t s = static_cast<cudaStream_t>(stream);
        int r = enter(const_cast<int64_t *>(send), s, err);
        if (r != LDA_OK) return r;
        void *p[kMaxPeers];
        g_->ptrs(p);
        for (int q = 0; q < world_ && r == LDA_OK; ++q) {
            if (p[q] == recv + static_cast<size_t>(q) * n) continue;  // this rank's slice, in place
            cudaError_t ce = cudaMemcpyPeerAsync(recv + static_cast<size_t>(q) * n, dev_, p[q], g_->device(q),
                                                 n * sizeof(int64_t), s);
            if (ce == cudaSuccess) ce = cudaStreamSynchronize(s);
            if (ce != cudaSuccess) r = cuda_fail("peer all-gather copy", ce, err);
        }
        return leave(r, err);
    }

  private:
    // the caller's buffer is final once its stream drains; publish it and
    // wait for every rank (first call: enable P2P to the other ranks' GPUs)
    int enter(void *buf, cudaStream_t s, std::string &err) {
        cudaError_t ce = cudaStreamSynchronize(s);
        if (ce != cudaSuccess) {
            g_->mark_broken();
            return cuda_fail("peer collective (stream)", ce, err);
        }
        g_->set_ptr(rank_, buf);
        int r = g_->barrier(err);
        if (r != LDA_OK) return r;
        if (!p2p_done_) {
            for (int q = 0; q < world_; ++q) {
                const int dq = g_->device(q);
                if (dq == dev_) continue;
                int can = 0;
                cudaDeviceCanAccessPeer(&can, dev_, dq);
                if (!can) {
                    g_->mark_broken();
                    err = "peer group: device " + std::to_string(dev_) + " cannot access device " +
                          std::to_string(dq) + " (no P2P)";
                    return LDA_ECUDA;
                }
                ce = cudaDeviceEnablePeerAccess(dq, 0);
                if (ce == cudaErrorPeerAccessAlreadyEnabled) {
                    cudaGetLastError();
                    ce = cudaSuccess;
                }
                if (ce != cudaSuccess) {
                    g_->mark_broken();
                    return cuda_fail("cudaDeviceEnablePeerAccess", ce, err);
                }
            }
            p2p_done_ = true;
        }
        return LDA_OK;
    }
    // last barrier: no rank touches its buffer again until every peer has
    // finished reading it
    int leave(int r, std::string &err) {
        if (r != LDA_OK) {
            g_->mark_broken();
            return r;
        }
        return g_->barrier(err);
    }
    int cuda_fail(const char *what, cudaError_t ce, std::string &err) {
        err = std::string(what) + ": " + cudaGetErrorString(ce);
        return LDA_ECUDA;
    }

    // slice q of n elements: [lo(q), lo(q+1)), boundaries on multiples of
    // 16 bytes so the kernels move 16-byte vectors
    int allreduce(void *buf, size_t n, size_t esz, int is_f64, void *stream, std::string &err) {
        cudaStream_t s = static_cast<cudaStream_t>(stream);
        int r = enter(buf, s, err);
        if (r != LDA_OK) return r;
        void *p[kMaxPeers];
        g_->ptrs(p);
        // reduce-scatter (in place: rank q writes only slice q of its own
        // buffer, which no other rank reads in this phase)
        int e = launch_peer_reduce_scatter(p, world_, rank_, buf, n, esz, is_f64, s);
        cudaError_t ce = e == 0 ? cudaStreamSynchronize(s) : static_cast<cudaError_t>(e);
        if (ce != cudaSuccess) {
            g_->mark_broken();
            return cuda_fail("peer reduce-scatter", ce, err);
        }
        r = g_->barrier(err);
        if (r != LDA_OK) return r;
        // all-gather: every other slice from its owner
        e = launch_peer_all_gather(p, world_, rank_, buf, n, esz, s);
        ce = e == 0 ? cudaStreamSynchronize(s) : static_cast<cudaError_t>(e);
        if (ce != cudaSuccess) r = cuda_fail("peer all-gather", ce, err);
        return leave(r, err);
    }

    std::shared_ptr<PeerGroup> g_;
    int dev_ = 0;
    bool p2p_done_ = false;
};

}  // namespace

int make_peer_comm(const std::shared_ptr<PeerGroup> &g, int rank, int device, std::unique_ptr<Comm> &out,
                   std::string &err) {
    int r = g->join(rank, device, err);
    if (r != LDA_OK) return r;
    out.reset(new PeerComm(g, rank, device));
    return LDA_OK;
}

}  // namespace lda

// Diagnostic (include/lda.h): the NCCL backend end to end with one rank on
// `device` -- dlopen + symbols, ncclGetUniqueId, ncclCommInitRank, the three
// collectives the library issues (in place, on a stream), ncclCommDestroy.
// With one rank every collective is the identity, which is checked.
extern "C" int lda_debug_nccl_selftest(int32_t device, char *msg, int32_t msg_cap) {
    std::string err;
    auto out = [&](int code, const std::string &m) {
        if (msg && msg_cap > 0) {
            std::strncpy(msg, m.c_str(), static_cast<size_t>(msg_cap) - 1);
            msg[msg_cap - 1] = '\0';
        }
        return code;
    };
    unsigned char uid[128];
    int r = lda::nccl_unique_id(uid, err);
    if (r != LDA_OK) return out(r, err);
    std::unique_ptr<lda::Comm> comm;
    r = lda::make_nccl_comm(0, 1, uid, device, comm, err);
    if (r != LDA_OK) return out(r, err);
    const size_t n = 1000;
    int32_t *di = nullptr;
    double *dd = nullptr;
    int64_t *dg = nullptr;
    cudaStream_t s = nullptr;
    cudaError_t ce = cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    if (ce == cudaSuccess) ce = cudaMalloc(&di, n * sizeof(int32_t));
    if (ce == cudaSuccess) ce = cudaMalloc(&dd, n * sizeof(double));
    if (ce == cudaSuccess) ce = cudaMalloc(&dg, 2 * n * sizeof(int64_t));
    std::vector<int32_t> hi(n), hi2(n);
    std::vector<double> hd(n), hd2(n);
    std::vector<int64_t> hg(n), hg2(n);
    for (size_t i = 0; i < n; ++i) {
        hi[i] = static_cast<int32_t>(i * 7919 % 1000003) - 5;
        hd[i] = 0.5 * static_cast<double>(i) - 3.25;
        hg[i] = static_cast<int64_t>(i) * 1000000007LL;
    }
    if (ce == cudaSuccess) ce = cudaMemcpy(di, hi.data(), n * sizeof(int32_t), cudaMemcpyHostToDevice);
    if (ce == cudaSuccess) ce = cudaMemcpy(dd, hd.data(), n * sizeof(double), cudaMemcpyHostToDevice);
    if (ce == cudaSuccess) ce = cudaMemcpy(dg, hg.data(), n * sizeof(int64_t), cudaMemcpyHostToDevice);
    if (ce == cudaSuccess && r == LDA_OK) r = comm->allreduce_i32(di, n, s, err);
    if (ce == cudaSuccess && r == LDA_OK) r = comm->allreduce_f64(dd, n, s, err);
    if (ce == cudaSuccess && r == LDA_OK) r = comm->allgather_i64(dg, dg + n, n, s, err);
    if (ce == cudaSuccess && r == LDA_OK) ce = cudaStreamSynchronize(s);
    if (ce == cudaSuccess && r == LDA_OK) ce = cudaMemcpy(hi2.data(), di, n * sizeof(int32_t), cudaMemcpyDeviceToHost);
    if (ce == cudaSuccess && r == LDA_OK) ce = cudaMemcpy(hd2.data(), dd, n * sizeof(double), cudaMemcpyDeviceToHost);
    if (ce == cudaSuccess && r == LDA_OK)
        ce = cudaMemcpy(hg2.data(), dg + n, n * sizeof(int64_t), cudaMemcpyDeviceToHost);
    if (di) cudaFree(di);
    if (dd) cudaFree(dd);
    if (dg) cudaFree(dg);
    if (s) cudaStreamDestroy(s);
    const std::string name = comm->name();
    comm.reset();
    if (ce != cudaSuccess) return out(LDA_ECUDA, cudaGetErrorString(ce));
    if (r != LDA_OK) return out(r, err);
    if (hi2 != hi || hd2 != hd || hg2 != hg) return out(LDA_ENCCL, "one-rank collectives changed the data");
    return out(LDA_OK, name + ": one-rank allreduce(int32), allreduce(fp64), allgather(int64) ok");
}
