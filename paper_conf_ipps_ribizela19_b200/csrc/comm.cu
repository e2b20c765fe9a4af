// comm.cu -- NCCL and in-process implementations of ss_comm::ShardComm
// (comm.cuh).  NCCL is resolved with dlopen on first use (SS_NCCL_LIB, else
// the libnccl.so.2 already loaded by the process -- torch's -- else the
// system's), so libsampleselect.so itself has no link-time NCCL dependency.
#include <dlfcn.h>

#include <algorithm>

#include <condition_variable>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <vector>

#include "comm.cuh"

// ---------------------------------------------------------------- NCCL -----
namespace {

// The few NCCL declarations used (nccl.h, NCCL 2.x ABI).
typedef struct ncclComm* ncclComm_t;
typedef struct { char internal[128]; } ncclUniqueId;
typedef int ncclResult_t;   // ncclSuccess = 0
enum { nccl_Sum = 0, nccl_Uint32 = 3, nccl_Uint64 = 5 };

struct NcclApi {
    bool ok = false;
    std::string why;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi& nccl() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        const char* env = std::getenv("SS_NCCL_LIB");
        void* h = nullptr;
        if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);   // torch's, if loaded
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            api.why = std::string("cannot load libnccl.so.2: ") + dlerror();
            return;
        }
        api.GetUniqueId = (ncclResult_t(*)(ncclUniqueId*))dlsym(h, "ncclGetUniqueId");
        api.CommInitRank = (ncclResult_t(*)(ncclComm_t*, int, ncclUniqueId, int))dlsym(h, "ncclCommInitRank");
        api.CommDestroy = (ncclResult_t(*)(ncclComm_t))dlsym(h, "ncclCommDestroy");
        api.AllReduce = (ncclResult_t(*)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t))dlsym(
            h, "ncclAllReduce");
        api.GetErrorString = (const char* (*)(ncclResult_t))dlsym(h, "ncclGetErrorString");
        if (!api.GetUniqueId || !api.CommInitRank || !api.CommDestroy || !api.AllReduce || !api.GetErrorString) {
            api.why = "libnccl.so.2 lacks an expected symbol";
            return;
        }
        api.ok = true;
    });
    return api;
}

std::string nccl_err(ncclResult_t r) {
    NcclApi& a = nccl();
    return a.GetErrorString ? a.GetErrorString(r) : ("NCCL error " + std::to_string(r));
}

class NcclComm : public ss_comm::ShardComm {
public:
    NcclComm(ncclComm_t c, int n, int r) : comm_(c), n_(n), r_(r) {}
    ~NcclComm() override {
        if (comm_) nccl().CommDestroy(comm_);
    }
    int nranks() const override { return n_; }
    int rank() const override { return r_; }
    bool capturable() const override { return true; }
    ss_status allreduce_sum(const void* send, void* recv, size_t count, int elem_bytes, cudaStream_t st,
                            std::string& err) override {
        const ncclResult_t r = nccl().AllReduce(send, recv, count, elem_bytes == 8 ? nccl_Uint64 : nccl_Uint32,
                                                nccl_Sum, comm_, st);
        if (r) {
            err = "ncclAllReduce: " + nccl_err(r);
            return SS_ERR_NCCL;
        }
        return SS_OK;
    }

private:
    ncclComm_t comm_;
    int n_, r_;
};

}  // namespace

// ---------------------------------------------------- in-process group -----
struct ss_local_group {
    int n = 0;
    std::mutex mu;
    std::condition_variable cv;
    int waiting = 0;
    unsigned long long gen = 0;
    std::vector<const void*> slots;
    void barrier() {
        std::unique_lock<std::mutex> lk(mu);
        const unsigned long long g = gen;
        if (++waiting == n) {
            waiting = 0;
            ++gen;
            cv.notify_all();
        } else {
            cv.wait(lk, [&] { return gen != g; });
        }
    }
};

namespace {

constexpr int LOCAL_MAX = 16;
struct SrcList { const void* p[LOCAL_MAX]; int n; };

template <typename U>
__global__ void local_sum_kernel(SrcList src, U* __restrict__ dst, size_t count) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < count; i += (size_t)gridDim.x * blockDim.x) {
        U acc = 0;
        for (int q = 0; q < src.n; ++q) acc += reinterpret_cast<const U*>(src.p[q])[i];
        dst[i] = acc;
    }
}

// Ranks are host threads of one process (contexts on one device, or on
// peer-accessible devices): each collective synchronises the caller's stream,
// publishes its send buffer, meets the others at a barrier, sums every rank's
// buffer into its own receive buffer, and meets them again before anyone may
// reuse its send buffer.  Not capturable (host barriers).
class LocalComm : public ss_comm::ShardComm {
public:
    LocalComm(ss_local_group* g, int r) : g_(g), r_(r) {}
    int nranks() const override { return g_->n; }
    int rank() const override { return r_; }
    bool capturable() const override { return false; }
    ss_status allreduce_sum(const void* send, void* recv, size_t count, int elem_bytes, cudaStream_t st,
                            std::string& err) override {
        cudaError_t e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) {
            err = std::string("local allreduce: ") + cudaGetErrorString(e);
            return SS_ERR_CUDA;
        }
        // a separate copy of the input when in-place: others read `send`
        const void* src = send;
        void* tmp = nullptr;
        if (send == recv && count) {
            if ((e = cudaMalloc(&tmp, count * elem_bytes)) != cudaSuccess ||
                (e = cudaMemcpy(tmp, send, count * elem_bytes, cudaMemcpyDeviceToDevice)) != cudaSuccess) {
                cudaFree(tmp);
                err = std::string("local allreduce: ") + cudaGetErrorString(e);
                return SS_ERR_CUDA;
            }
            src = tmp;
        }
        g_->slots[r_] = src;
        g_->barrier();
        SrcList l{};
        l.n = g_->n;
        for (int q = 0; q < l.n; ++q) l.p[q] = g_->slots[q];
        if (count) {
            const unsigned blocks = (unsigned)std::min<size_t>((count + 255) / 256, 1024);
            if (elem_bytes == 8) local_sum_kernel<unsigned long long><<<blocks, 256, 0, st>>>(
                l, (unsigned long long*)recv, count);
            else local_sum_kernel<unsigned><<<blocks, 256, 0, st>>>(l, (unsigned*)recv, count);
        }
        e = cudaGetLastError();
        const cudaError_t e2 = cudaStreamSynchronize(st);
        g_->barrier();   // every rank has read every send buffer
        cudaFree(tmp);
        if (e == cudaSuccess) e = e2;
        if (e != cudaSuccess) {
            err = std::string("local allreduce: ") + cudaGetErrorString(e);
            return SS_ERR_CUDA;
        }
        return SS_OK;
    }

private:
    ss_local_group* g_;
    int r_;
};

}  // namespace

namespace ss_comm {

ss_status nccl_unique_id(char out[128], std::string& err) {
    NcclApi& a = nccl();
    if (!a.ok) {
        err = a.why;
        return SS_ERR_NCCL;
    }
    ncclUniqueId id;
    const ncclResult_t r = a.GetUniqueId(&id);
    if (r) {
        err = "ncclGetUniqueId: " + nccl_err(r);
        return SS_ERR_NCCL;
    }
    std::memcpy(out, id.internal, 128);
    return SS_OK;
}

ShardComm* make_nccl_comm(const char id[128], int nranks, int rank, int device, ss_status* rc, std::string& err) {
    NcclApi& a = nccl();
    if (!a.ok) {
        err = a.why;
        *rc = SS_ERR_NCCL;
        return nullptr;
    }
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(device);
    ncclUniqueId uid;
    std::memcpy(uid.internal, id, 128);
    ncclComm_t comm = nullptr;
    const ncclResult_t r = a.CommInitRank(&comm, nranks, uid, rank);
    if (prev >= 0) cudaSetDevice(prev);
    if (r) {
        err = "ncclCommInitRank: " + nccl_err(r);
        *rc = SS_ERR_NCCL;
        return nullptr;
    }
    ShardComm* c = new (std::nothrow) NcclComm(comm, nranks, rank);
    if (!c) {
        a.CommDestroy(comm);
        *rc = SS_ERR_OUT_OF_MEMORY;
        return nullptr;
    }
    *rc = SS_OK;
    return c;
}

ss_status local_group_create(int nranks, ss_local_group** out) {
    if (!out || nranks < 1 || nranks > LOCAL_MAX) return SS_ERR_INVALID_ARGUMENT;
    ss_local_group* g = new (std::nothrow) ss_local_group();
    if (!g) return SS_ERR_OUT_OF_MEMORY;
    g->n = nranks;
    g->slots.assign(nranks, nullptr);
    *out = g;
    return SS_OK;
}

void local_group_destroy(ss_local_group* g) { delete g; }

ShardComm* make_local_comm(ss_local_group* g, int rank, int /*device*/, ss_status* rc, std::string& err) {
    if (!g || rank < 0 || rank >= g->n) {
        err = "bad local group or rank";
        *rc = SS_ERR_INVALID_ARGUMENT;
        return nullptr;
    }
    ShardComm* c = new (std::nothrow) LocalComm(g, rank);
    *rc = c ? SS_OK : SS_ERR_OUT_OF_MEMORY;
    return c;
}

}  // namespace ss_comm
