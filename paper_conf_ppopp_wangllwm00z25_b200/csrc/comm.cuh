// comm.cuh — collectives used by the multi-GPU phase-1 driver (§4.3).
//
// One process per GPU.  The product backend is NCCL (loaded with dlopen, so
// single-GPU use never needs it): label slices are exchanged with grouped
// ncclBroadcast calls (an in-place allgatherv — edge-balanced ranges have
// unequal sizes and global vertex ids must stay contiguous), sparse deltas and
// partial coarse graphs with the same allgatherv, counters with ncclAllReduce.
//
// A loopback backend runs P "ranks" as threads of one process on one device
// (device-to-device copies + a host barrier).  It exists so the partitioned
// algorithm can be tested on the single GPU this project's CI provides; it is
// selected only by a uid made with gala_loopback_unique_id (test hook).
#pragma once
#include <dlfcn.h>
#include <nccl.h>

#include <condition_variable>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <vector>

struct Comm {
    int rank = 0, world = 1;
    virtual ~Comm() {}
    // recv[displs[r] .. displs[r] + counts[r]) <- rank r's send (bytes); device buffers on `st`
    virtual void allgatherv(const void* send, void* recv, const std::vector<size_t>& counts,
                            const std::vector<size_t>& displs, cudaStream_t st) = 0;
    // in-place elementwise sum of int64 device buffer
    virtual void allreduce_sum_i64(int64_t* buf, size_t count, cudaStream_t st) = 0;
    // host scalar from every rank (synchronises)
    virtual std::vector<int64_t> allgather_host(int64_t x, cudaStream_t st) = 0;
    // this rank failed mid-run: release peers blocked in a collective (they raise CommError)
    virtual void abort() {}
};

// ------------------------------------------------------------------ NCCL (dlopen)
struct NcclApi {
    void* h = nullptr;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    bool load() {
        if (h) return true;
        const char* names[] = {"libnccl.so.2", "libnccl.so"};
        for (const char* nm : names) {
            h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
            if (h) break;
        }
        if (!h) return false;
#define NCCL_SYM(f) f = reinterpret_cast<decltype(f)>(dlsym(h, "nccl" #f))
        NCCL_SYM(GetUniqueId); NCCL_SYM(CommInitRank); NCCL_SYM(CommDestroy); NCCL_SYM(AllReduce);
        NCCL_SYM(AllGather); NCCL_SYM(Broadcast); NCCL_SYM(GroupStart); NCCL_SYM(GroupEnd); NCCL_SYM(GetErrorString);
#undef NCCL_SYM
        return GetUniqueId && CommInitRank && CommDestroy && AllReduce && AllGather && Broadcast && GroupStart &&
               GroupEnd && GetErrorString;
    }
};
static NcclApi& nccl_api() {
    static NcclApi a;
    return a;
}

struct CommError {
    std::string msg;
};

struct NcclComm : Comm {
    ncclComm_t comm = nullptr;
    NcclApi& api;
    NcclComm(const void* uid, int r, int w) : api(nccl_api()) {
        rank = r;
        world = w;
        ncclUniqueId id;
        memcpy(&id, uid, sizeof(id));
        ck(api.CommInitRank(&comm, w, id, r));
    }
    ~NcclComm() override {
        if (comm) api.CommDestroy(comm);
    }
    void ck(ncclResult_t r) {
        if (r != ncclSuccess) throw CommError{std::string("NCCL: ") + api.GetErrorString(r)};
    }
    void allgatherv(const void* send, void* recv, const std::vector<size_t>& counts, const std::vector<size_t>& displs,
                    cudaStream_t st) override {
        ck(api.GroupStart());
        for (int r = 0; r < world; ++r) {
            if (!counts[r]) continue;
            ck(api.Broadcast(r == rank ? send : nullptr, static_cast<char*>(recv) + displs[r], counts[r], ncclChar, r,
                             comm, st));
        }
        ck(api.GroupEnd());
    }
    void allreduce_sum_i64(int64_t* buf, size_t count, cudaStream_t st) override {
        ck(api.AllReduce(buf, buf, count, ncclInt64, ncclSum, comm, st));
    }
    int64_t* scratch = nullptr;   // world + 1 int64, allocated once
    int64_t* hscratch = nullptr;  // pinned mirror
    std::vector<int64_t> allgather_host(int64_t x, cudaStream_t st) override {
        if (!scratch) {
            cudaMalloc(&scratch, sizeof(int64_t) * (world + 1));
            cudaMallocHost(&hscratch, sizeof(int64_t) * (world + 1));
        }
        hscratch[world] = x;
        cudaMemcpyAsync(scratch + world, hscratch + world, sizeof(int64_t), cudaMemcpyHostToDevice, st);
        ck(api.AllGather(scratch + world, scratch, 1, ncclInt64, comm, st));
        cudaMemcpyAsync(hscratch, scratch, sizeof(int64_t) * world, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        return std::vector<int64_t>(hscratch, hscratch + world);
    }
};

// ------------------------------------------------------------------ loopback (test hook)
struct LoopShared {
    int world = 0;
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    long long generation = 0;
    std::vector<const void*> ptr;
    std::vector<cudaEvent_t> ev;
    std::vector<int64_t> scal;
    bool aborted = false;
    void barrier();
    void abort() {
        std::lock_guard<std::mutex> lk(mu);
        aborted = true;
        cv.notify_all();
    }
};
struct CommError;
inline void LoopShared::barrier() {
    std::unique_lock<std::mutex> lk(mu);
    long long gen = generation;
    if (aborted) throw CommError{"loopback: a peer rank failed"};
    if (++arrived == world) {
        arrived = 0;
        ++generation;
        cv.notify_all();
    } else {
        cv.wait(lk, [&] { return generation != gen || aborted; });
        if (generation == gen) throw CommError{"loopback: a peer rank failed"};
    }
}
static std::mutex g_loop_mu;
static std::map<std::string, std::shared_ptr<LoopShared>> g_loops;

__global__ void k_sum_rows_i64(int64_t* out, const int64_t* in, size_t count, int world) {
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (size_t)gridDim.x * blockDim.x) {
        int64_t s = 0;
        for (int r = 0; r < world; ++r) s += in[(size_t)r * count + i];
        out[i] = s;
    }
}

struct LoopComm : Comm {
    std::shared_ptr<LoopShared> sh;
    void abort() override { sh->abort(); }
    LoopComm(const void* uid, int r, int w) {
        rank = r;
        world = w;
        std::string key(static_cast<const char*>(uid), 128);
        std::lock_guard<std::mutex> lk(g_loop_mu);
        auto& s = g_loops[key];
        if (!s) {
            s = std::make_shared<LoopShared>();
            s->world = w;
            s->ptr.assign(w, nullptr);
            s->ev.assign(w, nullptr);
            s->scal.assign(w, 0);
        }
        sh = s;
        cudaEventCreateWithFlags(&sh->ev[r], cudaEventDisableTiming);
    }
    ~LoopComm() override {}
    // publish `p` and an event marking this rank's stream position, wait for all
    void publish(const void* p, cudaStream_t st) {
        sh->ptr[rank] = p;
        cudaEventRecord(sh->ev[rank], st);
        sh->barrier();
        for (int r = 0; r < world; ++r)
            if (r != rank) cudaStreamWaitEvent(st, sh->ev[r], 0);
    }
    void finish(cudaStream_t st) {   // nobody proceeds until every rank's reads are ordered
        sh->barrier();
        cudaEventRecord(sh->ev[rank], st);
        sh->barrier();
        for (int r = 0; r < world; ++r)
            if (r != rank) cudaStreamWaitEvent(st, sh->ev[r], 0);
        sh->barrier();
    }
    void allgatherv(const void* send, void* recv, const std::vector<size_t>& counts, const std::vector<size_t>& displs,
                    cudaStream_t st) override {
        publish(send, st);
        for (int r = 0; r < world; ++r)
            if (counts[r])
                cudaMemcpyAsync(static_cast<char*>(recv) + displs[r], sh->ptr[r], counts[r], cudaMemcpyDeviceToDevice, st);
        finish(st);
    }
    int64_t* tmp = nullptr;
    size_t tmp_cap = 0;
    void allreduce_sum_i64(int64_t* buf, size_t count, cudaStream_t st) override {
        if (tmp_cap < count * world) {
            cudaStreamSynchronize(st);
            if (tmp) cudaFree(tmp);
            tmp_cap = count * world + 64;
            cudaMalloc(&tmp, sizeof(int64_t) * tmp_cap);
        }
        publish(buf, st);
        for (int r = 0; r < world; ++r)
            cudaMemcpyAsync(tmp + (size_t)r * count, sh->ptr[r], sizeof(int64_t) * count, cudaMemcpyDeviceToDevice, st);
        finish(st);   // everyone has copied every buffer before anyone overwrites its own
        k_sum_rows_i64<<<(unsigned)std::min<size_t>((count + 255) / 256 + 1, 1024), 256, 0, st>>>(buf, tmp, count, world);
    }
    std::vector<int64_t> allgather_host(int64_t x, cudaStream_t st) override {
        cudaStreamSynchronize(st);
        sh->scal[rank] = x;
        sh->barrier();
        std::vector<int64_t> out = sh->scal;
        sh->barrier();
        return out;
    }
};
