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
    // peer memory (fabric.cuh): every rank passes one cudaMalloc'd device region and gets every
    // rank's region mapped into its address space (index = rank; its own pointer at `rank`).
    // Collective.  The mappings stay valid until release_region.
    virtual std::vector<void*> share_region(void* mine, cudaStream_t st) = 0;
    virtual void release_region(const std::vector<void*>& peers) { (void)peers; }
    // host-side rendezvous of ranks that share one process (loopback); a no-op across processes
    virtual void host_barrier() {}
    // may a kernel of this rank spin until the other ranks' kernels arrive (fabric device
    // barrier)?  Only when every rank has its own GPU: kernels of several ranks on ONE device
    // are not guaranteed to be co-resident (B200_PROFILING.md: Xid 109 when they are not), so
    // the loopback ranks meet on the host instead (stream sync + host barrier).
    virtual bool device_barrier_ok() const { return true; }
    // personalised exchange (bytes): send + sdispls[p] .. + scounts[p] goes to rank p, which
    // receives it at recv + its rdispls[this rank]; device buffers on `st`
    virtual void alltoallv(const void* send, const std::vector<size_t>& scounts, const std::vector<size_t>& sdispls,
                           void* recv, const std::vector<size_t>& rcounts, const std::vector<size_t>& rdispls,
                           cudaStream_t st) = 0;
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
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
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
        NCCL_SYM(Send); NCCL_SYM(Recv);
#undef NCCL_SYM
        return GetUniqueId && CommInitRank && CommDestroy && AllReduce && AllGather && Broadcast && GroupStart &&
               GroupEnd && GetErrorString && Send && Recv;
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
    void alltoallv(const void* send, const std::vector<size_t>& scounts, const std::vector<size_t>& sdispls, void* recv,
                   const std::vector<size_t>& rcounts, const std::vector<size_t>& rdispls, cudaStream_t st) override {
        ck(api.GroupStart());
        for (int p = 0; p < world; ++p) {
            if (scounts[p]) ck(api.Send(static_cast<const char*>(send) + sdispls[p], scounts[p], ncclChar, p, comm, st));
            if (rcounts[p]) ck(api.Recv(static_cast<char*>(recv) + rdispls[p], rcounts[p], ncclChar, p, comm, st));
        }
        ck(api.GroupEnd());
    }
    int64_t* scratch = nullptr;   // world + 1 int64, allocated once
    int64_t* hscratch = nullptr;  // pinned mirror
    void ensure_scratch() {
        if (scratch) return;
        if (cudaMalloc(&scratch, sizeof(int64_t) * (world + 1)) != cudaSuccess) {
            scratch = nullptr;
            throw CommError{"allgather_host: cudaMalloc failed"};
        }
        if (cudaMallocHost(&hscratch, sizeof(int64_t) * (world + 1)) != cudaSuccess) {
            cudaFree(scratch);
            scratch = nullptr;
            hscratch = nullptr;
            throw CommError{"allgather_host: cudaMallocHost failed"};
        }
    }
    std::vector<int64_t> allgather_host(int64_t x, cudaStream_t st) override {
        ensure_scratch();
        hscratch[world] = x;
        cudaMemcpyAsync(scratch + world, hscratch + world, sizeof(int64_t), cudaMemcpyHostToDevice, st);
        ck(api.AllGather(scratch + world, scratch, 1, ncclInt64, comm, st));
        cudaMemcpyAsync(hscratch, scratch, sizeof(int64_t) * world, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        return std::vector<int64_t>(hscratch, hscratch + world);
    }
    // CUDA IPC handles of every rank's region over one NCCL allgather; peers mapped with lazy
    // peer access (NVLink / NVSwitch P2P)
    std::vector<void*> share_region(void* mine, cudaStream_t st) override {
        std::vector<void*> out(world, nullptr);
        out[rank] = mine;
        if (world == 1) return out;
        cudaIpcMemHandle_t h;
        if (cudaIpcGetMemHandle(&h, mine) != cudaSuccess) throw CommError{"cudaIpcGetMemHandle failed"};
        const size_t hb = sizeof(cudaIpcMemHandle_t);
        char* dbuf = nullptr;
        if (cudaMalloc(&dbuf, hb * (world + 1)) != cudaSuccess) throw CommError{"share_region: cudaMalloc failed"};
        std::vector<char> hbuf(hb * world);
        cudaMemcpyAsync(dbuf + hb * world, &h, hb, cudaMemcpyHostToDevice, st);
        ncclResult_t r = api.AllGather(dbuf + hb * world, dbuf, hb, ncclChar, comm, st);
        cudaMemcpyAsync(hbuf.data(), dbuf, hb * world, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        cudaFree(dbuf);
        ck(r);
        for (int p = 0; p < world; ++p) {
            if (p == rank) continue;
            cudaIpcMemHandle_t hp;
            memcpy(&hp, hbuf.data() + hb * p, hb);
            if (cudaIpcOpenMemHandle(&out[p], hp, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
                throw CommError{"cudaIpcOpenMemHandle failed (no P2P path between the GPUs?)"};
        }
        return out;
    }
    void release_region(const std::vector<void*>& peers) override {
        for (int p = 0; p < (int)peers.size(); ++p)
            if (p != rank && peers[p]) cudaIpcCloseMemHandle(peers[p]);
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
    std::vector<std::vector<size_t>> displs;   // alltoallv: every rank's send displacements
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
            s->displs.assign(w, {});
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
    void alltoallv(const void* send, const std::vector<size_t>& scounts, const std::vector<size_t>& sdispls, void* recv,
                   const std::vector<size_t>& rcounts, const std::vector<size_t>& rdispls, cudaStream_t st) override {
        (void)scounts;
        sh->displs[rank] = sdispls;
        publish(send, st);
        for (int p = 0; p < world; ++p)
            if (rcounts[p])
                cudaMemcpyAsync(static_cast<char*>(recv) + rdispls[p], static_cast<const char*>(sh->ptr[p]) + sh->displs[p][rank],
                                rcounts[p], cudaMemcpyDeviceToDevice, st);
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
    void host_barrier() override { sh->barrier(); }
    bool device_barrier_ok() const override { return world == 1; }
    // same process, same device: the peers' regions are plain device pointers
    std::vector<void*> share_region(void* mine, cudaStream_t st) override {
        cudaStreamSynchronize(st);
        sh->ptr[rank] = mine;
        sh->barrier();
        std::vector<void*> out(world);
        for (int r = 0; r < world; ++r) out[r] = const_cast<void*>(sh->ptr[r]);
        sh->barrier();
        return out;
    }
};
