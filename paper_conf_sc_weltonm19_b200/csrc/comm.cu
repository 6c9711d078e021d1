// comm.cu -- the exchange steps of a sharded run:
// an all-gather of fixed-size per-rank blocks and a u64 sum all-reduce, both
// stream-ordered on the log's stream.
//
// Two transports:
//   * NCCL (the product path across GPUs): a communicator owned by the log, created in
//     ffm_log_create from the caller's ncclUniqueId; collectives are enqueued on the
//     log's stream (NVLink / NVSwitch; no host round trip).  libnccl.so.2 is opened at
//     run time (the one the process already loaded, e.g. torch's), so the library does
//     not need NCCL to load or to run single-GPU logs.
//   * caller callbacks (ffm_comm_ops): host buffers staged through pinned memory -- for
//     transports NCCL refuses, e.g. several ranks sharing one GPU in tests.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <string.h>

#include <algorithm>
#include <string>

#include "ffm_comm.h"

namespace ffm {

namespace {

// the NCCL C API subset used here (nccl.h: ncclUint64 = 5, ncclUint8 = 1, ncclSum = 0)
struct NcclId {
    char internal[128];
};
constexpr int kNcclUint8 = 1, kNcclUint64 = 5, kNcclSum = 0;

struct NcclApi {
    bool loaded = false;
    std::string why;
    int (*GetUniqueId)(NcclId*) = nullptr;
    int (*CommInitRank)(void**, int, NcclId, int) = nullptr;
    int (*AllGather)(const void*, void*, size_t, int, void*, cudaStream_t) = nullptr;
    int (*AllReduce)(const void*, void*, size_t, int, int, void*, cudaStream_t) = nullptr;
    int (*CommDestroy)(void*) = nullptr;
    int (*CommAbort)(void*) = nullptr;
    const char* (*GetErrorString)(int) = nullptr;
};

NcclApi& nccl() {
    static NcclApi api;
    static bool tried = false;
    if (tried) return api;
    tried = true;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);   // the process's NCCL (torch's), if loaded
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW);
    if (!h) {
        api.why = std::string("cannot open libnccl.so.2: ") + dlerror();
        return api;
    }
    auto sym = [&](const char* n) {
        void* p = dlsym(h, n);
        if (!p && api.why.empty()) api.why = std::string("libnccl.so.2 lacks ") + n;
        return p;
    };
    api.GetUniqueId = (int (*)(NcclId*))sym("ncclGetUniqueId");
    api.CommInitRank = (int (*)(void**, int, NcclId, int))sym("ncclCommInitRank");
    api.AllGather = (int (*)(const void*, void*, size_t, int, void*, cudaStream_t))sym("ncclAllGather");
    api.AllReduce = (int (*)(const void*, void*, size_t, int, int, void*, cudaStream_t))sym("ncclAllReduce");
    api.CommDestroy = (int (*)(void*))sym("ncclCommDestroy");
    api.CommAbort = (int (*)(void*))sym("ncclCommAbort");
    api.GetErrorString = (const char* (*)(int))sym("ncclGetErrorString");
    api.loaded = api.why.empty();
    return api;
}

int nccl_fail(Comm& c, const char* what, int r) {
    c.err = std::string(what) + ": " + (nccl().GetErrorString ? nccl().GetErrorString(r) : "NCCL error");
    return FFM_E_COMM;
}

int cuda_fail(Comm& c, const char* what, cudaError_t e) {
    c.err = std::string(what) + ": " + cudaGetErrorString(e);
    cudaGetLastError();
    return FFM_E_CUDA;
}

// pinned staging for the callback transport
int stage(Comm& c, size_t bytes) {
    if (bytes <= c.h_stage_bytes) return FFM_OK;
    const size_t nb = std::max<size_t>(bytes, 2 * c.h_stage_bytes);
    if (c.h_stage) cudaFreeHost(c.h_stage);
    c.h_stage = nullptr;
    c.h_stage_bytes = 0;
    cudaError_t e = cudaHostAlloc(&c.h_stage, nb, cudaHostAllocDefault);
    if (e != cudaSuccess) return cuda_fail(c, "cudaHostAlloc(comm staging)", e);
    c.h_stage_bytes = nb;
    return FFM_OK;
}

}  // namespace

int comm_unique_id(void* out) {
    NcclApi& api = nccl();
    if (!api.loaded) return FFM_E_COMM;
    NcclId id;
    if (api.GetUniqueId(&id) != 0) return FFM_E_COMM;
    memcpy(out, &id, sizeof(id));
    return FFM_OK;
}

int comm_init(Comm& c, int world, int rank, const void* nccl_id, const ffm_comm_ops* ops) {
    c.world = world;
    c.rank = rank;
    if (!nccl_id && !ops) return FFM_OK;   // a single log: no transport
    if (ops) {
        if (!ops->allgather || !ops->allreduce_u64) {
            c.err = "ffm_comm_ops with a NULL function";
            return FFM_E_INVAL;
        }
        c.ops = *ops;
        c.has_ops = true;
        return FFM_OK;
    }
    NcclApi& api = nccl();
    if (!api.loaded) {
        c.err = api.why;
        return FFM_E_COMM;
    }
    NcclId id;
    memcpy(&id, nccl_id, sizeof(id));
    int r = api.CommInitRank(&c.nccl, world, id, rank);   // collective over the world
    if (r != 0) {
        c.nccl = nullptr;
        return nccl_fail(c, "ncclCommInitRank", r);
    }
    return FFM_OK;
}

void comm_destroy(Comm& c) {
    if (c.nccl) nccl().CommDestroy(c.nccl);
    c.nccl = nullptr;
    if (c.h_stage) cudaFreeHost(c.h_stage);
    c.h_stage = nullptr;
    c.h_stage_bytes = 0;
}

int comm_allgather(Comm& c, const void* send, void* recv, size_t bytes, cudaStream_t st) {
    if (!c.nccl && !c.has_ops) {   // no transport: a world of one, local copy
        if (bytes && send != recv) {
            cudaError_t e = cudaMemcpyAsync(recv, send, bytes, cudaMemcpyDeviceToDevice, st);
            if (e != cudaSuccess) return cuda_fail(c, "allgather copy", e);
        }
        return FFM_OK;
    }
    c.bytes_moved += bytes * (uint64_t)c.world;
    if (!c.has_ops) {
        int r = nccl().AllGather(send, recv, bytes, kNcclUint8, c.nccl, st);
        return r ? nccl_fail(c, "ncclAllGather", r) : FFM_OK;
    }
    const size_t tot = bytes * (size_t)c.world;
    int s = stage(c, bytes + tot);
    if (s) return s;
    uint8_t* hs = (uint8_t*)c.h_stage;
    uint8_t* hr = hs + bytes;
    cudaError_t e;
    if (bytes && (e = cudaMemcpyAsync(hs, send, bytes, cudaMemcpyDeviceToHost, st)) != cudaSuccess)
        return cuda_fail(c, "allgather D2H", e);
    if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return cuda_fail(c, "allgather sync", e);
    if (c.ops.allgather(c.ops.ctx, hs, hr, bytes) != 0) {
        c.err = "ffm_comm_ops.allgather failed";
        return FFM_E_COMM;
    }
    if (tot && (e = cudaMemcpyAsync(recv, hr, tot, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_fail(c, "allgather H2D", e);
    if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return cuda_fail(c, "allgather sync", e);
    return FFM_OK;
}

int comm_allreduce_u64(Comm& c, uint64_t* buf, size_t n, cudaStream_t st) {
    if ((!c.nccl && !c.has_ops) || n == 0) return FFM_OK;
    c.bytes_moved += 8 * (uint64_t)n;
    if (!c.has_ops) {
        int r = nccl().AllReduce(buf, buf, n, kNcclUint64, kNcclSum, c.nccl, st);
        return r ? nccl_fail(c, "ncclAllReduce", r) : FFM_OK;
    }
    int s = stage(c, 8 * n);
    if (s) return s;
    cudaError_t e;
    if ((e = cudaMemcpyAsync(c.h_stage, buf, 8 * n, cudaMemcpyDeviceToHost, st)) != cudaSuccess)
        return cuda_fail(c, "allreduce D2H", e);
    if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return cuda_fail(c, "allreduce sync", e);
    if (c.ops.allreduce_u64(c.ops.ctx, (uint64_t*)c.h_stage, n) != 0) {
        c.err = "ffm_comm_ops.allreduce_u64 failed";
        return FFM_E_COMM;
    }
    if ((e = cudaMemcpyAsync(buf, c.h_stage, 8 * n, cudaMemcpyHostToDevice, st)) != cudaSuccess)
        return cuda_fail(c, "allreduce H2D", e);
    if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return cuda_fail(c, "allreduce sync", e);
    return FFM_OK;
}

}  // namespace ffm
