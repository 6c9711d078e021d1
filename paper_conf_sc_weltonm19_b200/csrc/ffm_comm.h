// ffm_comm.h -- exchange transport of sharded runs (comm.cu).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "../../include/ffm.h"

namespace ffm {

struct Comm {
    int world = 1, rank = 0;
    void* nccl = nullptr;        // ncclComm_t owned by the log (NCCL transport)
    ffm_comm_ops ops{};          // caller transport (host buffers)
    bool has_ops = false;
    void* h_stage = nullptr;     // pinned staging (caller transport)
    size_t h_stage_bytes = 0;
    uint64_t bytes_moved = 0;    // bytes received by this rank's collectives (stats)
    std::string err;
};

int comm_unique_id(void* out128);
// Neither nccl_id (128-byte ncclUniqueId) nor ops: no transport (a single log).  Else the
// given transport, for any world size (a world of one runs the collective path alone).
int comm_init(Comm& c, int world, int rank, const void* nccl_id, const ffm_comm_ops* ops);
void comm_destroy(Comm& c);
// recv[world * bytes] = every rank's send[bytes], rank-major (device buffers, on st).
int comm_allgather(Comm& c, const void* send, void* recv, size_t bytes, cudaStream_t st);
// buf[n] (device) = sum over ranks, mod 2^64 (on st).
int comm_allreduce_u64(Comm& c, uint64_t* buf, size_t n, cudaStream_t st);

}  // namespace ffm
