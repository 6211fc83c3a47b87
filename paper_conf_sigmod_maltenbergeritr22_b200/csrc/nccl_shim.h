// nccl_shim.h - run-time loaded NCCL point-to-point (exchange mode 4), internal.
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>

#include <string>
#include <vector>

namespace msort {

struct NcclState {
    std::vector<ncclComm_t> comms;  // single process: one per distinct device; dist: one (this rank's)
};

// one send or receive of `bytes` bytes with comm rank `peer`, on `stream`
struct P2POp {
    bool send;
    const void* buf;
    size_t bytes;
    int peer;
    int comm;  // index into NcclState::comms
    cudaStream_t stream;
};

int nccl_version();  // 0 if libnccl cannot be loaded
bool nccl_unique_id(void* out /* NCCL_UNIQUE_ID_BYTES */, std::string* err);
bool nccl_init_all(NcclState& s, const int* devs, int ndev, std::string* err);
bool nccl_init_rank(NcclState& s, int nranks, const void* id, int rank, std::string* err);
void nccl_destroy(NcclState& s);
// ncclGroupStart; the ops in order; ncclGroupEnd.  Matching sends / receives
// between two comm ranks pair up in posting order (NCCL p2p semantics).
bool nccl_group(const NcclState& s, const std::vector<P2POp>& ops, std::string* err);

}  // namespace msort
