// comm.cuh — transport interface of the block-sharded multi-GPU check (comm.cu).
#pragma once
#include <cuda_runtime.h>

#include "common.cuh"

namespace bc {

// Stream-ordered collectives over the ranks of one check.  Sizes in bytes; every rank passes the same
// size tables.  Return a bc_status.
struct Comm {
  int rank = 0, world = 1;
  virtual ~Comm() {}
  // recv = concatenation over ranks r of the bytes[r] bytes each rank sends
  virtual int allgatherv(const void* send, void* recv, const u64* bytes, cudaStream_t st) = 0;
  // sbytes[r] bytes from send + soff[r] go to rank r; rbytes[r] bytes from rank r land at recv + roff[r]
  virtual int alltoallv(const void* send, const u64* sbytes, const u64* soff, void* recv, const u64* rbytes,
                        const u64* roff, cudaStream_t st) = 0;
};

struct LocalGroup;
LocalGroup* local_group_create(int world);
void local_group_destroy(LocalGroup* g);
Comm* make_local_comm(LocalGroup* g, int rank, int dev);
Comm* make_nccl_comm(const void* id128, int rank, int world, int* status);
int nccl_unique_id(void* out128);
// all[r * n + i] = rank r's mine[i] (host arrays); dev_tmp: (1 + world) * n u64 of device scratch
int allgather_u64(Comm* c, const u64* mine, int n, u64* all, u64* dev_tmp, cudaStream_t st);

}  // namespace bc
