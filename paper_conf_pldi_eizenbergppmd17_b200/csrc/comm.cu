// comm.cu — transport of the block-sharded multi-GPU check (SURVEY.md §8 row e).
//
// Two implementations of one small stream-ordered interface (variable all-gather, all-to-all):
//   NcclComm  : NCCL over NVLink 5 / NVSwitch, one process per GPU; the ncclUniqueId is made by
//               bc_nccl_unique_id() on rank 0 and broadcast by the caller (torch.distributed).  The
//               library is dlopen'ed (the copy torch already loaded, else libnccl.so.2), so libbc has
//               no link-time NCCL dependency and shares the process's NCCL.
//   LocalComm : the ranks are contexts of one process, one host thread each (bc_group_create_local);
//               transfers are cudaMemcpyPeerAsync between the ranks' buffers around two host
//               barriers.  It runs the same data plane on one GPU (tests) or on several.
#include <dlfcn.h>
#include <nccl.h>

#include <condition_variable>
#include <cstring>
#include <mutex>
#include <vector>

#include "comm.cuh"

namespace bc {

// ------------------------------------------------------------------------------ NCCL
struct NcclApi {
  bool ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Broadcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
};

static NcclApi* nccl_api() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);  // the copy torch loaded
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
#define BC_SYM(f) api.f = reinterpret_cast<decltype(api.f)>(dlsym(h, "nccl" #f))
    BC_SYM(GetUniqueId);
    BC_SYM(CommInitRank);
    BC_SYM(CommDestroy);
    BC_SYM(GroupStart);
    BC_SYM(GroupEnd);
    BC_SYM(Send);
    BC_SYM(Recv);
    BC_SYM(Broadcast);
#undef BC_SYM
    api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.GroupStart && api.GroupEnd && api.Send &&
             api.Recv && api.Broadcast;
  });
  return api.ok ? &api : nullptr;
}

struct NcclComm : Comm {
  ncclComm_t c = nullptr;
  NcclApi* api = nullptr;
  ~NcclComm() override {
    if (c && api) api->CommDestroy(c);
  }
  int allgatherv(const void* send, void* recv, const u64* bytes, cudaStream_t st) override {
    u64 off = 0;
    if (api->GroupStart() != ncclSuccess) return BC_ERR_NCCL;
    for (int r = 0; r < world; ++r) {
      char* dst = (char*)recv + off;
      if (bytes[r] &&
          api->Broadcast(r == rank ? send : dst, dst, bytes[r], ncclChar, r, c, st) != ncclSuccess) {
        api->GroupEnd();
        return BC_ERR_NCCL;
      }
      off += bytes[r];
    }
    return api->GroupEnd() == ncclSuccess ? BC_OK : BC_ERR_NCCL;
  }
  int alltoallv(const void* send, const u64* sbytes, const u64* soff, void* recv, const u64* rbytes, const u64* roff,
                cudaStream_t st) override {
    if (api->GroupStart() != ncclSuccess) return BC_ERR_NCCL;
    for (int r = 0; r < world; ++r) {
      if (sbytes[r] && api->Send((const char*)send + soff[r], sbytes[r], ncclChar, r, c, st) != ncclSuccess) {
        api->GroupEnd();
        return BC_ERR_NCCL;
      }
      if (rbytes[r] && api->Recv((char*)recv + roff[r], rbytes[r], ncclChar, r, c, st) != ncclSuccess) {
        api->GroupEnd();
        return BC_ERR_NCCL;
      }
    }
    return api->GroupEnd() == ncclSuccess ? BC_OK : BC_ERR_NCCL;
  }
};

int nccl_unique_id(void* out128) {
  NcclApi* api = nccl_api();
  if (!api) return BC_ERR_NCCL;
  ncclUniqueId id;
  if (api->GetUniqueId(&id) != ncclSuccess) return BC_ERR_NCCL;
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  memcpy(out128, &id, sizeof(id));
  return BC_OK;
}

Comm* make_nccl_comm(const void* id128, int rank, int world, int* status) {
  NcclApi* api = nccl_api();
  if (!api) {
    *status = BC_ERR_NCCL;
    return nullptr;
  }
  ncclUniqueId id;
  memcpy(&id, id128, sizeof(id));
  NcclComm* c = new NcclComm();
  c->api = api;
  c->rank = rank;
  c->world = world;
  if (api->CommInitRank(&c->c, world, id, rank) != ncclSuccess) {
    c->c = nullptr;
    delete c;
    *status = BC_ERR_NCCL;
    return nullptr;
  }
  *status = BC_OK;
  return c;
}

// ------------------------------------------------------------------------- in-process group
struct LocalGroup {
  int world = 0;
  std::mutex m;
  std::condition_variable cv;
  int arrived = 0;
  u64 gen = 0;
  struct Slot {
    const void* send = nullptr;
    const u64* sbytes = nullptr;
    const u64* soff = nullptr;
    int dev = 0;
  };
  std::vector<Slot> slot;
  void barrier() {
    std::unique_lock<std::mutex> lk(m);
    const u64 g = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g; });
    }
  }
};

struct LocalComm : Comm {
  LocalGroup* g = nullptr;
  int dev = 0;
  int allgatherv(const void* send, void* recv, const u64* bytes, cudaStream_t st) override {
    g->slot[rank] = {send, nullptr, nullptr, dev};
    cudaStreamSynchronize(st);  // the send buffer is complete before a peer reads it
    g->barrier();
    u64 off = 0;
    for (int r = 0; r < world; ++r) {
      if (bytes[r]) cudaMemcpyPeerAsync((char*)recv + off, dev, g->slot[r].send, g->slot[r].dev, bytes[r], st);
      off += bytes[r];
    }
    const cudaError_t e = cudaStreamSynchronize(st);
    g->barrier();  // every peer is done reading my send buffer
    return e == cudaSuccess ? BC_OK : BC_ERR_CUDA;
  }
  int alltoallv(const void* send, const u64* sbytes, const u64* soff, void* recv, const u64* rbytes, const u64* roff,
                cudaStream_t st) override {
    g->slot[rank] = {send, sbytes, soff, dev};
    cudaStreamSynchronize(st);
    g->barrier();
    for (int r = 0; r < world; ++r) {
      const LocalGroup::Slot& p = g->slot[r];
      if (rbytes[r]) cudaMemcpyPeerAsync((char*)recv + roff[r], dev, (const char*)p.send + p.soff[rank], p.dev, rbytes[r], st);
    }
    const cudaError_t e = cudaStreamSynchronize(st);
    g->barrier();
    return e == cudaSuccess ? BC_OK : BC_ERR_CUDA;
  }
};

LocalGroup* local_group_create(int world) {
  LocalGroup* g = new LocalGroup();
  g->world = world;
  g->slot.resize(world);
  return g;
}
void local_group_destroy(LocalGroup* g) { delete g; }

Comm* make_local_comm(LocalGroup* g, int rank, int dev) {
  LocalComm* c = new LocalComm();
  c->g = g;
  c->rank = rank;
  c->world = g->world;
  c->dev = dev;
  return c;
}

// ------------------------------------------------------------------------- helpers
int allgather_u64(Comm* c, const u64* mine, int n, u64* all, u64* dev_tmp, cudaStream_t st) {
  // dev_tmp holds (1 + world) * n u64: [mine][all]
  cudaMemcpyAsync(dev_tmp, mine, n * sizeof(u64), cudaMemcpyHostToDevice, st);
  std::vector<u64> bytes(c->world, (u64)n * sizeof(u64));
  int s = c->allgatherv(dev_tmp, dev_tmp + n, bytes.data(), st);
  if (s) return s;
  cudaMemcpyAsync(all, dev_tmp + n, (size_t)c->world * n * sizeof(u64), cudaMemcpyDeviceToHost, st);
  return cudaStreamSynchronize(st) == cudaSuccess ? BC_OK : BC_ERR_CUDA;
}

}  // namespace bc
