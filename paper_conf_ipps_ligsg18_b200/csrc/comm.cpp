// comm.cpp — NCCL over NVLink/NVSwitch for the multi-GPU modes.
//
// NCCL is loaded at run time (dlopen "libnccl.so.2") so the library loads and
// the single-GPU path works without it.  Under PyTorch the already-loaded
// torch NCCL is reused (same soname).  The 128-byte unique id is created on
// rank 0 (ptas_get_unique_id) and broadcast by the caller (torch.distributed).
#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
#include <mutex>

#include "engine.h"

struct ptas_comm {
    ncclComm_t comm;
    int rank;
    int world;
    int device;
};

namespace {

struct NcclApi {
    bool ok = false;
    decltype(&ncclGetUniqueId) getUniqueId = nullptr;
    decltype(&ncclCommInitRank) commInitRank = nullptr;
    decltype(&ncclAllGather) allGather = nullptr;
    decltype(&ncclAllReduce) allReduce = nullptr;
    decltype(&ncclBroadcast) broadcast = nullptr;
    decltype(&ncclCommDestroy) commDestroy = nullptr;
    decltype(&ncclSend) send = nullptr;
    decltype(&ncclRecv) recv = nullptr;
};

NcclApi *nccl()
{
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) return;
        api.getUniqueId = (decltype(api.getUniqueId))dlsym(h, "ncclGetUniqueId");
        api.commInitRank = (decltype(api.commInitRank))dlsym(h, "ncclCommInitRank");
        api.allGather = (decltype(api.allGather))dlsym(h, "ncclAllGather");
        api.allReduce = (decltype(api.allReduce))dlsym(h, "ncclAllReduce");
        api.broadcast = (decltype(api.broadcast))dlsym(h, "ncclBroadcast");
        api.commDestroy = (decltype(api.commDestroy))dlsym(h, "ncclCommDestroy");
        api.send = (decltype(api.send))dlsym(h, "ncclSend");
        api.recv = (decltype(api.recv))dlsym(h, "ncclRecv");
        api.ok = api.getUniqueId && api.commInitRank && api.allGather && api.allReduce && api.broadcast &&
                 api.commDestroy;
    });
    return &api;
}

}  // namespace

extern "C" int ptas_get_unique_id(void *out128)
{
    if (!out128) return PTAS_EINVAL;
    NcclApi *a = nccl();
    if (!a->ok) return PTAS_ENCCL;
    ncclUniqueId id;
    if (a->getUniqueId(&id) != ncclSuccess) return PTAS_ENCCL;
    static_assert(sizeof(id) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(out128, &id, sizeof(id));
    return PTAS_OK;
}

extern "C" int ptas_comm_init(ptas_comm **c, int32_t rank, int32_t world, const void *unique_id128,
                              int32_t device)
{
    if (!c || !unique_id128 || world < 1 || rank < 0 || rank >= world) return PTAS_EINVAL;
    NcclApi *a = nccl();
    if (!a->ok) return PTAS_ENCCL;
    if (device < 0) {
        if (cudaGetDevice(&device) != cudaSuccess) return PTAS_ECUDA;
    }
    if (cudaSetDevice(device) != cudaSuccess) return PTAS_ECUDA;
    ncclUniqueId id;
    std::memcpy(&id, unique_id128, sizeof(id));
    ptas_comm *pc = new ptas_comm();
    if (a->commInitRank(&pc->comm, world, id, rank) != ncclSuccess) {
        delete pc;
        return PTAS_ENCCL;
    }
    pc->rank = rank;
    pc->world = world;
    pc->device = device;
    *c = pc;
    return PTAS_OK;
}

extern "C" int ptas_comm_destroy(ptas_comm *c)
{
    if (!c) return PTAS_EINVAL;
    NcclApi *a = nccl();
    int rc = PTAS_OK;
    if (a->ok && a->commDestroy(c->comm) != ncclSuccess) rc = PTAS_ENCCL;
    delete c;
    return rc;
}

namespace ptas {

int comm_rank(const ptas_comm *c) { return c ? c->rank : 0; }
int comm_world(const ptas_comm *c) { return c ? c->world : 1; }

// In-place all-gather: recv holds world * bytes_per_rank bytes; rank r's
// block is recv + r * bytes_per_rank (send may point there).
int comm_allgather(ptas_comm *c, const void *send, void *recv, size_t bytes_per_rank, cudaStream_t st)
{
    NcclApi *a = nccl();
    if (!a->ok || !c) return PTAS_ENCCL;
    if (a->allGather(send, recv, bytes_per_rank, ncclUint8, c->comm, st) != ncclSuccess)
        return PTAS_ENCCL;
    return PTAS_OK;
}

// In-place min over the ranks of `count` int32 values (status agreement).
int comm_allreduce_min_i32(ptas_comm *c, int32_t *d_buf, size_t count, cudaStream_t st)
{
    NcclApi *a = nccl();
    if (!a->ok || !c) return PTAS_ENCCL;
    if (a->allReduce(d_buf, d_buf, count, ncclInt32, ncclMin, c->comm, st) != ncclSuccess) return PTAS_ENCCL;
    return PTAS_OK;
}

// In-place broadcast of `bytes` bytes from `root`.
int comm_broadcast(ptas_comm *c, void *d_buf, size_t bytes, int root, cudaStream_t st)
{
    NcclApi *a = nccl();
    if (!a->ok || !c) return PTAS_ENCCL;
    if (a->broadcast(d_buf, d_buf, bytes, ncclUint8, root, c->comm, st) != ncclSuccess) return PTAS_ENCCL;
    return PTAS_OK;
}

// Point-to-point: `bytes` bytes to / from rank `peer` (stream-ordered; the
// slab/halo pipeline's halo of one chunk).
int comm_send(ptas_comm *c, const void *d_buf, size_t bytes, int peer, cudaStream_t st)
{
    NcclApi *a = nccl();
    if (!a->ok || !a->send || !c) return PTAS_ENCCL;
    if (a->send(d_buf, bytes, ncclUint8, peer, c->comm, st) != ncclSuccess) return PTAS_ENCCL;
    return PTAS_OK;
}

int comm_recv(ptas_comm *c, void *d_buf, size_t bytes, int peer, cudaStream_t st)
{
    NcclApi *a = nccl();
    if (!a->ok || !a->recv || !c) return PTAS_ENCCL;
    if (a->recv(d_buf, bytes, ncclUint8, peer, c->comm, st) != ncclSuccess) return PTAS_ENCCL;
    return PTAS_OK;
}

}  // namespace ptas
