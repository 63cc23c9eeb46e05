// group.cu -- native multi-GPU path: one process per GPU, the
// outer items sharded by contiguous ranges (cudanp_shard_range; outer items
// are independent), each rank computes its shard with the NP
// kernels and the shards are gathered to rank 0 by NCCL point-to-point calls
// enqueued on the caller's stream right behind the kernel.
//
// The survey sketched one process driving every device (ncclCommInitAll);
// the build contract is one process per GPU, so a group is one rank of an
// NCCL communicator built with ncclCommInitRank from a unique id that rank 0
// creates and the caller distributes (any channel: torch.distributed,
// sockets, a file).  NCCL is loaded at run time (dlopen of libnccl.so.2 --
// the one torch already loaded, if any), so the library still loads on
// hosts without NCCL or a GPU; only the group calls need it.
#include <dlfcn.h>
#include <nccl.h>

#include "common.cuh"

namespace cudanp {

struct NcclApi {
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
  bool ok = false;
};

static const NcclApi& nccl() {
  static NcclApi api = [] {
    NcclApi a;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return a;
    a.GetUniqueId = (decltype(a.GetUniqueId))dlsym(h, "ncclGetUniqueId");
    a.CommInitRank = (decltype(a.CommInitRank))dlsym(h, "ncclCommInitRank");
    a.CommDestroy = (decltype(a.CommDestroy))dlsym(h, "ncclCommDestroy");
    a.Send = (decltype(a.Send))dlsym(h, "ncclSend");
    a.Recv = (decltype(a.Recv))dlsym(h, "ncclRecv");
    a.GroupStart = (decltype(a.GroupStart))dlsym(h, "ncclGroupStart");
    a.GroupEnd = (decltype(a.GroupEnd))dlsym(h, "ncclGroupEnd");
    a.GetErrorString = (decltype(a.GetErrorString))dlsym(h, "ncclGetErrorString");
    a.ok = a.GetUniqueId && a.CommInitRank && a.CommDestroy && a.Send && a.Recv && a.GroupStart &&
           a.GroupEnd && a.GetErrorString;
    return a;
  }();
  return api;
}

static int nccl_fail(ncclResult_t r, const char* what) {
  set_error("%s: %s", what, nccl().GetErrorString ? nccl().GetErrorString(r) : "NCCL error");
  return CUDANP_ERR_NCCL;
}

static int need_nccl() {
  if (nccl().ok) return CUDANP_OK;
  set_error("libnccl.so.2 could not be loaded (dlopen) or lacks a required symbol");
  return CUDANP_ERR_NCCL;
}

}  // namespace cudanp

using namespace cudanp;

struct cudanp_group {
  ncclComm_t comm;
  int nranks, rank, device;
};

extern "C" {

int cudanp_group_unique_id(void* id_out) {
  if (!id_out) return fail_invalid("id_out is NULL");
  if (int rc = need_nccl()) return rc;
  ncclUniqueId id;
  ncclResult_t r = nccl().GetUniqueId(&id);
  if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
  memcpy(id_out, &id, sizeof(id));
  return CUDANP_OK;
}

int cudanp_group_create(const void* id, int nranks, int rank, cudanp_group** out) {
  if (!id || !out) return fail_invalid("id or out is NULL");
  if (nranks < 1 || rank < 0 || rank >= nranks) return fail_invalid("nranks / rank");
  if (int rc = need_nccl()) return rc;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return check_launch("cudaGetDevice");
  ncclUniqueId uid;
  memcpy(&uid, id, sizeof(uid));
  ncclComm_t comm = nullptr;
  ncclResult_t r = nccl().CommInitRank(&comm, nranks, uid, rank);
  if (r != ncclSuccess) return nccl_fail(r, "ncclCommInitRank");
  *out = new cudanp_group{comm, nranks, rank, dev};
  return CUDANP_OK;
}

int cudanp_group_destroy(cudanp_group* g) {
  if (!g) return CUDANP_OK;
  ncclResult_t r = nccl().CommDestroy(g->comm);
  delete g;
  return r == ncclSuccess ? CUDANP_OK : nccl_fail(r, "ncclCommDestroy");
}

int cudanp_group_rank(const cudanp_group* g, int* rank, int* nranks) {
  if (!g) return fail_invalid("group is NULL");
  if (rank) *rank = g->rank;
  if (nranks) *nranks = g->nranks;
  return CUDANP_OK;
}

int cudanp_group_gather(cudanp_group* g, const void* local, void* root_buf, int64_t n_total,
                        int dtype, void* stream) {
  if (!g) return fail_invalid("group is NULL");
  if (dtype != CUDANP_F32 && dtype != CUDANP_I32) return fail_invalid("dtype");
  if (n_total < 0) return fail_invalid("negative size");
  int64_t b = 0, e = 0;
  cudanp_shard_range(n_total, g->nranks, g->rank, &b, &e);
  if (e > b && !local) return fail_invalid("local is NULL");
  if (g->rank == 0 && n_total > 0 && !root_buf) return fail_invalid("root_buf is NULL on rank 0");
  cudaStream_t st = (cudaStream_t)stream;
  const ncclDataType_t dt = dtype == CUDANP_F32 ? ncclFloat32 : ncclInt32;
  const size_t esz = 4;
  if (g->rank == 0 && e > b && (char*)root_buf + b * esz != local) {
    if (cudaMemcpyAsync((char*)root_buf + b * esz, local, (e - b) * esz, cudaMemcpyDeviceToDevice, st) !=
        cudaSuccess)
      return check_launch("gather: root's own shard");
  }
  if (g->nranks == 1) return CUDANP_OK;
  ncclResult_t r = nccl().GroupStart();
  if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
  if (g->rank == 0) {
    for (int k = 1; k < g->nranks; ++k) {
      int64_t bk = 0, ek = 0;
      cudanp_shard_range(n_total, g->nranks, k, &bk, &ek);
      if (ek > bk) {
        r = nccl().Recv((char*)root_buf + bk * esz, (size_t)(ek - bk), dt, k, g->comm, st);
        if (r != ncclSuccess) break;
      }
    }
  } else if (e > b) {
    r = nccl().Send(local, (size_t)(e - b), dt, 0, g->comm, st);
  }
  ncclResult_t r2 = nccl().GroupEnd();
  if (r != ncclSuccess) return nccl_fail(r, "ncclSend/ncclRecv");
  if (r2 != ncclSuccess) return nccl_fail(r2, "ncclGroupEnd");
  return CUDANP_OK;
}

int cudanp_sharded_tmv(cudanp_group* g, const float* A_shard, int64_t lda, const float* x,
                       float* y_shard, float* y_root, int64_t n_outer_total, int64_t n_inner, int S,
                       int dist, int map, void* stream) {
  if (!g) return fail_invalid("group is NULL");
  int64_t b = 0, e = 0;
  if (int rc = cudanp_shard_range(n_outer_total, g->nranks, g->rank, &b, &e)) return rc;
  if (int rc = cudanp_tmv(A_shard, lda, x, y_shard, e - b, n_inner, S, dist, map, stream)) return rc;
  return cudanp_group_gather(g, y_shard, y_root, n_outer_total, CUDANP_F32, stream);
}

int cudanp_sharded_batched_loop_reduce(cudanp_group* g, const void* in_shard, const void* init_shard,
                                       void* out_shard, void* out_root, int64_t n_outer_total,
                                       int64_t n_inner, int dtype, int op, int S, int dist, int map,
                                       void* stream) {
  if (!g) return fail_invalid("group is NULL");
  int64_t b = 0, e = 0;
  if (int rc = cudanp_shard_range(n_outer_total, g->nranks, g->rank, &b, &e)) return rc;
  if (int rc = cudanp_batched_loop_reduce(in_shard, init_shard, out_shard, e - b, n_inner, dtype, op,
                                          S, dist, map, stream))
    return rc;
  return cudanp_group_gather(g, out_shard, out_root, n_outer_total, dtype, stream);
}

}  // extern "C"
