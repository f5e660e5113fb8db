// In-library NCCL transport of the halo exchange (SURVEY.md §8(b) nccl_comm,
// §8(e)): pack -> one NCCL group of per-peer ncclSend / ncclRecv over
// NVLink / NVSwitch -> unpack, all on the caller's stream (CUDA-graph
// capturable).  libnccl.so.2 is opened at first use (the process's NCCL —
// torch's bundled 2.28 when torch is loaded — so libpcgcn keeps no link-time
// NCCL dependency and still loads on machines without it); a missing NCCL
// is reported as PCGCN_ENCCL.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "kernels.h"
#include "plan_internal.h"

namespace pcgcn {
namespace {

typedef int nccl_result;
struct nccl_uid { char internal[128]; };
typedef void* nccl_comm;
constexpr int NCCL_FLOAT32 = 7;

struct NcclApi {
  bool ok = false;
  std::string why;
  nccl_result (*get_unique_id)(nccl_uid*) = nullptr;
  nccl_result (*comm_init_rank)(nccl_comm*, int, nccl_uid, int) = nullptr;
  nccl_result (*comm_destroy)(nccl_comm) = nullptr;
  nccl_result (*group_start)() = nullptr;
  nccl_result (*group_end)() = nullptr;
  nccl_result (*send)(const void*, size_t, int, int, nccl_comm, cudaStream_t) = nullptr;
  nccl_result (*recv)(void*, size_t, int, int, nccl_comm, cudaStream_t) = nullptr;
  const char* (*error_string)(nccl_result) = nullptr;
};

NcclApi& api() {
  static NcclApi a;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) { a.why = "libnccl.so.2 not found"; return; }
    auto sym = [&](const char* n) { return dlsym(h, n); };
    a.get_unique_id = reinterpret_cast<decltype(a.get_unique_id)>(sym("ncclGetUniqueId"));
    a.comm_init_rank = reinterpret_cast<decltype(a.comm_init_rank)>(sym("ncclCommInitRank"));
    a.comm_destroy = reinterpret_cast<decltype(a.comm_destroy)>(sym("ncclCommDestroy"));
    a.group_start = reinterpret_cast<decltype(a.group_start)>(sym("ncclGroupStart"));
    a.group_end = reinterpret_cast<decltype(a.group_end)>(sym("ncclGroupEnd"));
    a.send = reinterpret_cast<decltype(a.send)>(sym("ncclSend"));
    a.recv = reinterpret_cast<decltype(a.recv)>(sym("ncclRecv"));
    a.error_string = reinterpret_cast<decltype(a.error_string)>(sym("ncclGetErrorString"));
    a.ok = a.get_unique_id && a.comm_init_rank && a.comm_destroy && a.group_start && a.group_end && a.send &&
           a.recv && a.error_string;
    if (!a.ok) a.why = "libnccl.so.2 lacks a required symbol";
  });
  return a;
}

pcgcn_status nccl_fail(nccl_result r, const char* where) {
  set_error(std::string(where) + ": " + (api().error_string ? api().error_string(r) : "nccl error"));
  return PCGCN_ENCCL;
}

}  // namespace
}  // namespace pcgcn

using namespace pcgcn;

extern "C" {

pcgcn_status pcgcn_nccl_unique_id(void* id128) {
  if (!id128) { set_error("null id buffer"); return PCGCN_EINVAL; }
  if (!api().ok) { set_error(api().why); return PCGCN_ENCCL; }
  nccl_uid id;
  nccl_result r = api().get_unique_id(&id);
  if (r != 0) return nccl_fail(r, "ncclGetUniqueId");
  std::memcpy(id128, id.internal, 128);
  return PCGCN_OK;
}

pcgcn_status pcgcn_nccl_comm_init(const void* id128, int32_t rank, int32_t world, void** comm_out) {
  if (!id128 || !comm_out || world < 1 || rank < 0 || rank >= world) { set_error("bad id/rank/world"); return PCGCN_EINVAL; }
  if (!api().ok) { set_error(api().why); return PCGCN_ENCCL; }
  nccl_uid id;
  std::memcpy(id.internal, id128, 128);
  nccl_comm c = nullptr;
  nccl_result r = api().comm_init_rank(&c, world, id, rank);
  if (r != 0) return nccl_fail(r, "ncclCommInitRank");
  *comm_out = c;
  return PCGCN_OK;
}

void pcgcn_nccl_comm_destroy(void* comm) {
  if (comm && api().ok) api().comm_destroy(static_cast<nccl_comm>(comm));
}

pcgcn_status pcgcn_halo_exchange(pcgcn_plan_t p, float* Y, int64_t ldy, int32_t w, float* sendbuf, float* recvbuf,
                                 void* comm, void* stream) {
  if (!p || !p->d.built) { set_error("plan has no device structures"); return PCGCN_EINVAL; }
  const int32_t W = p->opts.world, me = p->opts.rank;
  if (W == 1) return PCGCN_OK;
  if (!comm) { set_error("halo_exchange: nccl_comm is NULL on a sharded plan"); return PCGCN_EINVAL; }
  if (!api().ok) { set_error(api().why); return PCGCN_ENCCL; }
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  pcgcn_status st = pcgcn_halo_pack(p, Y, ldy, w, sendbuf, stream);
  if (st != PCGCN_OK) return st;
  nccl_result r = api().group_start();
  if (r != 0) return nccl_fail(r, "ncclGroupStart");
  int64_t so = 0, ro = 0;
  for (int32_t q = 0; q < W; ++q) {
    if (q == me) continue;
    const int64_t ns = int64_t(p->halo_send[q].size()), nr = int64_t(p->halo_recv[q].size());
    if (ns > 0 && (r = api().send(sendbuf + so * w, size_t(ns * w), NCCL_FLOAT32, q, static_cast<nccl_comm>(comm), s)) != 0)
      break;
    if (nr > 0 && (r = api().recv(recvbuf + ro * w, size_t(nr * w), NCCL_FLOAT32, q, static_cast<nccl_comm>(comm), s)) != 0)
      break;
    so += ns;
    ro += nr;
  }
  nccl_result r2 = api().group_end();
  if (r != 0) return nccl_fail(r, "ncclSend/ncclRecv");
  if (r2 != 0) return nccl_fail(r2, "ncclGroupEnd");
  return pcgcn_halo_unpack(p, recvbuf, Y, ldy, w, stream);
}

}  // extern "C"
