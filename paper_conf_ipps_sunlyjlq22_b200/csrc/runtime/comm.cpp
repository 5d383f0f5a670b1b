// comm.cpp -- multi-GPU plumbing.
// One process per GPU; the grid is slab-decomposed along the slowest axis.
// NCCL (2.28, the torch-bundled library) owns the exchange.
#include <nccl.h>

#include <cstring>

#include "internal.h"

namespace smart_rt {

struct Comm {
  ncclComm_t nc = nullptr;
  int rank = 0, nranks = 1;
  bool owner = true;
};

void comm_destroy(Comm* c) {
  if (!c) return;
  if (c->owner && c->nc) ncclCommDestroy(c->nc);
  delete c;
}

int comm_attach(stencil_plan_s* child, const stencil_plan_s* parent) {
  Comm* c = new Comm(*parent->comm);
  c->owner = false;
  child->comm = c;
  return STENCIL_OK;
}

int comm_allreduce_max(stencil_plan_s* P, float* v, int n) {
  float* d = nullptr;
  SM_CUDA(cudaMalloc(&d, sizeof(float) * n));
  SM_CUDA(cudaMemcpyAsync(d, v, sizeof(float) * n, cudaMemcpyHostToDevice, P->stream));
  ncclResult_t r = ncclAllReduce(d, d, n, ncclFloat32, ncclMax, P->comm->nc, P->stream);
  if (r != ncclSuccess) {
    cudaFree(d);
    SM_FAIL(STENCIL_E_NCCL, "ncclAllReduce: %s", ncclGetErrorString(r));
  }
  SM_CUDA(cudaMemcpyAsync(v, d, sizeof(float) * n, cudaMemcpyDeviceToHost, P->stream));
  SM_CUDA(cudaStreamSynchronize(P->stream));
  cudaFree(d);
  return STENCIL_OK;
}

}  // namespace smart_rt

using namespace smart_rt;

extern "C" int stencil_nccl_unique_id(uint8_t* id) {
  clear_error();
  if (!id) SM_FAIL(STENCIL_E_INVAL, "null id");
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  ncclUniqueId u;
  ncclResult_t r = ncclGetUniqueId(&u);
  if (r != ncclSuccess) SM_FAIL(STENCIL_E_NCCL, "ncclGetUniqueId: %s", ncclGetErrorString(r));
  memcpy(id, &u, sizeof u);
  return STENCIL_OK;
}

extern "C" int stencil_plan_set_comm(stencil_plan_t P, const uint8_t* id, int rank, int nranks) {
  clear_error();
  if (!P || !id) SM_FAIL(STENCIL_E_INVAL, "null argument");
  if (nranks < 1 || rank < 0 || rank >= nranks) SM_FAIL(STENCIL_E_INVAL, "bad rank/nranks");
  SM_FAIL(STENCIL_E_STATE, "multi-GPU slab decomposition is not enabled in this build");
}
