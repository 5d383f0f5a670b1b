// p2p.cpp -- the fused, device-initiated halo transport (
// north star: "an r-deep halo exchange per time step ... over NVLink").
// The edge kernels store the planes a neighbour needs straight into its ghost
// planes (peer memory, see smart::Grid::peer_lo/peer_hi in the kernels) and a
// one-thread kernel publishes an epoch in the neighbour's flag word; the
// neighbour's next edge kernels wait for it (run_group in api.cpp). This file
// holds registration and CUDA IPC; the epoch counter is word 2 of the flag buffer.
#include <cstring>
#include <map>
#include <mutex>

#include "internal.h"

using namespace smart_rt;

namespace smart_rt {
int slab_setup_ext(stencil_plan_s* P, int rank, int nranks, int transport);
int preload_kernels(stencil_plan_s* P);
}

static bool bufs_ok(const stencil_p2p_buffers_t* b) { return b && b->in && b->out && b->flags && b->owned_planes > 0; }

extern "C" int stencil_plan_set_p2p(stencil_plan_t P, int rank, int nranks, const stencil_p2p_buffers_t* self,
                                    const stencil_p2p_buffers_t* lo, const stencil_p2p_buffers_t* hi) {
  clear_error();
  if (!P) SM_FAIL(STENCIL_E_INVAL, "null plan");
  if (nranks < 1 || rank < 0 || rank >= nranks) SM_FAIL(STENCIL_E_INVAL, "bad rank/nranks");
  if (!bufs_ok(self)) SM_FAIL(STENCIL_E_INVAL, "self: in, out, flags and owned_planes are required");
  if (self->owned_planes != P->dims[0]) SM_FAIL(STENCIL_E_INVAL, "self->owned_planes != dims[0]");
  if ((rank > 0) != (lo != nullptr) || (rank < nranks - 1) != (hi != nullptr))
    SM_FAIL(STENCIL_E_INVAL, "lo is required exactly when rank > 0, hi exactly when rank < nranks - 1");
  if ((lo && !bufs_ok(lo)) || (hi && !bufs_ok(hi))) SM_FAIL(STENCIL_E_INVAL, "incomplete neighbour buffers");
  if ((uintptr_t)self->flags % 8) SM_FAIL(STENCIL_E_INVAL, "flags must be 8-byte aligned");
  SM_TRY(slab_setup_ext(P, rank, nranks, TR_P2P));
  if ((lo && lo->owned_planes < 2 * P->ghost) || (hi && hi->owned_planes < 2 * P->ghost)) {
    comm_destroy(P->comm);
    P->comm = nullptr;
    P->ghost = 0;
    P->vdims[0] = P->dims[0];
    SM_FAIL(STENCIL_E_INVAL, "neighbour slab thinner than 2 * ghost planes");
  }
  Comm* c = P->comm;
  c->self = *self;
  if (lo) { c->lo = *lo; c->has_lo = true; }
  if (hi) { c->hi = *hi; c->has_hi = true; }
  // every kernel loaded before any run enqueues a flag wait (preload_kernels)
  return preload_kernels(P);
}

extern "C" int stencil_ipc_get_handle(const void* dev_ptr, uint8_t* handle, int64_t* offset) {
  clear_error();
  if (!dev_ptr || !handle || !offset) SM_FAIL(STENCIL_E_INVAL, "null argument");
  static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
  CUdeviceptr base = 0;
  size_t size = 0;
  // the allocation that contains dev_ptr (torch's caching allocator sub-allocates)
  cudaPointerAttributes at;
  SM_CUDA(cudaPointerGetAttributes(&at, dev_ptr));
  if (at.type != cudaMemoryTypeDevice) SM_FAIL(STENCIL_E_INVAL, "not device memory");
  typedef CUresult (*range_fn)(CUdeviceptr*, size_t*, CUdeviceptr);
  static range_fn range = nullptr;
  if (!range) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !p)
      SM_FAIL(STENCIL_E_CUDA, "cuMemGetAddressRange unavailable");
    range = reinterpret_cast<range_fn>(p);
  }
  if (range(&base, &size, (CUdeviceptr)dev_ptr) != CUDA_SUCCESS) SM_FAIL(STENCIL_E_CUDA, "cuMemGetAddressRange failed");
  cudaIpcMemHandle_t h;
  SM_CUDA(cudaIpcGetMemHandle(&h, (void*)base));
  memcpy(handle, &h, sizeof h);
  *offset = (int64_t)((CUdeviceptr)dev_ptr - base);
  return STENCIL_OK;
}

extern "C" int stencil_ipc_open_handle(const uint8_t* handle, int64_t offset, void** dev_ptr) {
  clear_error();
  if (!handle || !dev_ptr || offset < 0) SM_FAIL(STENCIL_E_INVAL, "bad argument");
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof h);
  void* base = nullptr;
  SM_CUDA(cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess));
  *dev_ptr = (char*)base + offset;
  return STENCIL_OK;
}

extern "C" int stencil_ipc_close(void* dev_ptr, int64_t offset) {
  clear_error();
  if (!dev_ptr) SM_FAIL(STENCIL_E_INVAL, "null pointer");
  SM_CUDA(cudaIpcCloseMemHandle((char*)dev_ptr - offset));
  return STENCIL_OK;
}
