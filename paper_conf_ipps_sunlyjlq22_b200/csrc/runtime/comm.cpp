// comm.cpp -- multi-GPU plumbing. Not in the
// paper (every measurement there is one stencil on one GPU);
// required by the north star: "the grid is slab-decomposed along the outermost
// dimension, with an r-deep halo exchange per time step done as NCCL send/recv
// over NVLink and overlapped with interior compute".
//
// One process per GPU; NCCL (2.28, torch-bundled) owns the exchange. Ghost
// planes are whole contiguous z-planes, so no packing is needed.
#include <nccl.h>

#include <cstring>

#include "internal.h"

namespace smart_rt {

void comm_destroy(Comm* c) {
  if (!c) return;
  if (c->owner && c->nccl) ncclCommDestroy((ncclComm_t)c->nccl);
  if (c->stream) cudaStreamDestroy(c->stream);
  if (c->ev_edge) cudaEventDestroy(c->ev_edge);
  if (c->ev_comm) cudaEventDestroy(c->ev_comm);
  if (c->edge_stream) cudaStreamDestroy(c->edge_stream);
  if (c->ev_main) cudaEventDestroy(c->ev_main);
  if (c->red_buf) cudaFree(c->red_buf);
  delete c;
}

int comm_create_stream_events(Comm* c) {
  SM_CUDA(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
  SM_CUDA(cudaEventCreateWithFlags(&c->ev_edge, cudaEventDisableTiming));
  SM_CUDA(cudaEventCreateWithFlags(&c->ev_comm, cudaEventDisableTiming));
  SM_CUDA(cudaEventCreateWithFlags(&c->ev_main, cudaEventDisableTiming));
  int lo = 0, hi = 0;   // numerically lower = higher priority
  SM_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
  SM_CUDA(cudaStreamCreateWithPriority(&c->edge_stream, cudaStreamNonBlocking, hi));
  return STENCIL_OK;
}

// Local plane ranges of one exchange for a launch whose stencil reaches zlo_g
// planes below and zhi_g above (tl fused steps x extents):
//   out = {recv_lo_begin, recv_lo_count, send_lo_begin, send_lo_count,
//          send_hi_begin, send_hi_count, recv_hi_begin, recv_hi_count}
// Owned planes are [G, G+n). Rank k-1 needs my first zhi_g owned planes as its
// upper ghosts; rank k+1 needs my last zlo_g owned planes as its lower ghosts.
void slab_halo(int G, int n, int zlo_g, int zhi_g, int rank, int nranks, int64_t out[8]) {
  const bool lo = rank > 0, hi = rank < nranks - 1;
  out[0] = G - zlo_g;  out[1] = lo ? zlo_g : 0;
  out[2] = G;          out[3] = lo ? zhi_g : 0;
  out[4] = G + n - zlo_g; out[5] = hi ? zlo_g : 0;
  out[6] = G + n;      out[7] = hi ? zhi_g : 0;
}

// A failed peer or network error surfaces asynchronously in NCCL: check the
// communicator before every exchange and after the label all-reduce.
int comm_check_async(const Comm* c) {
  if (!c || c->transport != TR_NCCL || !c->nccl) return STENCIL_OK;
  ncclResult_t ar = ncclSuccess;
  const ncclResult_t r = ncclCommGetAsyncError((ncclComm_t)c->nccl, &ar);
  if (r != ncclSuccess) SM_FAIL(STENCIL_E_NCCL, "ncclCommGetAsyncError: %s", ncclGetErrorString(r));
  if (ar != ncclSuccess && ar != ncclInProgress)
    SM_FAIL(STENCIL_E_NCCL, "NCCL communicator failed asynchronously: %s", ncclGetErrorString(ar));
  return STENCIL_OK;
}

int comm_exchange_nccl(stencil_plan_s* P, void* buf, int tl) {
  Comm* c = P->comm;
  SM_TRY(comm_check_async(c));
  const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
  const size_t plane = (size_t)P->vdims[1] * P->vdims[2];
  int64_t h[8];
  slab_halo(P->ghost, (int)P->dims[0], tl * P->pat.zlo, tl * P->pat.zhi, c->rank, c->nranks, h);
  ncclComm_t nc = (ncclComm_t)c->nccl;
  const ncclDataType_t dt = elem == 8 ? ncclFloat64 : ncclFloat32;
  char* b = (char*)buf;
  ncclResult_t r = ncclGroupStart();
  if (h[1]) r = r == ncclSuccess ? ncclRecv(b + h[0] * plane * elem, h[1] * plane, dt, c->rank - 1, nc, c->stream) : r;
  if (h[3]) r = r == ncclSuccess ? ncclSend(b + h[2] * plane * elem, h[3] * plane, dt, c->rank - 1, nc, c->stream) : r;
  if (h[5]) r = r == ncclSuccess ? ncclSend(b + h[4] * plane * elem, h[5] * plane, dt, c->rank + 1, nc, c->stream) : r;
  if (h[7]) r = r == ncclSuccess ? ncclRecv(b + h[6] * plane * elem, h[7] * plane, dt, c->rank + 1, nc, c->stream) : r;
  ncclResult_t r2 = ncclGroupEnd();
  if (r != ncclSuccess || r2 != ncclSuccess)
    SM_FAIL(STENCIL_E_NCCL, "halo send/recv: %s", ncclGetErrorString(r != ncclSuccess ? r : r2));
  return STENCIL_OK;
}

int comm_attach(stencil_plan_s* child, const stencil_plan_s* parent) {
  Comm* c = new Comm();
  c->transport = parent->comm->transport;
  c->rank = parent->comm->rank;
  c->nranks = parent->comm->nranks;
  c->nccl = parent->comm->nccl;
  c->owner = false;
  c->peers = parent->comm->peers;
  int rc = comm_create_stream_events(c);
  if (rc != STENCIL_OK) { comm_destroy(c); return rc; }
  child->comm = c;
  child->ghost = parent->ghost;
  child->vdims[0] = parent->vdims[0];
  return STENCIL_OK;
}

int comm_allreduce_max(stencil_plan_s* P, float* v, int n) {
  Comm* c = P->comm;
  if (c->transport != TR_NCCL) return STENCIL_OK;
  if (n < 1 || n > 64) SM_FAIL(STENCIL_E_INVAL, "all-reduce of %d values", n);
  SM_TRY(comm_check_async(c));
  if (!c->red_buf) SM_CUDA(cudaMalloc(&c->red_buf, sizeof(float) * 64));   // once per communicator
  float* d = c->red_buf;
  SM_CUDA(cudaMemcpyAsync(d, v, sizeof(float) * n, cudaMemcpyHostToDevice, P->stream));
  ncclResult_t r = ncclAllReduce(d, d, n, ncclFloat32, ncclMax, (ncclComm_t)c->nccl, P->stream);
  if (r != ncclSuccess) SM_FAIL(STENCIL_E_NCCL, "ncclAllReduce: %s", ncclGetErrorString(r));
  SM_CUDA(cudaMemcpyAsync(v, d, sizeof(float) * n, cudaMemcpyDeviceToHost, P->stream));
  SM_CUDA(cudaStreamSynchronize(P->stream));
  SM_TRY(comm_check_async(c));
  return STENCIL_OK;
}

}  // namespace smart_rt

using namespace smart_rt;

// Ghost depth used for every slab: 4 * order planes (TB launches of up to 4
// fused steps need tl * extent <= 4 * order).
static int slab_ghost(const stencil_plan_s* P) { return 4 * P->order; }

static int slab_setup(stencil_plan_s* P, int rank, int nranks, int transport) {
  if (P->ndim != 3) SM_FAIL(STENCIL_E_INVAL, "slab decomposition needs a 3-D grid");
  if (P->comm) SM_FAIL(STENCIL_E_STATE, "plan already has a communicator");
  const int G = slab_ghost(P);
  const int tt = P->var.tt;
  if ((P->oc & STENCIL_OC_TB) && tt > 4) SM_FAIL(STENCIL_E_INVAL, "tb_steps <= 4 with a communicator");
  if (P->dims[0] < 2 * G) SM_FAIL(STENCIL_E_INVAL, "slab of %lld planes < 2 * ghost (%d)", (long long)P->dims[0], 2 * G);
  Comm* c = new Comm();
  c->transport = transport;
  c->rank = rank;
  c->nranks = nranks;
  int rc = comm_create_stream_events(c);
  if (rc != STENCIL_OK) { comm_destroy(c); return rc; }
  P->comm = c;
  P->ghost = G;
  P->vdims[0] = P->dims[0] + 2 * G;
  P->tmaps.clear();
  free_host_path_buffers(P);   // stencil_run_host sized them for the old view
  return STENCIL_OK;
}

namespace smart_rt {
int slab_setup_ext(stencil_plan_s* P, int rank, int nranks, int transport) {
  return slab_setup(P, rank, nranks, transport);
}
}  // namespace smart_rt

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
  SM_TRY(slab_setup(P, rank, nranks, TR_NCCL));
  ncclUniqueId u;
  memcpy(&u, id, sizeof u);
  ncclComm_t nc = nullptr;
  ncclResult_t r = ncclCommInitRank(&nc, nranks, u, rank);
  if (r != ncclSuccess) {
    comm_destroy(P->comm);
    P->comm = nullptr;
    P->ghost = 0;
    P->vdims[0] = P->dims[0];
    SM_FAIL(STENCIL_E_NCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
  }
  P->comm->nccl = nc;
  return STENCIL_OK;
}

extern "C" int stencil_plan_set_nccl_comm(stencil_plan_t P, void* nccl_comm, int rank, int nranks) {
  clear_error();
  if (!P || !nccl_comm) SM_FAIL(STENCIL_E_INVAL, "null argument");
  if (nranks < 1 || rank < 0 || rank >= nranks) SM_FAIL(STENCIL_E_INVAL, "bad rank/nranks");
  int n = 0, r = 0;
  if (ncclCommCount((ncclComm_t)nccl_comm, &n) != ncclSuccess || ncclCommUserRank((ncclComm_t)nccl_comm, &r) != ncclSuccess ||
      n != nranks || r != rank)
    SM_FAIL(STENCIL_E_INVAL, "communicator does not match rank %d of %d", rank, nranks);
  SM_TRY(slab_setup(P, rank, nranks, TR_NCCL));
  P->comm->nccl = nccl_comm;
  P->comm->owner = false;
  return STENCIL_OK;
}

extern "C" int stencil_plan_share_comm(stencil_plan_t P, stencil_plan_t src) {
  clear_error();
  if (!P || !src || !src->comm || src->comm->transport != TR_NCCL)
    SM_FAIL(STENCIL_E_INVAL, "source plan has no NCCL communicator");
  return stencil_plan_set_nccl_comm(P, src->comm->nccl, src->comm->rank, src->comm->nranks);
}

extern "C" int stencil_plans_link_loopback(stencil_plan_t* plans, int nranks) {
  clear_error();
  if (!plans || nranks < 1) SM_FAIL(STENCIL_E_INVAL, "bad arguments");
  for (int k = 0; k < nranks; ++k) {
    if (!plans[k]) SM_FAIL(STENCIL_E_INVAL, "null plan %d", k);
    if (plans[k]->oc != plans[0]->oc || plans[k]->dtype != plans[0]->dtype ||
        plans[k]->dims[1] != plans[0]->dims[1] || plans[k]->dims[2] != plans[0]->dims[2] ||
        plans[k]->pat.nnz != plans[0]->pat.nnz)
      SM_FAIL(STENCIL_E_INVAL, "loopback plans must share stencil, OC, dtype and plane shape");
  }
  std::vector<stencil_plan_s*> v(plans, plans + nranks);
  for (int k = 0; k < nranks; ++k) {
    SM_TRY(slab_setup(plans[k], k, nranks, TR_LOOPBACK));
    plans[k]->comm->peers = v;
  }
  return STENCIL_OK;
}

extern "C" int stencil_plan_ghost_planes(stencil_plan_t P) { return P ? P->ghost : -1; }

extern "C" int stencil_slab_halo(int ghost, int64_t n, int zlo_g, int zhi_g, int rank, int nranks, int64_t* out) {
  clear_error();
  if (!out || nranks < 1 || rank < 0 || rank >= nranks || zlo_g < 0 || zhi_g < 0 || zlo_g > ghost ||
      zhi_g > ghost || n < 2 * ghost)
    SM_FAIL(STENCIL_E_INVAL, "bad slab halo arguments");
  slab_halo(ghost, (int)n, zlo_g, zhi_g, rank, nranks, out);
  return STENCIL_OK;
}
