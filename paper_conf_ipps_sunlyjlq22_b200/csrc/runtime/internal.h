// internal.h -- private declarations of the StencilMART B200 runtime (C++).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <map>
#include <memory>
#include <string>
#include <vector>

#include "../../../include/stencil.h"

namespace smart_rt {

// ----------------------------------------------------------------- errors
void set_error(const char* fmt, ...) __attribute__((format(printf, 1, 2)));
void clear_error();

#define SM_FAIL(code, ...)         \
  do {                             \
    ::smart_rt::set_error(__VA_ARGS__); \
    return (code);                 \
  } while (0)

#define SM_CUDA(call)                                                                    \
  do {                                                                                   \
    cudaError_t e_ = (call);                                                             \
    if (e_ != cudaSuccess)                                                               \
      SM_FAIL(STENCIL_E_CUDA, "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_),    \
              __FILE__, __LINE__);                                                       \
  } while (0)

#define SM_TRY(call)          \
  do {                        \
    int rc_ = (call);         \
    if (rc_ != STENCIL_OK) return rc_; \
  } while (0)

extern std::atomic<uint64_t> g_launches;

// ------------------------------------------------- driver API entry points
struct Driver {
  CUresult (*moduleLoadData)(CUmodule*, const void*);
  CUresult (*moduleUnload)(CUmodule);
  CUresult (*moduleGetFunction)(CUfunction*, CUmodule, const char*);
  CUresult (*funcSetAttribute)(CUfunction, CUfunction_attribute, int);
  CUresult (*funcGetAttribute)(int*, CUfunction_attribute, CUfunction);
  CUresult (*launchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                           unsigned, CUstream, void**, void**);
  CUresult (*tensorMapEncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                   const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                   const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                   CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  CUresult (*getErrorString)(CUresult, const char**);
  CUresult (*occupancy)(int*, CUfunction, int, size_t);   // cuOccupancyMaxActiveBlocksPerMultiprocessor
};
int get_driver(const Driver** out);
const char* cu_errstr(CUresult r);

// ---------------------------------------------------------------- pattern
// The stencil in the 3-D kernel view: offsets in lexicographic (dz,dy,dx)
// order, coefficients as given (fp64) -- rounded to the dtype at codegen.
struct Pattern {
  int nnz = 0;
  std::vector<int> dz, dy, dx;
  std::vector<double> c;
  int zlo = 0, zhi = 0, ylo = 0, yhi = 0, xlo = 0, xhi = 0;
};

// One kernel template instantiation.
enum Family { FAM_NAIVE = 0, FAM_TILED = 1, FAM_STREAM = 2, FAM_STREAM_TB = 3 };

struct Variant {
  int family = FAM_NAIVE;
  int bx = 32, by = 4, bz = 1, vx = 1, m = 1;
  bool cm = false;
  int tt = 1;
  bool rt = false;
  int ns = 1;
  bool tma = false;
  int chunk = 0;         // runtime argument (streaming)
  int ws_threads = 0;    // warp-specialised ST_TB_RT kernel: CTA size (tbrt_threads)
  long long sy = 0, sz = 0;   // row / plane strides baked into the kernel (0 = run time)
  int reg_lo = 0, reg_hi = 0; // k_stream_tb_rt register split (setmaxnreg; 0 = off)
  bool xshift = false;        // k_stream_tb_rt: per-step ring geometry with aligned windows
  bool splitmid = false;      // k_stream_tb_rt: even/odd-split rows in the last intermediate ring
  int midvx = 0;              // k_stream_tb_rt: columns per thread of the intermediate steps (0 = vx)
  bool fullw = false;         // k_stream_tb_rt: scalar-column stage tiles span whole ring rows (TbRtStage::FULLW)
  int mid_rows_set = 0;       // k_stream_tb_rt: rows of the intermediate tiles when > 0 (else mid_rows' rule)
  int mid_slots_set = 0;      // k_stream_tb_rt: slots of each stage ring when > 0 (else 2)
  int tiled_mid = 0;          // k_tiled (TB): rows of the 1 x n intermediate-step register tiles (0 = scalar)
  bool tiled_full = false;    // k_tiled (TB): those tiles span the buffer's whole rows (TiledCfg::FULL)
  int tiled_mvx = 1;          // k_tiled (TB): columns of those tiles (1, or vx with tiled_full)
  bool flat = false;          // 2-D streaming view [ny][1][nx]: every plane is one row
  bool xm = false;            // merging (BM/CM, factor m) along x instead of y (2-D streaming view)
  std::string name_expr(const char* desc) const;
  int rows() const { return xm ? by : by * m; }          // output rows of a CTA tile
  int tpx() const { return xm ? bx / vx / m : bx / vx; }  // threads along x (streaming families)
  int threads() const;
  int smem_bytes(const Pattern& p, int elem) const;
  int mid_rows(const Pattern& p, int elem) const;
  int mid_slots() const;
  int tbrt_threads(const Pattern& p, int elem) const;
  int tbrt_threads(const Pattern& p, int elem, int* first_last_warp) const;
  bool regsplit_fits(const Pattern& p, int elem, int kernel_regs) const;
};

// Compiled module cache (per process): key = generated source.
struct Kernel {
  CUfunction fn = nullptr;
  int regs = 0;
  int local_bytes = 0;
};
// spill_bytes (optional): ptxas spill stores + loads of the kernel (-1 unknown)
int compile_variant(const Pattern& pat, int dtype, const Variant& v, std::string* lowered,
                    std::vector<char>* cubin, int* spill_bytes = nullptr);
int load_kernel(const std::string& key_src, const std::vector<char>& cubin, const std::string& lowered,
                int smem, Kernel* out);
std::string generate_source(const Pattern& pat, int dtype, const Variant& v);
int count_window_loads(const Pattern& pat, int elem, const Variant& v);

// ---------------------------------------------------------------- kernels
// Grid descriptor passed by value to the NVRTC kernels (layout must match
// smart::Grid in stencil_kernels.cuh).
struct GridArg {
  int nz, ny, nx;
  long long sy, sz;
  int uz0, uz1, uy0, uy1, ux0, ux1;
  int cz0, cz1, cy0, cy1, cx0, cx1;
  int vec_ok;
  long long peer_lo, peer_hi;                     // P2P: mirror stores (layout of smart::Grid)
  int mlo0, mlo1, mhi0, mhi1, shift_lo, shift_hi;
};

// AOT kernels (aot_kernels.cu)
int launch_frame_copy(const void* src, void* dst, int elem, const GridArg& g, cudaStream_t s);
int launch_fill(void* dst, int dtype, const int64_t box[3], const int64_t org[3], const int64_t gdim[3],
                uint64_t seed, int kind, cudaStream_t s);

// ---------------------------------------------------------------- comm
// Slab decomposition along the slowest axis. A plan with a
// communicator owns `n = dims[0]` planes stored after G ghost planes, followed
// by G more: the device array has n + 2G planes. Transport: NCCL send/recv
// between processes, or LOOPBACK (all slabs as plans of one process, halos by
// cudaMemcpyAsync -- the multi-GPU schedule exercised on one device).
enum Transport { TR_NONE = 0, TR_NCCL = 1, TR_LOOPBACK = 2, TR_P2P = 3 };

struct Comm {
  int transport = TR_NONE;
  int rank = 0, nranks = 1;
  bool owner = true;                 // owns the NCCL communicator
  void* nccl = nullptr;              // ncclComm_t
  cudaStream_t stream = nullptr;     // comm stream (owned per plan)
  cudaEvent_t ev_edge = nullptr;     // edge planes of dst written (main stream)
  cudaEvent_t ev_comm = nullptr;     // halo exchange into dst done (comm stream)
  cudaStream_t edge_stream = nullptr;  // high-priority stream of the edge-plane kernels
  cudaEvent_t ev_main = nullptr;     // main stream reached the edge launch (previous interior done)
  float* red_buf = nullptr;          // device buffer of the label all-reduce (64 floats, owned)
  std::vector<stencil_plan_s*> peers;  // LOOPBACK: plans of all ranks (index = rank)
  const void* cur = nullptr;         // LOOPBACK: buffer this rank is exchanging (for peers)
  // P2P (fused halo): registered grids of this rank and its neighbours
  stencil_p2p_buffers_t self{}, lo{}, hi{};
  bool has_lo = false, has_hi = false;
};
// P2P transport: word 2 of a rank's flag buffer is its epoch counter (device)
int launch_p2p_signal(uint32_t* flag_a, uint32_t* flag_b, uint32_t* ctr, cudaStream_t s);
int preload_aot_kernels();
int launch_fma_probe(int dtype, long long iters, int blocks_per_sm, void* sink, double* flops, cudaStream_t s);
int launch_p2p_wait(const uint32_t* flag_a, const uint32_t* flag_b, const uint32_t* ctr, cudaStream_t s);
void comm_destroy(Comm* c);
int comm_create_stream_events(Comm* c);
// Halo plane ranges (local plane indices) of a launch fusing `tl` steps.
void slab_halo(int ghost, int n, int zlo_g, int zhi_g, int rank, int nranks, int64_t out[8]);
int comm_exchange_nccl(stencil_plan_s* P, void* buf, int tl);
int comm_allreduce_max(stencil_plan_s* P, float* v, int n);
int comm_check_async(const Comm* c);   // asynchronous NCCL errors (ncclCommGetAsyncError)
void free_host_path_buffers(stencil_plan_s* P);

// ---------------------------------------------------------------- plan
struct stencil_plan_impl;

}  // namespace smart_rt

struct stencil_plan_s {
  // user-facing definition
  int ndim = 3;
  int64_t dims[3] = {0, 0, 0};   // as given (2-D: dims[0..1])
  int order = 1;
  int dtype = STENCIL_F64;
  uint32_t oc = 0;
  stencil_params_t params{};    // resolved
  std::vector<uint8_t> access;
  std::vector<double> coeffs;

  // kernel view (3-D)
  smart_rt::Pattern pat;
  int64_t vdims[3] = {0, 0, 0};  // view extents nz, ny, nx (with ghosts: n + 2G planes)
  int frame[3] = {0, 0, 0};      // frame widths per view axis
  int ghost = 0;                 // G: ghost planes on each side of the slab (0 = no slab)
  smart_rt::Variant var;
  std::string src;               // generated source of the main variant
  std::string lowered;
  std::vector<char> cubin;
  smart_rt::Kernel kern;
  bool loaded = false;
  // remainder variant for TB (steps % T)
  std::map<int, smart_rt::Kernel> tb_rem;

  // execution state
  cudaStream_t stream = nullptr;
  void* ws = nullptr;
  size_t ws_bytes = 0;
  std::map<const void*, CUtensorMap> tmaps;

  // host end-to-end buffers
  void* h_in_dev = nullptr;
  void* h_out_dev = nullptr;
  void* h_ws_dev = nullptr;
  size_t h_bytes = 0;                // size of each of the three host-path buffers
  cudaStream_t h2d_stream = nullptr, d2h_stream = nullptr;   // pipelined stencil_run_host
  std::vector<cudaEvent_t> h2d_ev, cmp_ev;
  int host_chunks = 0;           // chunks of the last stencil_run_host (0 = not pipelined)

  // rows of the last OC sweep (stencil_sweep_rows)
  std::vector<stencil_sweep_row_t> sweep_rows;

  // kernel timing (stencil_plan_set_timing)
  bool timing = false;
  std::vector<cudaEvent_t> ev_pool;      // pairs: [2i] before, [2i+1] after launch i
  size_t ev_used = 0;

  // CUDA graph of one stencil_run (single-domain plans): the launch sequence of
  // the last (in, out, workspace, steps), captured at its second identical call
  cudaGraphExec_t g_exec = nullptr;
  cudaStream_t g_stream = nullptr;     // capture stream (the caller's may be the legacy stream)
  const void* g_in = nullptr;
  void* g_out = nullptr;
  void* g_ws = nullptr;
  int g_steps = -1, g_calls = 0;
  uint64_t g_nlaunch = 0;              // kernels per replay (stencil_launch_count)

  // multi-GPU
  smart_rt::Comm* comm = nullptr;

  ~stencil_plan_s();
};
