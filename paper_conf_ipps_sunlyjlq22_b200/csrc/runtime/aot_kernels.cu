// aot_kernels.cu -- pattern-independent kernels compiled ahead of time (nvcc,
// sm_100a): the frame copy of the ping-pong setup and the
// device side of the counter-based input generator (reading C-3).
#include <algorithm>

#include "internal.h"

namespace smart_rt {

namespace {

// Frame = points outside the update box. Three disjoint groups are
// enumerated so only frame points are touched:
//   A: whole planes z < uz0 or z >= uz1
//   B: planes uz0..uz1-1, whole rows y < uy0 or y >= uy1
//   C: planes uz0..uz1-1, rows uy0..uy1-1, columns x < ux0 or x >= ux1
template <class W>
__global__ void k_frame_copy(const W* __restrict__ src, W* __restrict__ dst, GridArg g) {
  const long long nzA = (long long)g.uz0 + (g.nz - g.uz1);
  const long long nyB = (long long)g.uy0 + (g.ny - g.uy1);
  const long long nxC = (long long)g.ux0 + (g.nx - g.ux1);
  const long long midz = g.uz1 - g.uz0, midy = g.uy1 - g.uy0;
  const long long nA = nzA * g.ny * g.nx;
  const long long nB = midz * nyB * g.nx;
  const long long nC = midz * midy * nxC;
  const long long total = nA + nB + nC;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    long long z, y, x;
    if (i < nA) {
      x = i % g.nx;
      y = (i / g.nx) % g.ny;
      long long zz = i / ((long long)g.nx * g.ny);
      z = zz < g.uz0 ? zz : g.uz1 + (zz - g.uz0);
    } else if (i < nA + nB) {
      long long k = i - nA;
      x = k % g.nx;
      long long yy = (k / g.nx) % nyB;
      z = g.uz0 + k / ((long long)g.nx * nyB);
      y = yy < g.uy0 ? yy : g.uy1 + (yy - g.uy0);
    } else {
      long long k = i - nA - nB;
      long long xx = k % nxC;
      y = g.uy0 + (k / nxC) % midy;
      z = g.uz0 + k / (nxC * midy);
      x = xx < g.ux0 ? xx : g.ux1 + (xx - g.ux0);
    }
    const long long p = z * g.sz + y * g.sy + x;
    dst[p] = src[p];
  }
}

// The same frame with 32-bit index arithmetic (counts < 2^31), as two kinds of
// work in one launch: blocks [0, nb_rows) copy the rows that lie wholly in the
// frame (groups A and B: one warp per row, coalesced along x), the others the
// x-edge columns of the remaining rows (group C: one thread per element). The
// 64-bit div/mod per element of k_frame_copy cost C2 (512^3 fp64) ~100 us per
// run, 4.5% of its step.
template <class W>
__global__ void __launch_bounds__(256) k_frame_rows(const W* __restrict__ src, W* __restrict__ dst, GridArg g,
                                                    int nb_rows) {
  const int nzA = g.uz0 + (g.nz - g.uz1), nyB = g.uy0 + (g.ny - g.uy1), nxC = g.ux0 + (g.nx - g.ux1);
  const int midz = g.uz1 - g.uz0, midy = g.uy1 - g.uy0;
  if ((int)blockIdx.x < nb_rows) {
    const int nA = nzA * g.ny, nrows = nA + midz * nyB;
    const int lane = threadIdx.x & 31;
    for (int r = blockIdx.x * 8 + (threadIdx.x >> 5); r < nrows; r += nb_rows * 8) {
      int z, y;
      if (r < nA) {
        const int zz = r / g.ny;
        y = r - zz * g.ny;
        z = zz < g.uz0 ? zz : g.uz1 + (zz - g.uz0);
      } else {
        const int k = r - nA, zi = k / nyB, yy = k - zi * nyB;
        z = g.uz0 + zi;
        y = yy < g.uy0 ? yy : g.uy1 + (yy - g.uy0);
      }
      const long long p = z * g.sz + y * g.sy;
      for (int x = lane; x < g.nx; x += 32) dst[p + x] = src[p + x];
    }
    return;
  }
  if (nxC == 0) return;
  const int nC = midz * midy * nxC;
  const int nb = gridDim.x - nb_rows;
  for (int i = (blockIdx.x - nb_rows) * 256 + threadIdx.x; i < nC; i += nb * 256) {
    const int row = i / nxC, xx = i - row * nxC;
    const int zi = row / midy, y = g.uy0 + (row - zi * midy);
    const int x = xx < g.ux0 ? xx : g.ux1 + (xx - g.ux0);
    const long long p = (g.uz0 + zi) * g.sz + y * g.sy + x;
    dst[p] = src[p];
  }
}

__device__ __forceinline__ unsigned long long mix64(unsigned long long x) {
  unsigned long long z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

template <class T>
__device__ __forceinline__ T value_of(unsigned long long h, int kind);

template <>
__device__ __forceinline__ double value_of<double>(unsigned long long h, int kind) {
  if (kind == 0) return __longlong_as_double((long long)((h >> 12) | 0x3FF0000000000000ull));
  return (double)((long long)((h >> 53) % 2047ull) - 1023);
}
template <>
__device__ __forceinline__ float value_of<float>(unsigned long long h, int kind) {
  if (kind == 0) return __uint_as_float((unsigned)((h >> 41) | 0x3F800000ull));
  return (float)((long long)((h >> 53) % 2047ull) - 1023);
}

template <class T>
__global__ void k_fill(T* __restrict__ dst, long long bz, long long by, long long bx, long long oz,
                       long long oy, long long ox, long long gy, long long gx, unsigned long long key,
                       int kind) {
  const long long total = bz * by * bx;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const long long x = i % bx, y = (i / bx) % by, z = i / (bx * by);
    const unsigned long long gidx =
        (unsigned long long)(((oz + z) * gy + (oy + y)) * gx + (ox + x));
    dst[i] = value_of<T>(mix64(gidx ^ key), kind);
  }
}

// P2P transport (fused halo): publish / await an epoch in neighbours' flag
// words. The rank's own epoch counter lives in its flag buffer (word 2, zeroed
// with the buffer), so a new buffer always starts a new count -- a host-side
// counter keyed by address would outlive a freed buffer whose address the
// allocator hands out again, and the ranks would wait for different epochs.
// The signal runs after the edge kernels in stream order: it advances the
// counter, then a system-scope fence + release store makes the edge kernels'
// peer stores visible before the flag. The wait spins on acquire loads (one
// thread, sleeping between polls) until both neighbours reached the rank's
// current epoch, so later kernels on the stream see their planes.
__global__ void k_p2p_signal(unsigned* a, unsigned* b, unsigned* ctr) {
  const unsigned v = *ctr + 1;
  *ctr = v;
  __threadfence_system();
  if (a) asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(a), "r"(v) : "memory");
  if (b) asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(b), "r"(v) : "memory");
}

__device__ __forceinline__ unsigned ld_acquire_sys(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__global__ void k_p2p_wait(const unsigned* a, const unsigned* b, const unsigned* ctr) {
  const unsigned v = *ctr;
  // epochs grow monotonically (wrap-safe comparison)
  if (a) while ((int)(ld_acquire_sys(a) - v) < 0) __nanosleep(128);
  if (b) while ((int)(ld_acquire_sys(b) - v) < 0) __nanosleep(128);
}

// FMA throughput probe: the measured denominator of the "alu" roofline of
// FMA-bound stencils (the paper lists each GPU's FP64 peak,
// P:L222-L225). Every thread runs NACC independent fma chains x <- x*a + b for
// iters x 8 steps (|a| < 1 keeps them bounded); the conditional store keeps the
// chains live. FMAs per launch = blocks * 256 * iters * 8 * NACC. a and b are
// compile-time immediates, as the stencil coefficients are in the generated
// kernels: with both in registers the same loop measured 34.2 instead of 37.0
// TFLOP/s fp64 on B200 (register-operand DFMA does not reach the pipe's rate).
template <class T, int NACC>
__global__ void __launch_bounds__(256) k_fma_probe(T* sink, long long iters) {
  T x[NACC];
#pragma unroll
  for (int k = 0; k < NACC; ++k) x[k] = T(threadIdx.x + k) * T(1e-3);
  for (long long i = 0; i < iters; ++i) {
#pragma unroll
    for (int u = 0; u < 8; ++u)
#pragma unroll
      for (int k = 0; k < NACC; ++k) x[k] = fma(x[k], T(0.9990234375), T(0.0009765625));
  }
  T s = T(0);
#pragma unroll
  for (int k = 0; k < NACC; ++k) s += x[k];
  if (s == T(-12345)) sink[0] = s;
}

int grid_for(long long n) {
  long long b = (n + 255) / 256;
  const long long cap = 148LL * 16;
  if (b > cap) b = cap;
  if (b < 1) b = 1;
  return (int)b;
}

}  // namespace

int launch_frame_copy(const void* src, void* dst, int elem, const GridArg& g, cudaStream_t s) {
  const long long vol = (long long)g.nz * g.ny * g.nx;
  const long long inner = (long long)(g.uz1 - g.uz0) * (g.uy1 - g.uy0) * (g.ux1 - g.ux0);
  const long long n = vol - inner;
  if (n <= 0) return STENCIL_OK;
  const long long rows = ((long long)g.uz0 + (g.nz - g.uz1)) * g.ny +
                         (long long)(g.uz1 - g.uz0) * (g.uy0 + (g.ny - g.uy1));
  if (vol < (1LL << 31)) {
    const long long nc = n - rows * g.nx;                            // group C elements
    const int nbr = (int)std::min<long long>((rows + 7) / 8, 148LL * 8);
    const int nbc = (int)std::min<long long>((nc + 255) / 256, 148LL * 8);
    if (elem == 8)
      k_frame_rows<unsigned long long><<<nbr + nbc, 256, 0, s>>>((const unsigned long long*)src,
                                                                 (unsigned long long*)dst, g, nbr);
    else
      k_frame_rows<unsigned><<<nbr + nbc, 256, 0, s>>>((const unsigned*)src, (unsigned*)dst, g, nbr);
    g_launches.fetch_add(1);
    SM_CUDA(cudaGetLastError());
    return STENCIL_OK;
  }
  if (elem == 8)
    k_frame_copy<unsigned long long><<<grid_for(n), 256, 0, s>>>(
        (const unsigned long long*)src, (unsigned long long*)dst, g);
  else
    k_frame_copy<unsigned><<<grid_for(n), 256, 0, s>>>((const unsigned*)src, (unsigned*)dst, g);
  g_launches.fetch_add(1);
  SM_CUDA(cudaGetLastError());
  return STENCIL_OK;
}

int launch_fill(void* dst, int dtype, const int64_t box[3], const int64_t org[3], const int64_t gdim[3],
                uint64_t seed, int kind, cudaStream_t s) {
  const long long n = box[0] * box[1] * box[2];
  if (n <= 0) return STENCIL_OK;
  const unsigned long long key = (unsigned long long)seed * 0xD1B54A32D192ED03ull;
  if (dtype == STENCIL_F64)
    k_fill<double><<<grid_for(n), 256, 0, s>>>((double*)dst, box[0], box[1], box[2], org[0], org[1],
                                                org[2], gdim[1], gdim[2], key, kind);
  else
    k_fill<float><<<grid_for(n), 256, 0, s>>>((float*)dst, box[0], box[1], box[2], org[0], org[1],
                                               org[2], gdim[1], gdim[2], key, kind);
  g_launches.fetch_add(1);
  SM_CUDA(cudaGetLastError());
  return STENCIL_OK;
}

int launch_p2p_signal(uint32_t* a, uint32_t* b, uint32_t* ctr, cudaStream_t s) {
  if (!a && !b) return STENCIL_OK;
  k_p2p_signal<<<1, 1, 0, s>>>(a, b, ctr);
  g_launches.fetch_add(1);
  SM_CUDA(cudaGetLastError());
  return STENCIL_OK;
}

int launch_p2p_wait(const uint32_t* a, const uint32_t* b, const uint32_t* ctr, cudaStream_t s) {
  if (!a && !b) return STENCIL_OK;
  k_p2p_wait<<<1, 1, 0, s>>>(a, b, ctr);
  g_launches.fetch_add(1);
  SM_CUDA(cudaGetLastError());
  return STENCIL_OK;
}

// Force-load the pattern-independent kernels a slab run launches. With CUDA's
// lazy module loading a kernel is loaded at its first launch, and that load can
// wait on the context; several P2P slab plans of one process enqueue spinning
// k_p2p_wait kernels on their streams, so a first k_frame_copy launch behind one
// of them deadlocked (found by the sanitizer pass's in-process P2P case).
int preload_aot_kernels() {
  cudaFuncAttributes a;
  SM_CUDA(cudaFuncGetAttributes(&a, k_frame_copy<unsigned long long>));
  SM_CUDA(cudaFuncGetAttributes(&a, k_frame_copy<unsigned>));
  SM_CUDA(cudaFuncGetAttributes(&a, k_frame_rows<unsigned long long>));
  SM_CUDA(cudaFuncGetAttributes(&a, k_frame_rows<unsigned>));
  SM_CUDA(cudaFuncGetAttributes(&a, k_p2p_signal));
  SM_CUDA(cudaFuncGetAttributes(&a, k_p2p_wait));
  return STENCIL_OK;
}

int launch_fma_probe(int dtype, long long iters, int blocks_per_sm, void* sink, double* flops, cudaStream_t s) {
  int dev = 0, nsm = 0;
  SM_CUDA(cudaGetDevice(&dev));
  SM_CUDA(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  const int blocks = nsm * blocks_per_sm;
  constexpr int NACC = 12;
  if (dtype == STENCIL_F64)
    k_fma_probe<double, NACC><<<blocks, 256, 0, s>>>((double*)sink, iters);
  else
    k_fma_probe<float, NACC><<<blocks, 256, 0, s>>>((float*)sink, iters);
  g_launches.fetch_add(1);
  SM_CUDA(cudaGetLastError());
  *flops = 2.0 * blocks * 256.0 * (double)iters * 8.0 * NACC;
  return STENCIL_OK;
}

}  // namespace smart_rt
