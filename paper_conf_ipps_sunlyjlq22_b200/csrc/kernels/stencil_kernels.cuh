// stencil_kernels.cuh -- hand-written sm_100a kernel templates, one family per
// optimization combination (OC) of StencilMART Table I.
//
// This header is compiled at plan-creation time by NVRTC (runtime/codegen.cpp)
// together with a generated stencil descriptor `S` that bakes in the offsets
// and coefficients of one stencil (the paper generates "stencil programs",
// P:L25). The descriptor holds only data; all logic is here.
//
// Descriptor contract (generated):
//   typedef <float|double> T;
//   static constexpr int NNZ, ZLO, ZHI, YLO, YHI, XLO, XHI, NZ, NY, NX;
//       neighbour extents: dz in [-ZLO, ZHI], NZ = ZLO + ZHI + 1, etc.
//   static __device__ constexpr int idx(int zi, int yi, int xi);
//       coefficient index of offset (zi-ZLO, yi-YLO, xi-XLO) or -1 if not accessed;
//       indices are the lexicographic (dz,dy,dx) rank of the offset.
//   static __device__ constexpr T coef(int i);
//   static constexpr int NOPS; static __device__ constexpr unsigned op(int i);
//       the variant's op table (see run_gather / run_scatter).
//   static constexpr int MIDR;  slots of each intermediate-stage ring of k_stream_tb_rt.
//   static constexpr int RTSHIFT;  1: retiming queues rotate by register
//       shifts (one plane body) instead of NZ unrolled bodies (large tables).
//
// Arithmetic contract (SURVEY C-4): every output
// is ONE fused-multiply-add chain acc = fma(c_o, u[p+o], acc) starting from 0
// over the offsets in lexicographic (dz,dy,dx) order. Every kernel below keeps
// that order per output, so all OCs produce bitwise identical grids.
//
// Frame rule (C-1): points outside the update box keep their value;
// kernels only write outputs inside the compute box (a sub-box of the update
// box); the frame of the output buffer is copied once by the runtime.

namespace smart {

typedef long long i64;

struct alignas(64) TmaDesc { unsigned long long v[16]; };   // CUtensorMap, opaque

struct Grid {
  int nz, ny, nx;                    // array extents (elements)
  i64 sy, sz;                        // element strides of y and z
  int uz0, uz1, uy0, uy1, ux0, ux1;  // update box: points inside are updated
  int cz0, cz1, cy0, cy1, cx0, cx1;  // compute box: outputs written by this launch
  int vec_ok;                        // 1 if rows are VX-aligned (vector stores allowed)
  // P2P halo transport (fused halo): output planes z in
  // [mlo0, mlo1) are also stored to plane z + shift_lo of the lower
  // neighbour's buffer peer_lo, planes in [mhi0, mhi1) to plane z + shift_hi of
  // the upper neighbour's buffer peer_hi (peer memory over NVLink; same
  // y/x layout). Empty ranges for every launch but the slab-edge ones.
  long long peer_lo, peer_hi;
  int mlo0, mlo1, mhi0, mhi1, shift_lo, shift_hi;
};

// Remote copy of local output plane z (nullptr when z is not mirrored): the
// address of element `off` of plane z in the neighbour's buffer.
template <class T>
__device__ __forceinline__ T* mirror_plane(const Grid& g, int z) {
  if (z >= g.mlo0 && z < g.mlo1) return reinterpret_cast<T*>(g.peer_lo) + (i64)(z + g.shift_lo) * g.sz;
  if (z >= g.mhi0 && z < g.mhi1) return reinterpret_cast<T*>(g.peer_hi) + (i64)(z + g.shift_hi) * g.sz;
  return nullptr;
}

// ---------------------------------------------------------------------------
// small PTX helpers
// ---------------------------------------------------------------------------
__device__ __forceinline__ unsigned smem_u32(const void* p) {
  return static_cast<unsigned>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
               :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
// One arrival per warp (S::ELECT barriers count warps, not threads): the warp's
// shared-memory reads / writes are ordered before lane 0's release-arrive by
// __syncwarp, so a waiter that acquires the phase sees all of them. 32 lanes
// arriving on one mbarrier word are 32 shared-memory atomics; one is enough.
template <bool ELECT>
__device__ __forceinline__ void warp_arrive(unsigned long long* bar) {
  if constexpr (ELECT) {
    __syncwarp();
    if ((threadIdx.x & 31) == 0) mbar_arrive(bar);
  } else {
    mbar_arrive(bar);
  }
}
// wait with a suspend-time hint: the warp sleeps in the barrier unit instead of
// spinning through issue slots (warp-specialised pipelines wait a lot)
__device__ __forceinline__ void mbar_wait_sleep(unsigned long long* bar, unsigned parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n\t"
      "@!P1 bra WAIT_%=;\n\t}"
      :: "r"(smem_u32(bar)), "r"(parity), "r"(0x989680u) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAIT_%=;\n\t}"
      :: "r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void tma_load_3d(void* dst, const TmaDesc* desc, unsigned long long* bar,
                                            int x, int y, int z) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4}], [%5];"
      :: "r"(smem_u32(dst)), "l"(reinterpret_cast<unsigned long long>(desc)),
         "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar)) : "memory");
}
// warp-role register redistribution (warpgroup-aligned, sm_90a+/sm_100a)
template <int N> __device__ __forceinline__ void setmaxnreg_dec() {
  asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" :: "n"(N));
}
template <int N> __device__ __forceinline__ void setmaxnreg_inc() {
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" :: "n"(N));
}
__device__ __forceinline__ void tma_prefetch_desc(const TmaDesc* desc) {
  asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<unsigned long long>(desc)) : "memory");
}
template <int BYTES>
__device__ __forceinline__ void cp_async_zfill(void* dst, const void* src, bool valid) {
  static_assert(BYTES == 4 || BYTES == 8 || BYTES == 16, "cp.async size");
  asm volatile("cp.async.ca.shared.global [%0], [%1], %2, %3;"
               :: "r"(smem_u32(dst)), "l"(src), "n"(BYTES), "r"(valid ? BYTES : 0) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" :: "n"(N) : "memory"); }
// arrive on `bar` once every cp.async this thread issued so far has landed
// (the barrier's expected count includes this arrival: .noinc)
__device__ __forceinline__ void cp_async_mbar_arrive(unsigned long long* bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" :: "r"(smem_u32(bar)) : "memory");
}

// ---------------------------------------------------------------------------
// vector access: VX consecutive elements, 128-bit (or 64-bit) accesses
// ---------------------------------------------------------------------------
template <class T, int VX> struct Vec { T e[VX]; };

template <class T, int VX>
__device__ __forceinline__ void lds_vec(const T* p, T (&w)[VX]) {
  if constexpr (sizeof(T) * VX == 16) {
    const float4 q = *reinterpret_cast<const float4*>(p);
    const T* t = reinterpret_cast<const T*>(&q);
#pragma unroll
    for (int e = 0; e < VX; ++e) w[e] = t[e];
  } else if constexpr (sizeof(T) * VX == 32) {
    const float4 q0 = reinterpret_cast<const float4*>(p)[0];
    const float4 q1 = reinterpret_cast<const float4*>(p)[1];
    const T* t0 = reinterpret_cast<const T*>(&q0);
    const T* t1 = reinterpret_cast<const T*>(&q1);
#pragma unroll
    for (int e = 0; e < VX / 2; ++e) { w[e] = t0[e]; w[e + VX / 2] = t1[e]; }
  } else if constexpr (sizeof(T) * VX == 8) {
    const float2 q = *reinterpret_cast<const float2*>(p);
    const T* t = reinterpret_cast<const T*>(&q);
#pragma unroll
    for (int e = 0; e < VX; ++e) w[e] = t[e];
  } else {
#pragma unroll
    for (int e = 0; e < VX; ++e) w[e] = p[e];
  }
}

template <class T, int VX>
__device__ __forceinline__ void stg_vec(T* p, const T (&w)[VX]) {
  if constexpr (sizeof(T) * VX == 16) {
    float4 q;
    T* t = reinterpret_cast<T*>(&q);
#pragma unroll
    for (int e = 0; e < VX; ++e) t[e] = w[e];
    *reinterpret_cast<float4*>(p) = q;
  } else if constexpr (sizeof(T) * VX == 8) {
    float2 q;
    T* t = reinterpret_cast<T*>(&q);
#pragma unroll
    for (int e = 0; e < VX; ++e) t[e] = w[e];
    *reinterpret_cast<float2*>(p) = q;
  } else {
#pragma unroll
    for (int e = 0; e < VX; ++e) p[e] = w[e];
  }
}

__device__ __forceinline__ double fma_t(double a, double b, double c) { return __fma_rn(a, b, c); }
__device__ __forceinline__ float fma_t(float a, float b, float c) { return __fmaf_rn(a, b, c); }

// packed op (fp32 only, emitted by the generator): a0 += c*w0, a1 += c*w1 as one
// FFMA2 -- per lane an ordinary RN fma, so results are bitwise those of fma_t
__device__ __forceinline__ void fma2_t(float c, float w0, float w1, float& a0, float& a1) {
  const float2 r = __ffma2_rn(make_float2(w0, w1), make_float2(c, c), make_float2(a0, a1));
  a0 = r.x;
  a1 = r.y;
}
__device__ __forceinline__ void fma2_t(double, double, double, double&, double&) {}   // never emitted

// ---------------------------------------------------------------------------
// compile-time pattern predicates (fold to constants after unrolling)
// ---------------------------------------------------------------------------
template <class S>
__device__ __forceinline__ constexpr int cidx(int zi, int yi, int xi) {
  return (zi < 0 || zi >= S::NZ || yi < 0 || yi >= S::NY || xi < 0 || xi >= S::NX) ? -1
                                                                                   : S::idx(zi, yi, xi);
}

// compile-time loop: f(IC<B>{}), ..., f(IC<E-1>{})
template <int V> struct IC { static constexpr int value = V; };
template <int B, int E, class F>
__device__ __forceinline__ void static_for(F&& f) {
  if constexpr (B < E) {
    f(IC<B>{});
    static_for<B + 1, E>(f);
  }
}

// ---------------------------------------------------------------------------
// Window loaders.  `get(j, kv, w)` fills w[VX] with the elements at relative
// row j and columns [kv*VX, kv*VX+VX) of one plane.
// ---------------------------------------------------------------------------
template <class T, int VX, int LD>
struct SmemPlane {                    // shared memory, compile-time row pitch
  const T* p;                          // element (row 0, col 0) of this thread
  __device__ __forceinline__ void get(int j, int kv, T (&w)[VX]) const {
    lds_vec<T, VX>(p + j * LD + kv * VX, w);
  }
};

// Even/odd-split rows (k_stream_tb_rt, S::SPLITMID; fp64, VX = 2): column c of
// a row lives at (c & 1) * SO + (c >> 1), rows SP elements apart. A thread's
// x-neighbour columns then come from contiguous 8-byte loads (the odd array for
// c - 1, the even one for c + 2) instead of 8-byte halves of 16-byte vectors at
// a 16-byte stride, which cost a 16-byte vector's shared-memory wavefronts for
// half the data. The odd array's offset SO is chosen so that a half-warp phase
// of 8-byte stores from 16 consecutive columns c0.. puts its 8 even and 8 odd
// values on disjoint banks: the odd block starts SO - (c0 & 1) elements after
// the even one, which must be 64 bytes past a multiple of 128, i.e. SO = 8 +
// (c0 & 1) (mod 16) for fp64; c0's parity is the same for every phase that lies
// within one tile row (K below). With SO = LX/2 = 34 the two halves overlapped
// on up to 14 banks: 17 M of C2's 24 M bank-conflict wavefronts per launch.
template <class T, int SP, int SO>
struct SplitPlane {
  const T* p;                          // even array of row 0 at the thread's first output vector
  __device__ __forceinline__ void get(int j, int kv, T (&w)[2]) const {
    w[0] = p[j * SP + kv];
    w[1] = p[j * SP + SO + kv];
  }
};
template <int SP, int SO>
__device__ __forceinline__ int split_idx(int row, int col) {
  return row * SP + (col & 1) * SO + (col >> 1);
}
// odd-array offset >= lx / 2, == 8 + (k & 1) (mod 16), k = column parity of the
// stores' phases; and the row pitch
__host__ __device__ constexpr int split_off(int lx, int k) {
  return lx / 2 + ((8 + (k & 1) - (lx / 2) % 16) + 32) % 16;
}
__host__ __device__ constexpr int split_pitch(int lx, int k) { return split_off(lx, k) + lx / 2 + 1; }
// full-width stage tiles (FULLW, tile rows MI ring rows apart): a phase that
// crosses from tile row cy to cy+1 continues the banks of its first part when
// MI * SP = LX/2 (mod 16 words); solvable for odd MI
__host__ __device__ constexpr int split_pitch_full(int lx, int so, int mi) {
  for (int sp = so + lx / 2; sp < so + lx / 2 + 16; ++sp)
    if (((mi * sp - lx / 2) % 16 + 16) % 16 == 0) return sp;
  return so + lx / 2 + (16 - so % 16) % 16;
}

template <class T, int VX, int NROW>
struct GlobalPlane {                  // global memory through the read-only path
  const T* p;                          // element (plane z+dz, col 0) -- rows via rowoff
  const i64* rowoff;                   // NROW clamped row offsets, index j + YLO
  int yshift;                          // = YLO
  __device__ __forceinline__ void get(int j, int kv, T (&w)[VX]) const {
    const T* q = p + rowoff[j + yshift] + kv * VX;
#pragma unroll
    for (int e = 0; e < VX; ++e) w[e] = __ldg(q + e);
  }
};

// Stage the LX x LY box of plane z at (X0, Y0) into shared memory with
// element-wise cp.async, zero fill outside the array (what the TMA box does):
// the staging path of the streaming TB kernels when the rows are not 16-byte
// multiples (no tensor map can describe them) or the box exceeds 256. NT
// threads, this one is t.
template <class T, int LX, int LY, int NT>
__device__ __forceinline__ void stage_plane_cp_async(T* dst, const T* in, const Grid& g, int X0, int Y0, int z,
                                                     int t) {
  const bool zok = z >= 0 && z < g.nz;
  const T* plane = in + (i64)(zok ? z : 0) * g.sz;
  for (int i = t; i < LX * LY; i += NT) {
    const int lx = i % LX, ly = i / LX;
    const int gx = X0 + lx, gy = Y0 + ly;
    const bool ok = zok && gx >= 0 && gx < g.nx && gy >= 0 && gy < g.ny;
    cp_async_zfill<sizeof(T)>(dst + i, ok ? plane + (i64)gy * g.sy + gx : in, ok);
  }
}

// ---------------------------------------------------------------------------
// Compute on a thread tile of M rows x VX columns, driven by the op table of
// the generated descriptor (S::NOPS, S::op(i); built by runtime/codegen.cpp).
//   BM: outputs at rows 0..M-1 (adjacent, "block merging").
//   CM: output m at row m*BY (a fixed distance, "cyclic merging").
// An op is either a window LOAD of VX consecutive values of one plane, or an
// FMA of one loaded value into one accumulator:
//   LOAD (bit31 = 0): zi = op & 15, row j = ((op >> 4) & 255) - 128,
//                     vector kv = ((op >> 12) & 4095) - 2048  (columns [kv*VX, kv*VX+VX))
//   FMA  (bit31 = 1): coefficient id = op & 1023, element e = (op >> 10) & 3,
//                     output column v = (op >> 12) & 3, output row m = (op >> 14) & 7,
//                     slice zi = (op >> 17) & 15; bit 30 (fp32 only): packed pair,
//                     columns v, v+1 from elements e, e+1 (one FFMA2)
// The generator emits each value once per window and, per accumulator, the
// FMAs in lexicographic (dz, dy, dx) order.
// run_gather:  out plane z reads plane z + zi - ZLO through pl[zi].
// run_scatter: retiming. pl is input plane p; slice zi adds into the
//              partial sums of output plane p - (zi - ZLO), kept in
//              acc[(U + NZ - zi) % NZ] (a register queue rotated at compile time).
// ---------------------------------------------------------------------------
// O: the op table (S itself for the main table, S::Mid for the intermediate
// fused steps of k_stream_tb).
template <class S, class O, int VX, int M, class L>
__device__ __forceinline__ void run_gather_ops(const L (&pl)[S::NZ], typename S::T (&acc)[M][VX]) {
  typedef typename S::T T;
  T w[VX];
#pragma unroll
  for (int i = 0; i < O::NOPS; ++i) {
    const unsigned op = O::op(i);
    if (!(op >> 31)) {
      pl[op & 15].get(int((op >> 4) & 255) - 128, int((op >> 12) & 4095) - 2048, w);
    } else if (op & 0x40000000u) {
      T* a = &acc[(op >> 14) & 7][(op >> 12) & 3];
      fma2_t(S::coef(op & 1023), w[(op >> 10) & 3], w[((op >> 10) & 3) + 1], a[0], a[1]);
    } else {
      T& a = acc[(op >> 14) & 7][(op >> 12) & 3];
      a = fma_t(S::coef(op & 1023), w[(op >> 10) & 3], a);
    }
  }
}

template <class S, int VX, int M, class L>
__device__ __forceinline__ void run_gather(const L (&pl)[S::NZ], typename S::T (&acc)[M][VX]) {
  run_gather_ops<S, S, VX, M>(pl, acc);
}

template <class S, class O, int VX, int M, int U, class L>
__device__ __forceinline__ void run_scatter_ops(const L& pl, typename S::T (&acc)[S::NZ][M][VX]) {
  typedef typename S::T T;
  constexpr int NZ = S::NZ;
  T w[VX];
#pragma unroll
  for (int i = 0; i < O::NOPS; ++i) {
    const unsigned op = O::op(i);
    if (!(op >> 31)) {
      pl.get(int((op >> 4) & 255) - 128, int((op >> 12) & 4095) - 2048, w);
    } else if (op & 0x40000000u) {
      const int zi = (op >> 17) & 15;
      T* a = &acc[(U + NZ - zi) % NZ][(op >> 14) & 7][(op >> 12) & 3];
      fma2_t(S::coef(op & 1023), w[(op >> 10) & 3], w[((op >> 10) & 3) + 1], a[0], a[1]);
    } else {
      const int zi = (op >> 17) & 15;
      T& a = acc[(U + NZ - zi) % NZ][(op >> 14) & 7][(op >> 12) & 3];
      a = fma_t(S::coef(op & 1023), w[(op >> 10) & 3], a);
    }
  }
}

template <class S, int VX, int M, int U, class L>
__device__ __forceinline__ void run_scatter(const L& pl, typename S::T (&acc)[S::NZ][M][VX]) {
  run_scatter_ops<S, S, VX, M, U>(pl, acc);
}

// Store a thread tile (rows given by the merge mode) into global memory,
// masked to the compute box; 128-bit stores when the whole vector is inside.
// XS > 0: the M outputs are merged along x instead (2-D streaming views), XS
// columns apart, all in row y0.
template <class T, int VX, int M, bool CM, int BYS, int XS = 0>
__device__ __forceinline__ void store_tile(T* __restrict__ out, const Grid& g, int z, int y0, int x0,
                                           const T (&acc)[M][VX]) {
  T* const rp = mirror_plane<T>(g, z);
  if constexpr (XS > 0) {
    if (y0 < g.cy0 || y0 >= g.cy1) return;
    T* row = out + z * g.sz + y0 * g.sy;
#pragma unroll
    for (int m = 0; m < M; ++m) {
      const int xm = x0 + m * XS;
      if (xm >= g.cx0 && xm + VX <= g.cx1 && g.vec_ok) {
        stg_vec<T, VX>(row + xm, acc[m]);
        if (rp) stg_vec<T, VX>(rp + y0 * g.sy + xm, acc[m]);
      } else {
#pragma unroll
        for (int v = 0; v < VX; ++v)
          if (xm + v >= g.cx0 && xm + v < g.cx1) {
            row[xm + v] = acc[m][v];
            if (rp) rp[y0 * g.sy + xm + v] = acc[m][v];
          }
      }
    }
    return;
  }
  const bool full_x = (x0 >= g.cx0) && (x0 + VX <= g.cx1) && g.vec_ok;
#pragma unroll
  for (int m = 0; m < M; ++m) {
    const int y = CM ? y0 + m * BYS : y0 + m;
    if (y < g.cy0 || y >= g.cy1) continue;
    T* row = out + z * g.sz + y * g.sy;
    if (full_x) {
      stg_vec<T, VX>(row + x0, acc[m]);
      if (rp) stg_vec<T, VX>(rp + y * g.sy + x0, acc[m]);
    } else {
#pragma unroll
      for (int v = 0; v < VX; ++v)
        if (x0 + v >= g.cx0 && x0 + v < g.cx1) {
          row[x0 + v] = acc[m][v];
          if (rp) rp[y * g.sy + x0 + v] = acc[m][v];
        }
    }
  }
}

// The same store with the plane-invariant part hoisted: streaming kernels
// build it once per thread and store one tile per plane. SY / SZ: the row and
// plane strides baked into the kernel by the generator (S::SY, S::SZ; 0 = take
// them from the Grid at run time) -- compile-time strides turn the per-plane
// address arithmetic into immediates (no 64-bit multiplies, no constant-bank
// reloads in the loop).
template <class T, int VX, int M, bool CM, int BYS, i64 SY = 0, i64 SZ = 0, int XS = 0>
struct TileStore {
  T* base;             // element (plane 0, row y0, column x0)
  i64 sz_, rs_;        // plane stride, stride between the tile's rows (run-time strides)
  unsigned rows;       // bit m: row m inside the compute box (XS > 0: output m's vector wholly inside)
  bool full;           // whole vectors inside the compute box (XS > 0: row y0 inside)
  int x0, cx0, cx1;
  __device__ __forceinline__ i64 sz() const { return SZ ? SZ : sz_; }
  __device__ __forceinline__ i64 rs() const { return SY ? (CM ? BYS : 1) * SY : rs_; }
  __device__ __forceinline__ TileStore(T* out, const Grid& g, int y0, int x0_) {
    x0 = x0_; cx0 = g.cx0; cx1 = g.cx1;
    base = out + (i64)y0 * (SY ? SY : g.sy) + x0;
    sz_ = g.sz;
    rs_ = (CM ? BYS : 1) * g.sy;
    rows = 0;
    if constexpr (XS > 0) {      // merged along x (2-D streaming views)
      full = y0 >= g.cy0 && y0 < g.cy1;
#pragma unroll
      for (int m = 0; m < M; ++m)
        if (x0 + m * XS >= g.cx0 && x0 + m * XS + VX <= g.cx1 && g.vec_ok) rows |= 1u << m;
      return;
    }
    full = (x0 >= g.cx0) && (x0 + VX <= g.cx1) && g.vec_ok;
#pragma unroll
    for (int m = 0; m < M; ++m) {
      const int y = CM ? y0 + m * BYS : y0 + m;
      if (y >= g.cy0 && y < g.cy1) rows |= 1u << m;
    }
  }
  // the same tile also into the neighbour's buffer when plane z is mirrored
  // (P2P halo transport); `out` is the launch's output grid (kernel parameter)
  __device__ __forceinline__ void store(int z, const T (&acc)[M][VX], const Grid& g, const T* out) const {
    store_at(base + (i64)z * sz(), acc);
    if (T* rp = mirror_plane<T>(g, z)) store_at(rp + (base - out), acc);
  }
  __device__ __forceinline__ void store_at(T* p, const T (&acc)[M][VX]) const {
    if constexpr (XS > 0) {
      if (!full) return;
#pragma unroll
      for (int m = 0; m < M; ++m) {
        if (rows & (1u << m)) {
          stg_vec<T, VX>(p + m * XS, acc[m]);
        } else {
#pragma unroll
          for (int v = 0; v < VX; ++v)
            if (x0 + m * XS + v >= cx0 && x0 + m * XS + v < cx1) p[m * XS + v] = acc[m][v];
        }
      }
      return;
    }
    if (full) {
#pragma unroll
      for (int m = 0; m < M; ++m)
        if (rows & (1u << m)) stg_vec<T, VX>(p + m * rs(), acc[m]);
    } else {
#pragma unroll
      for (int m = 0; m < M; ++m) {
        if (!(rows & (1u << m))) continue;
#pragma unroll
        for (int v = 0; v < VX; ++v)
          if (x0 + v >= cx0 && x0 + v < cx1) p[m * rs() + v] = acc[m][v];
      }
    }
  }
};

// acc[d] <- acc[d+1], acc[NZ-1] <- 0 (register moves after full unrolling)
template <class T, int NZ, int M, int VX>
__device__ __forceinline__ void shift_queue(T (&acc)[NZ][M][VX]) {
#pragma unroll
  for (int d = 0; d + 1 < NZ; ++d)
#pragma unroll
    for (int m = 0; m < M; ++m)
#pragma unroll
      for (int v = 0; v < VX; ++v) acc[d][m][v] = acc[d + 1][m][v];
#pragma unroll
  for (int m = 0; m < M; ++m)
#pragma unroll
    for (int v = 0; v < VX; ++v) acc[NZ - 1][m][v] = T(0);
}

template <class T, int VX, int M>
__device__ __forceinline__ void zero_acc(T (&acc)[M][VX]) {
#pragma unroll
  for (int m = 0; m < M; ++m)
#pragma unroll
    for (int v = 0; v < VX; ++v) acc[m][v] = T(0);
}

// ===========================================================================
// OC base / BM / CM with smem = 0: "each GPU thread works on a single output
// point", or on M merged points. Neighbours are read from global
// memory through L1 (ld.global.nc). Grid: (x tiles, y tiles, planes).
// ===========================================================================
template <class S, int BX, int BY, int M, bool CM>
__global__ void __launch_bounds__(BX * BY)
k_naive(const typename S::T* __restrict__ in, typename S::T* __restrict__ out, Grid g) {
  typedef typename S::T T;
  constexpr int NROW = CM ? (M - 1) * BY + S::NY : M + S::NY - 1;
  const int x = g.cx0 + blockIdx.x * BX + threadIdx.x;
  const int y0 = CM ? g.cy0 + blockIdx.y * BY * M + threadIdx.y
                    : g.cy0 + (blockIdx.y * BY + threadIdx.y) * M;
  const int z = g.cz0 + blockIdx.z;
  if (x >= g.cx1 || y0 >= g.cy1) return;
  i64 rowoff[NROW];
#pragma unroll
  for (int j = 0; j < NROW; ++j) {
    int y = y0 + j - S::YLO;
    y = y < g.ny - 1 ? y : g.ny - 1;   // rows past the box only feed masked outputs
    rowoff[j] = (i64)y * g.sy;
  }
  T acc[M][1];
  zero_acc<T, 1, M>(acc);
  GlobalPlane<T, 1, NROW> pl[S::NZ];
#pragma unroll
  for (int zi = 0; zi < S::NZ; ++zi) pl[zi] = {in + (i64)(z + zi - S::ZLO) * g.sz + x, rowoff, S::YLO};
  run_gather<S, 1, M>(pl, acc);
#pragma unroll
  for (int m = 0; m < M; ++m) {
    const int y = CM ? y0 + m * BY : y0 + m;
    if (y < g.cy1) {
      out[(i64)z * g.sz + (i64)y * g.sy + x] = acc[m][0];
      if (T* rp = mirror_plane<T>(g, z)) rp[(i64)y * g.sy + x] = acc[m][0];
    }
  }
}

// ===========================================================================
// Tiled kernel: OC base / BM / CM with smem = 1 (spatial tiling), and
// TB without ST: an (x,y,z) output tile plus a TT*extent halo is
// staged once in shared memory (one 3-D TMA box, or cp.async when the rows
// are not TMA-aligned), then TT time steps are computed in shared memory
// (ping-pong), each intermediate step on a region shrunk by the extent, with
// the frame re-imposed; the last step goes to global memory.
// ===========================================================================
template <class S, int BX, int BY, int BZ, int VX, int M, bool CM, int TT>
struct TiledCfg {
  typedef typename S::T T;
  static constexpr int ALN = (16 / (int)sizeof(T)) > VX ? (16 / (int)sizeof(T)) : VX;
  // smem column of the tile's x origin; a multiple of ALN so the TMA box starts
  // on a 16-byte boundary (cp.async.bulk.tensor faults on a misaligned x start)
  static constexpr int XOFF = ((TT * S::XLO + ALN - 1) / ALN) * ALN;
  static constexpr int LX = ((XOFF + BX + TT * S::XHI + ALN - 1) / ALN) * ALN;
  static constexpr int LY = BY * M + TT * (S::YLO + S::YHI);
  static constexpr int LZ = BZ + TT * (S::ZLO + S::ZHI);
  static constexpr int BUF = ((LX * LY * LZ * (int)sizeof(T) + 127) / 128) * 128 / (int)sizeof(T);
  static constexpr int NBUF = TT > 1 ? 2 : 1;
  // S::TMID > 0: intermediate steps in 1 x TMID register tiles (op table S::Mid,
  // gather); the last tile of a column may read TMID - 1 rows past the buffer
  static constexpr int PAD = (TT > 1 && S::TMID > 0) ? ((S::TMID * LX * (int)sizeof(T) + 127) / 128) * 128 / (int)sizeof(T) : 0;
  // S::TFULL: the intermediate tiles span the buffer's whole rows (column 0 reads
  // XLO elements before the first row: front pad)
  static constexpr bool FULL = TT > 1 && S::TMID > 0 && S::TFULL;
  static constexpr int PADF = FULL ? 128 / (int)sizeof(T) : 0;
  static constexpr int SMEM = (NBUF * BUF + PAD + PADF) * (int)sizeof(T) + 128;
  static constexpr int THREADS = (BX / VX) * BY;
};

template <class S, int BX, int BY, int BZ, int VX, int M, bool CM, int TT, bool TMA>
__global__ void __launch_bounds__((BX / VX) * BY)
k_tiled(const typename S::T* __restrict__ in, typename S::T* __restrict__ out, Grid g,
        const __grid_constant__ TmaDesc tmap) {
  typedef typename S::T T;
  typedef TiledCfg<S, BX, BY, BZ, VX, M, CM, TT> C;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  T* buf0 = reinterpret_cast<T*>(smem_raw) + C::PADF;
  T* buf1 = buf0 + C::BUF;
  unsigned long long* bar =
      reinterpret_cast<unsigned long long*>(smem_raw + (C::NBUF * C::BUF + C::PAD + C::PADF) * sizeof(T));

  const int tid = threadIdx.y * (BX / VX) + threadIdx.x;
  const int xa = (g.cx0 / C::ALN) * C::ALN;            // aligned x origin of the tile grid
  const int xb = xa + blockIdx.x * BX;
  const int yb = g.cy0 + blockIdx.y * BY * M;
  const int zb = g.cz0 + blockIdx.z * BZ;
  // region origin (array coordinates) of the staged box
  const int X0 = xb - C::XOFF, Y0 = yb - TT * S::YLO, Z0 = zb - TT * S::ZLO;

  if constexpr (TMA) {
    if (tid == 0) {
      tma_prefetch_desc(&tmap);
      mbar_init(bar, 1);
      fence_mbar_init();
    }
    __syncthreads();
    if (tid == 0) {
      mbar_expect_tx(bar, C::LX * C::LY * C::LZ * (unsigned)sizeof(T));
      tma_load_3d(buf0, &tmap, bar, X0, Y0, Z0);
    }
    mbar_wait(bar, 0);
  } else {
    const int n = C::LX * C::LY * C::LZ;
    for (int i = tid; i < n; i += C::THREADS) {
      const int lx = i % C::LX, ly = (i / C::LX) % C::LY, lz = i / (C::LX * C::LY);
      const int gx = X0 + lx, gy = Y0 + ly, gz = Z0 + lz;
      const bool ok = gx >= 0 && gx < g.nx && gy >= 0 && gy < g.ny && gz >= 0 && gz < g.nz;
      const T* src = ok ? in + (i64)gz * g.sz + (i64)gy * g.sy + gx : in;
      cp_async_zfill<sizeof(T)>(buf0 + i, src, ok);
    }
    cp_async_commit();
    cp_async_wait<0>();
    __syncthreads();
  }

  // intermediate fused steps s = 1 .. TT-1 (temporal blocking); the step
  // loop is unrolled at compile time so the region extents are constants (the
  // point -> (x, y, z) decomposition is then multiply-shift, not runtime division)
  T* src = buf0;
  T* dst = buf1;
  static_for<1, TT>([&](auto sc) {
    constexpr int s = decltype(sc)::value;
    constexpr int hz0 = (TT - s) * S::ZLO, hz1 = (TT - s) * S::ZHI;
    constexpr int hy0 = (TT - s) * S::YLO, hy1 = (TT - s) * S::YHI;
    constexpr int hx0 = (TT - s) * S::XLO, hx1 = (TT - s) * S::XHI;
    constexpr int RX = BX + hx0 + hx1, RY = BY * M + hy0 + hy1, RZ = BZ + hz0 + hz1;
    if constexpr (S::TMID > 0) {
      // 1 x MT register tiles: neighbouring lanes take neighbouring columns, so
      // every shared-memory access is a contiguous warp access, and each loaded
      // value feeds up to MT outputs of the column
      // C::FULL: the tiles cover every column of the buffer rows (LX), so the
      // lanes of a 16-lane phase read consecutive words even where the phase
      // crosses a row end (conflict-free when (MT - 1) * LX = 0 mod 16 words);
      // the extra columns compute don't-care values the last step never reads
      // S::TMVX = 2 (with FULL): MV = 2 columns per tile, 16-byte vector loads
      // and stores -- a radius-2 row window is 3 vectors for 2 columns instead
      // of 5 scalars for 1 (the rows start 16-byte aligned: XOFF and LX are
      // multiples of ALN)
      constexpr int MT = S::TMID, MV = C::FULL ? S::TMVX : 1, NTY = (RY + MT - 1) / MT;
      constexpr int TX = C::FULL ? C::LX / MV : RX, X1 = C::FULL ? C::XOFF : hx0, NT = TX * NTY * RZ;
      for (int t = tid; t < NT; t += C::THREADS) {
        const int rx = t % TX, ty = (t / TX) % NTY, rz = t / (TX * NTY);
        const int gx = xb - X1 + rx * MV, gy0 = yb - hy0 + ty * MT, gz = zb - hz0 + rz;
        const int lb = ((gz - Z0) * C::LY + (gy0 - Y0)) * C::LX + (gx - X0);
        T acc[MT][MV];
        zero_acc<T, MV, MT>(acc);
        SmemPlane<T, MV, C::LX> pl[S::NZ];
#pragma unroll
        for (int zi = 0; zi < S::NZ; ++zi) pl[zi].p = src + lb + (zi - S::ZLO) * C::LY * C::LX;
        run_gather_ops<S, typename S::Mid, MV, MT>(pl, acc);
        const bool zok = gz >= 0 && gz < g.nz, zupd = gz >= g.uz0 && gz < g.uz1;
        const bool vfast = MV > 1 && zupd && gx >= g.ux0 && gx + MV <= g.ux1;   // whole vector updated
#pragma unroll
        for (int m = 0; m < MT; ++m) {
          const int gy = gy0 + m;
          if (!zok || ty * MT + m >= RY || gy < 0 || gy >= g.ny) continue;
          const int li = lb + m * C::LX;
          const bool yupd = gy >= g.uy0 && gy < g.uy1;
          if (vfast && yupd) {
            stg_vec<T, MV>(dst + li, acc[m]);
            continue;
          }
#pragma unroll
          for (int v = 0; v < MV; ++v) {
            const int x = gx + v;
            if (x < 0 || x >= g.nx) continue;
            dst[li + v] = (zupd && yupd && x >= g.ux0 && x < g.ux1) ? acc[m][v] : src[li + v];
          }
        }
      }
      __syncthreads();
      T* t = src; src = dst; dst = t;
      return;
    }
    constexpr int n = RX * RY * RZ;
    for (int i = tid; i < n; i += C::THREADS) {
      const int rx = i % RX, ry = (i / RX) % RY, rz = i / (RX * RY);
      const int gx = xb - hx0 + rx, gy = yb - hy0 + ry, gz = zb - hz0 + rz;
      if (gx < 0 || gx >= g.nx || gy < 0 || gy >= g.ny || gz < 0 || gz >= g.nz) continue;
      const int li = ((gz - Z0) * C::LY + (gy - Y0)) * C::LX + (gx - X0);
      const bool upd = gz >= g.uz0 && gz < g.uz1 && gy >= g.uy0 && gy < g.uy1 && gx >= g.ux0 && gx < g.ux1;
      if (!upd) { dst[li] = src[li]; continue; }
      T acc = T(0);
#pragma unroll
      for (int zi = 0; zi < S::NZ; ++zi)
#pragma unroll
        for (int yi = 0; yi < S::NY; ++yi)
#pragma unroll
          for (int xi = 0; xi < S::NX; ++xi) {
            const int id = cidx<S>(zi, yi, xi);
            if (id >= 0)
              acc = fma_t(S::coef(id),
                          src[li + ((zi - S::ZLO) * C::LY + (yi - S::YLO)) * C::LX + (xi - S::XLO)], acc);
          }
      dst[li] = acc;
    }
    __syncthreads();
    T* t = src; src = dst; dst = t;
  });

  // final step: thread tile M x VX per plane, BZ planes
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int row0 = TT * S::YLO + (CM ? ty : ty * M);    // smem row of the first output
  const int col0 = C::XOFF + tx * VX;
  const int x0 = xb + tx * VX;
  const int y0 = yb + (CM ? ty : ty * M);
#pragma unroll 1
  for (int zz = 0; zz < BZ; ++zz) {
    const int z = zb + zz;
    if (z >= g.cz1) break;
    T acc[M][VX];
    zero_acc<T, VX, M>(acc);
    SmemPlane<T, VX, C::LX> pl[S::NZ];
#pragma unroll
    for (int zi = 0; zi < S::NZ; ++zi)
      pl[zi].p = src + ((TT * S::ZLO + zz + zi - S::ZLO) * C::LY + row0) * C::LX + col0;
    run_gather<S, VX, M>(pl, acc);
    store_tile<T, VX, M, CM, BY>(out, g, z, y0, x0, acc);
  }
}

// ===========================================================================
// Streaming kernel: OC ST and its combinations with BM/CM/RT/PR.
// A CTA owns an (x,y) tile of BX x (BY*M) outputs and a z-chunk of `chunk`
// output planes (concurrent streaming). Input planes (tile + halo)
// stream through a ring of shared-memory slots, each staged by one 2-D TMA box
// (cp.async when rows are not TMA-aligned) signalled on an mbarrier.
//   RT = false: gather form; the ring holds the NZ planes of the window and
//               every output plane reads all its slices from shared memory.
//   RT = true:  retiming: only the newest plane is needed; each value
//               loaded from it feeds every slice, accumulating into a register
//               queue of NZ partial-sum sets (one per live output plane).
//   NS:         planes in flight. NS = 1: the next plane is requested only
//               after the current one is consumed (no prefetching). NS >= 2:
//               prefetching: plane p+NS is requested while plane
//               p+1.. are computed, hiding the per-iteration barrier.
// ===========================================================================
// Thread-tile geometry shared by the streaming families. y-merge (3-D): a
// thread owns M rows (BM adjacent, CM BY apart) of VX columns. x-merge
// (S::XM, 2-D streaming views whose planes are single rows): M vectors of one
// row, adjacent (BM) or BX/M columns apart (CM).
template <class S, int BX, int BY, int VX, int M, bool CM>
struct TileGeom {
  static constexpr int MY = S::XM ? 1 : M;                    // rows of the tile
  static constexpr int TPX = S::XM ? BX / VX / M : BX / VX;   // threads along x
  static constexpr int XS = S::XM ? (CM ? BX / M : VX) : 0;   // columns between merged outputs
  static constexpr int XSTEP = S::XM && !CM ? VX * M : VX;   // columns between threads
  static __device__ __forceinline__ int row(int ty) { return S::XM || CM ? ty : ty * M; }
};

template <class S, int BX, int BY, int VX, int M, bool CM, bool RT, int NS>
struct StreamCfg {
  typedef typename S::T T;
  typedef TileGeom<S, BX, BY, VX, M, CM> TG;
  static constexpr int ALN = (16 / (int)sizeof(T)) > VX ? (16 / (int)sizeof(T)) : VX;
  static constexpr int XOFF = ((S::XLO + ALN - 1) / ALN) * ALN;   // 16-byte aligned box start
  static constexpr int LX = ((XOFF + BX + S::XHI + ALN - 1) / ALN) * ALN;
  static constexpr int LY = BY * TG::MY + S::YLO + S::YHI;
  static constexpr int PLANE = ((LX * LY * (int)sizeof(T) + 127) / 128) * 128 / (int)sizeof(T);
  static constexpr int NRING = (RT ? 1 : S::NZ) + NS - 1;
  static constexpr int SMEM = NRING * PLANE * (int)sizeof(T) + 8 * NRING + 128;
  static constexpr int THREADS = TG::TPX * BY;
};

template <class S, int BX, int BY, int VX, int M, bool CM, bool RT, int NS, bool TMA>
__global__ void __launch_bounds__(StreamCfg<S, BX, BY, VX, M, CM, RT, NS>::THREADS)
k_stream(const typename S::T* __restrict__ in, typename S::T* __restrict__ out, Grid g, int chunk,
         const __grid_constant__ TmaDesc tmap) {
  typedef typename S::T T;
  typedef StreamCfg<S, BX, BY, VX, M, CM, RT, NS> C;
  typedef typename C::TG TG;
  constexpr int NZ = S::NZ;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  T* ring = reinterpret_cast<T*>(smem_raw);
  unsigned long long* bar = reinterpret_cast<unsigned long long*>(smem_raw + C::NRING * C::PLANE * sizeof(T));

  const int tid = threadIdx.y * TG::TPX + threadIdx.x;
  const int xa = (g.cx0 / C::ALN) * C::ALN;
  const int xb = xa + blockIdx.x * BX;
  const int yb = g.cy0 + blockIdx.y * BY * TG::MY;
  const int zs = g.cz0 + blockIdx.z * chunk;
  const int ze = min(zs + chunk, g.cz1);
  const int pfirst = zs - S::ZLO;
  const int nit = (ze - zs) + NZ - 1;                  // planes pfirst .. pfirst+nit-1
  const int X0 = xb - C::XOFF, Y0 = yb - S::YLO;

  auto issue = [&](int it) {                            // request plane pfirst+it into its slot
    const int slot = it % C::NRING;
    T* dst = ring + slot * C::PLANE;
    if constexpr (TMA) {
      if (tid == 0) {
        mbar_expect_tx(&bar[slot], C::LX * C::LY * (unsigned)sizeof(T));
        tma_load_3d(dst, &tmap, &bar[slot], X0, Y0, pfirst + it);
      }
    } else {
      const int gz = pfirst + it;
      const T* plane = in + (i64)gz * g.sz;
      for (int i = tid; i < C::LX * C::LY; i += C::THREADS) {
        const int lx = i % C::LX, ly = i / C::LX;
        const int gx = X0 + lx, gy = Y0 + ly;
        const bool ok = gx >= 0 && gx < g.nx && gy >= 0 && gy < g.ny;
        cp_async_zfill<sizeof(T)>(dst + i, ok ? plane + (i64)gy * g.sy + gx : in, ok);
      }
    }
  };
  auto wait_plane = [&](int it) {
    if constexpr (TMA) {
      mbar_wait(&bar[it % C::NRING], (unsigned)((it / C::NRING) & 1));
    } else {
      cp_async_wait<NS - 1>();
      __syncthreads();
    }
  };

  if constexpr (TMA) {
    if (tid == 0) {
      tma_prefetch_desc(&tmap);
      for (int s = 0; s < C::NRING; ++s) mbar_init(&bar[s], 1);
      fence_mbar_init();
    }
    __syncthreads();
  }
  // prologue: planes 0 .. NS-2 in flight. Plane it+NS-1 goes to the slot of
  // plane it-W (W = window: NZ for gather, 1 for RT), last read in iteration
  // it-1 and released by that iteration's closing barrier.
#pragma unroll 1
  for (int it = 0; it < NS - 1; ++it) {
    if (it < nit) issue(it);
    if constexpr (!TMA) cp_async_commit();
  }

  const int tx = threadIdx.x, ty = threadIdx.y;
  const int row0 = S::YLO + TG::row(ty);
  const int col0 = C::XOFF + tx * TG::XSTEP;
  const int x0 = xb + tx * TG::XSTEP;
  const int y0 = yb + TG::row(ty);
  const TileStore<T, VX, M, CM, BY, S::SY, S::SZ, TG::XS> ts(out, g, y0, x0);

  if constexpr (RT && S::RTSHIFT) {
    // large op tables (high-order stencils): one copy of the plane body and a
    // register shift of the queue per plane (NZ*M*VX moves against NNZ*M*VX
    // FMAs) -- NZ unrolled copies would overflow the instruction cache.
    // acc[d] = partial sums of the output plane completing d planes from now.
    T acc[NZ][M][VX];
#pragma unroll
    for (int q = 0; q < NZ; ++q) zero_acc<T, VX, M>(acc[q]);
#pragma unroll 1
    for (int it = 0; it < nit; ++it) {
      if (it + NS - 1 < nit) issue(it + NS - 1);
      if constexpr (!TMA) cp_async_commit();
      wait_plane(it);
      SmemPlane<T, VX, C::LX> pl{ring + (it % C::NRING) * C::PLANE + row0 * C::LX + col0};
      run_scatter<S, VX, M, NZ - 1>(pl, acc);           // slice zi -> acc[NZ-1-zi]
      const int z = pfirst + it - S::ZHI;               // output completed by this plane
      if (z >= zs) ts.store(z, acc[0], g, out);
      shift_queue<T, NZ, M, VX>(acc);
      __syncthreads();                                  // slot it%NRING may be refilled
    }
  } else if constexpr (RT) {
    T acc[NZ][M][VX];
#pragma unroll
    for (int q = 0; q < NZ; ++q) zero_acc<T, VX, M>(acc[q]);
#pragma unroll 1
    for (int itb = 0; itb < nit; itb += NZ) {
      // unrolled by NZ so that the register-queue rotation is compile-time
      static_for<0, NZ>([&](auto ic) {
        constexpr int U = decltype(ic)::value;
        const int it = itb + U;
        if (it < nit) {
          if (it + NS - 1 < nit) issue(it + NS - 1);
          if constexpr (!TMA) cp_async_commit();
          wait_plane(it);
          zero_acc<T, VX, M>(acc[U]);                    // output plane pfirst+it+ZLO starts
          SmemPlane<T, VX, C::LX> pl{ring + (it % C::NRING) * C::PLANE + row0 * C::LX + col0};
          run_scatter<S, VX, M, U>(pl, acc);
          const int z = pfirst + it - S::ZHI;             // output completed by this plane
          if (z >= zs) ts.store(z, acc[(U + 1) % NZ], g, out);
          __syncthreads();                                // slot it%NRING may be refilled
        }
      });
    }
  } else {
#pragma unroll 1
    for (int it = 0; it < nit; ++it) {
      if (it + NS - 1 < nit) issue(it + NS - 1);
      if constexpr (!TMA) cp_async_commit();
      wait_plane(it);
      if (it >= NZ - 1) {
        const int z = pfirst + it - S::ZHI;
        T acc[M][VX];
        zero_acc<T, VX, M>(acc);
        SmemPlane<T, VX, C::LX> pl[NZ];
#pragma unroll
        for (int zi = 0; zi < NZ; ++zi)                  // plane z + zi - ZLO
          pl[zi].p = ring + ((it - (NZ - 1) + zi) % C::NRING) * C::PLANE + row0 * C::LX + col0;
        run_gather<S, VX, M>(pl, acc);
        ts.store(z, acc, g, out);
      }
      __syncthreads();                                    // oldest slot may be refilled
    }
  }
}

// ===========================================================================
// Streaming + temporal blocking: OC ST_TB and its combinations (
// the AN5D-style pipeline of [15]). A CTA streams one (x,y) tile through TT
// time steps at once: input planes (tile + TT*extent halo) arrive by TMA;
// stage s = 1..TT-1 computes plane p - s*ZHI of time step s on the tile
// expanded by (TT-s)*extent and keeps it in its own shared-memory ring of NZ
// planes; the last stage writes output plane p - TT*ZHI to global memory.
// Halos are recomputed redundantly (the paper's "redundantly loading from
// adjacent blocks"); the frame is re-imposed at every stage. Every ring uses
// the input plane geometry, so (x,y) has the same offset in all of them.
// Intermediate stages are computed in VX x MI register tiles (gather, op
// table S::Mid); the last stage uses the M x VX register tile (BM/CM) in
// gather form, or in the retiming (RT) scatter form with its register queue of
// partial sums.
// ===========================================================================
template <class S, int BX, int BY, int VX, int M, bool CM, bool RT, int NS, int TT>
struct StreamTbCfg {
  typedef typename S::T T;
  typedef TileGeom<S, BX, BY, VX, M, CM> TG;
  static constexpr int ALN = (16 / (int)sizeof(T)) > VX ? (16 / (int)sizeof(T)) : VX;
  // Column geometry. Without S::XSHIFT every ring uses the input plane's
  // geometry (column c = global xb - XOFF + c, XOFF rounded up to ALN). With
  // S::XSHIFT the ring of step s (s = 0: the TMA input) starts exactly at the
  // left edge of the region step s+1 needs: xoff(s) = (TT - s) * XLO. A thread
  // tile of step s+1 then begins XLO columns into its source row, so its
  // window (XLO left, XHI right) starts on a vector boundary and the op table's
  // vectors are shifted by XSH = XLO mod VX: a radius-1 fp64 window with VX = 2
  // is 2 aligned 128-bit loads instead of 3 (one a half-used neighbour vector),
  // and every output vector still lands aligned in its own ring.
  static constexpr int XOFF = S::XSHIFT ? TT * S::XLO : ((TT * S::XLO + ALN - 1) / ALN) * ALN;
  static __device__ __forceinline__ constexpr int xoff(int s) { return S::XSHIFT ? (TT - s) * S::XLO : XOFF; }
  static constexpr int LX = ((XOFF + BX + TT * S::XHI + ALN - 1) / ALN) * ALN;
  static constexpr int LY = BY * TG::MY + TT * (S::YLO + S::YHI);
  static constexpr int PLANE = ((LX * LY * (int)sizeof(T) + 127) / 128) * 128 / (int)sizeof(T);
  static constexpr int NIN = S::NZ + NS - 1;          // input ring (stage 0)
  static constexpr int NMID = S::NZ;                  // ring of each stage 1..TT-1
  static constexpr int MI = S::MI;                    // rows of an intermediate-stage thread tile
  // intermediate tiles are rounded to VX x MI, so their (discarded) edge values
  // read up to VX elements before a plane and MI rows after it: pad both ends
  static constexpr int PADF = 128 / (int)sizeof(T);
  static constexpr int PADB = ((MI * LX + ALN) * (int)sizeof(T) + 127) / 128 * 128 / (int)sizeof(T);
  static constexpr int SMEM = (PADF + (NIN + (TT - 1) * NMID) * PLANE + PADB) * (int)sizeof(T) + 8 * NIN + 128;
  static constexpr int THREADS = TG::TPX * BY;
};

template <class S, int BX, int BY, int VX, int M, bool CM, bool RT, int NS, int TT>
__global__ void __launch_bounds__(StreamTbCfg<S, BX, BY, VX, M, CM, RT, NS, TT>::THREADS)
k_stream_tb(const typename S::T* __restrict__ in, typename S::T* __restrict__ out, Grid g, int chunk,
            const __grid_constant__ TmaDesc tmap) {
  typedef typename S::T T;
  typedef StreamTbCfg<S, BX, BY, VX, M, CM, RT, NS, TT> C;
  typedef typename C::TG TG;
  constexpr int NZ = S::NZ;
  constexpr int MI = C::MI;
  static_assert(TT >= 2, "k_stream_tb needs TT >= 2");
  extern __shared__ __align__(128) unsigned char smem_raw[];
  T* ring0 = reinterpret_cast<T*>(smem_raw) + C::PADF;
  T* mid = ring0 + C::NIN * C::PLANE;                  // stage s ring: mid + (s-1)*NZ*PLANE
  unsigned long long* bar = reinterpret_cast<unsigned long long*>(
      smem_raw + (C::PADF + (C::NIN + (TT - 1) * C::NMID) * C::PLANE + C::PADB) * sizeof(T));

  const int tid = threadIdx.y * TG::TPX + threadIdx.x;
  const int xa = (g.cx0 / C::ALN) * C::ALN;
  const int xb = xa + blockIdx.x * BX;
  const int yb = g.cy0 + blockIdx.y * BY * TG::MY;
  const int zs = g.cz0 + blockIdx.z * chunk;
  const int ze = min(zs + chunk, g.cz1);
  const int pin0 = zs - TT * S::ZLO;                   // first input plane
  const int nit = (ze - zs) + TT * (NZ - 1);
  const int X0 = xb - C::XOFF, Y0 = yb - TT * S::YLO;

  auto issue = [&](int it) {
    const int slot = it % C::NIN;
    if constexpr (S::TMA) {
      if (tid == 0) {
        mbar_expect_tx(&bar[slot], C::LX * C::LY * (unsigned)sizeof(T));
        tma_load_3d(ring0 + slot * C::PLANE, &tmap, &bar[slot], X0, Y0, pin0 + it);
      }
    } else {   // rows not TMA-aligned (or box > 256): element-wise cp.async, zero fill outside
      stage_plane_cp_async<T, C::LX, C::LY, C::THREADS>(ring0 + slot * C::PLANE, in, g, X0, Y0, pin0 + it, tid);
    }
  };
  // plane pointer of stage k (0 = input) holding plane q
  auto stage_plane = [&](int k, int q) -> T* {
    const int idx = q - (zs - (TT - k) * S::ZLO);
    return k == 0 ? ring0 + (idx % C::NIN) * C::PLANE : mid + ((k - 1) * NZ + idx % NZ) * C::PLANE;
  };

  if (S::TMA && tid == 0) {
    tma_prefetch_desc(&tmap);
    for (int s = 0; s < C::NIN; ++s) mbar_init(&bar[s], 1);
    fence_mbar_init();
  }
  __syncthreads();
#pragma unroll 1
  for (int it = 0; it < NS - 1; ++it) {
    if (it < nit) issue(it);
    if constexpr (!S::TMA) cp_async_commit();
  }

  // Intermediate fused step s (1..TT-1) of iteration it: plane q = p - s*ZHI
  // on region R_s (tile expanded by (TT-s)*extent), computed in VX x MI
  // register tiles with the S::Mid op table; values outside R_s, the array or
  // the update box are masked / copied (frame re-imposed).
  auto mid_stage = [&](int it, auto sc) {
    constexpr int s = decltype(sc)::value;
    constexpr int HX0 = (TT - s) * S::XLO, HX1 = (TT - s) * S::XHI;
    constexpr int HY0 = (TT - s) * S::YLO, HY1 = (TT - s) * S::YHI;
    constexpr int TXL = ((HX0 + VX - 1) / VX) * VX;
    constexpr int NTX = (TXL + BX + HX1 + VX - 1) / VX;
    constexpr int RY = BY * TG::MY + HY0 + HY1;
    constexpr int NTY = (RY + MI - 1) / MI;
    if (it < s * (NZ - 1)) return;
    const int q = pin0 + it - s * S::ZHI;
    if (q < 0 || q >= g.nz) return;                   // outside the array: never consumed
    T* dst = stage_plane(s, q);
    const T* ctr = stage_plane(s - 1, q);
    const T* src[NZ];
#pragma unroll
    for (int zi = 0; zi < NZ; ++zi) src[zi] = stage_plane(s - 1, q + zi - S::ZLO);
    const bool zupd = q >= g.uz0 && q < g.uz1;
    const int rx0 = xb - HX0, rx1 = xb + BX + HX1, ry0 = yb - HY0, ry1 = yb + BY * TG::MY + HY1;
    for (int t = tid; t < NTX * NTY; t += C::THREADS) {
      const int gx0 = xb - TXL + (t % NTX) * VX, gy0 = ry0 + (t / NTX) * MI;
      const int lbase = (gy0 - Y0) * C::LX + (gx0 - X0);
      T acc[MI][VX];
      zero_acc<T, VX, MI>(acc);
      SmemPlane<T, VX, C::LX> pl[NZ];
#pragma unroll
      for (int zi = 0; zi < NZ; ++zi) pl[zi].p = src[zi] + lbase;
      run_gather_ops<S, typename S::Mid, VX, MI>(pl, acc);
#pragma unroll
      for (int m = 0; m < MI; ++m) {
        const int gy = gy0 + m;
        if (gy >= ry1 || gy < 0 || gy >= g.ny) continue;
        const bool rowupd = zupd && gy >= g.uy0 && gy < g.uy1;
        const int li = lbase + m * C::LX;
        if (rowupd && gx0 >= rx0 && gx0 + VX <= rx1 && gx0 >= g.ux0 && gx0 + VX <= g.ux1) {
          stg_vec<T, VX>(dst + li, acc[m]);             // whole vector interior
        } else {
#pragma unroll
          for (int v = 0; v < VX; ++v) {
            const int gx = gx0 + v;
            if (gx < rx0 || gx >= rx1 || gx < 0 || gx >= g.nx) continue;
            const bool upd = rowupd && gx >= g.ux0 && gx < g.ux1;
            dst[li + v] = upd ? acc[m][v] : ctr[li + v];
          }
        }
      }
    }
  };

  const int tx = threadIdx.x, ty = threadIdx.y;
  const int row0 = TT * S::YLO + TG::row(ty);
  const int col0 = C::XOFF + tx * TG::XSTEP;
  const int x0 = xb + tx * TG::XSTEP;
  const int y0 = yb + TG::row(ty);

  // one pipeline iteration up to (excluding) the last stage
  auto front = [&](int it) {
    if (it + NS - 1 < nit) issue(it + NS - 1);
    if constexpr (S::TMA) {
      mbar_wait(&bar[it % C::NIN], (unsigned)((it / C::NIN) & 1));
    } else {
      cp_async_commit();
      cp_async_wait<NS - 1>();
      __syncthreads();
    }
    static_for<1, TT>([&](auto sc) {
      mid_stage(it, sc);
      __syncthreads();
    });
  };

  if constexpr (RT) {
    T acc[NZ][M][VX];
#pragma unroll
    for (int q = 0; q < NZ; ++q) zero_acc<T, VX, M>(acc[q]);
    // the last stage consumes stage TT-1 plane q = p - (TT-1)*ZHI, produced
    // from iteration (TT-1)*(NZ-1) on; its index j = it - (TT-1)*(NZ-1).
    constexpr int J0 = (TT - 1) * (NZ - 1);
#pragma unroll 1
    for (int it = 0; it < nit; ++it) {
      front(it);
      if (it >= J0) {
        // rotation index of this stage-(TT-1) plane; each branch below uses
        // compile-time queue indices, so the partial sums stay in registers
        const int ur = (it - J0) % NZ;
        const int q = pin0 + it - (TT - 1) * S::ZHI;
        SmemPlane<T, VX, C::LX> pl{stage_plane(TT - 1, q) + row0 * C::LX + col0};
        const int z = q - S::ZHI;
        if constexpr (S::RTSHIFT) {                      // one body + register shift (see k_stream)
          (void)ur;
          run_scatter<S, VX, M, NZ - 1>(pl, acc);
          if (z >= zs) store_tile<T, VX, M, CM, BY, TG::XS>(out, g, z, y0, x0, acc[0]);
          shift_queue<T, NZ, M, VX>(acc);
        } else {
          static_for<0, NZ>([&](auto ic) {
            constexpr int UR = decltype(ic)::value;
            if (ur == UR) {
              zero_acc<T, VX, M>(acc[UR]);
              run_scatter<S, VX, M, UR>(pl, acc);
              if (z >= zs) store_tile<T, VX, M, CM, BY, TG::XS>(out, g, z, y0, x0, acc[(UR + 1) % NZ]);
            }
          });
        }
      }
      __syncthreads();
    }
  } else {
#pragma unroll 1
    for (int it = 0; it < nit; ++it) {
      front(it);
      if (it >= TT * (NZ - 1)) {
        const int z = pin0 + it - TT * S::ZHI;
        T acc[M][VX];
        zero_acc<T, VX, M>(acc);
        SmemPlane<T, VX, C::LX> pl[NZ];
#pragma unroll
        for (int zi = 0; zi < NZ; ++zi) pl[zi].p = stage_plane(TT - 1, z + zi - S::ZLO) + row0 * C::LX + col0;
        run_gather<S, VX, M>(pl, acc);
        store_tile<T, VX, M, CM, BY, TG::XS>(out, g, z, y0, x0, acc);
      }
      __syncthreads();
    }
  }
}

// ===========================================================================
// Streaming + temporal blocking with retiming in EVERY fused step: the OCs
// ST_TB_RT and their BM/CM/PR combinations.
// Retiming (split partial sums) lets each stage consume only the NEWEST plane
// of the stage below it: stage s keeps, per thread tile, a register queue of
// NZ partial-sum planes; when input plane q of stage s-1 arrives, every value
// of its window is scattered into the NZ live outputs, and output plane
// q - ZHI completes and is written to stage s's shared-memory plane. A stage
// therefore reads ONE plane window from shared memory per output tile (the
// gather pipeline k_stream_tb reads NZ), so shared-memory traffic per fused
// step is about that of one ST sweep while HBM traffic is divided by TT.
//
// Warp-specialised pipeline (no CTA-wide barrier in the loop):
//   warp 0, lane 0  producer: TMA loads of input planes into an NR-slot ring
//                   (NS = planes in flight: PR; NS = 1 is "no prefetching";
//                   NR = NS + ZHI because stage 1 keeps input plane j - ZHI
//                   until iteration j: it is the frame source of the stage-1
//                   plane completed then);
//   group s=1..TT-1 one VX x MI register tile per thread over region R_s
//                   (the output tile expanded by (TT-s)*extent), op table
//                   S::Mid in scatter form; writes stage-s planes into an
//                   MR-slot ring (S::MIDR);
//   group TT        the M x VX (BM/CM) output tile of k_stream, scatter form,
//                   stores to HBM.
// Hand-offs are mbarriers: full[slot] (count = producer threads; TMA: tx
// bytes) and empty[slot] (count = consumer threads), parity = use count & 1.
// Groups run decoupled; a group waits only when its input is not ready or
// its output slot is still being read.
//
// Tile values outside R_s are computed from don't-care inputs and never feed
// a valid output, so they are stored unmasked (inside the plane buffer).
// Frame points (outside the update box) keep their value at every fused step
// (the frame never changes, C-1): stage 1 takes it from the input
// plane still held in the ring, later stages from the launch's input grid. Canonical order (C-4): partial sums receive slices in
// ascending dz and, in each slice, FMAs in (dy,dx) order -- bitwise equal to
// every other OC.
// ===========================================================================
template <class S, int BX, int BY, int VX, int M, int TT, int MI, int s>
struct TbRtStage {
  static constexpr int MY = S::XM ? 1 : M;                 // rows of the output tile
  static constexpr int HX0 = (TT - s) * S::XLO, HX1 = (TT - s) * S::XHI;
  static constexpr int HY0 = (TT - s) * S::YLO, HY1 = (TT - s) * S::YHI;
  // tile x origin = xb - TXL (S::XSHIFT: exactly the region's left edge, see StreamTbRtCfg)
  // intermediate steps use thread tiles of S::MVX x MI (S::MVX = 1: scalar
  // columns, so every shared-memory access of the stage is a contiguous 8-byte
  // warp access instead of 16-byte vectors with half-used neighbours)
  static constexpr int VXM = S::MVX;
  // S::FULLW (scalar columns, rounded geometry): the stage's tiles span every
  // column of the ring rows (pitch LXF, the TMA box width). A 16-lane phase
  // that crosses from tile row cy to cy+1 then jumps (MI - 1) * LXF words, so
  // with (MI - 1) * LXF = 0 mod 16 (C2: MI = 5, LXF = 68) no load phase puts
  // two tile rows on the same banks (row-straddling phases of 66-column tile
  // rows in a 68-element pitch replayed up to 2 wavefronts each). The extra
  // columns are computed from don't-care neighbours and never feed a valid
  // output.
  static constexpr bool FULLW = S::FULLW && !S::XSHIFT && VXM == 1;
  static constexpr int ALNF = (16 / (int)sizeof(typename S::T)) > VX ? (16 / (int)sizeof(typename S::T)) : VX;
  static constexpr int XOFFF = ((TT * S::XLO + ALNF - 1) / ALNF) * ALNF;
  static constexpr int LXF = ((XOFFF + BX + TT * S::XHI + ALNF - 1) / ALNF) * ALNF;
  static constexpr int TXL = FULLW ? XOFFF : S::XSHIFT ? HX0 : ((HX0 + VXM - 1) / VXM) * VXM;
  static constexpr int NTX = FULLW ? LXF : (TXL + BX + HX1 + VXM - 1) / VXM;
  static constexpr int RY = BY * MY + HY0 + HY1;
  static constexpr int NTY = (RY + MI - 1) / MI;
  // S::WALIGN == 2: tile rows padded to whole half-warps (idle lanes), so no
  // 16-lane phase of a shared-memory access spans two tile rows
  static constexpr int NTXP = S::WALIGN == 2 ? (NTX + 15) / 16 * 16 : NTX;
  static constexpr int NT = NTXP * NTY;
  static constexpr int W = (NT + 31) / 32;                 // warps of group s
};

// first warp of group s (1..TT; group TT = the last stage); warp 0 = producer
template <class S, int BX, int BY, int VX, int M, int TT, int MI, int s>
struct TbRtWarp0 {
  static constexpr int value =
      TbRtWarp0<S, BX, BY, VX, M, TT, MI, s - 1>::value + TbRtStage<S, BX, BY, VX, M, TT, MI, s - 1>::W;
};
template <class S, int BX, int BY, int VX, int M, int TT, int MI>
struct TbRtWarp0<S, BX, BY, VX, M, TT, MI, 1> { static constexpr int value = 1; };

template <class S, int BX, int BY, int VX, int M, bool CM, int NS, int TT>
struct StreamTbRtCfg {
  typedef typename S::T T;
  typedef TileGeom<S, BX, BY, VX, M, CM> TG;
  static constexpr int ALN = (16 / (int)sizeof(T)) > VX ? (16 / (int)sizeof(T)) : VX;
  // Column geometry. Without S::XSHIFT every ring uses the input plane's
  // geometry (column c = global xb - XOFF + c, XOFF rounded up to ALN). With
  // S::XSHIFT the ring of step s (s = 0: the TMA input) starts exactly at the
  // left edge of the region step s+1 needs: xoff(s) = (TT - s) * XLO. A thread
  // tile of step s+1 then begins XLO columns into its source row, so its
  // window (XLO left, XHI right) starts on a vector boundary and the op table's
  // vectors are shifted by XSH = XLO mod VX: a radius-1 fp64 window with VX = 2
  // is 2 aligned 128-bit loads instead of 3 (one a half-used neighbour vector),
  // and every output vector still lands aligned in its own ring.
  static constexpr int XOFF = S::XSHIFT ? TT * S::XLO : ((TT * S::XLO + ALN - 1) / ALN) * ALN;
  static __device__ __forceinline__ constexpr int xoff(int s) { return S::XSHIFT ? (TT - s) * S::XLO : XOFF; }
  static constexpr int LX = ((XOFF + BX + TT * S::XHI + ALN - 1) / ALN) * ALN;
  static constexpr int LY = BY * TG::MY + TT * (S::YLO + S::YHI);
  // even/odd-split last ring (S::SPLITMID; only without XSHIFT): its own row
  // pitch SP, odd arrays at SO; K = ring column of stage TT-1's tile column 0
  static constexpr int MVS = S::MVX;
  static constexpr int K = XOFF - ((S::XLO + MVS - 1) / MVS) * MVS;
  // FULLW: a phase may span two tile rows, so rows must continue each other's
  // banks (split_pitch_full) besides the even/odd halves (SO = 8 mod 16, the
  // phases start on even columns)
  static constexpr bool FW = S::FULLW && !S::XSHIFT && MVS == 1;
  static constexpr int SO = split_off(LX, FW ? 0 : K);
  static constexpr int MI = S::MI;
  static constexpr int SP = !S::SPLITMID ? LX : FW ? split_pitch_full(LX, SO, MI) : split_pitch(LX, K);
  // slot stride: the plane plus the rows a VX x MI intermediate tile of the last
  // tile row reads past it (discarded values) -- without the gap those reads fall
  // into the next slot while the producer refills it (a benign data race that
  // compute-sanitizer racecheck reports on the cp.async path)
  static constexpr int PLANE = (((SP > LX ? SP : LX) * LY + MI * LX + ALN) * (int)sizeof(T) + 127) / 128 * 128 /
                               (int)sizeof(T);
  static constexpr int PADF = 128 / (int)sizeof(T);
  static constexpr int PADB = ((MI * LX + ALN) * (int)sizeof(T) + 127) / 128 * 128 / (int)sizeof(T);
  static constexpr int NR = NS + S::ZHI;                     // input ring slots
  static constexpr int MR = S::MIDR;                         // slots of each stage ring
  static constexpr int ELEMS = PADF + (NR + MR * (TT - 1)) * PLANE + PADB;
  static constexpr int NBAR = 2 * NR + 2 * MR * (TT - 1);
  static constexpr int SMEM = ELEMS * (int)sizeof(T) + 8 * NBAR + 128;
  static constexpr int FT = TG::TPX * BY;                   // last-stage tiles
  static constexpr int WF = (FT + 31) / 32;
  // register split (S::REG_LO > 0): producer + intermediate stages give
  // registers to the last stage (setmaxnreg); role boundaries are then
  // warpgroup-aligned by idle padding warps
  static constexpr bool SPLIT = S::REG_LO > 0;
  static constexpr int WL0 = TbRtWarp0<S, BX, BY, VX, M, TT, MI, TT>::value;
  static constexpr int WL = SPLIT ? (WL0 + 3) / 4 * 4 : WL0;   // first last-stage warp
  static constexpr int NW = SPLIT ? (WL + WF + 3) / 4 * 4 : WL + WF;
  static constexpr int THREADS = 32 * NW;
};

template <class S, int BX, int BY, int VX, int M, bool CM, int NS, int TT>
__global__ void __launch_bounds__(StreamTbRtCfg<S, BX, BY, VX, M, CM, NS, TT>::THREADS, S::MINB)
k_stream_tb_rt(const typename S::T* __restrict__ in, typename S::T* __restrict__ out, Grid g, int chunk,
               const __grid_constant__ TmaDesc tmap) {
  typedef typename S::T T;
  typedef StreamTbRtCfg<S, BX, BY, VX, M, CM, NS, TT> C;
  constexpr int NZ = S::NZ;
  constexpr int MI = C::MI;
  constexpr int NR = C::NR, MR = C::MR;
  static_assert(TT >= 2, "k_stream_tb_rt needs TT >= 2");
  extern __shared__ __align__(128) unsigned char smem_raw[];
  T* sbase = reinterpret_cast<T*>(smem_raw);
  T* ring0 = sbase + C::PADF;
  T* mid = ring0 + NR * C::PLANE;                      // stage s slot b: mid + (MR*(s-1)+b)*PLANE
  unsigned long long* bars = reinterpret_cast<unsigned long long*>(smem_raw + C::ELEMS * sizeof(T));
  // bars: full_in[NR], empty_in[NR], then per stage s=1..TT-1: full_s[MR], empty_s[MR]
  unsigned long long* full_in = bars;
  unsigned long long* empty_in = bars + NR;
  auto full_s = [&](int s) { return bars + 2 * NR + 2 * MR * (s - 1); };
  auto empty_s = [&](int s) { return bars + 2 * NR + 2 * MR * (s - 1) + MR; };

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  constexpr int AL = S::ELECT ? 1 : 32;                // arrivals per consumer warp
  const int xa = (g.cx0 / C::ALN) * C::ALN;
  const int xb = xa + blockIdx.x * BX;
  const int yb = g.cy0 + blockIdx.y * BY * C::TG::MY;
  const int zs = g.cz0 + blockIdx.z * chunk;
  const int ze = min(zs + chunk, g.cz1);
  const int pin0 = zs - TT * S::ZLO;                   // first input plane
  const int nin = (ze - zs) + TT * (NZ - 1);           // planes each stage consumes
  const int X0 = xb - C::XOFF, Y0 = yb - TT * S::YLO;

  // stage planes start defined (their unwritten corners only feed discarded outputs)
  for (int i = tid; i < C::ELEMS; i += C::THREADS) sbase[i] = T(0);
  if (tid == 0) {
    if constexpr (S::TMA) tma_prefetch_desc(&tmap);
    for (int q = 0; q < NR; ++q) {
      mbar_init(&full_in[q], S::TMA ? 1 : 32);   // cp.async: one arrival per producer lane
      mbar_init(&empty_in[q], AL * TbRtStage<S, BX, BY, VX, M, TT, MI, 1>::W);
    }
    static_for<1, TT>([&](auto sc) {
      constexpr int s = decltype(sc)::value;
      constexpr int WN = s + 1 < TT ? TbRtStage<S, BX, BY, VX, M, TT, MI, s + 1>::W : C::WF;
      for (int b = 0; b < MR; ++b) {
        mbar_init(&full_s(s)[b], AL * TbRtStage<S, BX, BY, VX, M, TT, MI, s>::W);
        mbar_init(&empty_s(s)[b], AL * WN);
      }
    });
    fence_mbar_init();
  }
  fence_proxy_async();                                  // generic zero-fill before async-proxy writes
  __syncthreads();
  if constexpr (C::SPLIT) {
    if (warp < C::WL) setmaxnreg_dec<S::REG_LO>();
    else setmaxnreg_inc<S::REG_HI>();
  }

  // ------------------------------------------------------------ producer
  if (warp == 0) {
    if constexpr (S::TMA) {
      if (tid == 0) {
        int slot = 0;
        unsigned ph = 0;                                 // (j / NR) & 1
#pragma unroll 1
        for (int j = 0; j < nin; ++j) {
          if (j >= NR) mbar_wait_sleep(&empty_in[slot], ph ^ 1u);
          mbar_expect_tx(&full_in[slot], C::LX * C::LY * (unsigned)sizeof(T));
          tma_load_3d(ring0 + slot * C::PLANE, &tmap, &full_in[slot], X0, Y0, pin0 + j);
          if (++slot == NR) { slot = 0; ph ^= 1u; }
        }
      }
    } else {
      // rows not TMA-aligned: the whole warp stages planes with cp.async, one
      // commit group per plane, NS planes in flight; plane j - (NS-1) is
      // published (a plain release-arrive by every lane) once cp.async.wait_group
      // says its group has landed -- the classic multistage cp.async pipeline
      // (compute-sanitizer racecheck flagged the variant that published with
      // cp.async.mbarrier.arrive.noinc; this form is clean)
      int slot = 0;
      unsigned ph = 0;
#pragma unroll 1
      for (int j = 0; j < nin; ++j) {
        if (j >= NR) mbar_wait_sleep(&empty_in[slot], ph ^ 1u);
        stage_plane_cp_async<T, C::LX, C::LY, 32>(ring0 + slot * C::PLANE, in, g, X0, Y0, pin0 + j, tid);
        cp_async_commit();
        if (j >= NS - 1) {
          cp_async_wait<NS - 1>();
          __threadfence_block();                         // landed copies ordered before the release
          mbar_arrive(&full_in[(j - (NS - 1)) % NR]);
        }
        if (++slot == NR) { slot = 0; ph ^= 1u; }
      }
      cp_async_wait<0>();
      __threadfence_block();
      for (int j = nin - (NS - 1) > 0 ? nin - (NS - 1) : 0; j < nin; ++j) mbar_arrive(&full_in[j % NR]);
    }
    return;
  }

  // ------------------------------------------------------------ intermediate stages
  bool done = false;
  static_for<1, TT>([&](auto sc) {
    constexpr int s = decltype(sc)::value;
    typedef TbRtStage<S, BX, BY, VX, M, TT, MI, s> G;
    constexpr int W0 = TbRtWarp0<S, BX, BY, VX, M, TT, MI, s>::value;
    if (done || warp < W0 || warp >= W0 + G::W) return;
    done = true;
    constexpr int XO_R = C::xoff(s - 1), XO_W = C::xoff(s);   // source / own ring geometry
    constexpr int MV = G::VXM;
    constexpr bool XOVER = XO_W - G::TXL + G::NTX * MV > C::LX;
    const int t = tid - 32 * W0;
    bool act = t < G::NT;
    // tile (column cx, row cy) of thread t. S::WALIGN: the first NXM columns of
    // every tile row (a multiple of 32) are whole warps of one tile row, the
    // remaining NTX - NXM columns of all rows go to the last warp(s); otherwise
    // row-major over NTX columns, where a warp straddling two tile rows hits
    // the same banks twice (a third shared-memory wavefront per access)
    constexpr int NXM = S::WALIGN == 1 ? (G::NTX / 32) * 32 : 0, NXE = G::NTXP - NXM;
    const int cx = t < NXM * G::NTY ? t % (NXM ? NXM : 1) : NXM + (t - NXM * G::NTY) % NXE;
    const int cy = t < NXM * G::NTY ? t / (NXM ? NXM : 1) : (t - NXM * G::NTY) / NXE;
    if (cx >= G::NTX) act = false;                              // (WALIGN == 2 padding lanes)
    const int gx0 = xb - G::TXL + cx * MV;
    const int gy0 = yb - G::HY0 + cy * MI;
    const int lb_r = (gy0 - Y0) * C::LX + (gx0 - xb + XO_R);   // tile origin in the source ring
    const int lrow = gy0 - Y0, lcol = gx0 - xb + XO_W;
    const int lb = lrow * C::LX + lcol;                         // ... in the stage's own ring
    const int ry1 = yb + BY * G::MY + G::HY1;
    // rows: bit m = writable (inside R_s rows and the array), bit 8+m = inside the update box
    unsigned rows = 0, allup = 1;
#pragma unroll
    for (int m = 0; m < MI; ++m) {
      const int gy = gy0 + m;
      const bool wr = gy < ry1 && gy >= 0 && gy < g.ny;
      const bool up = gy < ry1 && gy >= g.uy0 && gy < g.uy1;
      rows |= (wr ? 1u << m : 0u) | (up ? 1u << (8 + m) : 0u);
      allup &= (gy >= ry1 || up) ? 1u : 0u;
    }
    const bool xfast = gx0 >= g.ux0 && gx0 + MV <= g.ux1 && (!XOVER || gx0 - xb + XO_W + MV <= C::LX);
    const bool fast = act && xfast && allup;
    unsigned long long* fin = s == 1 ? full_in : full_s(s - 1);
    unsigned long long* ein = s == 1 ? empty_in : empty_s(s - 1);
    constexpr int DIN = s == 1 ? NR : MR;
    T acc[NZ][MI][MV];
#pragma unroll
    for (int q = 0; q < NZ; ++q) zero_acc<T, MV, MI>(acc[q]);
    // NZ unrolled plane bodies (compile-time queue rotation), or one body and
    // a register shift of the queue for large op tables (S::RTSHIFT)
    constexpr int UNR = S::RTSHIFT ? 1 : NZ;
    // ring slots and mbarrier phases advance incrementally (the input ring has
    // NS + ZHI slots, generally not a power of two: j % NR and j / NR per plane
    // cost a dozen integer instructions on every stage warp's critical path)
    int si = 0, so = 0, sf = (NR - S::ZHI % NR) % NR;   // slots of planes j, j (own ring), j - ZHI
    unsigned pin = 0, pout = 0;                          // phases (j / DIN) & 1, (j / MR) & 1
#pragma unroll 1
    for (int jb = 0; jb < nin; jb += UNR) {
      static_for<0, UNR>([&](auto ic) {
        constexpr int U = S::RTSHIFT ? NZ - 1 : decltype(ic)::value;
        const int j = jb + decltype(ic)::value;
        if (j >= nin) return;
        const T* src = s == 1 ? ring0 + si * C::PLANE : mid + (MR * (s - 2) + si) * C::PLANE;
        mbar_wait_sleep(&fin[si], pin);
        if constexpr (!S::RTSHIFT) zero_acc<T, MV, MI>(acc[U]);   // a new output plane starts
        if (act) {
          SmemPlane<T, MV, C::LX> pl{src + lb_r - S::XSH};
          run_scatter_ops<S, typename S::Mid, MV, MI, U>(pl, acc);
        }
        if (s > 1) warp_arrive<S::ELECT>(&ein[si]);      // input slot read (stage 1: below)
        T* dst = mid + (MR * (s - 1) + so) * C::PLANE;
        if (j >= MR) mbar_wait_sleep(&empty_s(s)[so], pout ^ 1u);
        const int zo = pin0 + j - s * S::ZHI;            // plane completed now
        // stage 1: input plane zo (= index j - ZHI) is still in the ring
        const T* fr = ring0 + sf * C::PLANE + lb_r;
        const bool zin = zo >= 0 && zo < g.nz;
        const bool zupd = zo >= g.uz0 && zo < g.uz1;
        const T(&res)[MI][MV] = acc[(U + 1) % NZ];
        constexpr bool SPL = S::SPLITMID && s == TT - 1;  // the ring the last stage reads
        if (zupd && fast) {                              // interior: vector stores (don't-care
#pragma unroll                                          // values past R_s stay in the buffer)
          for (int m = 0; m < MI; ++m)
            if (rows & (1u << m)) {
              if constexpr (SPL) {
#pragma unroll
                for (int v = 0; v < MV; ++v) dst[split_idx<C::SP, C::SO>(lrow + m, lcol + v)] = res[m][v];
              } else {
                stg_vec<T, MV>(dst + lb + m * C::LX, res[m]);
              }
            }
        } else if (zin && act) {                         // frame / edge tiles
#pragma unroll
          for (int m = 0; m < MI; ++m) {
            if (!(rows & (1u << m))) continue;
            const bool rowupd = zupd && (rows & (1u << (8 + m)));
            T* d = dst + lb + m * C::LX;
            if (rowupd && xfast && !SPL) {
              stg_vec<T, MV>(d, res[m]);
            } else {
              const T* frame = in + (i64)zo * g.sz + (i64)(gy0 + m) * g.sy;
#pragma unroll
              for (int v = 0; v < MV; ++v) {
                const int gx = gx0 + v;
                if (gx < 0 || gx >= g.nx || gx - xb + XO_W >= C::LX) continue;
                const bool upd = rowupd && gx >= g.ux0 && gx < g.ux1;
                const T val = upd ? res[m][v] : (s == 1 ? fr[m * C::LX + v] : __ldg(frame + gx));
                if constexpr (SPL) dst[split_idx<C::SP, C::SO>(lrow + m, lcol + v)] = val;
                else d[v] = val;
              }
            }
          }
        }
        if (s == 1 && j >= S::ZHI) warp_arrive<S::ELECT>(&ein[sf]);   // frame source released
        warp_arrive<S::ELECT>(&full_s(s)[so]);           // stage-s plane written
        if constexpr (S::RTSHIFT) shift_queue<T, NZ, MI, MV>(acc);
        if (++si == DIN) { si = 0; pin ^= 1u; }
        if (++so == MR) { so = 0; pout ^= 1u; }
        if (++sf == NR) sf = 0;
      });
    }
  });
  if (done || warp < C::WL || warp >= C::WL + C::WF) return;   // (idle padding warps)

  // ------------------------------------------------------------ last stage
  {
    const int q = tid - 32 * C::WL;
    const bool act = q < C::FT;
    typedef typename C::TG TG;
    const int tx = q % TG::TPX, ty = q / TG::TPX;
    const int row0 = TT * S::YLO + TG::row(ty);
    const int col0 = C::xoff(TT - 1) + tx * TG::XSTEP - S::XSH;   // window start in the last ring
    const int x0 = xb + tx * TG::XSTEP;
    const int y0 = yb + TG::row(ty);
    const TileStore<T, VX, M, CM, BY, S::SY, S::SZ, TG::XS> ts(out, g, y0, x0);
    unsigned long long* fin = full_s(TT - 1);
    unsigned long long* ein = empty_s(TT - 1);
    T acc[NZ][M][VX];
#pragma unroll
    for (int u = 0; u < NZ; ++u) zero_acc<T, VX, M>(acc[u]);
    constexpr int UNR = S::RTSHIFT ? 1 : NZ;
#pragma unroll 1
    for (int jb = 0; jb < nin; jb += UNR) {
      static_for<0, UNR>([&](auto ic) {
        constexpr int U = S::RTSHIFT ? NZ - 1 : decltype(ic)::value;
        const int j = jb + decltype(ic)::value;
        if (j >= nin) return;
        const int si = j % MR;
        mbar_wait_sleep(&fin[si], (unsigned)((j / MR) & 1));
        if constexpr (!S::RTSHIFT) zero_acc<T, VX, M>(acc[U]);
        if (act) {
          const T* pm = mid + (MR * (TT - 2) + si) * C::PLANE;
          if constexpr (S::SPLITMID) {
            SplitPlane<T, C::SP, C::SO> pl{pm + row0 * C::SP + (col0 >> 1)};
            run_scatter<S, VX, M, U>(pl, acc);
          } else {
            SmemPlane<T, VX, C::LX> pl{pm + row0 * C::LX + col0};
            run_scatter<S, VX, M, U>(pl, acc);
          }
        }
        warp_arrive<S::ELECT>(&ein[si]);
        const int z = pin0 + j - TT * S::ZHI;
        if (act && z >= zs) ts.store(z, acc[(U + 1) % NZ], g, out);
        if constexpr (S::RTSHIFT) shift_queue<T, NZ, M, VX>(acc);
      });
    }
  }
}

}  // namespace smart
