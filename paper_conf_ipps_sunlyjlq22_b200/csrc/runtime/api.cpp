// api.cpp -- the C ABI of include/stencil.h: validation, pattern ingestion,
// OC lattice, parameter settings, launch configuration and the time loop.
// SURVEY §8(a) rows a1 (pattern ingestion), a2 (OC validation + settings),
// a4 (frame / ping-pong setup), a5 (dispatch to the OC kernel family) and a6
// (time loop). Citations: PAPER.md line numbers (P:L<n>).
#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "internal.h"

namespace smart_rt {

std::atomic<uint64_t> g_launches{0};

// ----------------------------------------------------------------- errors
static thread_local std::string t_err;

void set_error(const char* fmt, ...) {
  char buf[4096];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  t_err = buf;
}
void clear_error() { t_err.clear(); }

// ------------------------------------------------------------- driver API
static Driver g_drv;
static int g_drv_state = 0;   // 0 unknown, 1 ok, -1 failed
static std::mutex g_drv_mu;

template <class F>
static bool entry(const char* name, F* fp) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess ||
      !p)
    return false;
  *fp = reinterpret_cast<F>(p);
  return true;
}

int get_driver(const Driver** out) {
  std::lock_guard<std::mutex> lk(g_drv_mu);
  if (g_drv_state == 0) {
    bool ok = entry("cuModuleLoadData", &g_drv.moduleLoadData) && entry("cuModuleUnload", &g_drv.moduleUnload) &&
              entry("cuModuleGetFunction", &g_drv.moduleGetFunction) &&
              entry("cuFuncSetAttribute", &g_drv.funcSetAttribute) &&
              entry("cuFuncGetAttribute", &g_drv.funcGetAttribute) && entry("cuLaunchKernel", &g_drv.launchKernel) &&
              entry("cuTensorMapEncodeTiled", &g_drv.tensorMapEncodeTiled) &&
              entry("cuGetErrorString", &g_drv.getErrorString) &&
              entry("cuOccupancyMaxActiveBlocksPerMultiprocessor", &g_drv.occupancy);
    g_drv_state = ok ? 1 : -1;
  }
  if (g_drv_state != 1) SM_FAIL(STENCIL_E_CUDA, "CUDA driver entry points unavailable (no GPU driver?)");
  *out = &g_drv;
  return STENCIL_OK;
}

const char* cu_errstr(CUresult r) {
  const char* s = nullptr;
  if (g_drv_state == 1 && g_drv.getErrorString) g_drv.getErrorString(r, &s);
  return s ? s : "unknown CUDA driver error";
}

// ------------------------------------------------------------ OC lattice
// Table I: BM xor CM; RT => ST; PR => ST.
static bool oc_valid(uint32_t oc) {
  if (oc >= 64) return false;
  const bool st = oc & STENCIL_OC_ST, bm = oc & STENCIL_OC_BM, cm = oc & STENCIL_OC_CM;
  const bool rt = oc & STENCIL_OC_RT, pr = oc & STENCIL_OC_PR;
  if (bm && cm) return false;
  if ((rt || pr) && !st) return false;
  return true;
}

static const char* oc_name_static(uint32_t oc) {
  static std::string names[64];
  static std::once_flag once;
  std::call_once(once, [] {
    const char* ab[6] = {"ST", "TB", "BM", "CM", "RT", "PR"};
    const uint32_t bit[6] = {STENCIL_OC_ST, STENCIL_OC_TB, STENCIL_OC_BM, STENCIL_OC_CM, STENCIL_OC_RT, STENCIL_OC_PR};
    for (uint32_t m = 0; m < 64; ++m) {
      std::string s;
      for (int k = 0; k < 6; ++k)
        if (m & bit[k]) s += (s.empty() ? "" : "_") + std::string(ab[k]);
      names[m] = s.empty() ? "base" : s;
    }
  });
  if (!oc_valid(oc)) return nullptr;
  return names[oc].c_str();
}

// ------------------------------------------------------ parameter space
static bool pow2(int v) { return v > 0 && (v & (v - 1)) == 0; }

static int family_of(uint32_t oc, int smem) {
  const bool st = oc & STENCIL_OC_ST, tb = oc & STENCIL_OC_TB;
  if (st) return tb ? FAM_STREAM_TB : FAM_STREAM;
  if (tb) return FAM_TILED;
  return smem ? FAM_TILED : FAM_NAIVE;
}

// Defaults (k = 0 setting) per OC and dtype.
static void default_params(uint32_t oc, int ndim, int dtype, stencil_params_t* p) {
  const int vmax = dtype == STENCIL_F64 ? 2 : 4;
  const bool merge = oc & (STENCIL_OC_BM | STENCIL_OC_CM);
  memset(p, 0, sizeof *p);
  p->smem = 0;
  p->merge = merge ? 2 : 1;
  p->tb_steps = (oc & STENCIL_OC_TB) ? 2 : 1;
  p->pr_stages = (oc & STENCIL_OC_PR) ? 2 : 1;
  p->stream_chunk = 0;   // auto
  const int fam = family_of(oc, 0);
  if (fam == FAM_NAIVE) {
    p->bx = 32; p->by = merge ? 4 : 8; p->bz = 1; p->vx = 1;
  } else if (fam == FAM_TILED) {
    p->vx = vmax; p->bx = 16 * vmax; p->by = merge ? 4 : 8; p->bz = (oc & STENCIL_OC_TB) ? 4 : 8;
    // 2-D tiles: 32 vectors wide, merge 4 rows per thread (measured on N2's
    // order-1 stencil, 8192^2 fp64, TB_BM: merge 4 -> 597 GStencil/s, merge 2 -> 547;
    // with register-tiled intermediate steps bx 64 -> 675, bx 32 -> 623; order 2:
    // 487 vs 436)
    if (ndim == 2) { p->bz = 1; p->bx = 32 * vmax; if (merge) p->merge = 4; }
    // 2-D TB with merging: 64 x 32 tiles (round 2, with the full-width 1 x 5
    // intermediate tiles; N2 same box: order 2 484 -> 527, order 1 642 -> 657
    // against 64 x 16)
    if (ndim == 2 && merge && (oc & STENCIL_OC_TB)) p->by = 8;
  } else if (fam == FAM_STREAM) {
    // wide, shallow tiles: many small CTAs keep more TMA planes in flight per SM
    // (measured on C2: 128x2 fp64 tiles reach 92% of the copy bandwidth)
    p->vx = vmax; p->bx = 64 * vmax; p->by = 2; p->bz = 1;
    // 2-D streams move one row per plane: one more row in flight (measured on N2's
    // order-3 / order-4 stencils, 8192^2 fp64: PR 4 +2.7% / +1.1% over PR 3)
    if (oc & STENCIL_OC_PR) p->pr_stages = ndim == 2 ? 4 : 3;
  } else if (oc & STENCIL_OC_RT) {
    // warp-specialised retiming pipeline (k_stream_tb_rt); measured on C2:
    // 64 x 32-row output tiles (8 threads x merge 4 rows), 3 planes in flight
    p->vx = vmax; p->bx = 32 * vmax; p->by = 8; p->bz = 1;
    if (merge) p->merge = 4;
    // without merging: 64 x 16 output tiles (one row per last-stage thread), so
    // the tile keeps its 1-row x/y halo small against its rows. Measured on C2
    // (round 2, same box, 10 steps): ST_TB_RT_PR 303 -> 437, ST_TB_RT (no
    // prefetching) 127 -> 210 GStencil/s against 64 x 8
    else if (ndim == 3) p->by = 16;
    // 4 planes in flight: the stage-1 warps waited on the input ring for 23% of
    // their ncu stall samples with 3 (round 2, C2 same box: 563 -> 585 GStencil/s
    // with 4; 6: 585; 8 no longer fits one CTA per SM)
    if (oc & STENCIL_OC_PR) p->pr_stages = 4;
  } else {
    p->vx = vmax; p->bx = 32 * vmax; p->by = merge ? 4 : 8; p->bz = 1;
  }
  if (ndim == 2 && (fam == FAM_STREAM || fam == FAM_STREAM_TB) && merge) {
    // 2-D streaming views merge along x (resolve_variant): 2 vectors of <= 16
    // bytes per thread and 32 threads per tile row -> 128-column tiles, whose
    // TMA box (with the halo) stays within 256 elements
    p->merge = 2;
    p->vx = std::min(vmax, 2);
    p->bx = 32 * p->vx * p->merge;
  }
}

// counter-based hash for the seeded settings sampler
static uint64_t mix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
template <size_t N>
static int pick(uint64_t& h, const int (&choices)[N]) {
  h = mix64(h);
  return choices[h % N];
}

static void sample_params(uint32_t oc, int ndim, int dtype, uint64_t seed, int k, stencil_params_t* p) {
  default_params(oc, ndim, dtype, p);
  if (k <= 0) return;
  uint64_t h = mix64(seed ^ ((uint64_t)oc << 32) ^ (uint64_t)k * 0x632BE59BD9B4E019ull);
  const bool merge = oc & (STENCIL_OC_BM | STENCIL_OC_CM);
  const bool st = oc & STENCIL_OC_ST, tb = oc & STENCIL_OC_TB;
  if (!st && !tb) { const int s[] = {0, 1}; p->smem = pick(h, s); }
  if (merge) { const int s[] = {2, 4, 8}; p->merge = pick(h, s); }
  if (tb) { const int s[] = {2, 4}; p->tb_steps = pick(h, s); }
  if (oc & STENCIL_OC_PR) { const int s[] = {2, 3, 4}; p->pr_stages = pick(h, s); }   // enum
  const int fam = family_of(oc, p->smem);
  if (fam == FAM_NAIVE) {
    const int sx[] = {32, 64, 128}, sy[] = {1, 2, 4, 8};
    p->bx = pick(h, sx); p->by = pick(h, sy); p->vx = 1;
  } else {
    const int vmax = dtype == STENCIL_F64 ? 2 : 4;
    const int sv[] = {1, 2, 4};
    p->vx = std::min(pick(h, sv), vmax);
    const int sx[] = {16, 32, 64, 128};
    p->bx = std::max(pick(h, sx) * p->vx / (p->vx > 2 ? 2 : 1), 8 * p->vx);
    const int sy[] = {2, 4, 8, 16};
    p->by = pick(h, sy);
    if (fam == FAM_TILED) { const int sz[] = {2, 4, 8}; p->bz = ndim == 2 ? 1 : pick(h, sz); }
    if (st) { const int sc[] = {0, 32, 64, 128, 256}; p->stream_chunk = pick(h, sc); }
  }
  // keep the CTA within 32..1024 threads
  while ((p->bx / std::max(p->vx, 1)) * p->by > 1024 && p->by > 1) p->by /= 2;
  while ((p->bx / std::max(p->vx, 1)) * p->by < 32) p->by *= 2;
}

// ------------------------------------------------------------- pattern
static int build_pattern(stencil_plan_s* P) {
  const int r = P->order, w = 2 * r + 1;
  const bool two = P->ndim == 2;
  const int tsize = two ? w * w : w * w * w;
  P->pat = Pattern();
  Pattern& pat = P->pat;
  int zlo = 0, zhi = 0, ylo = 0, yhi = 0, xlo = 0, xhi = 0;
  for (int t = 0; t < tsize; ++t) {
    if (!P->access[t]) continue;
    int a, b, c;   // slowest..fastest offsets of the user tensor
    if (two) { a = 0; b = t / w - r; c = t % w - r; }
    else { a = t / (w * w) - r; b = (t / w) % w - r; c = t % w - r; }
    pat.dz.push_back(a); pat.dy.push_back(b); pat.dx.push_back(c);
    pat.c.push_back(P->coeffs[t]);
    zlo = std::max(zlo, -a); zhi = std::max(zhi, a);
    ylo = std::max(ylo, -b); yhi = std::max(yhi, b);
    xlo = std::max(xlo, -c); xhi = std::max(xhi, c);
  }
  pat.nnz = (int)pat.c.size();
  pat.zlo = zlo; pat.zhi = zhi; pat.ylo = ylo; pat.yhi = yhi; pat.xlo = xlo; pat.xhi = xhi;
  return STENCIL_OK;
}

// The 3-D kernel view of the grid. 3-D: identity. 2-D [ny][nx]: non-streaming
// families see [1][ny][nx]; streaming families stream along y and see
// [ny][1][nx] (the streaming dimension is the slowest one, C-13).
static void build_view(stencil_plan_s* P, int fam) {
  const int r = P->order;
  if (P->ndim == 3) {
    for (int k = 0; k < 3; ++k) { P->vdims[k] = P->dims[k]; P->frame[k] = r; }
    return;
  }
  const bool stream = fam == FAM_STREAM || fam == FAM_STREAM_TB;
  Pattern& pat = P->pat;
  if (stream) {
    P->vdims[0] = P->dims[0]; P->vdims[1] = 1; P->vdims[2] = P->dims[1];
    P->frame[0] = r; P->frame[1] = 0; P->frame[2] = r;
    // (0, dy, dx) -> (dy, 0, dx)
    for (int i = 0; i < pat.nnz; ++i) { pat.dz[i] = pat.dy[i]; pat.dy[i] = 0; }
    pat.zlo = pat.ylo; pat.zhi = pat.yhi; pat.ylo = pat.yhi = 0;
  } else {
    P->vdims[0] = 1; P->vdims[1] = P->dims[0]; P->vdims[2] = P->dims[1];
    P->frame[0] = 0; P->frame[1] = r; P->frame[2] = r;
  }
}

// ---------------------------------------------------- variant + feasibility
struct TmaBox { int lx, ly, lz; };

static TmaBox tma_box(const Variant& v, const Pattern& p, int elem) {
  const int aln = std::max(16 / elem, v.vx);
  auto ru = [](int a, int b) { return (a + b - 1) / b * b; };
  if (v.family == FAM_TILED) {
    const int xoff = ru(v.tt * p.xlo, aln);
    return {ru(xoff + v.bx + v.tt * p.xhi, aln), v.rows() + v.tt * (p.ylo + p.yhi),
            v.bz + v.tt * (p.zlo + p.zhi)};
  }
  const int t = v.family == FAM_STREAM_TB ? v.tt : 1;   // stream: halo of t time steps
  const int xoff = v.xshift ? t * p.xlo : ru(t * p.xlo, aln);   // mirrors StreamTbRtCfg::XOFF
  return {ru(xoff + v.bx + t * p.xhi, aln), v.rows() + t * (p.ylo + p.yhi), 1};
}

// Register split of the warp-specialised ST_TB_RT kernel (setmaxnreg): the
// CTA runs alone on its SM (__launch_bounds__(THREADS, 1)), so every warp gets
// the same cap R0 = 64K / THREADS; the producer and intermediate-stage warps
// shrink to R0 - 8 and the last stage -- the pipeline's slowest stage, which
// spills at R0 -- grows by what they free. Measured on C2 (512^3 heat, fp64,
// T = 2, 896 threads, R0 = 72): 517 -> 530 GStencil/s with 64/88, no spills
// (56/112: 521). Applied only when aligning the roles to warpgroups costs at
// most 2 idle warps; ensure_loaded() drops the split if the compiled kernel
// holds fewer registers than the pool needs.
static void choose_regsplit(Variant* v, const Pattern& pat, int elem) {
  v->reg_lo = v->reg_hi = 0;
  if (const char* e = getenv("STENCIL_REGSPLIT")) {   // dev override: "lo,hi" (or "0,0" = off)
    if (sscanf(e, "%d,%d", &v->reg_lo, &v->reg_hi) != 2) v->reg_lo = v->reg_hi = 0;
    return;
  }
  int wl = 0;
  const int nw0 = v->tbrt_threads(pat, elem, &wl) / 32;
  v->reg_lo = 1;                                   // padded (warpgroup-aligned) layout
  const int nw = v->tbrt_threads(pat, elem, &wl) / 32;
  v->reg_lo = 0;
  if (nw * 32 > 1024 || nw > nw0 + 2 || wl >= nw) return;
  const int r0 = std::min(255, (65536 / (nw * 32)) / 8 * 8);
  const int lo = r0 - 8;
  if (lo < 40) return;
  const int hi = std::min(256, ((nw * r0 - wl * lo) / (nw - wl)) / 8 * 8);
  if (hi <= r0) return;
  v->reg_lo = lo;
  v->reg_hi = hi;
}

static int resolve_variant(stencil_plan_s* P) {
  const stencil_params_t& p = P->params;
  const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
  const int fam = family_of(P->oc, p.smem);
  Variant v;
  v.family = fam;
  v.bx = p.bx; v.by = p.by; v.bz = p.bz; v.vx = p.vx;
  v.m = (P->oc & (STENCIL_OC_BM | STENCIL_OC_CM)) ? p.merge : 1;   // merging only under BM / CM
  v.cm = (P->oc & STENCIL_OC_CM) != 0;
  v.tt = (P->oc & STENCIL_OC_TB) ? p.tb_steps : 1;
  v.rt = (P->oc & STENCIL_OC_RT) != 0;
  v.ns = (P->oc & STENCIL_OC_PR) ? p.pr_stages : 1;
  if (fam == FAM_NAIVE) { v.vx = 1; v.bz = 1; }
  if (fam == FAM_STREAM || fam == FAM_STREAM_TB) v.bz = 1;
  if (P->ndim == 2) {
    // 2-D streaming views [ny][1][nx]: a plane is one row, so BM / CM merge
    // along x, the only other axis (P:L63 names merging in the
    // innermost dimension as a real, coalescing-relevant choice)
    if (fam == FAM_STREAM || fam == FAM_STREAM_TB) { v.by = 1; v.flat = true; v.xm = v.m > 1; }
    else v.bz = 1;
  }
  if (v.vx != 1 && v.vx != 2 && v.vx != 4) SM_FAIL(STENCIL_E_INVAL, "vx must be 1, 2 or 4");
  if (v.vx * elem > 32) SM_FAIL(STENCIL_E_INVAL, "vx*sizeof(T) must be <= 32 bytes");
  if (!pow2(v.bx) || !pow2(v.by) || !pow2(v.bz) || !pow2(v.m) || v.bx < v.vx)
    SM_FAIL(STENCIL_E_INVAL, "tile parameters must be powers of two (bx=%d by=%d bz=%d merge=%d vx=%d)", v.bx,
            v.by, v.bz, v.m, v.vx);
  if (v.m > 8) SM_FAIL(STENCIL_E_INVAL, "merge factor must be <= 8");
  if (v.xm && v.bx < v.vx * v.m)
    SM_FAIL(STENCIL_E_OC_INFEASIBLE, "x-merge of %d vectors of %d needs a tile of >= %d columns (bx=%d)", v.m, v.vx,
            v.vx * v.m, v.bx);
  if (v.tt < 1 || v.tt > 8) SM_FAIL(STENCIL_E_INVAL, "tb_steps must be in 1..8");
  if (v.ns < 1 || v.ns > 8) SM_FAIL(STENCIL_E_INVAL, "pr_stages must be in 1..8");
  if (fam == FAM_STREAM_TB && v.rt && v.tt >= 2) {
    // aligned-window ring geometry (StreamTbRtCfg): possible when the shifted
    // input offset TT*XLO keeps the TMA box start 16-byte aligned; used when it
    // saves at least 15% of the window loads. Measured on C2 (512^3, fp64, T=2):
    // Algorithm-1 order-1 stencils 494 -> 537 GStencil/s (loads -20..-30%);
    // the heat star saves only 9% and spills more: 530 -> 512, so it keeps the
    // rounded geometry.
    const int aln = std::max(16 / elem, v.vx);
    const bool tma_ok = (v.tt * P->pat.xlo) % aln == 0;
    if (tma_ok && P->pat.xlo % v.vx != 0) {
      Variant vs = v;
      vs.xshift = true;
      const int l0 = count_window_loads(P->pat, elem, v), l1 = count_window_loads(P->pat, elem, vs);
      v.xshift = l1 <= 0.85 * l0;
    }
    // 8-row block-merged last stage on a radius-1 in-plane pattern (the setting
    // stencil_plan_create picks for C2-like stencils): measured with the rounded
    // geometry; the aligned windows would win on load counts but took C2 from 615
    // to 434 GStencil/s (they also rule out the scalar-column stage tiles)
    if (v.m == 8 && !v.cm && !v.xm && elem == 8 && P->pat.xlo <= 1 && P->pat.xhi <= 1 && P->pat.ylo <= 1 &&
        P->pat.yhi <= 1)
      v.xshift = false;
    if (const char* nx = getenv("STENCIL_XSHIFT")) v.xshift = tma_ok && atoi(nx) != 0;   // dev override
    // even/odd-split last intermediate ring (fp64, 16-byte vectors of 2, rounded geometry)
    v.splitmid = elem == 8 && v.vx == 2 && !v.xshift;
    if (const char* sp = getenv("STENCIL_SPLITMID")) v.splitmid = v.splitmid && atoi(sp) != 0;   // dev override
    // Scalar-column (1 x 4) intermediate tiles for radius-1 in-plane patterns in
    // the rounded geometry: the intermediate step's loads and stores become
    // contiguous 8-byte warp accesses (no half-used neighbour vectors). Measured
    // on C2 (heat, 512^3 fp64, same box): ST_TB_BM_RT_PR 545 -> 554 GStencil/s;
    // 1 x 6 / 1 x 8 tiles need 128 registers and lose (440 / 286).
    if (elem == 8 && v.vx == 2 && !v.xshift && P->pat.xlo <= 1 && P->pat.xhi <= 1 && P->pat.ylo <= 1 &&
        P->pat.yhi <= 1) {
      v.midvx = 1;
      if (v.tbrt_threads(P->pat, elem) > 1024) v.midvx = 0;
    }
    if (const char* mv = getenv("STENCIL_MID_VX"))   // dev override: intermediate-step columns per thread
      if (!v.xshift) v.midvx = std::max(0, std::min(v.vx, atoi(mv)));
    // scalar-column stage tiles over whole ring rows (TbRtStage::FULLW); with
    // 8-row last-stage tiles (merge 8, see stencil_plan_create) they come with
    // 1 x 5 stage tiles (conflict-free: (5 - 1) * LX = 0 mod 16 words) and
    // 3-slot stage rings. C2, same box, 10 steps (GStencil/s): the round-2
    // default (merge 4, 1 x 4 tiles, 2 slots) 590; merge 8 + these 603 (2
    // slots) / 615 (3 slots); merge 8 alone 579
    v.fullw = false;
    v.mid_rows_set = v.mid_slots_set = 0;
    if (v.midvx == 1 && !v.xshift && v.m == 8 && !v.cm && !v.xm) {
      v.fullw = true;
      v.mid_rows_set = 5;
      v.mid_slots_set = 3;
    }
    if (const char* fw = getenv("STENCIL_FULLW")) v.fullw = atoi(fw) != 0;   // dev override
    if (v.midvx != 1 || v.xshift) v.fullw = false;
    if (v.fullw && v.tbrt_threads(P->pat, elem) > 1024) v.fullw = false;
    choose_regsplit(&v, P->pat, elem);
    v.ws_threads = v.tbrt_threads(P->pat, elem);
  }
  if (fam == FAM_TILED && v.tt > 1) {
    // intermediate fused steps in 1 x 4 register tiles (k_tiled, S::TMID). Measured
    // (same box, TB_BM / TB): N2 order-1 8192^2 582 -> 673 / 391 -> 439, order-2
    // 423 -> 486, C2 heat 512^3 191 -> 240 / 138 -> 192 GStencil/s against one
    // point per thread; 1 x 2 is within +-4%, 1 x 8 loses
    // Round 2: the tiles span the buffer's whole rows (TiledCfg::FULL) and are
    // 1 x 5, so that no 16-lane phase of their loads and stores hits a bank twice
    // where it crosses a row end ((5 - 1) * LX = 0 mod 16 words for fp64 rows of
    // LX = 0 mod 4). ncu: the 1 x 4 tiles over the region's own columns put
    // 12.2 M bank-conflict replays into N2 order 2's 70.3 M shared wavefronts
    // per 2-step launch, with the L1/shared pipe 97% busy. Same box: N2 order 2
    // (TB_BM, 64 x 32 tiles) 499 -> 527, order 1 627 -> 657, C2 heat TB_BM 192 -> 226.
    v.tiled_mid = 5;
    v.tiled_full = true;
    if (const char* e = getenv("STENCIL_TILED_MID")) v.tiled_mid = std::max(0, std::min(8, atoi(e)));   // dev override (op tables encode M <= 8)
    if (const char* e = getenv("STENCIL_TILED_FULL")) v.tiled_full = atoi(e) != 0;   // dev override
    // 2-column (16-byte vector) tiles where they cut the window loads or the
    // instruction count: 3-D views and x-extent >= 3. Same box, 10 steps (TB_BM,
    // GStencil/s, 1 column -> 2): N2 order 2 517 -> 536, order 3 253 -> 286, C2
    // heat 217 -> 240, C5 order 2 (1024^3) 14.6 -> 22.3; the 2-D order-1 stencil
    // (x-extent 2) loses, 647 -> 575 (56 registers: 4 CTAs per SM instead of 5)
    v.tiled_mvx = (P->ndim == 3 || P->pat.xlo + P->pat.xhi >= 3) ? 2 : 1;
    if (const char* e = getenv("STENCIL_TILED_MVX")) v.tiled_mvx = atoi(e) == 2 ? 2 : 1;   // dev override
    if (!v.tiled_full || v.vx < v.tiled_mvx) v.tiled_mvx = 1;   // vector tiles need whole (aligned) rows
  }
  const int thr = v.threads();
  if (thr < 32 || thr > 1024)
    SM_FAIL(STENCIL_E_OC_INFEASIBLE, "CTA of %d threads outside 32..1024", thr);
  const int smem = v.smem_bytes(P->pat, elem);
  if (smem > 232448)
    SM_FAIL(STENCIL_E_OC_INFEASIBLE, "OC %s needs %d B of shared memory per CTA (> 227 KB)",
            oc_name_static(P->oc), smem);
  // TMA staging when rows are 16-byte multiples and the box fits 256^3
  v.tma = false;
  if (fam == FAM_TILED || fam == FAM_STREAM || fam == FAM_STREAM_TB) {
    const TmaBox b = tma_box(v, P->pat, elem);
    const bool rows_ok = (P->vdims[2] * elem) % 16 == 0;
    const char* notma = getenv("STENCIL_NO_TMA");   // dev / test override: cp.async staging
    v.tma = rows_ok && b.lx <= 256 && b.ly <= 256 && b.lz <= 256 && !(notma && atoi(notma));
  }
  // (streaming TB without TMA: the input planes are staged with element-wise
  // cp.async -- rows that are not 16-byte multiples, boxes wider than 256)
  if (fam == FAM_STREAM_TB && v.tt < 2) v.family = FAM_STREAM;
  v.chunk = p.stream_chunk;
  v.sy = P->vdims[2];                       // = make_grid's strides (contiguous view)
  v.sz = P->vdims[1] * P->vdims[2];
  if (const char* e = getenv("STENCIL_NO_BAKE"))   // dev override: run-time strides
    if (atoi(e)) v.sy = v.sz = 0;
  P->var = v;
  return STENCIL_OK;
}

static int validate_params(const stencil_params_t* p) {
  for (int k = 0; k < 3; ++k)
    if (p->reserved[k] != 0) SM_FAIL(STENCIL_E_INVAL, "stencil_params_t.reserved must be 0");
  if (p->smem < -1 || p->smem > 1) SM_FAIL(STENCIL_E_INVAL, "smem must be -1, 0 or 1");
  const int32_t* f = &p->bx;
  for (int k = 0; k < 8; ++k)
    if (f[k] < 0) SM_FAIL(STENCIL_E_INVAL, "negative parameter");
  return STENCIL_OK;
}

static void merge_params(const stencil_params_t* user, stencil_params_t* out) {
  if (!user) return;
  if (user->smem >= 0) out->smem = user->smem;
  if (user->bx) out->bx = user->bx;
  if (user->by) out->by = user->by;
  if (user->bz) out->bz = user->bz;
  if (user->vx) out->vx = user->vx;
  if (user->merge) out->merge = user->merge;
  if (user->stream_chunk) out->stream_chunk = user->stream_chunk;
  if (user->tb_steps) out->tb_steps = user->tb_steps;
  if (user->pr_stages) out->pr_stages = user->pr_stages;
}

// ------------------------------------------------------------ grid args
static GridArg make_grid(const stencil_plan_s* P, int elem_vx) {
  GridArg g{};
  g.nz = (int)P->vdims[0]; g.ny = (int)P->vdims[1]; g.nx = (int)P->vdims[2];
  g.sy = P->vdims[2];
  g.sz = P->vdims[1] * P->vdims[2];
  g.uz0 = P->frame[0]; g.uz1 = g.nz - P->frame[0];
  g.uy0 = P->frame[1]; g.uy1 = g.ny - P->frame[1];
  g.ux0 = P->frame[2]; g.ux1 = g.nx - P->frame[2];
  g.cz0 = g.uz0; g.cz1 = g.uz1; g.cy0 = g.uy0; g.cy1 = g.uy1; g.cx0 = g.ux0; g.cx1 = g.ux1;
  if (P->comm) {   // slab: frame only at the global z faces; compute the owned planes
    const int G = P->ghost, n = (int)P->dims[0], r = P->frame[0];
    g.uz0 = P->comm->rank == 0 ? G + r : 0;
    g.uz1 = P->comm->rank == P->comm->nranks - 1 ? G + n - r : g.nz;
    g.cz0 = std::max(G, g.uz0);
    g.cz1 = std::min(G + n, g.uz1);
  }
  g.vec_ok = (g.nx % elem_vx) == 0;
  return g;
}

static int ensure_loaded(stencil_plan_s* P) {
  if (P->loaded) return STENCIL_OK;
  const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
  if (P->cubin.empty()) SM_TRY(compile_variant(P->pat, P->dtype, P->var, &P->lowered, &P->cubin));
  SM_TRY(load_kernel(P->src, P->cubin, P->lowered, P->var.smem_bytes(P->pat, elem), &P->kern));
  if (!P->var.regsplit_fits(P->pat, elem, P->kern.regs)) {
    if (getenv("STENCIL_REGSPLIT"))
      SM_FAIL(STENCIL_E_OC_INFEASIBLE, "register split %d/%d does not fit %d regs/thread", P->var.reg_lo,
              P->var.reg_hi, P->kern.regs);
    // the kernel holds fewer registers than the split needs: recompile without it
    P->var.reg_lo = P->var.reg_hi = 0;
    P->var.ws_threads = P->var.tbrt_threads(P->pat, elem);
    P->src = generate_source(P->pat, P->dtype, P->var);
    P->cubin.clear();
    SM_TRY(compile_variant(P->pat, P->dtype, P->var, &P->lowered, &P->cubin));
    SM_TRY(load_kernel(P->src, P->cubin, P->lowered, P->var.smem_bytes(P->pat, elem), &P->kern));
  }
  P->loaded = true;
  return STENCIL_OK;
}

static int get_tmap(stencil_plan_s* P, const Variant& v, const void* buf, CUtensorMap** out) {
  auto it = P->tmaps.find(buf);
  if (it != P->tmaps.end() && v.family == P->var.family && v.tt == P->var.tt) {
    *out = &it->second;
    return STENCIL_OK;
  }
  const Driver* d = nullptr;
  SM_TRY(get_driver(&d));
  const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
  if (((uintptr_t)buf) % 16) SM_FAIL(STENCIL_E_INVAL, "TMA staging needs 16-byte aligned grid pointers");
  const TmaBox b = tma_box(v, P->pat, elem);
  CUtensorMap m;
  cuuint64_t gdim[3] = {(cuuint64_t)P->vdims[2], (cuuint64_t)P->vdims[1], (cuuint64_t)P->vdims[0]};
  cuuint64_t gstr[2] = {(cuuint64_t)(P->vdims[2] * elem), (cuuint64_t)(P->vdims[2] * P->vdims[1] * elem)};
  cuuint32_t box[3] = {(cuuint32_t)b.lx, (cuuint32_t)b.ly, (cuuint32_t)b.lz};
  cuuint32_t es[3] = {1, 1, 1};
  CUresult r = d->tensorMapEncodeTiled(&m, elem == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                                       3, const_cast<void*>(buf), gdim, gstr, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                       CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) SM_FAIL(STENCIL_E_CUDA, "cuTensorMapEncodeTiled: %s", cu_errstr(r));
  if (v.family == P->var.family && v.tt == P->var.tt) {
    P->tmaps[buf] = m;
    *out = &P->tmaps[buf];
  } else {
    static thread_local CUtensorMap tmp;
    tmp = m;
    *out = &tmp;
  }
  return STENCIL_OK;
}

// Default z-chunk of the streaming kernels (concurrent streaming).
// Columns that cannot fill the GPU (2-D grids stream along y with a single
// row of CTAs per x-tile: 64 tiles at 8192^2) are cut so that about one wave
// of CTAs is resident, counting at most 16 CTAs per SM: measured on the N2
// 2-D stencils (8192^2 fp64), chunks of ~200 rows run 1.2-1.3x faster than
// 512 (too few CTAs) and than 64-128 on order-1 stencils (too many concurrent
// streams). Otherwise: enough CTAs for ~8 per SM, chunks of at least 16
// planes (halo reuse); measured on C2, full-depth columns beat any split.
static int auto_chunk(const stencil_plan_s* P, const Variant& v, const Kernel& k, int threads, int smem,
                      int czlen, long long tiles_xy) {
  if (v.chunk > 0) return std::min(v.chunk, czlen);
  int nsm = 0, dev = 0, occ = 0;
  const Driver* d = nullptr;
  if (cudaGetDevice(&dev) == cudaSuccess &&
      cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && get_driver(&d) == 0 &&
      d->occupancy(&occ, k.fn, threads, (size_t)smem) == CUDA_SUCCESS && occ > 0) {
    const long long slots = (long long)nsm * std::min(occ, 16);
    if (tiles_xy * 2 < slots) {
      const long long nch = std::max(1LL, slots / tiles_xy);
      return std::min(czlen, std::max(32, (int)((czlen + nch - 1) / nch)));
    }
  }
  // enough CTAs for ~8 per SM, but chunks of at least 16 planes (halo reuse)
  long long target = 148LL * 8;
  int c = 1;
  while (c < czlen && tiles_xy * ((czlen + c - 1) / c) > target) c *= 2;
  (void)P;
  return std::max(std::min(c, czlen), std::min(16, czlen));
}

// Launch the main variant (or `k` for a TB remainder) for one application of
// the kernel: src -> dst over the compute box of g.
static int launch_sweep(stencil_plan_s* P, const Variant& v, const Kernel& k, const void* src, void* dst,
                        const GridArg& g) {
  const Driver* d = nullptr;
  SM_TRY(get_driver(&d));
  const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
  const int czlen = g.cz1 - g.cz0, cylen = g.cy1 - g.cy0, cxlen = g.cx1 - g.cx0;
  if (czlen <= 0 || cylen <= 0 || cxlen <= 0) return STENCIL_OK;
  const int aln = std::max(16 / elem, v.vx);
  unsigned gx, gy, gz, bx, by;
  int chunk = 0;
  CUtensorMap* tm = nullptr;
  CUtensorMap dummy;
  memset(&dummy, 0, sizeof dummy);
  void* args[5];
  const void* in = src;
  void* out = dst;
  GridArg gg = g;
  args[0] = (void*)&in;
  args[1] = (void*)&out;
  args[2] = (void*)&gg;
  int nargs = 3;
  if (v.family == FAM_NAIVE) {
    gx = (cxlen + v.bx - 1) / v.bx;
    gy = (cylen + v.by * v.m - 1) / (v.by * v.m);
    gz = czlen;
    bx = v.bx; by = v.by;
  } else {
    const int xa = (g.cx0 / aln) * aln;
    gx = (g.cx1 - xa + v.bx - 1) / v.bx;
    gy = (cylen + v.rows() - 1) / v.rows();
    bx = v.family == FAM_TILED ? v.bx / v.vx : v.tpx(); by = v.by;
    if (v.family == FAM_STREAM_TB && v.rt) { bx = v.threads(); by = 1; }   // warp-specialised, 1-D
    if (v.tma) SM_TRY(get_tmap(P, v, src, &tm));
    if (v.family == FAM_TILED) {
      gz = (czlen + v.bz - 1) / v.bz;
      args[3] = tm ? (void*)tm : (void*)&dummy;
      nargs = 4;
    } else {
      chunk = auto_chunk(P, v, k, (int)(bx * by), v.smem_bytes(P->pat, elem), czlen, (long long)gx * gy);
      gz = (czlen + chunk - 1) / chunk;
      args[3] = (void*)&chunk;
      args[4] = tm ? (void*)tm : (void*)&dummy;
      nargs = 5;
    }
  }
  (void)nargs;
  if (gy > 65535 || gz > 65535) SM_FAIL(STENCIL_E_OC_INFEASIBLE, "grid too large for this tile setting");
  const int smem = v.smem_bytes(P->pat, elem);
  if (P->timing) {
    if (P->ev_pool.size() < P->ev_used + 2) {
      for (int i = 0; i < 64; ++i) {
        cudaEvent_t e;
        SM_CUDA(cudaEventCreate(&e));
        P->ev_pool.push_back(e);
      }
    }
    SM_CUDA(cudaEventRecord(P->ev_pool[P->ev_used], P->stream));
  }
  CUresult r = d->launchKernel(k.fn, gx, gy, gz, bx, by, 1, smem, (CUstream)P->stream, args, nullptr);
  g_launches.fetch_add(1);
  if (r != CUDA_SUCCESS) SM_FAIL(STENCIL_E_CUDA, "cuLaunchKernel(%s): %s", P->lowered.c_str(), cu_errstr(r));
  if (P->timing) {
    SM_CUDA(cudaEventRecord(P->ev_pool[P->ev_used + 1], P->stream));
    P->ev_used += 2;
  }
  return STENCIL_OK;
}

static int get_tb_rem_kernel(stencil_plan_s* P, int tt, Variant* vout, Kernel* kout) {
  Variant v = P->var;
  v.tt = tt;
  v.reg_lo = v.reg_hi = 0;   // remainder launches are rare: no register split
  {
    // the aligned-window geometry needs a 16-byte aligned TMA box start (tt * XLO
    // elements); a remainder depth may not keep it (e.g. T = 4, remainder 3)
    const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
    const int aln = std::max(16 / elem, v.vx);
    if (tt < 2 || (tt * P->pat.xlo) % aln != 0) v.xshift = false;
  }
  if (v.family == FAM_STREAM_TB && tt == 1) v.family = FAM_STREAM;   // remainder of one step: plain ST
  const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
  if (v.family == FAM_STREAM_TB && v.rt) {
    v.ws_threads = v.tbrt_threads(P->pat, elem);
    if (v.ws_threads > 1024) SM_FAIL(STENCIL_E_OC_INFEASIBLE, "TB remainder CTA of %d threads", v.ws_threads);
  }
  if ((v.family == FAM_TILED || v.family == FAM_STREAM_TB) && v.tma) {
    const TmaBox b = tma_box(v, P->pat, elem);
    v.tma = b.lx <= 256 && b.ly <= 256 && b.lz <= 256;
  }
  *vout = v;
  auto it = P->tb_rem.find(tt);
  if (it != P->tb_rem.end()) { *kout = it->second; return STENCIL_OK; }
  std::string low;
  std::vector<char> bin;
  SM_TRY(compile_variant(P->pat, P->dtype, v, &low, &bin));
  Kernel k;
  SM_TRY(load_kernel(generate_source(P->pat, P->dtype, v), bin, low, v.smem_bytes(P->pat, elem), &k));
  if (!v.regsplit_fits(P->pat, elem, k.regs))
    SM_FAIL(STENCIL_E_OC_INFEASIBLE, "register split %d/%d does not fit %d regs/thread", v.reg_lo, v.reg_hi,
            k.regs);
  P->tb_rem[tt] = k;
  *kout = k;
  return STENCIL_OK;
}

int run_device(stencil_plan_s* P, const void* in, void* out, int steps);

// Compile and load every kernel a run of this plan can launch (the main one and
// the TB remainder kernels of depth 1..T-1, and the AOT frame-copy / flag
// kernels, which CUDA loads lazily at first launch) now. P2P registration calls it:
// several slab plans of ONE process (one GPU) enqueue spin-waiting flag kernels
// on their streams, and a module load inside a later plan's first run could then
// wait on the context behind a spin that only that run would release (seen as a
// hang of two in-process slabs whose kernels had not been loaded before).
int preload_kernels(stencil_plan_s* P) {
  SM_TRY(preload_aot_kernels());
  SM_TRY(ensure_loaded(P));
  const int T = P->var.family == FAM_TILED || P->var.family == FAM_STREAM_TB ? P->var.tt : 1;
  for (int tl = 1; tl < T; ++tl) {
    Variant v;
    Kernel k;
    SM_TRY(get_tb_rem_kernel(P, tl, &v, &k));
  }
  return STENCIL_OK;
}

}  // namespace smart_rt

using namespace smart_rt;

stencil_plan_s::~stencil_plan_s() {
  for (cudaEvent_t e : ev_pool) cudaEventDestroy(e);
  for (cudaEvent_t e : h2d_ev) cudaEventDestroy(e);
  for (cudaEvent_t e : cmp_ev) cudaEventDestroy(e);
  if (h2d_stream) cudaStreamDestroy(h2d_stream);
  if (d2h_stream) cudaStreamDestroy(d2h_stream);
  if (h_in_dev) cudaFree(h_in_dev);
  if (h_out_dev) cudaFree(h_out_dev);
  if (h_ws_dev) cudaFree(h_ws_dev);
  if (g_exec) cudaGraphExecDestroy(g_exec);
  if (g_stream) cudaStreamDestroy(g_stream);
  if (comm) comm_destroy(comm);
}

namespace smart_rt {

// Halo exchange into buffer bufs[k] of every local plan k (a7). NCCL: the
// plan's comm stream waits for the edge planes, then grouped send/recv with
// ranks +-1. LOOPBACK: each slab pulls its ghost planes from its neighbours'
// buffers with cudaMemcpyAsync after their edge planes are written.
static int exchange(const std::vector<stencil_plan_s*>& Ps, const std::vector<void*>& bufs, int tl) {
  for (size_t k = 0; k < Ps.size(); ++k) {
    stencil_plan_s* P = Ps[k];
    Comm* c = P->comm;
    if (c->transport == TR_NCCL) {
      SM_CUDA(cudaStreamWaitEvent(c->stream, c->ev_edge, 0));
      SM_TRY(comm_exchange_nccl(P, bufs[k], tl));
    } else {
      const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
      const size_t pb = (size_t)P->vdims[1] * P->vdims[2] * elem;
      int64_t h[8];
      slab_halo(P->ghost, (int)P->dims[0], tl * P->pat.zlo, tl * P->pat.zhi, c->rank, c->nranks, h);
      SM_CUDA(cudaStreamWaitEvent(c->stream, c->ev_edge, 0));
      if (h[1]) {   // lower ghosts <- rank-1's last zlo_g owned planes
        stencil_plan_s* Q = c->peers[c->rank - 1];
        int64_t hq[8];
        slab_halo(Q->ghost, (int)Q->dims[0], tl * Q->pat.zlo, tl * Q->pat.zhi, c->rank - 1, c->nranks, hq);
        SM_CUDA(cudaStreamWaitEvent(c->stream, Q->comm->ev_edge, 0));
        SM_CUDA(cudaMemcpyAsync((char*)bufs[k] + h[0] * pb, (const char*)bufs[k - 1] + hq[4] * pb, h[1] * pb,
                                cudaMemcpyDeviceToDevice, c->stream));
      }
      if (h[7]) {   // upper ghosts <- rank+1's first zhi_g owned planes
        stencil_plan_s* Q = c->peers[c->rank + 1];
        int64_t hq[8];
        slab_halo(Q->ghost, (int)Q->dims[0], tl * Q->pat.zlo, tl * Q->pat.zhi, c->rank + 1, c->nranks, hq);
        SM_CUDA(cudaStreamWaitEvent(c->stream, Q->comm->ev_edge, 0));
        SM_CUDA(cudaMemcpyAsync((char*)bufs[k] + h[6] * pb, (const char*)bufs[k + 1] + hq[2] * pb, h[7] * pb,
                                cudaMemcpyDeviceToDevice, c->stream));
      }
    }
    SM_CUDA(cudaEventRecord(c->ev_comm, c->stream));
  }
  return STENCIL_OK;
}

// main stream of plan k waits for the exchange that filled its ghosts and,
// for LOOPBACK, for its neighbours' copies out of its buffer
static int wait_exchange(const std::vector<stencil_plan_s*>& Ps) {
  for (stencil_plan_s* P : Ps) {
    Comm* c = P->comm;
    SM_CUDA(cudaStreamWaitEvent(P->stream, c->ev_comm, 0));
    if (c->transport == TR_LOOPBACK) {
      if (c->rank > 0) SM_CUDA(cudaStreamWaitEvent(P->stream, c->peers[c->rank - 1]->comm->ev_comm, 0));
      if (c->rank < c->nranks - 1) SM_CUDA(cudaStreamWaitEvent(P->stream, c->peers[c->rank + 1]->comm->ev_comm, 0));
    }
  }
  return STENCIL_OK;
}

// The time loop (a6) over a group of local plans: one plan on one GPU, one
// slab per process (NCCL), or all slabs of a LOOPBACK group. With slabs, each
// launch computes the edge planes first, starts the halo exchange of those
// planes on the comm stream and computes the interior meanwhile (a7).
static int run_group(const std::vector<stencil_plan_s*>& Ps, const std::vector<const void*>& ins,
                     const std::vector<void*>& outs, int steps) {
  const size_t np = Ps.size();
  stencil_plan_s* P0 = Ps[0];
  const bool slab = P0->comm != nullptr;
  for (size_t k = 0; k < np; ++k) {
    stencil_plan_s* P = Ps[k];
    if (!ins[k] || !outs[k]) SM_FAIL(STENCIL_E_INVAL, "null grid pointer");
    if (ins[k] == outs[k]) SM_FAIL(STENCIL_E_INVAL, "in and out must be distinct buffers");
    if ((uintptr_t)ins[k] % 16 || (uintptr_t)outs[k] % 16)
      SM_FAIL(STENCIL_E_INVAL, "grid pointers must be 16-byte aligned");
    if (P->var.tt != P0->var.tt || P->var.family != P0->var.family)
      SM_FAIL(STENCIL_E_INVAL, "plans of a group must use the same OC setting");
  }
  if (steps < 0) SM_FAIL(STENCIL_E_INVAL, "steps must be >= 0");
  if (steps == 0) {
    for (size_t k = 0; k < np; ++k) {
      const int elem = Ps[k]->dtype == STENCIL_F64 ? 8 : 4;
      const size_t bytes = (size_t)Ps[k]->vdims[0] * Ps[k]->vdims[1] * Ps[k]->vdims[2] * elem;
      SM_CUDA(cudaMemcpyAsync(outs[k], ins[k], bytes, cudaMemcpyDeviceToDevice, Ps[k]->stream));
    }
    return STENCIL_OK;
  }
  const int T = P0->var.family == FAM_TILED || P0->var.family == FAM_STREAM_TB ? P0->var.tt : 1;
  const int launches = (steps + T - 1) / T;
  const bool p2p = slab && P0->comm->transport == TR_P2P;
  std::vector<GridArg> gs(np);
  for (size_t k = 0; k < np; ++k) {
    stencil_plan_s* P = Ps[k];
    const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
    const size_t bytes = (size_t)P->vdims[0] * P->vdims[1] * P->vdims[2] * elem;
    if (launches >= 2 && (!P->ws || P->ws_bytes < bytes))
      SM_FAIL(STENCIL_E_STATE, "steps=%d needs a workspace of %zu bytes (stencil_plan_set_workspace)", steps, bytes);
    if (p2p) {
      const Comm* c = P->comm;
      if (c->transport != TR_P2P || ins[k] != c->self.in || outs[k] != c->self.out ||
          (launches >= 2 && P->ws != c->self.ws))
        SM_FAIL(STENCIL_E_STATE, "P2P slab plans run on their registered in/out/workspace buffers");
    }
    SM_TRY(ensure_loaded(P));
    gs[k] = make_grid(P, P->var.vx);
    if (p2p) continue;   // frame copy after the initial halo (below)
    // a4: frame of the input into every buffer the sweep writes (fixed thereafter)
    SM_TRY(launch_frame_copy(ins[k], outs[k], elem, gs[k], P->stream));
    if (launches >= 2) SM_TRY(launch_frame_copy(ins[k], P->ws, elem, gs[k], P->stream));
  }
  if (p2p) {
    // initial ghosts of `in`: push my edge planes into the neighbours' `in`
    // ghosts (whole planes, peer memory), publish, await theirs; then the
    // frame copy (ghost planes included) reads complete planes
    const int tl0 = std::min(T, steps);
    for (size_t k = 0; k < np; ++k) {
      stencil_plan_s* P = Ps[k];
      Comm* c = P->comm;
      const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
      const size_t pb = (size_t)P->vdims[1] * P->vdims[2] * elem;
      const int G = P->ghost, n = (int)P->dims[0];
      const int up = tl0 * P->pat.zhi, down = tl0 * P->pat.zlo;
      if (c->has_lo && up)
        SM_CUDA(cudaMemcpyAsync((char*)c->lo.in + (G + c->lo.owned_planes) * pb, (const char*)ins[k] + G * pb,
                                up * pb, cudaMemcpyDeviceToDevice, P->stream));
      if (c->has_hi && down)
        SM_CUDA(cudaMemcpyAsync((char*)c->hi.in + (G - down) * pb, (const char*)ins[k] + (G + n - down) * pb,
                                down * pb, cudaMemcpyDeviceToDevice, P->stream));
      SM_TRY(launch_p2p_signal(c->has_lo ? c->lo.flags + 1 : nullptr, c->has_hi ? c->hi.flags : nullptr,
                               c->self.flags + 2, P->stream));
      SM_TRY(launch_p2p_wait(c->has_lo ? c->self.flags : nullptr, c->has_hi ? c->self.flags + 1 : nullptr,
                             c->self.flags + 2, P->stream));
      SM_TRY(launch_frame_copy(ins[k], outs[k], elem, gs[k], P->stream));
      if (launches >= 2) SM_TRY(launch_frame_copy(ins[k], P->ws, elem, gs[k], P->stream));
    }
  } else if (slab) {   // ghosts of the input: neighbours' current owned planes
    std::vector<void*> b(np);
    for (size_t k = 0; k < np; ++k) {
      b[k] = const_cast<void*>(ins[k]);
      SM_CUDA(cudaEventRecord(Ps[k]->comm->ev_edge, Ps[k]->stream));
    }
    SM_TRY(exchange(Ps, b, std::min(T, steps)));
    SM_TRY(wait_exchange(Ps));
  }
  std::vector<const void*> src(ins);
  std::vector<void*> dst(np);
  for (int i = 0; i < launches; ++i) {
    const int tl = std::min(T, steps - i * T);
    const bool more = i + 1 < launches;
    const int tl_next = more ? std::min(T, steps - (i + 1) * T) : 0;
    for (size_t k = 0; k < np; ++k) dst[k] = ((launches - 1 - i) % 2 == 0) ? outs[k] : Ps[k]->ws;
    std::vector<Variant> vs(np);
    std::vector<Kernel> ks(np);
    for (size_t k = 0; k < np; ++k) {
      if (tl == T) { vs[k] = Ps[k]->var; ks[k] = Ps[k]->kern; }
      else SM_TRY(get_tb_rem_kernel(Ps[k], tl, &vs[k], &ks[k]));
    }
    if (p2p && more) {
      // fused halo: edge kernels also store the planes the neighbours need
      // into their ghost planes (same parity buffer), publish, compute the
      // interior, then await the neighbours before the next launch
      // edge depth: the planes the neighbours need next (tl_next steps) and
      // at least what this launch's interior would otherwise read from the
      // ghost planes (tl steps) -- those ghosts belong to the buffer the
      // neighbours' next edge launches overwrite once they have our signal
      const int E = std::max(tl, tl_next) * std::max(P0->pat.zlo, P0->pat.zhi);
      const bool to_out = (launches - 1 - i) % 2 == 0;
      for (size_t k = 0; k < np; ++k) {
        stencil_plan_s* P = Ps[k];
        Comm* c = P->comm;
        const int G = P->ghost, n = (int)P->dims[0];
        GridArg g = gs[k];
        if (c->has_lo) {
          g.peer_lo = (long long)(uintptr_t)(to_out ? c->lo.out : c->lo.ws);
          g.mlo0 = G; g.mlo1 = G + tl_next * P->pat.zhi; g.shift_lo = (int)c->lo.owned_planes;
        }
        if (c->has_hi) {
          g.peer_hi = (long long)(uintptr_t)(to_out ? c->hi.out : c->hi.ws);
          g.mhi0 = G + n - tl_next * P->pat.zlo; g.mhi1 = G + n; g.shift_hi = -n;
        }
        const int c0 = g.cz0, c1 = g.cz1;
        if (c1 - c0 > 2 * E) {
          g.cz1 = c0 + E;
          SM_TRY(launch_sweep(P, vs[k], ks[k], src[k], dst[k], g));
          g.cz0 = c1 - E; g.cz1 = c1;
          SM_TRY(launch_sweep(P, vs[k], ks[k], src[k], dst[k], g));
        } else {
          SM_TRY(launch_sweep(P, vs[k], ks[k], src[k], dst[k], g));
        }
        SM_TRY(launch_p2p_signal(c->has_lo ? c->lo.flags + 1 : nullptr, c->has_hi ? c->hi.flags : nullptr,
                                 c->self.flags + 2, P->stream));
        GridArg gi = gs[k];
        if (gi.cz1 - gi.cz0 > 2 * E) {
          gi.cz0 += E; gi.cz1 -= E;
          SM_TRY(launch_sweep(P, vs[k], ks[k], src[k], dst[k], gi));
        }
        SM_TRY(launch_p2p_wait(c->has_lo ? c->self.flags : nullptr, c->has_hi ? c->self.flags + 1 : nullptr,
                               c->self.flags + 2, P->stream));
      }
    } else if (slab && more) {
      // The edge planes (the ones the neighbours need next) run on a
      // high-priority stream concurrently with the interior: they start once
      // the main stream has finished the previous launch (its interior read
      // the planes they overwrite) and the previous exchange (main waited for
      // it); the interior of this launch needs neither of them, and the next
      // launch sees them through the exchange event.
      const int E = tl_next * std::max(P0->pat.zlo, P0->pat.zhi);
      for (size_t k = 0; k < np; ++k) {   // edge planes first
        stencil_plan_s* P = Ps[k];
        Comm* c = P->comm;
        GridArg g = gs[k];
        const int c0 = g.cz0, c1 = g.cz1;
        cudaStream_t main_stream = P->stream;
        const char* ser = getenv("STENCIL_EDGE_SERIAL");   // dev override: edges on the main stream
        cudaStream_t es = (ser && atoi(ser)) ? main_stream : c->edge_stream;
        SM_CUDA(cudaEventRecord(c->ev_main, main_stream));
        SM_CUDA(cudaStreamWaitEvent(es, c->ev_main, 0));
        P->stream = es;
        int rc = STENCIL_OK;
        if (c1 - c0 > 2 * E) {
          g.cz1 = c0 + E;
          rc = launch_sweep(P, vs[k], ks[k], src[k], dst[k], g);
          g.cz0 = c1 - E; g.cz1 = c1;
          if (rc == STENCIL_OK) rc = launch_sweep(P, vs[k], ks[k], src[k], dst[k], g);
        } else {
          rc = launch_sweep(P, vs[k], ks[k], src[k], dst[k], g);
        }
        P->stream = main_stream;
        if (rc != STENCIL_OK) return rc;
        SM_CUDA(cudaEventRecord(c->ev_edge, es));
        if (c1 - c0 <= 2 * E) SM_CUDA(cudaStreamWaitEvent(main_stream, c->ev_edge, 0));   // no interior
      }
      SM_TRY(exchange(Ps, dst, tl_next));
      for (size_t k = 0; k < np; ++k) {   // interior overlaps the exchange
        GridArg g = gs[k];
        if (g.cz1 - g.cz0 > 2 * E) {
          g.cz0 += E; g.cz1 -= E;
          SM_TRY(launch_sweep(Ps[k], vs[k], ks[k], src[k], dst[k], g));
        }
      }
      SM_TRY(wait_exchange(Ps));
    } else {
      for (size_t k = 0; k < np; ++k) SM_TRY(launch_sweep(Ps[k], vs[k], ks[k], src[k], dst[k], gs[k]));
    }
    for (size_t k = 0; k < np; ++k) src[k] = dst[k];
  }
  SM_CUDA(cudaGetLastError());
  return STENCIL_OK;
}

// End to end with host buffers, pipelined over z-chunks (views with enough
// planes, no slab). Chunk k's input planes [Z_{k-1}, Z_k) go up on a copy
// stream; then, on the plan's stream, launch i of the time loop (fusing up to
// T steps) computes the planes it can now reach, [Z_{k-1} - sk_i, Z_k - sk_i)
// with the skew sk_i = (i+1)*T*E (E = max z extent; the first chunk starts at
// 0, the last runs to the top) -- a time-skewed wavefront that computes every
// (launch, plane) exactly once -- and the planes that became final,
// [Z_{k-1} - sk_last, Z_k - sk_last), go down on a second copy stream. The
// H2D of chunk k+1, the sweep of chunk k and the D2H of chunk k-1 overlap
// (PCIe is full duplex) instead of running back to back.
// Correctness: launch i reads the buffer of launch i-1 on
// [lo - t_i*zlo, hi + t_i*zhi); its top is <= Z_k - sk_{i-1}, already computed;
// its bottom is >= Z_{k-1} - sk_i - T*E = Z_{k-1} - sk_{i+1}, at or above
// everything an earlier chunk's launch i+1 wrote into that same-parity buffer,
// so nothing it needs was overwritten; final planes below Z_k - sk_last are
// never written again (later chunks write above Z_k - sk_i >= Z_k - sk_last);
// frame points are time-invariant. Same kernels and per-point order as
// stencil_run: bitwise equal results. *done = false: the plan does not qualify.
static int run_host_pipelined(stencil_plan_s* P, const void* hin, void* hout, int steps, bool* done) {
  *done = false;
  // chunk axis: the slowest view axis, or y for the 2-D tiled/naive views [1][ny][nx]
  const bool yax = P->vdims[0] == 1;
  const int nz = (int)(yax ? P->vdims[1] : P->vdims[0]);
  const int E = yax ? std::max(P->pat.ylo, P->pat.yhi) : std::max(P->pat.zlo, P->pat.zhi);
  if (P->comm || steps < 1 || P->timing || nz < 64) return STENCIL_OK;
  const int T = P->var.family == FAM_TILED || P->var.family == FAM_STREAM_TB ? P->var.tt : 1;
  const int launches = (steps + T - 1) / T;
  const long long skew = (long long)launches * T * E;
  // up to 16 chunks (shorter fill and drain) of >= 32 planes and more than
  // twice the skew (the wavefront must stay well inside a chunk)
  const int K = (int)std::min<long long>(16, nz / std::max<long long>(32, 2 * skew + 1));
  if (K < 2) return STENCIL_OK;
  const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
  const size_t pb = (yax ? (size_t)P->vdims[2] : (size_t)P->vdims[1] * P->vdims[2]) * elem;   // bytes per plane / row
  // small grids: ~3 copies/launches of ~10 us per chunk outweigh the overlap
  // (C1 256^2 fp64: 0.10 ms unpipelined, 0.48 ms in 8 chunks); the pipeline
  // pays from tens of MB (copy time ~ bytes / 50 GB/s). Dev override for tests.
  const char* mb = getenv("STENCIL_PIPELINE_MIN_BYTES");
  const size_t min_bytes = mb ? (size_t)atoll(mb) : ((size_t)32 << 20);
  if (pb * (size_t)nz < min_bytes) return STENCIL_OK;
  SM_TRY(ensure_loaded(P));
  char* din = (char*)P->h_in_dev;
  char* dout = (char*)P->h_out_dev;
  char* dws = (char*)P->ws;
  if (!P->h2d_stream) SM_CUDA(cudaStreamCreateWithFlags(&P->h2d_stream, cudaStreamNonBlocking));
  if (!P->d2h_stream) SM_CUDA(cudaStreamCreateWithFlags(&P->d2h_stream, cudaStreamNonBlocking));
  while ((int)P->h2d_ev.size() < K) {
    cudaEvent_t a, b;
    SM_CUDA(cudaEventCreateWithFlags(&a, cudaEventDisableTiming));
    SM_CUDA(cudaEventCreateWithFlags(&b, cudaEventDisableTiming));
    P->h2d_ev.push_back(a);
    P->cmp_ev.push_back(b);
  }
  // On an error return, copies already queued still read / write the caller's
  // host buffers: drain every stream before handing control back.
  struct Drain {
    stencil_plan_s* P;
    bool armed = true;
    ~Drain() {
      if (!armed) return;
      cudaStreamSynchronize(P->h2d_stream);
      cudaStreamSynchronize(P->d2h_stream);
      cudaStreamSynchronize(P->stream);
    }
  } drain{P};
  // the copy streams start after everything queued on the plan's stream
  SM_CUDA(cudaEventRecord(P->cmp_ev[0], P->stream));
  SM_CUDA(cudaStreamWaitEvent(P->h2d_stream, P->cmp_ev[0], 0));
  SM_CUDA(cudaStreamWaitEvent(P->d2h_stream, P->cmp_ev[0], 0));
  const GridArg g = make_grid(P, P->var.vx);
  const int gc0 = yax ? g.cy0 : g.cz0, gc1 = yax ? g.cy1 : g.cz1;   // compute box along the chunk axis
  std::vector<Variant> vs(launches);
  std::vector<Kernel> ks(launches);
  for (int i = 0; i < launches; ++i) {
    const int tl = std::min(T, steps - i * T);
    if (tl == T) { vs[i] = P->var; ks[i] = P->kern; }
    else SM_TRY(get_tb_rem_kernel(P, tl, &vs[i], &ks[i]));
  }
  int d_done = 0;   // planes already sent down
  for (int k = 0; k < K; ++k) {
    const int z0 = (int)((long long)nz * k / K), z1 = (int)((long long)nz * (k + 1) / K);
    SM_CUDA(cudaMemcpyAsync(din + z0 * pb, (const char*)hin + z0 * pb, (z1 - z0) * pb, cudaMemcpyHostToDevice,
                            P->h2d_stream));
    SM_CUDA(cudaEventRecord(P->h2d_ev[k], P->h2d_stream));
    SM_CUDA(cudaStreamWaitEvent(P->stream, P->h2d_ev[k], 0));
    // a4 for these planes: the frame into every buffer the sweep writes
    GridArg gf = g;
    if (yax) {
      gf.ny = z1 - z0;
      gf.uy0 = std::min(std::max(g.uy0 - z0, 0), gf.ny);
      gf.uy1 = std::min(std::max(g.uy1 - z0, gf.uy0), gf.ny);
    } else {
      gf.nz = z1 - z0;
      gf.uz0 = std::min(std::max(g.uz0 - z0, 0), gf.nz);
      gf.uz1 = std::min(std::max(g.uz1 - z0, gf.uz0), gf.nz);
    }
    SM_TRY(launch_frame_copy(din + z0 * pb, dout + z0 * pb, elem, gf, P->stream));
    if (launches >= 2) SM_TRY(launch_frame_copy(din + z0 * pb, dws + z0 * pb, elem, gf, P->stream));
    const void* src = din;
    for (int i = 0; i < launches; ++i) {
      const int sk = (i + 1) * T * E;
      char* dst = ((launches - 1 - i) % 2 == 0) ? dout : dws;
      const int lo = std::max(gc0, k == 0 ? 0 : z0 - sk);
      const int hi = std::min(gc1, k == K - 1 ? nz : z1 - sk);
      if (hi > lo) {
        GridArg gl = g;
        if (yax) { gl.cy0 = lo; gl.cy1 = hi; } else { gl.cz0 = lo; gl.cz1 = hi; }
        SM_TRY(launch_sweep(P, vs[i], ks[i], src, dst, gl));
      }
      src = dst;
    }
    SM_CUDA(cudaEventRecord(P->cmp_ev[k], P->stream));
    const int d1 = k == K - 1 ? nz : std::max(d_done, (int)(z1 - skew));
    if (d1 > d_done) {
      SM_CUDA(cudaStreamWaitEvent(P->d2h_stream, P->cmp_ev[k], 0));
      SM_CUDA(cudaMemcpyAsync((char*)hout + d_done * pb, dout + d_done * pb, (d1 - d_done) * pb,
                              cudaMemcpyDeviceToHost, P->d2h_stream));
      d_done = d1;
    }
  }
  SM_CUDA(cudaGetLastError());
  SM_CUDA(cudaStreamSynchronize(P->d2h_stream));
  SM_CUDA(cudaStreamSynchronize(P->stream));
  drain.armed = false;
  P->host_chunks = K;
  *done = true;
  return STENCIL_OK;
}

void free_host_path_buffers(stencil_plan_s* P) {
  if (P->h_in_dev || P->h_out_dev || P->h_ws_dev) cudaDeviceSynchronize();   // no copy may still use them
  if (P->h_in_dev) cudaFree(P->h_in_dev);
  if (P->h_out_dev) cudaFree(P->h_out_dev);
  if (P->h_ws_dev) cudaFree(P->h_ws_dev);
  P->h_in_dev = P->h_out_dev = P->h_ws_dev = nullptr;
  P->h_bytes = 0;
}

// One stencil_run. Single-domain plans replay a CUDA graph of the run's launch
// sequence (frame copies, the ceil(steps/T) sweeps, TB remainder) once the same
// (in, out, workspace, steps) comes a second time: the first call runs eagerly
// (module loads, tensor maps), the second is captured on the plan's own stream
// and launched, later ones only launch the graph. Small grids are launch-bound
// (C1, 256^2: 12 launches of a few us each per run). Not used with kernel timing
// (per-launch events) or slabs (exchanges on other streams); opt-in (below).
// Off by default: measured on C1 (256^2, 10 steps, same box, twice each) the
// end-to-end step took 0.121-0.139 ms with graph replay against 0.107-0.111 ms
// with direct launches. STENCIL_GRAPHS=1 turns it on.
static bool graphs_enabled() {
  const char* e = getenv("STENCIL_GRAPHS");
  return e && atoi(e) != 0;
}

static void drop_graph(stencil_plan_s* P) {
  if (P->g_exec) cudaGraphExecDestroy(P->g_exec);
  P->g_exec = nullptr;
}

int run_device(stencil_plan_s* P, const void* in, void* out, int steps) {
  if (P->comm && P->comm->transport == TR_LOOPBACK)
    SM_FAIL(STENCIL_E_STATE, "a loopback slab runs with its group (stencil_run_group)");
  if (P->comm || P->timing || steps < 1 || !graphs_enabled()) return run_group({P}, {in}, {out}, steps);
  const bool same = P->g_in == in && P->g_out == out && P->g_ws == P->ws && P->g_steps == steps;
  if (same && P->g_exec) {
    SM_CUDA(cudaGraphLaunch(P->g_exec, P->stream));
    g_launches.fetch_add(P->g_nlaunch);
    return STENCIL_OK;
  }
  if (!same) {
    drop_graph(P);
    P->g_in = in; P->g_out = out; P->g_ws = P->ws; P->g_steps = steps; P->g_calls = 0;
  }
  if (++P->g_calls < 2) return run_group({P}, {in}, {out}, steps);
  if (!P->g_stream) SM_CUDA(cudaStreamCreateWithFlags(&P->g_stream, cudaStreamNonBlocking));
  cudaStream_t s0 = P->stream;
  SM_CUDA(cudaStreamBeginCapture(P->g_stream, cudaStreamCaptureModeThreadLocal));
  P->stream = P->g_stream;
  const uint64_t l0 = g_launches.load();
  int rc = run_group({P}, {in}, {out}, steps);
  P->stream = s0;
  cudaGraph_t graph = nullptr;
  const cudaError_t ce = cudaStreamEndCapture(P->g_stream, &graph);
  const uint64_t n = g_launches.load() - l0;
  g_launches.fetch_sub(n);                         // counted when the graph runs
  cudaError_t ie = cudaErrorUnknown;
  if (rc == STENCIL_OK && ce == cudaSuccess && graph) ie = cudaGraphInstantiate(&P->g_exec, graph, 0);
  if (graph) cudaGraphDestroy(graph);
  if (rc != STENCIL_OK || ce != cudaSuccess || ie != cudaSuccess) {
    (void)cudaGetLastError();
    P->g_exec = nullptr;
    P->g_calls = INT32_MIN;                        // no graph for this key; run eagerly
    if (rc != STENCIL_OK) return rc;
    return run_group({P}, {in}, {out}, steps);
  }
  P->g_nlaunch = n;
  SM_CUDA(cudaGraphLaunch(P->g_exec, P->stream));
  g_launches.fetch_add(n);
  return STENCIL_OK;
}

}  // namespace smart_rt

// =====================================================================
// C ABI
// =====================================================================
extern "C" {

const char* stencil_last_error(void) { return t_err.c_str(); }
uint64_t stencil_launch_count(void) { return g_launches.load(); }
int stencil_abi_version(void) { return STENCIL_ABI_VERSION; }

int stencil_oc_valid(uint32_t oc) { return oc_valid(oc) ? 1 : 0; }

int stencil_oc_list(uint32_t* ids) {
  int n = 0;
  for (uint32_t m = 0; m < 64; ++m)
    if (oc_valid(m)) {
      if (ids) ids[n] = m;
      ++n;
    }
  return n;
}

const char* stencil_oc_name(uint32_t oc) { return oc_name_static(oc); }

int stencil_sample_params(uint32_t oc, int ndim, stencil_dtype_t dtype, uint64_t seed, int k,
                          stencil_params_t* out) {
  clear_error();
  if (!out) SM_FAIL(STENCIL_E_INVAL, "null output");
  if (!oc_valid(oc)) SM_FAIL(STENCIL_E_OC_INVALID, "OC %u violates Table I", oc);
  if (ndim != 2 && ndim != 3) SM_FAIL(STENCIL_E_INVAL, "ndim must be 2 or 3");
  if (dtype != STENCIL_F32 && dtype != STENCIL_F64) SM_FAIL(STENCIL_E_INVAL, "bad dtype");
  sample_params(oc, ndim, dtype, seed, k, out);
  return STENCIL_OK;
}

int stencil_plan_create(stencil_plan_t* plan, int ndim, const int64_t* dims, int order, const uint8_t* access,
                        const double* coeffs, stencil_dtype_t dtype, uint32_t oc, const stencil_params_t* params) {
  clear_error();
  if (!plan) SM_FAIL(STENCIL_E_INVAL, "null plan pointer");
  *plan = nullptr;
  if (ndim != 2 && ndim != 3) SM_FAIL(STENCIL_E_INVAL, "ndim must be 2 or 3 (got %d)", ndim);
  if (order < 1 || order > 4) SM_FAIL(STENCIL_E_INVAL, "order must be in 1..4 (got %d)", order);
  if (!dims || !access || !coeffs) SM_FAIL(STENCIL_E_INVAL, "null dims/access/coeffs");
  if (dtype != STENCIL_F32 && dtype != STENCIL_F64) SM_FAIL(STENCIL_E_INVAL, "unknown dtype %d", (int)dtype);
  for (int k = 0; k < ndim; ++k) {
    if (dims[k] < 2 * order + 1)
      SM_FAIL(STENCIL_E_INVAL, "dims[%d]=%lld < 2*order+1=%d", k, (long long)dims[k], 2 * order + 1);
    if (dims[k] > (1LL << 30)) SM_FAIL(STENCIL_E_INVAL, "dims[%d] too large", k);
  }
  {
    long long vol = 1;
    for (int k = 0; k < ndim; ++k) vol *= dims[k];
    if (vol > (1LL << 36)) SM_FAIL(STENCIL_E_INVAL, "grid too large");
  }
  const int w = 2 * order + 1;
  const int tsize = ndim == 3 ? w * w * w : w * w;
  const int centre = tsize / 2;
  if (access[centre] != 1) SM_FAIL(STENCIL_E_INVAL, "the centre of the access tensor must be 1 (P:L135)");
  for (int t = 0; t < tsize; ++t) {
    if (access[t] > 1) SM_FAIL(STENCIL_E_INVAL, "access tensor must be binary (entry %d = %d)", t, access[t]);
    if (!access[t] && coeffs[t] != 0.0)
      SM_FAIL(STENCIL_E_INVAL, "coefficient %d is nonzero where access == 0", t);
    if (!std::isfinite(coeffs[t])) SM_FAIL(STENCIL_E_INVAL, "coefficient %d is not finite", t);
  }
  if (!oc_valid(oc)) SM_FAIL(STENCIL_E_OC_INVALID, "OC %u violates Table I (BM xor CM; RT, PR need ST)", oc);
  if (params) SM_TRY(validate_params(params));

  std::unique_ptr<stencil_plan_s> P(new stencil_plan_s());
  P->ndim = ndim;
  for (int k = 0; k < ndim; ++k) P->dims[k] = dims[k];
  P->order = order;
  P->dtype = dtype;
  P->oc = oc;
  P->access.assign(access, access + tsize);
  P->coeffs.assign(coeffs, coeffs + tsize);
  default_params(oc, ndim, dtype, &P->params);
  merge_params(params, &P->params);
  // parameters an OC does not have are reported at their neutral value
  if (!(oc & (STENCIL_OC_BM | STENCIL_OC_CM))) P->params.merge = 1;
  if (!(oc & STENCIL_OC_TB)) P->params.tb_steps = 1;
  if (!(oc & STENCIL_OC_PR)) P->params.pr_stages = 1;
  SM_TRY(build_pattern(P.get()));
  build_view(P.get(), family_of(oc, P->params.smem));
  // Default tiles shrink until the shared-memory footprint fits (high-order
  // stencils under TB need smaller tiles); user-given fields are kept.
  const bool user_bz = params && params->bz, user_by = params && params->by, user_bx = params && params->bx;
  // single-step 3-D streaming of an HBM-bound stencil with a tall y extent:
  // taller tiles, the 2*r halo rows each tile re-reads per plane would otherwise be
  // 2x its own rows (measured on C3, star25 r = 4, 768^3 fp32: ST_BM_RT_PR 454 ->
  // 600 GStencil/s, ST_CM_RT_PR 435 -> 614). FMA-bound stencils (>= 48 FMAs per
  // point) keep by 2: order-4 random 1024^3 fp64 54.2 (by 2) vs 50.1 (by 4).
  if (!user_by && ndim == 3 && family_of(oc, P->params.smem) == FAM_STREAM &&
      P->pat.ylo + P->pat.yhi >= 6 && P->pat.nnz < 48 && P->params.by < 4)
    P->params.by = 4;
  if (!user_bx && family_of(oc, P->params.smem) != FAM_NAIVE) {
    // keep the default halo tile within one TMA box (<= 256 elements per row)
    const int elem = dtype == STENCIL_F64 ? 8 : 4;
    for (;;) {
      Variant v;
      v.family = family_of(oc, P->params.smem);
      v.bx = P->params.bx; v.by = P->params.by; v.bz = P->params.bz; v.vx = P->params.vx;
      v.m = P->params.merge; v.tt = (oc & STENCIL_OC_TB) ? P->params.tb_steps : 1;
      if (tma_box(v, P->pat, elem).lx <= 256 || P->params.bx <= 8 * P->params.vx) break;
      P->params.bx /= 2;
    }
  }
  // TB-RT with block merging on a radius-1 in-plane star (C2's heat; the
  // scalar-column stage tiles of resolve_variant): 8-row last-stage tiles, 64 x
  // 32 outputs per CTA as before but 4 last-stage warps instead of 8 and 2.25
  // instead of 2.5 shared loads per output (round 2)
  const bool user_m = params && params->merge;
  bool try_m8 = !user_by && !user_m && ndim == 3 && family_of(oc, P->params.smem) == FAM_STREAM_TB &&
                (oc & STENCIL_OC_RT) && (oc & STENCIL_OC_BM) && dtype == STENCIL_F64 && P->params.by == 8 &&
                P->params.merge == 4;
  std::string first_err;   // the reason at the requested (or default) setting
  for (int attempt = 0;; ++attempt) {
    const int rc = resolve_variant(P.get());
    if (rc == STENCIL_E_OC_INFEASIBLE && first_err.empty()) first_err = t_err;
    const bool give_up = [&] {
      if (rc != STENCIL_E_OC_INFEASIBLE || attempt > 12) return true;
      stencil_params_t& q = P->params;
      if (!user_bz && q.bz > 1) q.bz /= 2;
      else if (!user_by && q.by > 1 && (q.bx / std::max(q.vx, 1)) * (q.by / 2) >= 32) q.by /= 2;
      else if (!user_bx && q.bx > 8 * q.vx) q.bx /= 2;
      else return true;
      return false;
    }();
    if (!give_up) continue;
    if (rc == STENCIL_E_OC_INFEASIBLE) SM_FAIL(rc, "%s (no smaller default tile fits either)", first_err.c_str());
    if (rc != STENCIL_OK) return rc;
    if (try_m8) {
      try_m8 = false;
      const char* nm = getenv("STENCIL_NO_M8");   // dev override (A/B against the round-1 setting)
      if (P->var.midvx == 1 && !P->var.xshift && !(nm && atoi(nm))) {
        const stencil_params_t keep = P->params;
        P->params.by = 4;
        P->params.merge = 8;
        if (resolve_variant(P.get()) == STENCIL_OK && P->var.fullw) break;
        P->params = keep;                                 // fall back to the measured round-1 setting
        if (resolve_variant(P.get()) != STENCIL_OK) return STENCIL_E_OC_INFEASIBLE;
      }
    }
    break;
  }
  clear_error();
  if (P->var.reg_lo > 0 && !getenv("STENCIL_REGSPLIT")) {
    // keep the register split only where it pays: the unsplit kernel spills,
    // the CTA is alone on its SM anyway (shared memory), and the split kernel
    // spills less (large op tables: the intermediate stages need their registers)
    const int elem = dtype == STENCIL_F64 ? 8 : 4;
    Variant v0 = P->var;
    v0.reg_lo = v0.reg_hi = 0;
    v0.ws_threads = v0.tbrt_threads(P->pat, elem);
    std::string low;
    std::vector<char> bin;
    int sp0 = -1, sp1 = -1;
    SM_TRY(compile_variant(P->pat, P->dtype, v0, &low, &bin, &sp0));
    const bool alone = 2 * (v0.smem_bytes(P->pat, elem) + 1024) > 228 * 1024;
    if (sp0 > 0 && alone) SM_TRY(compile_variant(P->pat, P->dtype, P->var, &low, &bin, &sp1));
    if (!(sp0 > 0 && alone && sp1 >= 0 && sp1 < sp0)) P->var = v0;
  }
  P->src = generate_source(P->pat, P->dtype, P->var);
  // kernel specialisation (host-only; module load is deferred to first use)
  SM_TRY(compile_variant(P->pat, P->dtype, P->var, &P->lowered, &P->cubin));
  *plan = P.release();
  return STENCIL_OK;
}

void stencil_plan_destroy(stencil_plan_t plan) { delete plan; }

int stencil_plan_set_stream(stencil_plan_t plan, void* s) {
  if (!plan) SM_FAIL(STENCIL_E_INVAL, "null plan");
  plan->stream = (cudaStream_t)s;
  return STENCIL_OK;
}

size_t stencil_plan_workspace_bytes(stencil_plan_t plan) {
  if (!plan) return 0;
  const int elem = plan->dtype == STENCIL_F64 ? 8 : 4;
  return (size_t)plan->vdims[0] * plan->vdims[1] * plan->vdims[2] * elem;
}

int stencil_plan_set_workspace(stencil_plan_t plan, void* p, size_t bytes) {
  if (!plan) SM_FAIL(STENCIL_E_INVAL, "null plan");
  if (p && bytes < stencil_plan_workspace_bytes(plan))
    SM_FAIL(STENCIL_E_INVAL, "workspace of %zu bytes < %zu", bytes, stencil_plan_workspace_bytes(plan));
  if ((uintptr_t)p % 16) SM_FAIL(STENCIL_E_INVAL, "workspace must be 16-byte aligned");
  plan->ws = p;
  plan->ws_bytes = bytes;
  return STENCIL_OK;
}

int stencil_plan_info(stencil_plan_t P, stencil_plan_info_t* info) {
  if (!P || !info) SM_FAIL(STENCIL_E_INVAL, "null argument");
  memset(info, 0, sizeof *info);
  info->ndim = P->ndim;
  info->order = P->order;
  info->nnz = P->pat.nnz;
  info->dtype = P->dtype;
  // extents in the user's axes
  const Pattern& p = P->pat;
  if (P->ndim == 2 && (P->var.family == FAM_STREAM || P->var.family == FAM_STREAM_TB)) {
    int e[6] = {0, 0, p.zlo, p.zhi, p.xlo, p.xhi};
    memcpy(info->ext, e, sizeof e);
  } else {
    int e[6] = {p.zlo, p.zhi, p.ylo, p.yhi, p.xlo, p.xhi};
    memcpy(info->ext, e, sizeof e);
  }
  info->oc = P->oc;
  info->params = P->params;
  info->kernel_family = P->var.family;
  const int elem = P->dtype == STENCIL_F64 ? 8 : 4;
  info->smem_bytes = P->var.smem_bytes(P->pat, elem);
  info->threads = P->var.threads();
  info->regs = P->kern.regs;
  info->uses_tma = P->var.tma ? 1 : 0;
  const GridArg g = make_grid(P, P->var.vx);   // points this plan updates per time step
  info->points = (long long)(g.cz1 - g.cz0) * (g.cy1 - g.cy0) * (g.cx1 - g.cx0);
  snprintf(info->kernel_name, sizeof info->kernel_name, "%s", P->lowered.c_str());
  info->reg_split[0] = P->var.reg_lo;
  info->reg_split[1] = P->var.reg_hi;
  info->xshift = P->var.xshift ? 1 : 0;
  info->host_chunks = P->host_chunks;
  return STENCIL_OK;
}

int stencil_plan_set_timing(stencil_plan_t P, int enable) {
  clear_error();
  if (!P) SM_FAIL(STENCIL_E_INVAL, "null plan");
  P->timing = enable != 0;
  P->ev_used = 0;
  return STENCIL_OK;
}

int stencil_plan_kernel_time(stencil_plan_t P, double* kernel_ms, int64_t* launches) {
  clear_error();
  if (!P || !kernel_ms || !launches) SM_FAIL(STENCIL_E_INVAL, "null argument");
  double tot = 0.0;
  if (P->ev_used) SM_CUDA(cudaEventSynchronize(P->ev_pool[P->ev_used - 1]));
  for (size_t i = 0; i + 1 < P->ev_used; i += 2) {
    float ms = 0.f;
    SM_CUDA(cudaEventElapsedTime(&ms, P->ev_pool[i], P->ev_pool[i + 1]));
    tot += ms;
  }
  *kernel_ms = tot;
  *launches = (int64_t)(P->ev_used / 2);
  P->ev_used = 0;
  return STENCIL_OK;
}

int stencil_run_group(stencil_plan_t* plans, int nplans, const void* const* ins, void* const* outs, int steps) {
  clear_error();
  if (!plans || !ins || !outs || nplans < 1) SM_FAIL(STENCIL_E_INVAL, "bad arguments");
  std::vector<stencil_plan_s*> ps(plans, plans + nplans);
  for (int k = 0; k < nplans; ++k) {
    if (!ps[k]) SM_FAIL(STENCIL_E_INVAL, "null plan %d", k);
    Comm* c = ps[k]->comm;
    if (nplans > 1 && (!c || c->transport != TR_LOOPBACK || c->nranks != nplans || c->rank != k ||
                       c->peers[k] != ps[k]))
      SM_FAIL(STENCIL_E_STATE, "plans must be one loopback group in rank order");
  }
  if (nplans == 1 && ps[0]->comm && ps[0]->comm->transport == TR_LOOPBACK && ps[0]->comm->nranks != 1)
    SM_FAIL(STENCIL_E_STATE, "a loopback slab runs with its whole group");
  return run_group(ps, std::vector<const void*>(ins, ins + nplans), std::vector<void*>(outs, outs + nplans), steps);
}

int stencil_run(stencil_plan_t plan, const void* in, void* out, int steps) {
  clear_error();
  if (!plan) SM_FAIL(STENCIL_E_INVAL, "null plan");
  return run_device(plan, in, out, steps);
}

int stencil_run_host(stencil_plan_t P, const void* in_host, void* out_host, int steps) {
  clear_error();
  if (!P || !in_host || !out_host) SM_FAIL(STENCIL_E_INVAL, "null argument");
  if (P->comm && P->comm->transport == TR_P2P)
    SM_FAIL(STENCIL_E_STATE, "P2P slab plans run only on their registered device buffers");
  const size_t bytes = stencil_plan_workspace_bytes(P);
  if (P->h_bytes < bytes) free_host_path_buffers(P);   // the view grew (slab ghosts): reallocate
  if (!P->h_in_dev) SM_CUDA(cudaMalloc(&P->h_in_dev, bytes));
  if (!P->h_out_dev) SM_CUDA(cudaMalloc(&P->h_out_dev, bytes));
  P->h_bytes = bytes;
  void* saved_ws = P->ws;
  size_t saved_b = P->ws_bytes;
  if (!P->ws || P->ws_bytes < bytes) {
    if (!P->h_ws_dev) SM_CUDA(cudaMalloc(&P->h_ws_dev, bytes));
    P->ws = P->h_ws_dev;
    P->ws_bytes = bytes;
  }
  {
    bool done = false;
    const char* np = getenv("STENCIL_NO_PIPELINE");   // dev override: unpipelined path
    P->host_chunks = 0;
    const int rc = (np && atoi(np)) ? STENCIL_OK : run_host_pipelined(P, in_host, out_host, steps, &done);
    if (rc != STENCIL_OK || done) {
      P->ws = saved_ws;
      P->ws_bytes = saved_b;
      return rc;
    }
  }
  SM_CUDA(cudaMemcpyAsync(P->h_in_dev, in_host, bytes, cudaMemcpyHostToDevice, P->stream));
  int rc = run_device(P, P->h_in_dev, P->h_out_dev, steps);
  P->ws = saved_ws;
  P->ws_bytes = saved_b;
  if (rc != STENCIL_OK) return rc;
  SM_CUDA(cudaMemcpyAsync(out_host, P->h_out_dev, bytes, cudaMemcpyDeviceToHost, P->stream));
  SM_CUDA(cudaStreamSynchronize(P->stream));
  return STENCIL_OK;
}

int stencil_fill_field(void* dev, stencil_dtype_t dtype, int ndim, const int64_t* box_dims, const int64_t* origin,
                       const int64_t* global_dims, uint64_t seed, int kind, void* stream) {
  clear_error();
  if (!dev || !box_dims || !global_dims) SM_FAIL(STENCIL_E_INVAL, "null argument");
  if (ndim < 1 || ndim > 3) SM_FAIL(STENCIL_E_INVAL, "ndim must be 1..3");
  if (dtype != STENCIL_F32 && dtype != STENCIL_F64) SM_FAIL(STENCIL_E_INVAL, "bad dtype");
  if (kind != 0 && kind != 1) SM_FAIL(STENCIL_E_INVAL, "kind must be 0 or 1");
  int64_t b[3] = {1, 1, 1}, o[3] = {0, 0, 0}, g[3] = {1, 1, 1};
  for (int k = 0; k < ndim; ++k) {
    b[3 - ndim + k] = box_dims[k];
    o[3 - ndim + k] = origin ? origin[k] : 0;
    g[3 - ndim + k] = global_dims[k];
    if (b[3 - ndim + k] < 0 || o[3 - ndim + k] < 0 || o[3 - ndim + k] + b[3 - ndim + k] > g[3 - ndim + k])
      SM_FAIL(STENCIL_E_INVAL, "box outside the global grid on axis %d", k);
  }
  return launch_fill(dev, dtype, b, o, g, seed, kind, (cudaStream_t)stream);
}

int stencil_fma_probe(stencil_dtype_t dtype, int64_t iters, int blocks_per_sm, void* sink, void* stream,
                      double* flops) {
  clear_error();
  if (!sink || !flops) SM_FAIL(STENCIL_E_INVAL, "null argument");
  if (dtype != STENCIL_F32 && dtype != STENCIL_F64) SM_FAIL(STENCIL_E_INVAL, "bad dtype");
  if (iters < 1 || blocks_per_sm < 1 || blocks_per_sm > 8) SM_FAIL(STENCIL_E_INVAL, "iters >= 1, blocks_per_sm in 1..8");
  return launch_fma_probe(dtype, iters, blocks_per_sm, sink, flops, (cudaStream_t)stream);
}

int stencil_slab_range(int64_t nz_global, int rank, int nranks, int64_t* z_begin, int64_t* z_end) {
  clear_error();
  if (nranks < 1 || rank < 0 || rank >= nranks || !z_begin || !z_end || nz_global < nranks)
    SM_FAIL(STENCIL_E_INVAL, "bad slab arguments");
  const int64_t base = nz_global / nranks, rem = nz_global % nranks;
  *z_begin = rank * base + std::min<int64_t>(rank, rem);
  *z_end = *z_begin + base + (rank < rem ? 1 : 0);
  return STENCIL_OK;
}

}  // extern "C"
