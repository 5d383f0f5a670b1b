// codegen.cpp -- kernel specialisation.
//
// The paper generates one "stencil program" per stencil and OC (P:L25,
// P:L234). Here the generated part is only DATA: a descriptor struct holding
// the offsets (as a dense index table over the stencil's bounding box) and the
// coefficients rounded to the plan dtype, written as exact hex-float literals.
// The hand-written kernel templates of kernels/stencil_kernels.cuh are compiled
// against it with NVRTC for sm_100a. Cubins are cached per process and on disk.
#include <nvrtc.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <mutex>
#include <sstream>

#include "internal.h"

namespace smart_rt {

#include "kernels_src.inc"   // static const char kKernelsSrc[] (generated at build time)

namespace {

std::mutex g_mu;
std::map<std::string, CUmodule> g_modules;          // source -> loaded module
std::map<std::string, std::pair<std::string, std::vector<char>>> g_cubins;  // source -> (lowered, cubin)
std::map<std::string, int> g_spills;                                          // source -> ptxas spill bytes

uint64_t fnv1a(const std::string& s) {
  uint64_t h = 1469598103934665603ull;
  for (unsigned char c : s) { h ^= c; h *= 1099511628211ull; }
  return h;
}

std::string cache_dir() {
  const char* d = getenv("STENCIL_CACHE_DIR");
  std::string dir;
  if (d && *d) dir = d;
  else {
    const char* home = getenv("HOME");
    dir = std::string(home && *home ? home : "/tmp") + "/.cache/stencilmart";
  }
  return dir;
}

void mkdirs(const std::string& path) {
  std::string cur;
  std::stringstream ss(path);
  std::string part;
  if (!path.empty() && path[0] == '/') cur = "/";
  while (std::getline(ss, part, '/')) {
    if (part.empty()) continue;
    cur += part + "/";
    mkdir(cur.c_str(), 0755);
  }
}

bool read_file(const std::string& p, std::vector<char>* out) {
  std::ifstream f(p, std::ios::binary);
  if (!f) return false;
  out->assign(std::istreambuf_iterator<char>(f), std::istreambuf_iterator<char>());
  return !out->empty();
}

void write_file_atomic(const std::string& p, const char* data, size_t n) {
  std::string tmp = p + ".tmp" + std::to_string(getpid());
  std::ofstream f(tmp, std::ios::binary);
  if (!f) return;
  f.write(data, (std::streamsize)n);
  f.close();
  rename(tmp.c_str(), p.c_str());
}

std::string hexfloat(double v, bool f32) {
  char buf[64];
  if (f32) {
    float x = (float)v;                       // round-to-nearest-even, once (C-19)
    if (x == 0.0f) return std::signbit(x) ? "-0.0f" : "0.0f";
    snprintf(buf, sizeof buf, "%af", (double)x);
  } else {
    if (v == 0.0) return std::signbit(v) ? "-0.0" : "0.0";
    snprintf(buf, sizeof buf, "%a", v);
  }
  return buf;
}

}  // namespace

std::string Variant::name_expr(const char* desc) const {
  char b[256];
  const char* tf = tma ? "true" : "false";
  const char* cmf = cm ? "true" : "false";
  switch (family) {
    case FAM_NAIVE:
      snprintf(b, sizeof b, "smart::k_naive<%s, %d, %d, %d, %s>", desc, bx, by, m, cmf);
      break;
    case FAM_TILED:
      snprintf(b, sizeof b, "smart::k_tiled<%s, %d, %d, %d, %d, %d, %s, %d, %s>", desc, bx, by, bz, vx, m,
               cmf, tt, tf);
      break;
    case FAM_STREAM:
      snprintf(b, sizeof b, "smart::k_stream<%s, %d, %d, %d, %d, %s, %s, %d, %s>", desc, bx, by, vx, m, cmf,
               rt ? "true" : "false", ns, tf);
      break;
    default:
      if (rt)   // retiming in every fused step (k_stream_tb_rt)
        snprintf(b, sizeof b, "smart::k_stream_tb_rt<%s, %d, %d, %d, %d, %s, %d, %d>", desc, bx, by, vx, m, cmf,
                 ns, tt);
      else
        snprintf(b, sizeof b, "smart::k_stream_tb<%s, %d, %d, %d, %d, %s, %s, %d, %d>", desc, bx, by, vx, m,
                 cmf, rt ? "true" : "false", ns, tt);
      break;
  }
  return b;
}

int Variant::threads() const {
  if (family == FAM_STREAM_TB && rt) return ws_threads;
  switch (family) {
    case FAM_NAIVE: return bx * by;
    default: return (family == FAM_TILED ? bx / vx : tpx()) * by;
  }
}

static int roundup(int a, int b) { return (a + b - 1) / b * b; }

// Rows of an intermediate-stage thread tile of k_stream_tb / k_stream_tb_rt
// (S::MI). 2 rows: measured on C2 (512^3 heat, fp64), 4-row tiles of the
// retiming pipeline need ~95 registers and lose 15% to the lower occupancy.
int Variant::mid_rows(const Pattern& p, int elem) const {
  (void)p; (void)elem;
  if (flat) return 1;          // 2-D streaming view: a plane is one row, taller tiles only waste lanes
  if (family == FAM_STREAM_TB && rt)
    if (const char* e = getenv("STENCIL_MID_ROWS")) return atoi(e);   // dev override
  if (mid_rows_set > 0) return mid_rows_set;
  return midvx == 1 ? 4 : 2;   // scalar-column intermediate tiles: 1 x 4
}

// Slots of each intermediate-stage ring of k_stream_tb_rt (S::MIDR).
int Variant::mid_slots() const {
  if (const char* e = getenv("STENCIL_MIDR")) return std::max(2, atoi(e));   // dev override
  return mid_slots_set > 0 ? mid_slots_set : 2;
}

// Mirrors StreamTbRtCfg::THREADS of stencil_kernels.cuh: one producer warp,
// ceil(NT_s / 32) warps per intermediate stage s, ceil(tiles / 32) last-stage warps.
int Variant::tbrt_threads(const Pattern& p, int elem) const {
  int wl = 0;
  return tbrt_threads(p, elem, &wl);
}

// Register split (setmaxnreg) of k_stream_tb_rt: warps [0, WL) shrink to
// reg_lo, the last stage [WL, NW) grows to reg_hi. The growth is served from
// the CTA's own allocation (regs/thread of the compiled kernel x NW warps), so
// the split must fit it -- otherwise setmaxnreg.inc would wait forever. Checked
// against the loaded kernel's register count before any launch.
bool Variant::regsplit_fits(const Pattern& p, int elem, int kernel_regs) const {
  if (reg_lo <= 0) return true;
  int wl = 0;
  const int nw = tbrt_threads(p, elem, &wl) / 32;
  if (reg_lo % 8 || reg_hi % 8 || reg_lo < 24 || reg_hi > 256 || reg_lo > kernel_regs || reg_hi < kernel_regs)
    return false;
  return (long)wl * reg_lo + (long)(nw - wl) * reg_hi <= (long)nw * kernel_regs;
}

int Variant::tbrt_threads(const Pattern& p, int elem, int* wl_out) const {
  const int mi = mid_rows(p, elem);
  int warps = 1;
  for (int s = 1; s < tt; ++s) {
    const int hx0 = (tt - s) * p.xlo, hx1 = (tt - s) * p.xhi;
    const int hy0 = (tt - s) * p.ylo, hy1 = (tt - s) * p.yhi;
    const int mvx = midvx > 0 ? midvx : vx;
    const int txl = xshift ? hx0 : roundup(hx0, mvx);
    int ntx = (txl + bx + hx1 + mvx - 1) / mvx;
    if (fullw) {                                  // TbRtStage::FULLW: the ring's whole rows
      const int aln = std::max(16 / elem, vx);
      ntx = roundup(roundup(tt * p.xlo, aln) + bx + tt * p.xhi, aln);
    }
    if (const char* wa = getenv("STENCIL_WALIGN"))   // dev: padded tile rows (TbRtStage::NTXP)
      if (atoi(wa) == 2) ntx = roundup(ntx, 16);
    const int nty = (rows() + hy0 + hy1 + mi - 1) / mi;
    warps += (ntx * nty + 31) / 32;
  }
  if (reg_lo > 0) warps = roundup(warps, 4);    // warpgroup-aligned roles (register split)
  *wl_out = warps;
  warps += (tpx() * by + 31) / 32;
  if (reg_lo > 0) warps = roundup(warps, 4);
  return 32 * warps;
}

// Mirrors TiledCfg / StreamCfg of stencil_kernels.cuh.
int Variant::smem_bytes(const Pattern& p, int elem) const {
  const int aln = std::max(16 / elem, vx);
  if (family == FAM_TILED) {
    const int xoff = roundup(tt * p.xlo, aln);
    const int lx = roundup(xoff + bx + tt * p.xhi, aln);
    const int ly = by * m + tt * (p.ylo + p.yhi);
    const int lz = bz + tt * (p.zlo + p.zhi);
    const int buf = roundup(lx * ly * lz * elem, 128) / elem;
    const int pad = tt > 1 && tiled_mid > 0 ? roundup(tiled_mid * lx * elem, 128) / elem : 0;   // TiledCfg::PAD
    const int padf = tt > 1 && tiled_mid > 0 && tiled_full ? 128 / elem : 0;                      // TiledCfg::PADF
    return ((tt > 1 ? 2 : 1) * buf + pad + padf) * elem + 128;
  }
  if (family == FAM_STREAM) {
    const int xoff = roundup(p.xlo, aln);
    const int lx = roundup(xoff + bx + p.xhi, aln);
    const int ly = rows() + p.ylo + p.yhi;
    const int plane = roundup(lx * ly * elem, 128) / elem;
    const int nz = p.zlo + p.zhi + 1;
    const int nring = (rt ? 1 : nz) + ns - 1;
    return nring * plane * elem + 8 * nring + 128;
  }
  if (family == FAM_STREAM_TB && rt) {   // mirrors StreamTbRtCfg
    const int xoff = xshift ? tt * p.xlo : roundup(tt * p.xlo, aln);
    const int lx = roundup(xoff + bx + tt * p.xhi, aln);
    const int ly = rows() + tt * (p.ylo + p.yhi);
    // even/odd-split last ring: row pitch split_pitch(lx, k) (stencil_kernels.cuh)
    const int mv = midvx > 0 ? midvx : vx;
    const int k = xoff - roundup(p.xlo, mv);
    const int so = lx / 2 + ((8 + ((fullw ? 0 : k) & 1) - (lx / 2) % 16) + 32) % 16;
    int sp = !splitmid ? lx : so + lx / 2 + 1;
    if (splitmid && fullw) {                      // split_pitch_full
      const int mi = mid_rows(p, elem);
      sp = so + lx / 2 + (16 - so % 16) % 16;
      for (int c = so + lx / 2; c < so + lx / 2 + 16; ++c)
        if (((mi * c - lx / 2) % 16 + 16) % 16 == 0) { sp = c; break; }
    }
    const int plane = roundup((std::max(lx, sp) * ly + mid_rows(p, elem) * lx + aln) * elem, 128) / elem;
    const int padf = 128 / elem;
    const int padb = roundup((mid_rows(p, elem) * lx + aln) * elem, 128) / elem;
    const int nr = ns + p.zhi, mr = mid_slots();
    return (padf + (nr + mr * (tt - 1)) * plane + padb) * elem + 8 * (2 * nr + 2 * mr * (tt - 1)) + 128;
  }
  if (family == FAM_STREAM_TB) {   // mirrors StreamTbCfg
    const int xoff = roundup(tt * p.xlo, aln);
    const int lx = roundup(xoff + bx + tt * p.xhi, aln);
    const int ly = rows() + tt * (p.ylo + p.yhi);
    const int plane = roundup(lx * ly * elem, 128) / elem;
    const int nz = p.zlo + p.zhi + 1;
    const int nin = nz + ns - 1;
    const int padf = 128 / elem;
    const int padb = roundup((mid_rows(p, elem) * lx + aln) * elem, 128) / elem;
    return (padf + (nin + (tt - 1) * nz) * plane + padb) * elem + 8 * nin + 128;
  }
  return 0;
}

// Op table of a variant (format documented at run_gather in stencil_kernels.cuh).
// Loops are ordered so that every accumulator receives its FMAs in
// lexicographic (dz, dy, dx) order -- the canonical chain of every OC.
// fp32 (`pair`): two FMAs that share a coefficient and feed adjacent output
// columns (v, v+1) from adjacent window elements (e, e+1), v and e even, become
// ONE packed op (bit 30) that the kernels issue as an FFMA2 (sm_100's packed
// fp32 FMA: two independent RN fmas, so every chain stays bitwise the same).
// The window's FMAs are emitted offset-major (dx ascending, then column), which
// keeps each accumulator's chain lexicographic and puts pair partners side by side.
static std::vector<uint32_t> encode_ops(const Pattern& pat, const Variant& v, bool pair) {
  const int NZ = pat.zlo + pat.zhi + 1, NY = pat.ylo + pat.yhi + 1, NX = pat.xlo + pat.xhi + 1;
  std::vector<int> idx((size_t)NZ * NY * NX, -1);
  for (int i = 0; i < pat.nnz; ++i)
    idx[((size_t)(pat.dz[i] + pat.zlo) * NY + pat.dy[i] + pat.ylo) * NX + pat.dx[i] + pat.xlo] = i;
  auto cidx = [&](int zi, int yi, int xi) {
    if (zi < 0 || zi >= NZ || yi < 0 || yi >= NY || xi < 0 || xi >= NX) return -1;
    return idx[((size_t)zi * NY + yi) * NX + xi];
  };
  const int VX = v.family == FAM_NAIVE ? 1 : v.vx;
  const int M = v.m, BY = v.by;
  const bool scatter = v.rt && (v.family == FAM_STREAM || v.family == FAM_STREAM_TB);
  // placement of merged output m relative to the thread's first output: rows
  // (y-merge: BM m, CM m*BY) or vectors (x-merge: BM m, CM m*BX/M/VX)
  const int KS = v.xm ? (v.cm ? v.bx / M / VX : 1) : 0;
  auto rsh = [&](int m) { return v.xm ? 0 : (v.cm ? m * BY : m); };
  auto csh = [&](int m) { return v.xm ? m * KS : 0; };
  // window vector kv covers columns [kv*VX - xsh, kv*VX - xsh + VX) relative to
  // the thread's first output column (xsh > 0: TB-RT aligned windows, StreamTbRtCfg)
  const int xsh = v.xshift ? pat.xlo % VX : 0;
  auto fdiv = [](int a, int b) { return a >= 0 ? a / b : -((-a + b - 1) / b); };
  const int KLO = fdiv(xsh - pat.xlo, VX), KHI = fdiv(VX - 1 + pat.xhi + xsh, VX);
  auto load = [](int zi, int j, int kv) {
    return (uint32_t)(zi & 15) | ((uint32_t)(j + 128) & 255) << 4 | ((uint32_t)(kv + 2048) & 4095) << 12;
  };
  auto fma = [](int id, int e, int vv, int m, int zi) {
    return 0x80000000u | (uint32_t)id | (uint32_t)e << 10 | (uint32_t)vv << 12 | (uint32_t)m << 14 |
           (uint32_t)zi << 17;
  };
  std::vector<uint32_t> ops, f;
  auto window = [&](int zsel, int j_rel, int kv, int zi_lo, int zi_hi, int m_lo, int m_hi) {
    // FMAs fed by window (row j_rel, vector kv) into outputs m_lo..m_hi-1
    f.clear();
    for (int zi = zi_lo; zi < zi_hi; ++zi)
      for (int m = m_lo; m < m_hi; ++m) {
        const int dyi = j_rel - rsh(m) + pat.ylo;
        // element e of this window feeds column vv of output m through offset
        // dx = (kv - csh(m))*VX + e - vv - xsh
        for (int d = kv * VX - xsh - (VX - 1); d <= kv * VX - xsh + VX - 1; ++d)
          for (int vv = 0; vv < VX; ++vv) {
            const int e = d - kv * VX + xsh + vv;
            if (e < 0 || e >= VX) continue;
            const int id = cidx(zi, dyi, d - csh(m) * VX + pat.xlo);
            if (id < 0) continue;
            if (pair && !(vv & 1) && !(e & 1) && vv + 1 < VX && e + 1 < VX) {
              f.push_back(fma(id, e, vv, m, zi) | 0x40000000u);   // columns vv, vv+1
              ++vv;
              continue;
            }
            f.push_back(fma(id, e, vv, m, zi));
          }
      }
    if (!f.empty()) {
      ops.push_back(load(zsel, j_rel, kv));
      ops.insert(ops.end(), f.begin(), f.end());
    }
  };
  // (windows are visited in (zi, row, vector) order, and each window emits its
  // FMAs in ascending dx: every accumulator's chain is lexicographic)
  if (v.xm && !v.cm) {           // x-BM: outputs share windows over M + extent vectors
    for (int zi = 0; zi < (scatter ? 1 : NZ); ++zi)
      for (int j = -pat.ylo; j <= pat.yhi; ++j)
        for (int kv = KLO; kv <= KHI + M - 1; ++kv)
          window(zi, j, kv, scatter ? 0 : zi, scatter ? NZ : zi + 1, 0, M);
  } else if (v.xm) {             // x-CM: separate windows per output, KS vectors apart
    for (int zi = 0; zi < (scatter ? 1 : NZ); ++zi)
      for (int m = 0; m < M; ++m)
        for (int j = -pat.ylo; j <= pat.yhi; ++j)
          for (int kv = KLO; kv <= KHI; ++kv)
            window(zi, j, kv + m * KS, scatter ? 0 : zi, scatter ? NZ : zi + 1, m, m + 1);
  } else if (!v.cm) {
    if (!scatter) {
      for (int zi = 0; zi < NZ; ++zi)
        for (int j = -pat.ylo; j < M + pat.yhi; ++j)
          for (int kv = KLO; kv <= KHI; ++kv) window(zi, j, kv, zi, zi + 1, 0, M);
    } else {
      for (int j = -pat.ylo; j < M + pat.yhi; ++j)
        for (int kv = KLO; kv <= KHI; ++kv) window(0, j, kv, 0, NZ, 0, M);
    }
  } else {
    if (!scatter) {
      for (int zi = 0; zi < NZ; ++zi)
        for (int m = 0; m < M; ++m)
          for (int j = -pat.ylo; j <= pat.yhi; ++j)
            for (int kv = KLO; kv <= KHI; ++kv) window(zi, m * BY + j, kv, zi, zi + 1, m, m + 1);
    } else {
      for (int m = 0; m < M; ++m)
        for (int j = -pat.ylo; j <= pat.yhi; ++j)
          for (int kv = KLO; kv <= KHI; ++kv) window(0, m * BY + j, kv, 0, NZ, m, m + 1);
    }
  }
  return ops;
}

// Window LOAD entries of a TB-RT variant's two op tables (last stage + the
// intermediate stages): the shared-memory vector loads per thread tile and plane.
int count_window_loads(const Pattern& pat, int elem, const Variant& v) {
  int n = 0;
  for (uint32_t op : encode_ops(pat, v, false)) n += !(op >> 31);
  Variant vm = v;
  vm.family = FAM_STREAM; vm.cm = false; vm.xm = false; vm.m = v.mid_rows(pat, elem);
  if (v.midvx > 0) vm.vx = v.midvx;
  for (uint32_t op : encode_ops(pat, vm, false)) n += !(op >> 31);
  return n;
}

std::string generate_source(const Pattern& pat, int dtype, const Variant& v) {
  const bool f32 = dtype == STENCIL_F32;
  const int NZ = pat.zlo + pat.zhi + 1, NY = pat.ylo + pat.yhi + 1, NX = pat.xlo + pat.xhi + 1;
  std::vector<int> idx((size_t)NZ * NY * NX, -1);
  for (int i = 0; i < pat.nnz; ++i) {
    const int zi = pat.dz[i] + pat.zlo, yi = pat.dy[i] + pat.ylo, xi = pat.dx[i] + pat.xlo;
    idx[((size_t)zi * NY + yi) * NX + xi] = i;
  }
  std::ostringstream o;
  o << "// generated stencil descriptor: nnz=" << pat.nnz << "\n";
  o << "#include \"stencil_kernels.cuh\"\n";
  o << "namespace gen {\n";
  o << "__device__ constexpr short g_idx[" << NZ << "][" << NY << "][" << NX << "] = {";
  for (int z = 0; z < NZ; ++z) {
    o << "{";
    for (int y = 0; y < NY; ++y) {
      o << "{";
      for (int x = 0; x < NX; ++x) o << idx[((size_t)z * NY + y) * NX + x] << (x + 1 < NX ? "," : "");
      o << "}" << (y + 1 < NY ? "," : "");
    }
    o << "}" << (z + 1 < NZ ? "," : "");
  }
  o << "};\n";
  const char* T = f32 ? "float" : "double";
  // (tried: fp64 coefficients in __constant__ memory instead of immediates --
  // ptxas then stages them through uniform registers with LDCU + R2UR and the
  // order-2 random kernel grew from 86 to 132 registers; the UMOV-materialised
  // immediates stay)
  // A DFMA takes a 32-bit immediate (the high word of the double); any other fp64
  // coefficient is materialised by two UMOVs into a uniform register, re-issued
  // when the 63 uniform registers run out -- on an order-4 random stencil (293
  // coefficients) 599 UMOVs per 1172 DFMAs per plane body. From the constant
  // bank ptxas loads two coefficients per LDCU.128 instead (176 per body).
  // Measured on C5's 1024^3 random stencils (ST_BM_RT_PR, same box): order 3
  // (163 coefficients) 93.0 -> 99.4 GStencil/s, order 4 (293) 54.9 -> 57.0,
  // order 2 (51) 242 -> 233, C4's box125 (dyadic, all immediates) 124 -> 109:
  // the constant bank pays only for large tables of non-immediate coefficients.
  int nonimm = 0;
  for (int i = 0; i < pat.nnz && !f32; ++i) {
    uint64_t bits;
    memcpy(&bits, &pat.c[i], sizeof bits);
    nonimm += (bits & 0xffffffffull) != 0;
  }
  bool cbank = !f32 && nonimm >= 128;
  if (const char* cb = getenv("STENCIL_CBANK")) cbank = atoi(cb) != 0;   // dev override
  o << (cbank ? "__constant__ " : "__device__ constexpr ") << T << " g_coef[" << pat.nnz << "] = {";
  for (int i = 0; i < pat.nnz; ++i) o << hexfloat(pat.c[i], f32) << (i + 1 < pat.nnz ? "," : "");
  o << "};\n";
  // Packed FFMA2 pairs for fp32 are off by default: measured on C3 (star25,
  // 768^3) they cut FMA instructions by 42% but raise registers 96 -> 151 and
  // run 2-7% slower (the kernel is not FMA-issue bound).
  const char* f2 = getenv("STENCIL_FFMA2");                            // dev override
  const bool pair = f32 && f2 && atoi(f2);
  const std::vector<uint32_t> ops = encode_ops(pat, v, pair);
  o << "__device__ constexpr unsigned g_ops[" << std::max<size_t>(ops.size(), 1) << "] = {";
  for (size_t i = 0; i < ops.size(); ++i) o << ops[i] << "u" << (i + 1 < ops.size() ? "," : "");
  if (ops.empty()) o << "0u";
  o << "};\n";
  std::vector<uint32_t> mops;
  const int mi = v.mid_rows(pat, f32 ? 4 : 8);
  const int tmid = v.family == FAM_TILED && v.tt > 1 ? v.tiled_mid : 0;
  if (tmid > 0) {                      // k_tiled intermediate steps: 1 x tmid tiles, gather
    Variant vm = v;
    vm.family = FAM_STREAM; vm.rt = false; vm.cm = false; vm.xm = false; vm.m = tmid; vm.vx = v.tiled_mvx;
    vm.xshift = false;
    mops = encode_ops(pat, vm, pair);
  }
  if (v.family == FAM_STREAM_TB) {     // intermediate fused steps: VX x MI tiles, gather or (RT) scatter
    Variant vm = v;
    vm.family = FAM_STREAM; vm.cm = false; vm.xm = false; vm.m = mi;
    if (v.midvx > 0) vm.vx = v.midvx;
    mops = encode_ops(pat, vm, pair);
  }
  o << "__device__ constexpr unsigned g_mops[" << std::max<size_t>(mops.size(), 1) << "] = {";
  for (size_t i = 0; i < mops.size(); ++i) o << mops[i] << "u" << (i + 1 < mops.size() ? "," : "");
  if (mops.empty()) o << "0u";
  o << "};\n";
  o << "struct S {\n  typedef " << T << " T;\n";
  o << "  static constexpr int MI = " << mi << ";\n";
  int minb = 1;   // __launch_bounds__ min blocks of k_stream_tb_rt
  if (const char* e = getenv("STENCIL_MINB")) minb = atoi(e);   // dev override
  o << "  static constexpr int MINB = " << minb << ";\n";
  o << "  static constexpr int MIDR = " << v.mid_slots() << ";\n";
  o << "  static constexpr int TMID = " << tmid << ";\n";
  o << "  static constexpr bool TFULL = " << (tmid > 0 && v.tiled_full ? "true" : "false") << ";\n";
  o << "  static constexpr int TMVX = " << (tmid > 0 ? v.tiled_mvx : 1) << ";\n";
  o << "  static constexpr int MVX = " << (v.midvx > 0 ? v.midvx : std::max(v.vx, 1)) << ";\n";
  o << "  static constexpr bool SPLITMID = " << (v.splitmid ? "true" : "false") << ";\n";
  o << "  static constexpr bool FULLW = " << (v.fullw ? "true" : "false") << ";\n";
  {   // k_stream_tb_rt hand-off details, off by default: measured on C2 (same box,
      // 2 runs each) elected-lane arrivals 552 -> 546 GStencil/s, warp-aligned
      // stage-1 tiles 552 -> 530, both 528 (dev overrides for A/B measurements)
    const char* el = getenv("STENCIL_ELECT");
    const char* wa = getenv("STENCIL_WALIGN");
    o << "  static constexpr bool ELECT = " << ((el ? atoi(el) : 0) ? "true" : "false") << ";\n";
    o << "  static constexpr int WALIGN = " << (wa ? atoi(wa) : 0) << ";\n";
  }
  o << "  static constexpr bool XM = " << (v.xm ? "true" : "false") << ";   // merge along x (2-D streaming)\n";
  o << "  static constexpr bool TMA = " << (v.tma ? "true" : "false") << ";   // streaming TB staging (else cp.async)\n";
  o << "  static constexpr bool XSHIFT = " << (v.xshift ? "true" : "false") << ";\n";
  o << "  static constexpr int XSH = " << (v.xshift ? pat.xlo % std::max(v.vx, 1) : 0) << ";\n";
  o << "  static constexpr int REG_LO = " << v.reg_lo << ", REG_HI = " << v.reg_hi << ";\n";
  o << "  static constexpr long long SY = " << v.sy << "LL, SZ = " << v.sz << "LL;   // baked strides\n";
  o << "  struct Mid {\n    static constexpr int NOPS = " << mops.size() << ";\n"
    << "    static __device__ __forceinline__ constexpr unsigned op(int i) { return g_mops[i]; }\n  };\n";
  o << "  static constexpr int NNZ = " << pat.nnz << ", ZLO = " << pat.zlo << ", ZHI = " << pat.zhi
    << ", YLO = " << pat.ylo << ", YHI = " << pat.yhi << ", XLO = " << pat.xlo << ", XHI = " << pat.xhi
    << ", NZ = " << NZ << ", NY = " << NY << ", NX = " << NX << ";\n";
  o << "  static __device__ __forceinline__ constexpr int idx(int z, int y, int x) { return g_idx[z][y][x]; }\n";
  o << "  static __device__ __forceinline__ " << (cbank ? "" : "constexpr ") << "T coef(int i) { return g_coef[i]; }\n";
  o << "  static constexpr int NOPS = " << ops.size() << ";\n";
  // retiming queue rotation: NZ unrolled plane bodies while they stay small,
  // register shifts beyond. Measured (B200, 512^3 / 768^3): the unrolled form
  // is instruction-cache bound on a 293-point order-4 stencil ('no_instructions'
  // the top stall; 27 -> 51 GStencil/s with shifts) and on an order-3 one
  // (55 -> 84); it wins on the 25-point star (567 vs 493, ops*NZ ~ 2100) and
  // the heat stencil. Crossover between ~2100 and ~2500 table entries x NZ.
  int rtshift = (long)ops.size() * NZ > 2300 ? 1 : 0;
  if (const char* e = getenv("STENCIL_RT_SHIFT")) rtshift = atoi(e);   // dev override
  o << "  static constexpr int RTSHIFT = " << rtshift << ";\n";
  o << "  static __device__ __forceinline__ constexpr unsigned op(int i) { return g_ops[i]; }\n";
  o << "};\n}  // namespace gen\n";
  o << "// variant: " << v.name_expr("gen::S") << "\n";
  return o.str();
}

// spill bytes (stores + loads) from the ptxas -v lines of an NVRTC log; -1 if absent
static int parse_spill(const std::string& log) {
  int total = -1;
  size_t pos = 0;
  while ((pos = log.find("bytes spill stores", pos)) != std::string::npos) {
    size_t b = log.rfind(',', pos);
    const int st = b == std::string::npos ? 0 : atoi(log.c_str() + b + 1);
    const size_t l = log.find("bytes spill loads", pos);
    size_t b2 = l == std::string::npos ? std::string::npos : log.rfind(',', l);
    const int ld = b2 == std::string::npos ? 0 : atoi(log.c_str() + b2 + 1);
    total = std::max(total, 0) + st + ld;
    pos += 8;
  }
  return total;
}

int compile_variant(const Pattern& pat, int dtype, const Variant& v, std::string* lowered,
                    std::vector<char>* cubin, int* spill_bytes) {
  const std::string src = generate_source(pat, dtype, v);
  int spill_dummy = 0;
  if (!spill_bytes) spill_bytes = &spill_dummy;
  const std::string expr = "&" + v.name_expr("gen::S");
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_cubins.find(src);
    if (it != g_cubins.end()) {
      *lowered = it->second.first;
      *cubin = it->second.second;
      *spill_bytes = g_spills[src];
      return STENCIL_OK;
    }
  }
  std::vector<const char*> optv = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", "-default-device",
                                   "--extra-device-vectorization", "--ptxas-options=-v"};
  static thread_local std::string maxreg_opt;
  if (const char* e = getenv("STENCIL_MAXRREG")) {   // dev override (register cap experiments)
    maxreg_opt = std::string("--maxrregcount=") + e;
    optv.push_back(maxreg_opt.c_str());
  }
  const char* const* opts = optv.data();
  const int nopt = (int)optv.size();
  int nv_major = 0, nv_minor = 0;
  nvrtcVersion(&nv_major, &nv_minor);
  std::string key_str = src + "|" + kKernelsSrc + "|";
  for (int i = 0; i < nopt; ++i) key_str += std::string(opts[i]) + " ";
  key_str += std::to_string(nv_major) + "." + std::to_string(nv_minor);
  char hname[32];
  snprintf(hname, sizeof hname, "%016llx", (unsigned long long)fnv1a(key_str));
  const std::string dir = cache_dir();
  const std::string base = dir + "/" + hname;

  // disk cache
  std::vector<char> bin, nm, sp;
  if (read_file(base + ".cubin", &bin) && read_file(base + ".name", &nm) && read_file(base + ".spill", &sp)) {
    *lowered = std::string(nm.begin(), nm.end());
    *cubin = bin;
    *spill_bytes = atoi(std::string(sp.begin(), sp.end()).c_str());
    std::lock_guard<std::mutex> lk(g_mu);
    g_cubins[src] = {*lowered, *cubin};
    g_spills[src] = *spill_bytes;
    return STENCIL_OK;
  }

  nvrtcProgram prog;
  const char* hdr_src[] = {kKernelsSrc};
  const char* hdr_name[] = {"stencil_kernels.cuh"};
  nvrtcResult r = nvrtcCreateProgram(&prog, src.c_str(), "stencil_gen.cu", 1, hdr_src, hdr_name);
  if (r != NVRTC_SUCCESS) SM_FAIL(STENCIL_E_NVRTC, "nvrtcCreateProgram: %s", nvrtcGetErrorString(r));
  nvrtcAddNameExpression(prog, expr.c_str());
  r = nvrtcCompileProgram(prog, nopt, opts);
  if (r != NVRTC_SUCCESS) {
    size_t ls = 0;
    nvrtcGetProgramLogSize(prog, &ls);
    std::string log(ls, '\0');
    nvrtcGetProgramLog(prog, &log[0]);
    nvrtcDestroyProgram(&prog);
    if (log.size() > 3000) log = log.substr(0, 3000) + "...";
    SM_FAIL(STENCIL_E_NVRTC, "NVRTC compile of %s failed: %s", expr.c_str(), log.c_str());
  }
  {
    size_t ls = 0;
    nvrtcGetProgramLogSize(prog, &ls);
    std::string log(ls, '\0');
    if (ls) nvrtcGetProgramLog(prog, &log[0]);
    *spill_bytes = parse_spill(log);
  }
  const char* low = nullptr;
  nvrtcGetLoweredName(prog, expr.c_str(), &low);
  *lowered = low ? low : "";
  size_t cs = 0;
  nvrtcGetCUBINSize(prog, &cs);
  cubin->resize(cs);
  nvrtcGetCUBIN(prog, cubin->data());
  nvrtcDestroyProgram(&prog);
  {
    std::lock_guard<std::mutex> lk(g_mu);
    g_cubins[src] = {*lowered, *cubin};
    g_spills[src] = *spill_bytes;
  }
  mkdirs(dir);
  write_file_atomic(base + ".cubin", cubin->data(), cubin->size());
  write_file_atomic(base + ".name", lowered->data(), lowered->size());
  const std::string spn = std::to_string(*spill_bytes);
  write_file_atomic(base + ".spill", spn.data(), spn.size());
  return STENCIL_OK;
}

int load_kernel(const std::string& key_src, const std::vector<char>& cubin, const std::string& lowered,
                int smem, Kernel* out) {
  const Driver* d = nullptr;
  SM_TRY(get_driver(&d));
  SM_CUDA(cudaFree(nullptr));   // make the primary context current
  CUmodule mod = nullptr;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_modules.find(key_src);
    if (it != g_modules.end()) mod = it->second;
  }
  if (!mod) {
    CUresult r = d->moduleLoadData(&mod, cubin.data());
    if (r != CUDA_SUCCESS) SM_FAIL(STENCIL_E_CUDA, "cuModuleLoadData: %s", cu_errstr(r));
    std::lock_guard<std::mutex> lk(g_mu);
    g_modules[key_src] = mod;
  }
  CUfunction fn = nullptr;
  CUresult r = d->moduleGetFunction(&fn, mod, lowered.c_str());
  if (r != CUDA_SUCCESS) SM_FAIL(STENCIL_E_CUDA, "cuModuleGetFunction(%s): %s", lowered.c_str(), cu_errstr(r));
  if (smem > 48 * 1024) {
    r = d->funcSetAttribute(fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, smem);
    if (r != CUDA_SUCCESS)
      SM_FAIL(STENCIL_E_OC_INFEASIBLE, "shared memory %d B not available: %s", smem, cu_errstr(r));
  }
  out->fn = fn;
  d->funcGetAttribute(&out->regs, CU_FUNC_ATTRIBUTE_NUM_REGS, fn);
  d->funcGetAttribute(&out->local_bytes, CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES, fn);
  return STENCIL_OK;
}

}  // namespace smart_rt
