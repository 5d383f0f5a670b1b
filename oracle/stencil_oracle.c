/*
 * oracle/stencil_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously correct CPU definition of one StencilMART stencil
 * sweep, in fp64. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library. It shares no
 * code, header, table or helper with the CUDA path
 * (paper_conf_ipps_sunlyjlq22_b200/csrc) and neither side includes the other.
 *
 * What it computes (§I: "A stencil computation sweeps a
 * computation grid and processes the fixed neighbors around each point to
 * update its value, where the extent of the neighbors along each dimension is
 * referred to as the stencil order"; §IV-B: the access pattern is a
 * binary tensor of size (2N+1)^d whose accessed neighbours and centre are 1):
 *
 *   S    = { o in [-r, r]^d : access[o] = 1 }
 *   u_{t+1}[p] = sum_{o in S, lexicographic (dz,dy,dx) order} c_o * u_t[p + o]
 *                for every p with r <= p_k < n_k - r on every axis,
 *   u_{t+1}[p] = u_t[p]   on the frame (any p_k < r or p_k >= n_k - r).
 *
 * The boundary rule is the paper-silent reading C-1 of DESIGN.md (P:L304 leaves
 * boundary conditions to future work). Accumulation is a plain sequential
 * sum "acc = acc + c*u" in fp64; this file is compiled with
 * -ffp-contract=off so no fused multiply-add is introduced.
 *
 * 2-D grids are treated as nz = 1 with no frame along z and dz = 0 only.
 * T steps ping-pong between `out` and a private buffer; steps = 0 copies.
 * OpenMP parallelises the outermost loop only (the cpu_baseline's "cores").
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* Returns 0 on success, -1 on a bad argument, -2 on allocation failure. */
int oracle_stencil_f64(int ndim, const int64_t *dims, int order,
                       const uint8_t *access, const double *coeffs,
                       const double *in, double *out, int steps, int nthreads)
{
    if ((ndim != 2 && ndim != 3) || order < 1 || steps < 0) return -1;
    int64_t n[3], f[3];
    if (ndim == 3) { n[0] = dims[0]; n[1] = dims[1]; n[2] = dims[2]; f[0] = order; }
    else           { n[0] = 1;       n[1] = dims[0]; n[2] = dims[1]; f[0] = 0; }
    f[1] = order; f[2] = order;
    const int64_t total = n[0] * n[1] * n[2];
    const int w = 2 * order + 1;

    /* the offset list S in lexicographic (dz, dy, dx) order */
    int nnz = 0;
    const int tsize = (ndim == 3) ? w * w * w : w * w;
    int64_t *off = (int64_t *)malloc(sizeof(int64_t) * tsize);
    double *cf = (double *)malloc(sizeof(double) * tsize);
    if (!off || !cf) { free(off); free(cf); return -2; }
    for (int t = 0; t < tsize; ++t) {
        if (!access[t]) continue;
        int dz, dy, dx;
        if (ndim == 3) { dz = t / (w * w) - order; dy = (t / w) % w - order; dx = t % w - order; }
        else           { dz = 0;                   dy = t / w - order;       dx = t % w - order; }
        off[nnz] = ((int64_t)dz * n[1] + dy) * n[2] + dx;
        cf[nnz] = coeffs[t];
        ++nnz;
    }

#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif

    if (steps == 0) {
        memcpy(out, in, sizeof(double) * total);
        free(off); free(cf);
        return 0;
    }
    double *tmp = (double *)malloc(sizeof(double) * total);
    if (!tmp) { free(off); free(cf); return -2; }

    /* the last step must land in `out` */
    const double *src = in;
    double *dst = (steps % 2 == 1) ? out : tmp;
    for (int s = 0; s < steps; ++s) {
#pragma omp parallel for schedule(static)
        for (int64_t z = 0; z < n[0]; ++z) {
            for (int64_t y = 0; y < n[1]; ++y) {
                for (int64_t x = 0; x < n[2]; ++x) {
                    const int64_t p = (z * n[1] + y) * n[2] + x;
                    const int frame = z < f[0] || z >= n[0] - f[0] ||
                                      y < f[1] || y >= n[1] - f[1] ||
                                      x < f[2] || x >= n[2] - f[2];
                    if (frame) { dst[p] = src[p]; continue; }
                    double acc = 0.0;
                    for (int i = 0; i < nnz; ++i) acc = acc + cf[i] * src[p + off[i]];
                    dst[p] = acc;
                }
            }
        }
        src = dst;
        dst = (dst == out) ? tmp : out;
    }
    free(tmp); free(off); free(cf);
    return 0;
}

/* Number of threads OpenMP would use (reported as cpu_baseline.cores). */
int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
