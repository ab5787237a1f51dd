/*
 * stencil_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU oracle for the iterative 3D star-stencil
 * sweep of Tang et al., "Optimizing and Auto-Tuning Iterative Stencil Loops for
 * GPUs with the In-Plane Method" (IPDPS 2013).  Only tests/, the smoke() entry
 * of __graft_entry__.py and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  It shares NO code, header, table or helper with the CUDA
 * product path under paper_conf_ipps_tangtkwkgtw13_b200/ and never includes
 * anything from there.
 *
 * What it computes (PAPER.md line numbers, "P:L<n>"):
 *   - Eq. (1), P:L59-64 (Sec. III-A): for every updated point
 *       out[i,j,k] = c0*in[i,j,k]
 *                  + sum_{m=1..r} c_m*(in[i+-m,j,k] + in[i,j+-m,k] + in[i,j,k+-m])
 *   - Fig. 1, P:L66-80 (ITERSTENCILLOOP): two grids, ComputeKernel(in,out),
 *     Swap(in,out), "return in" after the last swap.  The stop criterion
 *      is read as a fixed iteration count (reading R5).
 *   - Domain (paper silent, reading R1): the updated region is the
 *     interior nx*ny*nz (the LX*LY*LZ of P:L103); storage is the OUTER grid
 *     (nx+2r)*(ny+2r)*(nz+2r) whose r-wide shell is a frozen Dirichlet
 *     boundary: copied from the input, never computed.
 *
 * Precision: fp64 throughout (the paper fixes none; P:L218 only says results
 * were checked against a CPU result).  Summation order is the plain one of
 * Eq. (1) as written; no blocking, fusion or reordering.
 *
 * Layout of every array argument: dense outer grid, x fastest:
 *   a[((k)*(ny+2r) + j)*(nx+2r) + i],  i in [0,nx+2r), j in [0,ny+2r),
 *   k in [0,nz+2r); interior points are i,j,k in [r, n+r).
 *
 * Pins (tests/test_oracle.py): impulse response, sine-mode eigenvalues,
 * Dirichlet eigenvectors over T iterations, constant/linear fields,
 * finite-difference polynomial reproduction, a scalar simulation of the
 * paper's in-plane steps 1-6 on integer data, and hand-computed
 * values in tests/golden/.
 */
#include <stdlib.h>
#include <string.h>
#include <time.h>

#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_OK 0
#define ORACLE_EINVAL 1
#define ORACLE_ENOMEM 2

/* Index of outer point (i,j,k) in the dense outer array. */
static long idx3(long i, long j, long k, long px, long py) {
    return (k * py + j) * px + i;
}

/*
 * One application of Eq. (1) to every interior point: dst <- S(src).
 * Shell cells of dst are not touched.  Eq. (1) is summed exactly as printed:
 * c0*centre first, then for m = 1..r the term c_m * (six neighbours), the six
 * neighbours added in the order i-m, i+m, j-m, j+m, k-m, k+m.
 */
static void compute_kernel(const double *src, double *dst, long nx, long ny,
                           long nz, int r, const double *c, int nthreads) {
    const long px = nx + 2 * r, py = ny + 2 * r;
    long k;
    (void)nthreads;
#ifdef _OPENMP
#pragma omp parallel for num_threads(nthreads) schedule(static)
#endif
    for (k = r; k < nz + r; ++k) {
        for (long j = r; j < ny + r; ++j) {
            for (long i = r; i < nx + r; ++i) {
                double acc = c[0] * src[idx3(i, j, k, px, py)];
                for (int m = 1; m <= r; ++m) {
                    double nb = src[idx3(i - m, j, k, px, py)]
                              + src[idx3(i + m, j, k, px, py)]
                              + src[idx3(i, j - m, k, px, py)]
                              + src[idx3(i, j + m, k, px, py)]
                              + src[idx3(i, j, k - m, px, py)]
                              + src[idx3(i, j, k + m, px, py)];
                    acc += c[m] * nb;
                }
                dst[idx3(i, j, k, px, py)] = acc;
            }
        }
    }
}

/*
 * ITERSTENCILLOOP of Fig. 1 for a fixed number of iterations.
 *   in   : initial outer grid (read only)
 *   out  : result outer grid (written; shell == in's shell)
 *   c    : r+1 coefficients c0..cr (Eq. 1 is isotropic: one c_m for all axes)
 *   iters: number of Jacobi sweeps (>= 0); iters == 0 returns a copy of in.
 * Returns ORACLE_OK, ORACLE_EINVAL or ORACLE_ENOMEM.
 */
int oracle_sweep(const double *in, double *out, long nx, long ny, long nz,
                 int r, const double *c, int iters, int nthreads) {
    if (!in || !out || !c || nx < 1 || ny < 1 || nz < 1 || r < 1 || iters < 0)
        return ORACLE_EINVAL;
    if (nthreads < 1) nthreads = 1;
    const long n = (nx + 2 * r) * (ny + 2 * r) * (nz + 2 * r);
    double *a = (double *)malloc(sizeof(double) * (size_t)n);
    double *b = (double *)malloc(sizeof(double) * (size_t)n);
    if (!a || !b) { free(a); free(b); return ORACLE_ENOMEM; }
    /* in <- initial; both grids carry the same (frozen) shell. */
    memcpy(a, in, sizeof(double) * (size_t)n);
    memcpy(b, in, sizeof(double) * (size_t)n);
    for (int t = 0; t < iters; ++t) {
        compute_kernel(a, b, nx, ny, nz, r, c, nthreads);  /* ComputeKernel(in,out) */
        double *tmp = a; a = b; b = tmp;                    /* Swap(in,out) */
    }
    memcpy(out, a, sizeof(double) * (size_t)n);             /* return in */
    free(a);
    free(b);
    return ORACLE_OK;
}

/*
 * Per-axis ("anisotropic") generalisation of Eq. (1) -- DESIGN.md reading R3b.
 * The BASELINE north star asks for "symmetric per-axis coefficients": each
 * axis d in {x, y, z} has its own c_{d,m}, symmetric in +-m, so
 *     out[i,j,k] = c0*in[i,j,k]
 *                + sum_{m=1..r} ( cx_m*(in[i-m,j,k] + in[i+m,j,k])
 *                               + cy_m*(in[i,j-m,k] + in[i,j+m,k])
 *                               + cz_m*(in[i,j,k-m] + in[i,j,k+m]) )
 * which is Eq. (1) when cx = cy = cz.  Written out plainly, same
 * Fig. 1 loop and frozen shell as oracle_sweep.
 *   c: 1 + 3r values: c0, cx_1..cx_r, cy_1..cy_r, cz_1..cz_r
 */
static void compute_kernel_axes(const double *src, double *dst, long nx, long ny,
                                long nz, int r, const double *c, int nthreads) {
    const long px = nx + 2 * r, py = ny + 2 * r;
    const double *cx = c + 1, *cy = c + 1 + r, *cz = c + 1 + 2 * r;
    long k;
    (void)nthreads;
#ifdef _OPENMP
#pragma omp parallel for num_threads(nthreads) schedule(static)
#endif
    for (k = r; k < nz + r; ++k) {
        for (long j = r; j < ny + r; ++j) {
            for (long i = r; i < nx + r; ++i) {
                double acc = c[0] * src[idx3(i, j, k, px, py)];
                for (int m = 1; m <= r; ++m) {
                    acc += cx[m - 1] * (src[idx3(i - m, j, k, px, py)] + src[idx3(i + m, j, k, px, py)]);
                    acc += cy[m - 1] * (src[idx3(i, j - m, k, px, py)] + src[idx3(i, j + m, k, px, py)]);
                    acc += cz[m - 1] * (src[idx3(i, j, k - m, px, py)] + src[idx3(i, j, k + m, px, py)]);
                }
                dst[idx3(i, j, k, px, py)] = acc;
            }
        }
    }
}

/* Fig. 1 loop of the per-axis stencil; arguments as oracle_sweep except c (1 + 3r values). */
int oracle_sweep_axes(const double *in, double *out, long nx, long ny, long nz,
                      int r, const double *c, int iters, int nthreads) {
    if (!in || !out || !c || nx < 1 || ny < 1 || nz < 1 || r < 1 || iters < 0)
        return ORACLE_EINVAL;
    if (nthreads < 1) nthreads = 1;
    const long n = (nx + 2 * r) * (ny + 2 * r) * (nz + 2 * r);
    double *a = (double *)malloc(sizeof(double) * (size_t)n);
    double *b = (double *)malloc(sizeof(double) * (size_t)n);
    if (!a || !b) { free(a); free(b); return ORACLE_ENOMEM; }
    memcpy(a, in, sizeof(double) * (size_t)n);
    memcpy(b, in, sizeof(double) * (size_t)n);
    for (int t = 0; t < iters; ++t) {
        compute_kernel_axes(a, b, nx, ny, nz, r, c, nthreads);  /* ComputeKernel(in,out) */
        double *tmp = a; a = b; b = tmp;                         /* Swap(in,out) */
    }
    memcpy(out, a, sizeof(double) * (size_t)n);                  /* return in */
    free(a);
    free(b);
    return ORACLE_OK;
}

/*
 * Value of one interior point after `iters` sweeps, computed without sweeping
 * the whole grid.  After t sweeps an interior point depends only on inputs
 * within distance t*r along the star (Eq. 1 has radius r), so the sweep is run
 * on the sub-box [p - (iters+1)*r, p + (iters+1)*r] per axis, clipped to
 * the outer grid, whose outermost r layers are held frozen.  A frozen layer
 * that is not part of the true shell is stale after the first sweep, and the
 * error moves r cells per sweep, reaching depth (iters-1)*r < iters*r: the
 * centre point is exact.  Used for sampled parity at full problem sizes.
 *   in : full dense outer grid (nx+2r)(ny+2r)(nz+2r)
 *   (i,j,k) : INTERIOR coordinates, 0 <= i < nx etc.
 *   result : *value
 */
int oracle_point(const double *in, long nx, long ny, long nz, int r,
                 const double *c, int iters, long i, long j, long k,
                 double *value) {
    if (!in || !c || !value || nx < 1 || ny < 1 || nz < 1 || r < 1 || iters < 0)
        return ORACLE_EINVAL;
    if (i < 0 || i >= nx || j < 0 || j >= ny || k < 0 || k >= nz)
        return ORACLE_EINVAL;
    const long px = nx + 2 * r, py = ny + 2 * r;
    const long h = ((long)iters + 1) * r;
    /* outer coordinates of the point and of the clipped box [lo, hi] */
    const long oi = i + r, oj = j + r, ok = k + r;
    long lo[3], hi[3];
    const long o[3] = {oi, oj, ok};
    const long ext[3] = {nx + 2 * r, ny + 2 * r, nz + 2 * r};
    for (int d = 0; d < 3; ++d) {
        lo[d] = o[d] - h;
        hi[d] = o[d] + h;
        if (lo[d] < 0) lo[d] = 0;
        if (hi[d] > ext[d] - 1) hi[d] = ext[d] - 1;
    }
    /* the sub-box, seen as its own outer grid with an r-wide frozen shell */
    const long sx = hi[0] - lo[0] + 1 - 2 * r;
    const long sy = hi[1] - lo[1] + 1 - 2 * r;
    const long sz = hi[2] - lo[2] + 1 - 2 * r;
    if (sx < 1 || sy < 1 || sz < 1) return ORACLE_EINVAL;
    const long bx = sx + 2 * r, by = sy + 2 * r, bz = sz + 2 * r;
    double *box = (double *)malloc(sizeof(double) * (size_t)(bx * by * bz));
    double *res = (double *)malloc(sizeof(double) * (size_t)(bx * by * bz));
    if (!box || !res) { free(box); free(res); return ORACLE_ENOMEM; }
    for (long kk = 0; kk < bz; ++kk)
        for (long jj = 0; jj < by; ++jj)
            memcpy(&box[(kk * by + jj) * bx],
                   &in[idx3(lo[0], lo[1] + jj, lo[2] + kk, px, py)],
                   sizeof(double) * (size_t)bx);
    int rc = oracle_sweep(box, res, sx, sy, sz, r, c, iters, 1);
    if (rc == ORACLE_OK)
        *value = res[((ok - lo[2]) * by + (oj - lo[1])) * bx + (oi - lo[0])];
    free(box);
    free(res);
    return rc;
}

/* Threads the OpenMP runtime would use for nthreads <= 0 (all host cores). */
int oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* Wall-clock seconds of oracle_sweep, for bench.py's cpu_baseline leg. */
double oracle_time_sweep(const double *in, double *out, long nx, long ny,
                         long nz, int r, const double *c, int iters,
                         int nthreads) {
    struct timespec t0, t1;
    clock_gettime(CLOCK_MONOTONIC, &t0);
    int rc = oracle_sweep(in, out, nx, ny, nz, r, c, iters, nthreads);
    clock_gettime(CLOCK_MONOTONIC, &t1);
    if (rc != ORACLE_OK) return -1.0;
    return (double)(t1.tv_sec - t0.tv_sec) + 1e-9 * (double)(t1.tv_nsec - t0.tv_nsec);
}

/*
 * Application stencils with a second input grid (Sec. V, Table V, P:L284-321;
 * BASELINE config 3 "3D wave").  The paper names them and counts their grids
 * (Table V: "Poisson" reads 2 grids, writes 1) but prints no formulas
 * (reading R19), so the oracle states the plain definitions:
 *
 *   source (Poisson-type Jacobi iteration):  u_{t+1} = S(u_t) + d * f
 *   wave   (leapfrog):                       u_{n+1} = S(u_n) + d * u_{n-1}
 *
 * with S = Eq. (1) (compute_kernel above) and the extra term added to the
 * finished Eq. (1) value of the same interior point.  Shells are frozen: every
 * written grid carries the shell of `in` (source) or of `u` (wave).
 */
static void add_scaled(const double *g, double d, double *dst, long nx, long ny,
                       long nz, int r) {
    const long px = nx + 2 * r, py = ny + 2 * r;
    for (long k = r; k < nz + r; ++k)
        for (long j = r; j < ny + r; ++j)
            for (long i = r; i < nx + r; ++i)
                dst[idx3(i, j, k, px, py)] += d * g[idx3(i, j, k, px, py)];
}

/* iters sweeps u <- S(u) + d f from `in`; result in `out` (in, f read only). */
int oracle_source(const double *in, const double *f, double d, double *out,
                  long nx, long ny, long nz, int r, const double *c, int iters,
                  int nthreads) {
    if (!in || !f || !out || !c || nx < 1 || ny < 1 || nz < 1 || r < 1 || iters < 0)
        return ORACLE_EINVAL;
    if (nthreads < 1) nthreads = 1;
    const long n = (nx + 2 * r) * (ny + 2 * r) * (nz + 2 * r);
    double *a = (double *)malloc(sizeof(double) * (size_t)n);
    double *b = (double *)malloc(sizeof(double) * (size_t)n);
    if (!a || !b) { free(a); free(b); return ORACLE_ENOMEM; }
    memcpy(a, in, sizeof(double) * (size_t)n);
    memcpy(b, in, sizeof(double) * (size_t)n);
    for (int t = 0; t < iters; ++t) {
        compute_kernel(a, b, nx, ny, nz, r, c, nthreads);
        add_scaled(f, d, b, nx, ny, nz, r);
        double *tmp = a; a = b; b = tmp;
    }
    memcpy(out, a, sizeof(double) * (size_t)n);
    free(a);
    free(b);
    return ORACLE_OK;
}

/* iters leapfrog steps in place: (u_prev, u) = (state n-1, n) -> (n+iters-1, n+iters). */
int oracle_wave(double *u_prev, double *u, double d, long nx, long ny, long nz,
                int r, const double *c, int iters, int nthreads) {
    if (!u_prev || !u || !c || nx < 1 || ny < 1 || nz < 1 || r < 1 || iters < 0)
        return ORACLE_EINVAL;
    if (nthreads < 1) nthreads = 1;
    const long n = (nx + 2 * r) * (ny + 2 * r) * (nz + 2 * r);
    double *next = (double *)malloc(sizeof(double) * (size_t)n);
    if (!next) return ORACLE_ENOMEM;
    memcpy(next, u, sizeof(double) * (size_t)n);    /* shell of every state = u's shell */
    if (iters > 0) {
        /* u_prev takes u's shell too (reading R1: the boundary is frozen in time) */
        double *tmp = (double *)malloc(sizeof(double) * (size_t)n);
        if (!tmp) { free(next); return ORACLE_ENOMEM; }
        memcpy(tmp, u, sizeof(double) * (size_t)n);
        const long px = nx + 2 * r, py = ny + 2 * r;
        for (long k = r; k < nz + r; ++k)
            for (long j = r; j < ny + r; ++j)
                for (long i = r; i < nx + r; ++i)
                    tmp[idx3(i, j, k, px, py)] = u_prev[idx3(i, j, k, px, py)];
        memcpy(u_prev, tmp, sizeof(double) * (size_t)n);
        free(tmp);
    }
    for (int t = 0; t < iters; ++t) {
        compute_kernel(u, next, nx, ny, nz, r, c, nthreads);   /* next = S(u_n) */
        add_scaled(u_prev, d, next, nx, ny, nz, r);             /*      + d u_{n-1} */
        memcpy(u_prev, u, sizeof(double) * (size_t)n);          /* (u_{n-1}, u_n) <- (u_n, u_{n+1}) */
        memcpy(u, next, sizeof(double) * (size_t)n);
    }
    free(next);
    return ORACLE_OK;
}

/*
 * Table V application stencils with several grids: Div (3 inputs
 * -> 1 output) and Grad (1 input -> 3 outputs).  The paper benchmarks them but
 * takes their definitions from [17] (Christen's framework, not in
 * PAPER.md); reading R19 fixes them as the order-2r central first
 * derivatives with one coefficient set a_1..a_r (a_m multiplies the
 * difference f[+m] - f[-m]; for h = 1 the FD weights are
 * a_m = (-1)^(m+1) (r!)^2 / (m (r-m)! (r+m)!), e.g. r = 1: a_1 = 1/2):
 *   Div : out = sum_m a_m * ((u[i+m]-u[i-m]) + (v[j+m]-v[j-m]) + (w[k+m]-w[k-m]))
 *   Grad: gx = sum_m a_m * (f[i+m]-f[i-m]),  gy (j),  gz (k)
 * One application (no Fig. 1 loop: input and output grids differ in kind).
 * Interior points only; the shell of every output is set to 0.  Summed as
 * written: m = 1..r, the three differences in the order x, y, z.
 */
int oracle_div(const double *u, const double *v, const double *w, double *out, long nx, long ny, long nz,
               int r, const double *a, int nthreads) {
    if (!u || !v || !w || !out || !a || nx < 1 || ny < 1 || nz < 1 || r < 1) return ORACLE_EINVAL;
    if (nthreads < 1) nthreads = 1;
    const long px = nx + 2 * r, py = ny + 2 * r;
    memset(out, 0, sizeof(double) * (size_t)(px * py * (nz + 2 * r)));
    long k;
    (void)nthreads;
#ifdef _OPENMP
#pragma omp parallel for num_threads(nthreads) schedule(static)
#endif
    for (k = r; k < nz + r; ++k)
        for (long j = r; j < ny + r; ++j)
            for (long i = r; i < nx + r; ++i) {
                double acc = 0.0;
                for (int m = 1; m <= r; ++m) {
                    double d = (u[idx3(i + m, j, k, px, py)] - u[idx3(i - m, j, k, px, py)])
                             + (v[idx3(i, j + m, k, px, py)] - v[idx3(i, j - m, k, px, py)])
                             + (w[idx3(i, j, k + m, px, py)] - w[idx3(i, j, k - m, px, py)]);
                    acc += a[m - 1] * d;
                }
                out[idx3(i, j, k, px, py)] = acc;
            }
    return ORACLE_OK;
}

int oracle_grad(const double *f, double *gx, double *gy, double *gz, long nx, long ny, long nz, int r,
                const double *a, int nthreads) {
    if (!f || !gx || !gy || !gz || !a || nx < 1 || ny < 1 || nz < 1 || r < 1) return ORACLE_EINVAL;
    if (nthreads < 1) nthreads = 1;
    const long px = nx + 2 * r, py = ny + 2 * r;
    const size_t n = (size_t)(px * py * (nz + 2 * r));
    memset(gx, 0, sizeof(double) * n);
    memset(gy, 0, sizeof(double) * n);
    memset(gz, 0, sizeof(double) * n);
    long k;
    (void)nthreads;
#ifdef _OPENMP
#pragma omp parallel for num_threads(nthreads) schedule(static)
#endif
    for (k = r; k < nz + r; ++k)
        for (long j = r; j < ny + r; ++j)
            for (long i = r; i < nx + r; ++i) {
                double sx = 0.0, sy = 0.0, sz = 0.0;
                for (int m = 1; m <= r; ++m) {
                    sx += a[m - 1] * (f[idx3(i + m, j, k, px, py)] - f[idx3(i - m, j, k, px, py)]);
                    sy += a[m - 1] * (f[idx3(i, j + m, k, px, py)] - f[idx3(i, j - m, k, px, py)]);
                    sz += a[m - 1] * (f[idx3(i, j, k + m, px, py)] - f[idx3(i, j, k - m, px, py)]);
                }
                gx[idx3(i, j, k, px, py)] = sx;
                gy[idx3(i, j, k, px, py)] = sy;
                gz[idx3(i, j, k, px, py)] = sz;
            }
    return ORACLE_OK;
}
