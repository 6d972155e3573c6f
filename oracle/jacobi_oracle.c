/*
 * jacobi_oracle.c — plain, slow, obviously-correct CPU oracle for the CPU-Free Jacobi path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code, header,
 * table or constant generator with the CUDA path under paper_conf_sc_baydamirlibu24_b200/.
 *
 * What it computes (PAPER.md, /root/reference):
 *   - P:195-197 (§2.1): the Jacobi method for the Laplace equation  Δu = 0 on Ω \ ∂Ω,
 *     i.e. Dirichlet data on ∂Ω.  The formula is garbled in the text; reading R1
 *     takes the standard Jacobi sweep for the discrete Laplacian: the new value of every
 *     interior cell is the mean of its 4 (2D, "2D5pt") or 6 (3D, "3D7pt")
 *     face neighbours, no centre term.
 *   - P:355 (Listing 4.1): a fixed number of iterations `num_iterations`.
 *   - P:394 (§4.1.1): every iteration reads only values of the previous time step
 *     (out-of-place, double-buffered Jacobi — not Gauss-Seidel).
 *   - P:350 (Ch.4): slab decomposition does not change the result, so the oracle is the
 *     undecomposed global sweep.
 * Arithmetic (readings R2-R4): IEEE binary64, round-to-nearest-even, summed left
 * to right in the order x+1, x-1, y+1, y-1 (then z+1, z-1), then ONE multiplication by
 * 0.25 (2D) or by fl(1/6) = 0x1.5555555555555p-3 (3D).  Build with -ffp-contract=off and
 * without -ffast-math (no FMA, no FTZ/DAZ).
 *
 * Layout: row-major, x fastest, idx = (z*ny + y)*nx + x; 2D is nz == 1.  Extents include
 * the Dirichlet layer (reading R7).  Boundary cells are never written.
 *
 * The OpenMP pragma only splits the outermost loop across host threads; every cell update
 * is independent inside one sweep, so the result is bitwise identical for any thread count.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_C6 0x1.5555555555555p-3 /* fl(1/6), reading R3 */

/* One Jacobi sweep of the 2D 5-point stencil: b <- J(a) on interior cells. */
static void sweep_2d(int64_t nx, int64_t ny, const double *a, double *b, int nthreads)
{
    (void)nthreads;
#pragma omp parallel for num_threads(nthreads) schedule(static)
    for (int64_t y = 1; y < ny - 1; ++y) {
        for (int64_t x = 1; x < nx - 1; ++x) {
            int64_t c = y * nx + x;
            double e = a[c + 1];   /* x+1 */
            double w = a[c - 1];   /* x-1 */
            double n = a[c + nx];  /* y+1 */
            double s = a[c - nx];  /* y-1 */
            double sum = e + w;
            sum = sum + n;
            sum = sum + s;
            b[c] = 0.25 * sum;
        }
    }
}

/* One Jacobi sweep of the 3D 7-point stencil: b <- J(a) on interior cells. */
static void sweep_3d(int64_t nx, int64_t ny, int64_t nz, const double *a, double *b, int nthreads)
{
    (void)nthreads;
    const int64_t plane = nx * ny;
#pragma omp parallel for num_threads(nthreads) schedule(static)
    for (int64_t z = 1; z < nz - 1; ++z) {
        for (int64_t y = 1; y < ny - 1; ++y) {
            for (int64_t x = 1; x < nx - 1; ++x) {
                int64_t c = z * plane + y * nx + x;
                double sum = a[c + 1] + a[c - 1]; /* x+1, x-1 */
                sum = sum + a[c + nx];            /* y+1 */
                sum = sum + a[c - nx];            /* y-1 */
                sum = sum + a[c + plane];         /* z+1 */
                sum = sum + a[c - plane];         /* z-1 */
                b[c] = ORACLE_C6 * sum;
            }
        }
    }
}

/*
 * oracle_jacobi: run `iters` Jacobi iterations on the field `in` (nx*ny*nz doubles,
 * boundary included) and write the result to `out` (may alias `in`).
 * stencil: 5 (2D, nz must be 1) or 7 (3D, nz >= 3).  nthreads <= 0 means 1.
 * Returns 0 on success, -1 on invalid arguments, -5 if memory allocation fails.
 */
int oracle_jacobi(int64_t nx, int64_t ny, int64_t nz, int stencil, int64_t iters,
                  const double *in, double *out, int nthreads)
{
    if (nx < 3 || ny < 3 || iters < 0 || !in || !out) return -1;
    if (stencil == 5 && nz != 1) return -1;
    if (stencil == 7 && nz < 3) return -1;
    if (stencil != 5 && stencil != 7) return -1;
    if (nthreads <= 0) nthreads = 1;
    size_t n = (size_t)(nx * ny * nz);
    double *a = (double *)malloc(n * sizeof(double));
    double *b = (double *)malloc(n * sizeof(double));
    if (!a || !b) { free(a); free(b); return -5; }
    /* Both buffers start identical, boundary included (reading R10). */
    memcpy(a, in, n * sizeof(double));
    memcpy(b, in, n * sizeof(double));
    for (int64_t t = 0; t < iters; ++t) {
        if (stencil == 5) sweep_2d(nx, ny, a, b, nthreads);
        else              sweep_3d(nx, ny, nz, a, b, nthreads);
        double *tmp = a; a = b; b = tmp;  /* swap: the new field is the next "previous step" */
    }
    memcpy(out, a, n * sizeof(double));
    free(a);
    free(b);
    return 0;
}

/* Number of host threads OpenMP would use by default (1 without OpenMP). */
int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
