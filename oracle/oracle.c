/*
 * oracle.c — TEST INFRASTRUCTURE ONLY.  Plain, slow, obviously-correct CPU
 * implementation of the MAPS-Multi Window(2D) -> Structured-Injective hot path
 * (an iterated radius-r 2D stencil), written from the paper, never from the
 * CUDA path.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference leg may load this library.  It shares no
 * code, header, table or constant with paper_conf_sc_ben_nunlbr15_b200/.
 *
 * Citations are to /root/reference/PAPER.md lines ("P:L<n> §<sec>") and to
 * the readings listed in DESIGN.md §3 ("reading c<k>").
 *
 * What it computes
 *   Game of Life (§4: "each cell processes information from its 8
 *   neighbors", Window(2D) radius 1, WRAP (Fig 2a line 1); rule
 *   B3/S23 of Gardner [14], reading c1):
 *       N(y,x)  = sum over the 8 (dy,dx) != (0,0) of cell(G, y+dy, x+dx)
 *       G'(y,x) = (N == 3) || (G(y,x) && N == 2)
 *   applied synchronously n times (double buffering; reading
 *   c6).  Generation n is returned (reading c7); n = 0 returns the input
 *   normalised to 0/1 (reading c2: nonzero byte = alive).
 *
 *   Window convolution (Table 1 P:L87-88 "N-dimensional convolution"; the
 *   float case of BASELINE.json north_star), cross-correlation, radius r:
 *       acc = +0.0f
 *       for dy = -r..r: for dx = -r..r:
 *           acc = fmaf(W[(dy+r)(2r+1) + (dx+r)], cell(in, y+dy, x+dx), acc)
 *       out(y,x) = acc
 *   (readings c9, c11: no kernel flip, row-major taps, one correctly rounded
 *   fmaf per tap, RN-even).  A second variant accumulates in double for error
 *   reporting.
 *
 *   cell(G,y,x): boundary lookup per side (reading c3/c4/c5):
 *       WRAP  -> G[y mod h][x mod w] (mathematical mod, both sides of the axis)
 *       CLAMP -> G[clamp(y,0,h-1)][clamp(x,0,w-1)]
 *       ZERO  -> 0 outside the grid
 *   Each of the four sides takes its own mode so that tests can evaluate a
 *   sub-window ("cone") of a large grid with ZERO on cut sides; WRAP must be
 *   given for both sides of an axis or for neither.
 *
 * Build: gcc -O2 -fopenmp -ffp-contract=off -fPIC -shared (no -ffast-math; no
 * FTZ/DAZ) — see __init__.py.  OpenMP only parallelises over output rows; each
 * cell is evaluated exactly as written above.
 */
#include <math.h>
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_WRAP 0
#define ORACLE_CLAMP 1
#define ORACLE_ZERO 2

/* Mathematical modulus: result in [0, n). */
static int64_t mod_floor(int64_t i, int64_t n) {
    int64_t m = i % n;
    return m < 0 ? m + n : m;
}

/* Resolve one coordinate against its side modes.  Returns -1 if the cell is
 * outside under ZERO (value 0), else the in-range index. */
static int64_t resolve(int64_t i, int64_t n, int mode_lo, int mode_hi) {
    if (i >= 0 && i < n) return i;
    int mode = (i < 0) ? mode_lo : mode_hi;
    if (mode == ORACLE_WRAP) return mod_floor(i, n);
    if (mode == ORACLE_CLAMP) return i < 0 ? 0 : n - 1;
    return -1; /* ZERO */
}

static int check_modes(int top, int bottom, int left, int right) {
    int ok = 1;
    if ((top == ORACLE_WRAP) != (bottom == ORACLE_WRAP)) ok = 0;
    if ((left == ORACLE_WRAP) != (right == ORACLE_WRAP)) ok = 0;
    int m[4] = {top, bottom, left, right};
    for (int i = 0; i < 4; ++i)
        if (m[i] < 0 || m[i] > 2) ok = 0;
    return ok;
}

/* ---------------------------------------------------------------- Life */

static uint8_t life_cell(const uint8_t* G, int64_t w, int64_t h, int64_t y, int64_t x,
                         int top, int bottom, int left, int right) {
    int64_t yy = resolve(y, h, top, bottom);
    int64_t xx = resolve(x, w, left, right);
    if (yy < 0 || xx < 0) return 0;
    return G[yy * w + xx] != 0;
}

static void life_generation(const uint8_t* G, uint8_t* out, int64_t w, int64_t h,
                            int top, int bottom, int left, int right) {
#pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < h; ++y) {
        for (int64_t x = 0; x < w; ++x) {
            int N = 0;
            for (int dy = -1; dy <= 1; ++dy)
                for (int dx = -1; dx <= 1; ++dx) {
                    if (dy == 0 && dx == 0) continue;
                    N += life_cell(G, w, h, y + dy, x + dx, top, bottom, left, right);
                }
            int alive = G[y * w + x] != 0;
            out[y * w + x] = (uint8_t)((N == 3) || (alive && N == 2));
        }
    }
}

/* out <- generation n of `in` (h rows x w bytes, row-major, row stride w).
 * Returns 0, or -1 on invalid arguments / allocation failure. */
int oracle_life_ex(const uint8_t* in, uint8_t* out, int64_t w, int64_t h, int64_t n,
                   int top, int bottom, int left, int right) {
    if (w <= 0 || h <= 0 || n < 0 || !check_modes(top, bottom, left, right)) return -1;
    size_t cells = (size_t)w * (size_t)h;
    uint8_t* a = (uint8_t*)malloc(cells);
    uint8_t* b = (uint8_t*)malloc(cells);
    if (!a || !b) { free(a); free(b); return -1; }
    for (size_t i = 0; i < cells; ++i) a[i] = in[i] != 0;
    for (int64_t t = 0; t < n; ++t) {
        life_generation(a, b, w, h, top, bottom, left, right);
        uint8_t* tmp = a; a = b; b = tmp;
    }
    memcpy(out, a, cells);
    free(a);
    free(b);
    return 0;
}

int oracle_life(const uint8_t* in, uint8_t* out, int64_t w, int64_t h, int64_t n, int boundary) {
    return oracle_life_ex(in, out, w, h, n, boundary, boundary, boundary, boundary);
}

/* ---------------------------------------------------------- Convolution */

static float conv_cell(const float* G, int64_t w, int64_t h, int64_t y, int64_t x,
                       int top, int bottom, int left, int right) {
    int64_t yy = resolve(y, h, top, bottom);
    int64_t xx = resolve(x, w, left, right);
    if (yy < 0 || xx < 0) return 0.0f;
    return G[yy * w + xx];
}

static void conv_step_f32(const float* G, float* out, int64_t w, int64_t h, int r,
                          const float* W, int top, int bottom, int left, int right) {
    int k = 2 * r + 1;
#pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < h; ++y) {
        for (int64_t x = 0; x < w; ++x) {
            float acc = 0.0f;
            for (int dy = -r; dy <= r; ++dy)
                for (int dx = -r; dx <= r; ++dx)
                    acc = fmaf(W[(dy + r) * k + (dx + r)],
                               conv_cell(G, w, h, y + dy, x + dx, top, bottom, left, right), acc);
            out[y * w + x] = acc;
        }
    }
}

/* fp32, fixed tap order (reading c11).  Returns 0 or -1. */
int oracle_conv_ex(const float* in, float* out, int64_t w, int64_t h, int64_t n, int r,
                   const float* weights, int top, int bottom, int left, int right) {
    if (w <= 0 || h <= 0 || n < 0 || r < 0 || !check_modes(top, bottom, left, right)) return -1;
    size_t cells = (size_t)w * (size_t)h;
    float* a = (float*)malloc(cells * sizeof(float));
    float* b = (float*)malloc(cells * sizeof(float));
    if (!a || !b) { free(a); free(b); return -1; }
    memcpy(a, in, cells * sizeof(float));
    for (int64_t t = 0; t < n; ++t) {
        conv_step_f32(a, b, w, h, r, weights, top, bottom, left, right);
        float* tmp = a; a = b; b = tmp;
    }
    memcpy(out, a, cells * sizeof(float));
    free(a);
    free(b);
    return 0;
}

int oracle_conv(const float* in, float* out, int64_t w, int64_t h, int64_t n, int r,
                const float* weights, int boundary) {
    return oracle_conv_ex(in, out, w, h, n, r, weights, boundary, boundary, boundary, boundary);
}

/* fp64 accumulation (for error reporting): the field is carried in double
 * between iterations; weights are the same fp32 values widened. */
static void conv_step_f64(const double* G, double* out, int64_t w, int64_t h, int r,
                          const float* W, int top, int bottom, int left, int right) {
    int k = 2 * r + 1;
#pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < h; ++y) {
        for (int64_t x = 0; x < w; ++x) {
            double acc = 0.0;
            for (int dy = -r; dy <= r; ++dy)
                for (int dx = -r; dx <= r; ++dx) {
                    int64_t yy = resolve(y + dy, h, top, bottom);
                    int64_t xx = resolve(x + dx, w, left, right);
                    double v = (yy < 0 || xx < 0) ? 0.0 : G[yy * w + xx];
                    acc = fma((double)W[(dy + r) * k + (dx + r)], v, acc);
                }
            out[y * w + x] = acc;
        }
    }
}

int oracle_conv_f64_ex(const float* in, double* out, int64_t w, int64_t h, int64_t n, int r,
                       const float* weights, int top, int bottom, int left, int right) {
    if (w <= 0 || h <= 0 || n < 0 || r < 0 || !check_modes(top, bottom, left, right)) return -1;
    size_t cells = (size_t)w * (size_t)h;
    double* a = (double*)malloc(cells * sizeof(double));
    double* b = (double*)malloc(cells * sizeof(double));
    if (!a || !b) { free(a); free(b); return -1; }
    for (size_t i = 0; i < cells; ++i) a[i] = (double)in[i];
    for (int64_t t = 0; t < n; ++t) {
        conv_step_f64(a, b, w, h, r, weights, top, bottom, left, right);
        double* tmp = a; a = b; b = tmp;
    }
    memcpy(out, a, cells * sizeof(double));
    free(a);
    free(b);
    return 0;
}

int oracle_conv_f64(const float* in, double* out, int64_t w, int64_t h, int64_t n, int r,
                    const float* weights, int boundary) {
    return oracle_conv_f64_ex(in, out, w, h, n, r, weights, boundary, boundary, boundary, boundary);
}

/* ------------------------------------------------------ Window (3D) */

/* Window (3D) input pattern (§5.3: "each image in the batch is
 * separately convolved in three dimensions ... This corresponds to the Window
 * (3D) input memory access pattern, using the Structured Injective output";
 * Table 1 P:L87-88 "N-dimensional convolution").  A d x h
 * x w fp32 volume (plane-major: index (z*h + y)*w + x), cross-correlation with
 * (2r+1)^3 weights ordered (dz, dy, dx) row-major, one correctly rounded fmaf
 * per tap starting from +0.0f (the 3-D extension of reading c11, DESIGN.md
 * reading v1):
 *     acc = +0.0f
 *     for dz = -r..r: for dy = -r..r: for dx = -r..r:
 *         acc = fmaf(W[((dz+r)(2r+1) + (dy+r))(2r+1) + (dx+r)], cell(z+dz, y+dy, x+dx), acc)
 * cell() resolves each axis with its own side modes exactly as in 2-D. */
static float conv3_cell(const float* G, int64_t w, int64_t h, int64_t d, int64_t z, int64_t y, int64_t x,
                        const int* m) {
    int64_t zz = resolve(z, d, m[0], m[1]);
    int64_t yy = resolve(y, h, m[2], m[3]);
    int64_t xx = resolve(x, w, m[4], m[5]);
    if (zz < 0 || yy < 0 || xx < 0) return 0.0f;
    return G[(zz * h + yy) * w + xx];
}

static void conv3_step_f32(const float* G, float* out, int64_t w, int64_t h, int64_t d, int r, const float* W,
                           const int* m) {
    int k = 2 * r + 1;
#pragma omp parallel for schedule(static) collapse(2)
    for (int64_t z = 0; z < d; ++z)
        for (int64_t y = 0; y < h; ++y)
            for (int64_t x = 0; x < w; ++x) {
                float acc = 0.0f;
                for (int dz = -r; dz <= r; ++dz)
                    for (int dy = -r; dy <= r; ++dy)
                        for (int dx = -r; dx <= r; ++dx)
                            acc = fmaf(W[((dz + r) * k + (dy + r)) * k + (dx + r)],
                                       conv3_cell(G, w, h, d, z + dz, y + dy, x + dx, m), acc);
                out[(z * h + y) * w + x] = acc;
            }
}

/* n steps; modes[6] = (z lo, z hi, y lo, y hi, x lo, x hi).  Returns 0 or -1. */
int oracle_conv3d_ex(const float* in, float* out, int64_t w, int64_t h, int64_t d, int64_t n, int r,
                     const float* weights, const int* modes) {
    if (w <= 0 || h <= 0 || d <= 0 || n < 0 || r < 0 || !modes) return -1;
    if (!check_modes(modes[0], modes[1], modes[2], modes[3]) || !check_modes(modes[4], modes[5], modes[4], modes[5]))
        return -1;
    size_t cells = (size_t)w * (size_t)h * (size_t)d;
    float* a = (float*)malloc(cells * sizeof(float));
    float* b = (float*)malloc(cells * sizeof(float));
    if (!a || !b) { free(a); free(b); return -1; }
    memcpy(a, in, cells * sizeof(float));
    for (int64_t t = 0; t < n; ++t) {
        conv3_step_f32(a, b, w, h, d, r, weights, modes);
        float* tmp = a; a = b; b = tmp;
    }
    memcpy(out, a, cells * sizeof(float));
    free(a);
    free(b);
    return 0;
}

/* ------------------------------------------------------------ Histogram */

/* Reductive (Static) output pattern (§3.2; Fig 4 P:L359-403 §4.5.3,
 * "auto bin = *image_iter; hist_iter[bin] += 1"): the BINS-bin histogram of a
 * w x h image of u8 pixels, bin = pixel value (reading h1).  Counts are
 * 64-bit (reading h2).  Plain sequential loop over rows and columns; `pitch`
 * is the row stride in bytes (padding bytes are not pixels). */
int oracle_histogram(const uint8_t* img, int64_t w, int64_t h, int64_t pitch, int nbins, uint64_t* bins) {
    if (w < 0 || h < 0 || pitch < w || nbins != 256 || !bins) return -1;
    for (int b = 0; b < nbins; ++b) bins[b] = 0;
    for (int64_t y = 0; y < h; ++y)
        for (int64_t x = 0; x < w; ++x) bins[img[y * pitch + x]] += 1;
    return 0;
}

/* Histogram task over an fp32 field (reading h4): 256
 * bins over [0, 1), bin = floor(v * 256) evaluated in double (v * 256 is
 * exact), below 0 (and NaN) -> bin 0, at or above 256 -> bin 255. */
int oracle_histogram_f32(const float* img, int64_t w, int64_t h, int64_t pitch_floats, int nbins, uint64_t* bins) {
    if (w < 0 || h < 0 || pitch_floats < w || nbins != 256 || !bins) return -1;
    for (int b = 0; b < nbins; ++b) bins[b] = 0;
    for (int64_t y = 0; y < h; ++y)
        for (int64_t x = 0; x < w; ++x) {
            const double s = floor((double)img[y * pitch_floats + x] * 256.0);
            int b;
            if (!(s >= 0.0)) b = 0;
            else if (s > 255.0) b = 255;
            else b = (int)s;
            bins[b] += 1;
        }
    return 0;
}

/* Number of OpenMP threads the oracle will use (for the cpu_baseline record). */
int oracle_num_threads(void) {
    int n = 1;
#pragma omp parallel
    {
#pragma omp single
        n = omp_get_num_threads();
    }
    return n;
}
