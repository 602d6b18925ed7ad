/*
 * gen.c — seeded synthetic-input generators shared by the oracle tests and the
 * CUDA-path tests/bench (reading c12).  Holds NONE of the
 * method's arithmetic: it only fills host buffers with counter-based random
 * values so that both sides see identical inputs.
 *
 *   v(seed, i) = splitmix64(seed + i),  i = y*w + x over GLOBAL coordinates,
 *   so every rank can generate only its own rows.
 *   Life cell   = v >> 63                     (p = 0.5)
 *   f32 field   = (v >> 40) * 2^-24           in [0,1), exact in fp32
 *   weights t   = ((v_t >> 40) + 1) * 2^-24, normalised to sum 1 in double,
 *                 then rounded to f32 (non-negative, asymmetric)
 */
#include <stdint.h>

static inline uint64_t splitmix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

uint64_t mapsm_gen_splitmix64(uint64_t x) { return splitmix64(x); }

/* rows x w bytes starting at global row y0; row stride = pitch bytes. */
void mapsm_gen_life_u8(uint64_t seed, int64_t w, int64_t y0, int64_t rows, uint8_t* out,
                       int64_t pitch) {
#pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < rows; ++y) {
        uint64_t base = seed + (uint64_t)(y0 + y) * (uint64_t)w;
        uint8_t* o = out + y * pitch;
        for (int64_t x = 0; x < w; ++x) o[x] = (uint8_t)(splitmix64(base + (uint64_t)x) >> 63);
    }
}

/* rows x w floats starting at global row y0; row stride = pitch floats. */
void mapsm_gen_field_f32(uint64_t seed, int64_t w, int64_t y0, int64_t rows, float* out,
                         int64_t pitch) {
#pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < rows; ++y) {
        uint64_t base = seed + (uint64_t)(y0 + y) * (uint64_t)w;
        float* o = out + y * pitch;
        for (int64_t x = 0; x < w; ++x)
            o[x] = (float)(splitmix64(base + (uint64_t)x) >> 40) * (1.0f / 16777216.0f);
    }
}

/* (2r+1)^2 weights, row-major over (dy,dx). */
void mapsm_gen_weights_f32(uint64_t seed, int r, float* out) {
    int k = 2 * r + 1, taps = k * k;
    double raw[81 * 4], sum = 0.0;
    if (taps > 81 * 4) return;
    for (int t = 0; t < taps; ++t) {
        raw[t] = (double)((splitmix64(seed + (uint64_t)t) >> 40) + 1) * (1.0 / 16777216.0);
        sum += raw[t];
    }
    for (int t = 0; t < taps; ++t) out[t] = (float)(raw[t] / sum);
}

/* `taps` weights by the same recipe (Window(3D): (2r+1)^3, ordered (dz,dy,dx)). */
int mapsm_gen_weights_n_f32(uint64_t seed, int taps, float* out) {
    double raw[4096], sum = 0.0;
    if (taps < 1 || taps > 4096) return -1;
    for (int t = 0; t < taps; ++t) {
        raw[t] = (double)((splitmix64(seed + (uint64_t)t) >> 40) + 1) * (1.0 / 16777216.0);
        sum += raw[t];
    }
    for (int t = 0; t < taps; ++t) out[t] = (float)(raw[t] / sum);
    return 0;
}

/* u8 images for the histogram (Reductive-Static) path, rows [y0, y0+rows),
 * row stride `pitch` bytes.  kind 0: uniform, pixel = v >> 56.
 * kind 1: skewed ("natural-image-like" concentration around 128 that makes
 * bins collide): the mean of the 4 high bytes of v, rounded down. */
void mapsm_gen_image_u8(uint64_t seed, int64_t w, int64_t y0, int64_t rows, uint8_t* out, int64_t pitch,
                        int kind) {
#pragma omp parallel for schedule(static)
    for (int64_t y = 0; y < rows; ++y) {
        uint64_t base = seed + (uint64_t)(y0 + y) * (uint64_t)w;
        uint8_t* o = out + y * pitch;
        for (int64_t x = 0; x < w; ++x) {
            uint64_t v = splitmix64(base + (uint64_t)x);
            if (kind == 0) {
                o[x] = (uint8_t)(v >> 56);
            } else {
                unsigned s = (unsigned)((v >> 56) & 255) + (unsigned)((v >> 48) & 255) + (unsigned)((v >> 40) & 255) +
                             (unsigned)((v >> 32) & 255);
                o[x] = (uint8_t)(s / 4);
            }
        }
    }
}
