/*
 * spade_gen.h — seeded, counter-based synthetic POINT generator (input data only).
 *
 * This module holds none of the method's arithmetic: it only manufactures input coordinates.
 * It is the one piece both sides use — the CUDA product path gets its device-resident inputs
 * from gen_device.cu, the CPU oracle gets bit-identical samples from gen_host.c — so that a
 * 1 G-point shard generated on a GPU can be re-created for any index on the host.
 *
 * Every point is a pure function pt(kind, params, seed, global_index): integer-only
 * (splitmix64 + multiply-shift + Irwin-Hall sums), no libm, no state.
 *
 * Workload shapes: "taxi-like" clustered points mimic the
 * NYC Taxi pickups of PAPER.md Table 1: a Zipf-weighted mixture of Gaussian-ish clusters
 * (some sheared into streaks) plus a uniform background; "uniform" points fill a box.
 */
#ifndef SPADE_GEN_H
#define SPADE_GEN_H

#include <stdint.h>

#ifdef __CUDACC__
#define SG_FN __host__ __device__ static inline
#else
#define SG_FN static inline
#endif

#define SG_MAX_CLUSTERS 64

enum { SG_KIND_UNIFORM = 0, SG_KIND_TAXI = 1 };

typedef struct {
    int32_t kind;                 /* SG_KIND_* */
    int32_t ncl;                  /* clusters (taxi), <= SG_MAX_CLUSTERS */
    int32_t x0, y0;               /* box origin */
    int32_t w, h;                 /* box size: points in [x0, x0+w) x [y0, y0+h) */
    uint32_t bg_thresh;           /* taxi: background point iff (r0 >> 32) < bg_thresh */
    uint32_t cum[SG_MAX_CLUSTERS];/* taxi: cumulative cluster weights on a 2^32 scale */
    int32_t cx[SG_MAX_CLUSTERS], cy[SG_MAX_CLUSTERS];   /* cluster centres */
    int32_t sx[SG_MAX_CLUSTERS], sy[SG_MAX_CLUSTERS];   /* cluster spreads */
    int32_t shear[SG_MAX_CLUSTERS];                     /* streak shear, 1/256 units */
} sg_params;

SG_FN uint64_t sg_mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* k-th 64-bit random word of point `idx` under `seed`. */
SG_FN uint64_t sg_word(uint64_t seed, uint64_t idx, uint32_t k) {
    return sg_mix64(sg_mix64(seed ^ (0xD1B54A32D192ED03ull * (uint64_t)(k + 1))) ^ (idx * 0xA24BAED4963EE407ull));
}

/* uniform integer in [0, range) from 32 random bits (multiply-shift). */
SG_FN int64_t sg_below(uint32_t r, uint32_t range) { return (int64_t)(((uint64_t)r * range) >> 32); }

/* Irwin-Hall(4) centred sum of four 16-bit uniforms: range [-131070, 131070], sd ~ 37837. */
SG_FN int64_t sg_ih4(uint64_t r) {
    int64_t s = (int64_t)(r & 0xFFFF) + (int64_t)((r >> 16) & 0xFFFF) + (int64_t)((r >> 32) & 0xFFFF) +
                (int64_t)((r >> 48) & 0xFFFF);
    return s - 131070;
}

SG_FN int64_t sg_clamp(int64_t v, int64_t lo, int64_t hi) { return v < lo ? lo : (v > hi ? hi : v); }

/* The point with global index `idx`. */
SG_FN void sg_point(const sg_params* p, uint64_t seed, uint64_t idx, int32_t* ox, int32_t* oy) {
    uint64_t r0 = sg_word(seed, idx, 0);
    uint64_t r1 = sg_word(seed, idx, 1);
    int64_t x, y;
    if (p->kind == SG_KIND_UNIFORM || (uint32_t)(r0 >> 32) < p->bg_thresh) {
        x = p->x0 + sg_below((uint32_t)r1, (uint32_t)p->w);
        y = p->y0 + sg_below((uint32_t)(r1 >> 32), (uint32_t)p->h);
    } else {
        uint32_t u = (uint32_t)r0;
        int c = 0;
        while (c < p->ncl - 1 && u >= p->cum[c]) ++c;
        uint64_t r2 = sg_word(seed, idx, 2);
        int64_t dx = sg_ih4(r1) * p->sx[c] / 65536;         /* C division: truncation, both sides */
        int64_t dy = sg_ih4(r2) * p->sy[c] / 65536 + dx * p->shear[c] / 256;
        x = sg_clamp((int64_t)p->cx[c] + dx, p->x0, (int64_t)p->x0 + p->w - 1);
        y = sg_clamp((int64_t)p->cy[c] + dy, p->y0, (int64_t)p->y0 + p->h - 1);
    }
    *ox = (int32_t)x;
    *oy = (int32_t)y;
}

#endif /* SPADE_GEN_H */
