/*
 * pathtrace.c -- ORACLE (test infrastructure; see oracle.h).
 *
 * Config 4 (BASELINE.json configs[3]): a path tracer, the paper's
 * "pathtracer" benchmark (Table 2: spheres in a Cornell box,
 * Russian roulette, bounded bounces; "Loop trip count divergence"), whose
 * bounce loop is the inner loop of Fig. 2(b) and whose samples per pixel are
 * the coarsened outer loop:
 *
 *     for (s = 0; s < spp; s++) {          // outer loop, one sample per trip
 *       Prolog: camera ray of sample s
 *       for (b = 0; alive; b++) { L1: bounce() }   // divergent trip count
 *       Epilog: pixel += radiance
 *     }
 *
 * executed literally, one pixel after another, with a BRUTE-FORCE closest hit
 * over every triangle (the plain definition of "closest hit"; no BVH here).
 * DESIGN.md reading R7 fixes every operation; dot(a,b) = (ax*bx + ay*by) + az*bz.
 */
#include <math.h>
#include <string.h>
#include "oracle.h"

typedef struct { float x, y, z; } v3;
static v3 mk(float x, float y, float z) { v3 r = {x, y, z}; return r; }
static v3 sub(v3 a, v3 b) { return mk(a.x - b.x, a.y - b.y, a.z - b.z); }
static v3 add(v3 a, v3 b) { return mk(a.x + b.x, a.y + b.y, a.z + b.z); }
static v3 scl(v3 a, float s) { return mk(a.x * s, a.y * s, a.z * s); }
static float dot(v3 a, v3 b) { return (a.x * b.x + a.y * b.y) + a.z * b.z; }
static v3 cross(v3 a, v3 b) {
  return mk(a.y * b.z - a.z * b.y, a.z * b.x - a.x * b.z, a.x * b.y - a.y * b.x);
}
static v3 normalize(v3 a) {
  float inv = 1.0f / sqrtf(dot(a, a));
  return scl(a, inv);
}

#define PT_TMIN 1.0e-4f
#define PT_DET_EPS 1.0e-12f

/* Moller-Trumbore; returns 1 and *t on a hit with t > PT_TMIN */
static int mt_hit(const float* tri, v3 o, v3 d, float* t_out) {
  v3 v0 = mk(tri[0], tri[1], tri[2]);
  v3 e1 = sub(mk(tri[3], tri[4], tri[5]), v0);
  v3 e2 = sub(mk(tri[6], tri[7], tri[8]), v0);
  v3 pv = cross(d, e2);
  float det = dot(e1, pv);
  if (fabsf(det) < PT_DET_EPS) return 0;
  float inv = 1.0f / det;
  v3 tv = sub(o, v0);
  float u = dot(tv, pv) * inv;
  if (u < 0.0f || u > 1.0f) return 0;
  v3 qv = cross(tv, e1);
  float v = dot(d, qv) * inv;
  if (v < 0.0f || u + v > 1.0f) return 0;
  float t = dot(e2, qv) * inv;
  if (!(t > PT_TMIN)) return 0;
  *t_out = t;
  return 1;
}

int64_t or_pt_closest(const float* tris, uint32_t n_tris, const float o[3], const float d[3],
                      float* t_best) {
  v3 O = mk(o[0], o[1], o[2]), D = mk(d[0], d[1], d[2]);
  int64_t best = -1;
  float tb = INFINITY;
  for (uint32_t i = 0; i < n_tris; ++i) {
    float t;
    if (mt_hit(tris + 9ull * i, O, D, &t) && t < tb) {  /* ascending i: ties keep the smaller id */
      tb = t;
      best = i;
    }
  }
  *t_best = tb;
  return best;
}

static void onb(v3 n, v3* t1, v3* t2) {
  /* Duff et al. 2017, branchless orthonormal basis */
  float sign = copysignf(1.0f, n.z);
  float a = -1.0f / (sign + n.z);
  float b = n.x * n.y * a;
  *t1 = mk(1.0f + sign * n.x * n.x * a, sign * b, -sign * n.x);
  *t2 = mk(b, sign + n.y * n.y * a, -n.y);
}

static void draw(uint32_t event, uint64_t q, uint64_t seed, uint32_t u[4]) {
  uint32_t ctr[4] = {event, (uint32_t)OR_TAG_PT << 16, (uint32_t)q, (uint32_t)(q >> 32)};
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  or_philox4x32_10(ctr, key, u);
}

/* The direction half of a bounce (reading R7), after the hit: ng = the unit
 * geometric normal of the hit triangle, d = the incoming unit direction, u =
 * the bounce's Philox draw, ior = the material's index.  The shading normal n
 * is ng flipped to face the incoming ray; entering = the ray arrives on ng's
 * side.
 *   kind 0 diffuse:    cosine-weighted about n (Malley: a uniform point of the
 *                      unit disk, r = sqrt(U01(u0)), phi = 2 pi U01(u1), lifted
 *                      to the hemisphere), in the Duff et al. basis of n;
 *   kind 1 mirror:     d - 2 (d.n) n;
 *   kind 2 dielectric: eta = 1/ior entering, ior leaving; Schlick reflectance
 *                      F = r0 + (1 - r0)(1 - cos_i)^5, r0 = ((1-ior)/(1+ior))^2;
 *                      reflect if total internal reflection (k < 0) or
 *                      U01(u2) < F, else refract: eta d + (eta cos_i - sqrt(k)) n.
 * Exported so the tests can check each branch against float64 geometry. */
void or_pt_scatter(uint32_t kind, float ior, const float d_in[3], const float ng_in[3],
                   const uint32_t u[4], float d_out[3]) {
  v3 d = mk(d_in[0], d_in[1], d_in[2]), ng = mk(ng_in[0], ng_in[1], ng_in[2]);
  float cosd = dot(ng, d);
  int entering = cosd < 0.0f;
  v3 n = entering ? ng : scl(ng, -1.0f);                /* faces the incoming ray */
  if (kind == 0u) {                                     /* diffuse: cosine-weighted */
    float r1 = or_u01(u[0]);
    float rr = sqrtf(r1);
    float sp, cp;
    or_sr_sincos2pif(or_u01(u[1]), &sp, &cp);
    float lx = rr * cp, ly = rr * sp, lz = sqrtf(1.0f - r1);
    v3 t1, t2;
    onb(n, &t1, &t2);
    d = add(add(scl(t1, lx), scl(t2, ly)), scl(n, lz));
  } else if (kind == 1u) {                              /* mirror */
    d = sub(d, scl(n, 2.0f * dot(d, n)));
  } else {                                              /* dielectric */
    float eta = entering ? 1.0f / ior : ior;
    float cosi = -dot(d, n);
    float k = 1.0f - eta * eta * (1.0f - cosi * cosi);
    float r0 = (1.0f - ior) / (1.0f + ior);
    r0 = r0 * r0;
    float c5 = 1.0f - cosi;
    float fr = r0 + (1.0f - r0) * (c5 * c5 * c5 * c5 * c5);
    if (k < 0.0f || or_u01(u[2]) < fr) {
      d = sub(d, scl(n, 2.0f * dot(d, n)));             /* reflect */
    } else {
      d = add(scl(d, eta), scl(n, eta * cosi - sqrtf(k)));  /* refract */
    }
  }
  d_out[0] = d.x; d_out[1] = d.y; d_out[2] = d.z;
}

/* One path of sample id q for pixel (px, py).  rgb += radiance is done by
 * the caller; counters: [0] bounces (rays traced). */
static v3 trace_path(const or_pt_scene* sc, uint32_t px, uint32_t py, uint64_t q, uint64_t seed,
                     uint32_t width, uint32_t height, uint32_t max_depth, uint64_t* rays) {
  const float* cam = sc->cam;
  v3 eye = mk(cam[0], cam[1], cam[2]), fwd = mk(cam[3], cam[4], cam[5]);
  v3 right = mk(cam[6], cam[7], cam[8]), up = mk(cam[9], cam[10], cam[11]);
  float tan_half = cam[12], aspect = cam[13];
  uint32_t u[4];
  draw(0u, q, seed, u);
  float fx = ((float)px + or_u01(u[0])) / (float)width;
  float fy = ((float)py + or_u01(u[1])) / (float)height;
  float sx = (2.0f * fx - 1.0f) * tan_half * aspect;
  float sy = (1.0f - 2.0f * fy) * tan_half;
  v3 d = normalize(add(add(fwd, scl(right, sx)), scl(up, sy)));
  v3 o = eye;
  v3 thr = mk(1.0f, 1.0f, 1.0f), rad = mk(0.0f, 0.0f, 0.0f);
  for (uint32_t b = 0; b < max_depth; ++b) {
    float t;
    float oo[3] = {o.x, o.y, o.z}, dd[3] = {d.x, d.y, d.z};
    int64_t hit = or_pt_closest(sc->tris, sc->n_tris, oo, dd, &t);
    *rays += 1;
    if (hit < 0) break;                                   /* escaped: black background */
    const float* m = sc->mats + 8u * sc->mat[hit];
    uint32_t kind = (uint32_t)m[0];
    rad = add(rad, mk(thr.x * m[4], thr.y * m[5], thr.z * m[6]));   /* emission */
    if (kind == 3u) break;                                /* light: absorbs */
    const float* tri = sc->tris + 9ull * (uint64_t)hit;
    v3 v0 = mk(tri[0], tri[1], tri[2]);
    v3 e1 = sub(mk(tri[3], tri[4], tri[5]), v0);
    v3 e2 = sub(mk(tri[6], tri[7], tri[8]), v0);
    v3 ng = normalize(cross(e1, e2));
    v3 p = add(o, scl(d, t));
    draw(b + 1u, q, seed, u);
    float dd_in[3] = {d.x, d.y, d.z}, ng3[3] = {ng.x, ng.y, ng.z}, dout[3];
    or_pt_scatter(kind, m[7], dd_in, ng3, u, dout);
    d = mk(dout[0], dout[1], dout[2]);
    thr = mk(thr.x * m[1], thr.y * m[2], thr.z * m[3]);
    o = p;
    if (b >= 3u) {                                        /* Russian roulette */
      float pm = fmaxf(thr.x, fmaxf(thr.y, thr.z));
      float prr = fminf(0.95f, pm);
      if (!(or_u01(u[3]) < prr)) break;
      thr = mk(thr.x / prr, thr.y / prr, thr.z / prr);
    }
  }
  return rad;
}

void or_pt_render(const or_pt_scene* sc, uint32_t width, uint32_t height, uint32_t spp,
                  uint32_t max_depth, uint64_t seed, const uint32_t* pixels, uint32_t n_pixels,
                  float* rgb, uint64_t* counters) {
  for (uint32_t k = 0; k < n_pixels; ++k) {
    uint32_t pix = pixels ? pixels[k] : k;
    uint32_t px = pix % width, py = pix / width;
    v3 sum = mk(0.0f, 0.0f, 0.0f);
    for (uint32_t s = 0; s < spp; ++s) {
      uint64_t q = (uint64_t)pix * spp + s;
      v3 r = trace_path(sc, px, py, q, seed, width, height, max_depth, &counters[1]);
      sum = add(sum, r);
      counters[0] += 1;
    }
    rgb[3u * k + 0] = sum.x;
    rgb[3u * k + 1] = sum.y;
    rgb[3u * k + 2] = sum.z;
  }
}
