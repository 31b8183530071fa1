// pso_oracle.cpp — plain CPU oracle for FastPSO's hot path.
//
// TEST INFRASTRUCTURE ONLY (see pso_oracle.h).  Single-threaded, no blocking,
// no fusion: each function is one step of Alg. 1 in the paper's
// order, with the free choices fixed by the readings in DESIGN.md.
// Build: g++ -O3 -std=c++17 -ffp-contract=off -fPIC -shared.

#include "pso_oracle.h"

#include <cmath>
#include <cstdint>
#include <cstring>
#include <limits>
#include <vector>

namespace {

// ---------------------------------------------------------------------------
// Philox4x32-10 (Salmon, Moraes, Dror, Shaw, SC'11 "Parallel random numbers:
// as easy as 1, 2, 3"; Random123).  The paper draws with Thrust and
// does not name a generator; reading 6 fixes Philox4x32-10.
// ---------------------------------------------------------------------------
const uint32_t kM0 = 0xD2511F53u;  // round multipliers
const uint32_t kM1 = 0xCD9E8D57u;
const uint32_t kW0 = 0x9E3779B9u;  // Weyl key increments
const uint32_t kW1 = 0xBB67AE85u;

void philox(const uint32_t in[4], const uint32_t key[2], uint32_t out[4]) {
  uint32_t c0 = in[0], c1 = in[1], c2 = in[2], c3 = in[3];
  uint32_t k0 = key[0], k1 = key[1];
  for (int round = 0; round < 10; ++round) {
    if (round > 0) {  // key bump between rounds, none after the last
      k0 += kW0;
      k1 += kW1;
    }
    uint64_t p0 = (uint64_t)kM0 * (uint64_t)c0;
    uint64_t p1 = (uint64_t)kM1 * (uint64_t)c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

uint32_t word(uint64_t seed, uint32_t tag, uint32_t t, uint32_t i, uint32_t j) {
  const uint32_t ctr[4] = {j >> 2, i, t, tag};
  const uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  uint32_t out[4];
  philox(ctr, key, out);
  return out[j & 3u];
}

float uniform(uint32_t w) { return (float)(w >> 8) * 0x1p-24f; }

// ---------------------------------------------------------------------------
// Objectives, accumulated in double, k = j+1 is the 1-based dimension index.
// ---------------------------------------------------------------------------
const double kPi = 3.14159265358979323846;

double objective(int32_t obj, const float* x, int32_t d) {
  switch (obj) {
    case ORC_SPHERE: {  // f(x) = sum x_k^2
      double s = 0.0;
      for (int32_t j = 0; j < d; ++j) s += (double)x[j] * (double)x[j];
      return s;
    }
    case ORC_RASTRIGIN: {  // [20]: f(x) = 10 d + sum (x_k^2 - 10 cos(2 pi x_k))
      double s = 0.0;
      for (int32_t j = 0; j < d; ++j) {
        double xj = x[j];
        s += xj * xj + 10.0 - 10.0 * std::cos(2.0 * kPi * xj);
      }
      return s;
    }
    case ORC_ROSENBROCK: {  // [20]: sum_{k<d} 100 (x_{k+1} - x_k^2)^2 + (x_k - 1)^2
      double s = 0.0;
      for (int32_t j = 0; j + 1 < d; ++j) {
        double xj = x[j], xn = x[j + 1];
        double a = xn - xj * xj;
        double b = xj - 1.0;
        s += 100.0 * a * a + b * b;
      }
      return s;
    }
    case ORC_GRIEWANK: {  // 1/4000 sum x_k^2 - prod cos(x_k / sqrt(k)) + 1
      double s = 0.0, p = 1.0;
      for (int32_t j = 0; j < d; ++j) {
        double xj = x[j];
        s += xj * xj;
        p *= std::cos(xj / std::sqrt((double)(j + 1)));
      }
      return s / 4000.0 - p + 1.0;
    }
    case ORC_ACKLEY: {  // [20]: -20 exp(-0.2 sqrt(sum x^2 / d)) - exp(sum cos(2 pi x) / d) + 20 + e
      double s = 0.0, c = 0.0;
      for (int32_t j = 0; j < d; ++j) {
        double xj = x[j];
        s += xj * xj;
        c += std::cos(2.0 * kPi * xj);
      }
      return -20.0 * std::exp(-0.2 * std::sqrt(s / d)) - std::exp(c / d) + 20.0 +
             std::exp(1.0);
    }
    case ORC_EASOM: {  // -(-1)^d prod cos^2(x_k) exp(-sum (x_k - pi)^2)
      double p = 1.0, e = 0.0;
      for (int32_t j = 0; j < d; ++j) {
        double xj = x[j];
        double cj = std::cos(xj);
        p *= cj * cj;
        e += (xj - kPi) * (xj - kPi);
      }
      double sgn = (d % 2 == 0) ? 1.0 : -1.0;  // (-1)^d
      return -sgn * p * std::exp(-e);
    }
    default:
      return std::numeric_limits<double>::quiet_NaN();
  }
}

// ---------------------------------------------------------------------------
// One element of the swarm update: Eq. 1, Eq. 5,
// Eq. 2 and the domain clamp (reading 2).  Fixed fp32 order:
//   a = w*v; b = (c1*r1)*(pb-x); c = (c2*r2)*(g-x); v' = (a+b)+c
// ---------------------------------------------------------------------------
// Bounds of dimension j: Eq. 5's lower/upper velocity bound and the domain.
struct Bounds {
  float vlo, vhi, xlo, xhi;
};
inline Bounds bounds_of(const orc_params* p, int32_t j) {
  if (p->bounds) {
    const int32_t d = p->d;
    return Bounds{p->bounds[j], p->bounds[d + j], p->bounds[2 * d + j], p->bounds[3 * d + j]};
  }
  return Bounds{-p->vmax, p->vmax, p->lo, p->hi};
}

inline void move_element(const orc_params* p, const Bounds& bd, float r1, float r2, float pb,
                         float g, float* x, float* v) {
  float a = p->w * *v;
  float b = (p->c1 * r1) * (pb - *x);
  float c = (p->c2 * r2) * (g - *x);
  float vn = (a + b) + c;
  vn = std::fmin(std::fmax(vn, bd.vlo), bd.vhi);            // Eq. 5
  float xn = std::fmin(std::fmax(*x + vn, bd.xlo), bd.xhi);  // Eq. 2 + clamp
  *v = vn;
  *x = xn;
}

// Move, evaluate and pbest-update one row with global index gi (Alg. 1
// lines 14-16 then 5-9, rotated: reading 7).
void row_step(const orc_params* p, uint32_t t, const float* G, uint32_t gi,
              float* x, float* v, float* pb, float* pf, float* f) {
  const int32_t d = p->d;
  for (int32_t j = 0; j < d; ++j) {
    float r1 = uniform(word(p->seed, ORC_TAG_R1, t, gi, (uint32_t)j));
    float r2 = uniform(word(p->seed, ORC_TAG_R2, t, gi, (uint32_t)j));
    move_element(p, bounds_of(p, j), r1, r2, pb[j], G[j], &x[j], &v[j]);
  }
  float fi = (float)objective(p->objective, x, d);
  *f = fi;
  if (fi < *pf) {  // Alg. 1 line 7, strict; NaN never passes
    *pf = fi;
    std::memcpy(pb, x, sizeof(float) * (size_t)d);
  }
}

// Lexicographic (f, i) order used for the gbest reduction (reading 9).
inline bool lex_less(float fa, int64_t ia, float fb, int64_t ib) {
  return fa < fb || (fa == fb && ia < ib);
}

orc_state shard_view(const orc_state* s, int32_t d, int64_t begin, int64_t count) {
  orc_state v = *s;
  const int64_t off = begin - s->row_begin;
  v.row_begin = begin;
  v.nrows = count;
  v.X = s->X + off * d;
  v.V = s->V + off * d;
  v.PB = s->PB + off * d;
  v.pf = s->pf + off;
  v.f = s->f + off;
  return v;
}

}  // namespace

extern "C" {

void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  philox(ctr, key, out);
}

uint32_t orc_word(uint64_t seed, uint32_t tag, uint32_t t, uint32_t i, uint32_t j) {
  return word(seed, tag, t, i, j);
}

float orc_uniform(uint32_t w) { return uniform(w); }

void orc_words(uint64_t seed, uint32_t tag, uint32_t t, uint32_t i, uint32_t j0,
               int64_t m, uint32_t* out) {
  for (int64_t k = 0; k < m; ++k) out[k] = word(seed, tag, t, i, j0 + (uint32_t)k);
}

double orc_objective_f64(int32_t obj, const float* x, int32_t d) {
  return objective(obj, x, d);
}

float orc_objective(int32_t obj, const float* x, int32_t d) {
  return (float)objective(obj, x, d);
}

void orc_objective_rows(int32_t obj, const float* X, int64_t m, int32_t d, float* out) {
  for (int64_t i = 0; i < m; ++i) out[i] = (float)objective(obj, X + i * d, d);
}

// Reading 3: Eq. 5's bounds are user-defined; the default is
// the symmetric absolute bound [-1, 1], the value under which the oracle lands
// near the paper's Table 2 errors for both Sphere and Griewank.
float orc_default_vmax(float lo, float hi) {
  (void)lo;
  (void)hi;
  return 1.0f;
}

void orc_init_local(const orc_params* p, orc_state* s, float* cand_f, int64_t* cand_i,
                    float* cand_row) {
  const int32_t d = p->d;
  bool have = false;
  float bf = 0.0f;
  int64_t bi = 0;
  for (int64_t r = 0; r < s->nrows; ++r) {
    const int64_t gi = s->row_begin + r;
    float* x = s->X + r * d;
    float* v = s->V + r * d;
    for (int32_t j = 0; j < d; ++j) {  // Alg. 1 line 2, reading 4
      const Bounds bd = bounds_of(p, j);
      float ux = uniform(word(p->seed, ORC_TAG_X0, 0, (uint32_t)gi, (uint32_t)j));
      float uv = uniform(word(p->seed, ORC_TAG_V0, 0, (uint32_t)gi, (uint32_t)j));
      x[j] = std::fmin(std::fmax(bd.xlo + (bd.xhi - bd.xlo) * ux, bd.xlo), bd.xhi);
      v[j] = bd.vlo + (bd.vhi - bd.vlo) * uv;
    }
    float fi = (float)objective(p->objective, x, d);
    s->f[r] = fi;
    s->pf[r] = std::isnan(fi) ? std::numeric_limits<float>::infinity() : fi;  // reading 11
    std::memcpy(s->PB + r * d, x, sizeof(float) * (size_t)d);
    if (!have || lex_less(s->pf[r], gi, bf, bi)) {
      have = true;
      bf = s->pf[r];
      bi = gi;
    }
  }
  if (have) {
    *cand_f = bf;
    *cand_i = bi;
    std::memcpy(cand_row, s->PB + (bi - s->row_begin) * d, sizeof(float) * (size_t)d);
  } else {  // empty shard: never wins (reading 11: +inf, index past any row)
    *cand_f = std::numeric_limits<float>::infinity();
    *cand_i = std::numeric_limits<int64_t>::max();
  }
  s->t = 0;
}

void orc_step_local(const orc_params* p, orc_state* s, int* has_cand, float* cand_f,
                    int64_t* cand_i, float* cand_row) {
  const int32_t d = p->d;
  s->t += 1;
  const uint32_t t = (uint32_t)s->t;
  bool have = false;
  float bf = 0.0f;
  int64_t bi = 0;
  for (int64_t r = 0; r < s->nrows; ++r) {
    const int64_t gi = s->row_begin + r;
    row_step(p, t, s->G, (uint32_t)gi, s->X + r * d, s->V + r * d, s->PB + r * d,
             &s->pf[r], &s->f[r]);
    const float fi = s->f[r];
    if (fi < s->gf) {  // Alg. 1 line 10, strict
      if (!have || lex_less(fi, gi, bf, bi)) {
        have = true;
        bf = fi;
        bi = gi;
      }
    }
  }
  *has_cand = have ? 1 : 0;
  if (have) {
    *cand_f = bf;
    *cand_i = bi;
    std::memcpy(cand_row, s->PB + (bi - s->row_begin) * d, sizeof(float) * (size_t)d);
  }
}

void orc_merge(orc_state* s, int32_t d, int32_t k, const int* has, const float* cf,
               const int64_t* ci, const float* rows, int is_init) {
  int best = -1;
  for (int32_t r = 0; r < k; ++r) {
    if (!has[r]) continue;
    if (best < 0 || lex_less(cf[r], ci[r], cf[best], ci[best])) best = r;
  }
  if (best < 0) return;
  if (is_init || cf[best] < s->gf) {
    s->gf = cf[best];
    s->gi = ci[best];
    std::memcpy(s->G, rows + (size_t)best * d, sizeof(float) * (size_t)d);
  }
}

void orc_create(const orc_params* p, orc_state* s, int32_t nshards) {
  const int32_t d = p->d;
  if (nshards < 1) nshards = 1;
  std::vector<int> has(nshards);
  std::vector<float> cf(nshards);
  std::vector<int64_t> ci(nshards);
  std::vector<float> rows((size_t)nshards * d);
  for (int32_t r = 0; r < nshards; ++r) {
    const int64_t b = s->row_begin + (s->nrows * r) / nshards;
    const int64_t e = s->row_begin + (s->nrows * (r + 1)) / nshards;
    orc_state v = shard_view(s, d, b, e - b);
    orc_init_local(p, &v, &cf[r], &ci[r], rows.data() + (size_t)r * d);
    has[r] = (e > b) ? 1 : 0;
  }
  orc_merge(s, d, nshards, has.data(), cf.data(), ci.data(), rows.data(), 1);
  s->t = 0;
}

void orc_step(const orc_params* p, orc_state* s, int64_t iters, int32_t nshards) {
  const int32_t d = p->d;
  if (nshards < 1) nshards = 1;
  std::vector<int> has(nshards);
  std::vector<float> cf(nshards);
  std::vector<int64_t> ci(nshards);
  std::vector<float> rows((size_t)nshards * d);
  for (int64_t it = 0; it < iters; ++it) {
    for (int32_t r = 0; r < nshards; ++r) {
      const int64_t b = s->row_begin + (s->nrows * r) / nshards;
      const int64_t e = s->row_begin + (s->nrows * (r + 1)) / nshards;
      orc_state v = shard_view(s, d, b, e - b);  // shares G, gf, t with s
      orc_step_local(p, &v, &has[r], &cf[r], &ci[r], rows.data() + (size_t)r * d);
    }
    s->t += 1;
    orc_merge(s, d, nshards, has.data(), cf.data(), ci.data(), rows.data(), 0);
  }
}

void orc_rebest(const orc_params* p, orc_state* s) {
  const int32_t d = p->d;
  int64_t bi = -1;
  float bf = 0.0f;
  for (int64_t r = 0; r < s->nrows; ++r) {
    if (std::isnan(s->pf[r])) s->pf[r] = std::numeric_limits<float>::infinity();
    if (bi < 0 || s->pf[r] < bf) {  // ascending scan, strict: lowest index wins ties
      bi = r;
      bf = s->pf[r];
    }
  }
  if (bi < 0) return;
  s->gf = bf;
  s->gi = s->row_begin + bi;
  std::memcpy(s->G, s->PB + bi * d, sizeof(float) * (size_t)d);
}

void orc_rows_step(const orc_params* p, uint64_t t, const float* G, const int64_t* idx,
                   int64_t m, float* X, float* V, float* PB, float* pf, float* f) {
  const int32_t d = p->d;
  for (int64_t r = 0; r < m; ++r)
    row_step(p, (uint32_t)t, G, (uint32_t)idx[r], X + r * d, V + r * d, PB + r * d, &pf[r],
             &f[r]);
}

}  // extern "C"
