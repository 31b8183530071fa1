/*
 * pso_oracle.h — the plain CPU oracle for FastPSO's hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing in the product path (the CUDA library
 * under paper_conf_icpp_liuwc21_b200/) includes, links or calls this code,
 * and this code includes nothing from there.  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load it.
 *
 * It is a plain, slow, single-threaded C++17 implementation of the method as
 * the paper states it, compiled with -O3 -ffp-contract=off so every fp32
 * operation of the update is rounded exactly once, in the written order.
 *
 * Citations: P:Lnnn = /root/reference/PAPER.md line nnn.
 *   Alg. 1          PSO main loop (init; evaluate; pbest; gbest; move)
 *   Eq. 1         v' = w v + c1 l (pbest - p) + c2 g (gbest - p)
 *   Eq. 2         p' = p + v'
 *   Eq. 4         the same update on the n x d matrices V, P, L, G
 *   Eq. 5         velocity bound constraint (clamp)
 *   Sec 3.1            random init of positions/velocities, random L, G
 *   Sec 3.2        swarm evaluation (Sphere, Griewank, Easom built-ins)
 *   Sec 3.3        pbest update, gbest = argmin by reduction
 *   Sec 4.1        objective definitions and domains
 *   [20] Molga & Smutnicki (cited at P:L147): Rastrigin, Rosenbrock, Ackley
 * Every free choice the paper leaves open follows SURVEY.md 8(c) and is listed
 * in DESIGN.md ("Readings").
 */
#ifndef PSO_ORACLE_H
#define PSO_ORACLE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Objective ids.  The numbers are the interface values of the C ABI
 * (include/fastpso.h); the oracle defines its own copy. */
enum {
  ORC_SPHERE = 1,
  ORC_RASTRIGIN = 2,
  ORC_ROSENBROCK = 3,
  ORC_GRIEWANK = 4,
  ORC_ACKLEY = 5,
  ORC_EASOM = 6
};

/* Philox stream tags (reading 6). */
enum { ORC_TAG_R1 = 0, ORC_TAG_R2 = 1, ORC_TAG_X0 = 2, ORC_TAG_V0 = 3 };

typedef struct {
  int64_t n;          /* global swarm size (Alg. 1 input n) */
  int32_t d;          /* dimension */
  int32_t objective;  /* ORC_* */
  float w, c1, c2;    /* Alg. 1 inputs omega, c1, c2 */
  float lo, hi;       /* domain */
  float vmax;         /* velocity bound (Eq. 5), symmetric |v| <= vmax; reading 3 */
  uint64_t seed;      /* Philox key */
  const float* bounds; /* NULL, or 4*d floats [vlo | vhi | xlo | xhi] per dimension
                          (Eq. 5 per-dimension reading, NEXT-2); replaces vmax/lo/hi */
} orc_params;

/* Caller-owned state of one shard: global rows [row_begin, row_begin+nrows).
 * Dense row-major, d floats per row. */
typedef struct {
  int64_t row_begin, nrows;
  float* X;   /* positions P        nrows*d */
  float* V;   /* velocities V       nrows*d */
  float* PB;  /* pbest positions    nrows*d */
  float* pf;  /* pbest fitness      nrows   */
  float* f;   /* last evaluated fitness (perror of Alg. 1 line 6)  nrows */
  float* G;   /* gbest position     d       */
  float gf;   /* gbest fitness                      */
  int64_t gi; /* gbest global particle index        */
  uint64_t t; /* iteration counter (0 after create) */
} orc_state;

/* --- Philox4x32-10 (Salmon et al., Random123) and the stream layout ------- */
void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
/* word(tag, t, i, j) = Philox(ctr={j>>2, i, t, tag}, key={seed lo, seed hi})[j & 3] */
uint32_t orc_word(uint64_t seed, uint32_t tag, uint32_t t, uint32_t i, uint32_t j);
/* U(w) = (float)(w >> 8) * 2^-24, in [0, 1 - 2^-24] (reading 5) */
float orc_uniform(uint32_t w);
/* Fill out[k] = word(tag,t,i,j0+k) for k < m (bulk helper for tests). */
void orc_words(uint64_t seed, uint32_t tag, uint32_t t, uint32_t i, uint32_t j0,
               int64_t m, uint32_t* out);

/* --- Objectives (Sec 3.2; [20]) ------------------------------ */
/* Plain definition accumulated in double from the fp32 x; returns double. */
double orc_objective_f64(int32_t obj, const float* x, int32_t d);
/* The same, rounded once to fp32 (what the method compares). */
float orc_objective(int32_t obj, const float* x, int32_t d);
/* Evaluate m rows of a dense m x d matrix. */
void orc_objective_rows(int32_t obj, const float* X, int64_t m, int32_t d, float* out);

float orc_default_vmax(float lo, float hi);

/* --- Shard-level steps (what one GPU of a particle-split swarm does) ------ */
/* Alg. 1 lines 1-3 + first evaluation: X0, V0 from Philox; pf = F(X0)
 * (NaN -> +inf); PB = X0.  Returns the shard's best row: lowest global index
 * attaining min pf (every row is eligible).  cand_row receives PB of it. */
void orc_init_local(const orc_params* p, orc_state* s, float* cand_f,
                    int64_t* cand_i, float* cand_row);
/* One iteration: t += 1; move (Eq. 1, 5, 2 + domain clamp) for every element;
 * evaluate; pbest (strict <).  Candidate = lexicographic min (f_i, i) over
 * rows with f_i < gf (strict); *has_cand = 0 if none. */
void orc_step_local(const orc_params* p, orc_state* s, int* has_cand,
                    float* cand_f, int64_t* cand_i, float* cand_row);
/* Merge k shard candidates into the (replicated) gbest.  is_init: take the
 * lexicographic min unconditionally; else only if strictly below gf. */
void orc_merge(orc_state* s, int32_t d, int32_t k, const int* has,
               const float* cf, const int64_t* ci, const float* rows, int is_init);

/* --- Whole swarm, optionally as k virtual particle shards ---------------- */
void orc_create(const orc_params* p, orc_state* s, int32_t nshards);
void orc_step(const orc_params* p, orc_state* s, int64_t iters, int32_t nshards);
/* Recompute gf, gi, G from pf, PB (pf NaN -> +inf), as after create. */
void orc_rebest(const orc_params* p, orc_state* s);

/* Move + evaluate + pbest for m sampled rows with global indices idx[],
 * at iteration t (already incremented), with gbest position G.  Rows are
 * independent given G (Eq. 4), so this is exact for any subset. */
void orc_rows_step(const orc_params* p, uint64_t t, const float* G,
                   const int64_t* idx, int64_t m, float* X, float* V,
                   float* PB, float* pf, float* f);

#ifdef __cplusplus
}
#endif
#endif /* PSO_ORACLE_H */
