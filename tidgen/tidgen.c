/*
 * tidgen.c — seeded, counter-based synthetic SIFT-like descriptor generator.
 *
 * This module is SHARED INPUT PLUMBING: both the CPU oracle (oracle/) and the
 * CUDA path (paper_conf_icpp_wangzll21_b200/) are fed from it.  It holds none of
 * the method's arithmetic (no distances, no nearest neighbours, no ratio test,
 * no counting, no ranking) — it only draws u8 descriptors.
 *
 * Every output byte is a pure function of (seed, object id, keypoint, dim), so
 * any slice of a reference set or query batch can be regenerated independently
 * (by a shard, by a host thread, by the oracle) without storing it twice.
 *
 * Recipe:
 *   - K cluster centres, each an OpenCV-style u8 SIFT vector: 128 gamma(0.5)
 *     bins -> L2-normalise -> clip at 0.2 -> renormalise -> x512 -> round ->
 *     saturate to [0,255]  (the paper never states the encoding; ||x||2 ~ 512
 *     matches the Table 2 overflow boundary).
 *   - reference keypoint = sat_u8(round(centre_k + sigma * N(0,1))), k uniform.
 *   - query q plants n_planted noisy copies (sigma_p) of distinct keypoints of
 *     its target reference t(q) at random positions; the rest are fresh
 *     cluster draws.  Targets are distinct across a batch (t is a bijection
 *     q -> (q*stride + offset) mod R_total with gcd(stride, R_total) = 1).
 *   - N(0,1) is approximated by a rescaled Irwin–Hall(4) sum of 16-bit uniforms
 *     taken from one 64-bit hash (bounded |z| <= 3.47): cheap, deterministic,
 *     bit-identical for every consumer of this library.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

enum {
  ST_CENTRE = 1, ST_REF_K = 2, ST_REF = 3, ST_Q_PERM = 4, ST_Q_SRC = 5,
  ST_Q_NOISE = 6, ST_Q_K = 7, ST_Q = 8, ST_KPCOUNT = 9
};

static inline uint64_t mix64(uint64_t z) {
  z += 0x9e3779b97f4a7c15ULL;
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

static inline uint64_t h4(uint64_t seed, uint64_t stream, uint64_t a, uint64_t b) {
  return mix64(mix64(mix64(seed ^ (stream * 0xd1342543de82ef95ULL)) ^ a) ^ (b * 0x2545f4914f6cdd1dULL));
}

/* approx N(0,1): Irwin–Hall(4) on 16-bit uniforms, mean 4*32767.5, sd 65536/sqrt(3) */
static inline double gauss(uint64_t h) {
  double s = (double)(h & 0xffff) + (double)((h >> 16) & 0xffff) +
             (double)((h >> 32) & 0xffff) + (double)((h >> 48) & 0xffff);
  return (s - 131070.0) / 37837.22;
}

static inline uint8_t sat_round(double x) {
  double r = floor(x + 0.5);
  if (r < 0.0) return 0;
  if (r > 255.0) return 255;
  return (uint8_t)r;
}

/* One OpenCV-style SIFT centre (128 u8). */
static void make_centre(uint64_t seed, int k, uint8_t* out) {
  double g[128], ss = 0.0;
  for (int t = 0; t < 128; ++t) {
    double z = gauss(h4(seed, ST_CENTRE, (uint64_t)k, (uint64_t)t));
    g[t] = 0.5 * z * z;                   /* gamma(0.5, 1) */
    ss += g[t] * g[t];
  }
  double inv = ss > 0 ? 1.0 / sqrt(ss) : 0.0, ss2 = 0.0;
  for (int t = 0; t < 128; ++t) {
    g[t] *= inv;
    if (g[t] > 0.2) g[t] = 0.2;
    ss2 += g[t] * g[t];
  }
  double inv2 = ss2 > 0 ? 1.0 / sqrt(ss2) : 0.0;
  for (int t = 0; t < 128; ++t) out[t] = sat_round(g[t] * inv2 * 512.0);
}

void tidgen_centres(uint64_t seed, int32_t K, uint8_t* out /*[K][128]*/) {
  for (int k = 0; k < K; ++k) make_centre(seed, k, out + (size_t)k * 128);
}

/* Number of stored keypoints of reference r.  kp_min == m => all equal to m. */
int32_t tidgen_ref_kp_count(uint64_t seed, int64_t r, int32_t m, int32_t kp_min) {
  if (kp_min >= m) return m;
  return kp_min + (int32_t)(h4(seed, ST_KPCOUNT, (uint64_t)r, 0) % (uint64_t)(m - kp_min + 1));
}

static void ref_keypoint(uint64_t seed, const uint8_t* centres, int32_t K, double sigma,
                         int64_t r, int32_t i, uint8_t* out) {
  int k = (int)(h4(seed, ST_REF_K, (uint64_t)r, (uint64_t)i) % (uint64_t)K);
  const uint8_t* c = centres + (size_t)k * 128;
  uint64_t row = ((uint64_t)r << 12) | (uint64_t)i;
  for (int t = 0; t < 128; ++t)
    out[t] = sat_round((double)c[t] + sigma * gauss(h4(seed, ST_REF, row, (uint64_t)t)));
}

/*
 * References [first, first+count) of a set, each stored as m rows of 128 u8
 * (layout [count][m][128]).  Rows >= kp_count(r) are filled with `pad_byte`
 * (callers use this to prove padding is ignored).  kp_counts_out (nullable)
 * receives the per-reference keypoint counts.
 */
void tidgen_refs(uint64_t seed, int32_t K, double sigma, int64_t first, int64_t count,
                 int32_t m, int32_t kp_min, int32_t pad_byte,
                 uint8_t* out, int32_t* kp_counts_out) {
  uint8_t* centres = (uint8_t*)malloc((size_t)K * 128);
  tidgen_centres(seed, K, centres);
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t j = 0; j < count; ++j) {
    int64_t r = first + j;
    int32_t kc = tidgen_ref_kp_count(seed, r, m, kp_min);
    uint8_t* o = out + (size_t)j * m * 128;
    for (int32_t i = 0; i < kc; ++i) ref_keypoint(seed, centres, K, sigma, r, i, o + (size_t)i * 128);
    if (kc < m) memset(o + (size_t)kc * 128, pad_byte, (size_t)(m - kc) * 128);
    if (kp_counts_out) kp_counts_out[j] = kc;
  }
  free(centres);
}

static int64_t gcd64(int64_t a, int64_t b) { while (b) { int64_t t = a % b; a = b; b = t; } return a; }

/* Planted target of query q in a set of R_total references (a bijection on q mod R_total). */
int64_t tidgen_target(uint64_t seed, int64_t q, int64_t R_total) {
  if (R_total <= 0) return -1;
  int64_t stride = 1000003 % R_total;
  if (stride == 0) stride = 1;
  while (gcd64(stride, R_total) != 1) stride = (stride + 1) % R_total == 0 ? 1 : stride + 1;
  int64_t off = (int64_t)(mix64(seed ^ 0x51ed27) % (uint64_t)R_total);
  return (int64_t)(((__int128)q * stride + off) % R_total);
}

/* Fisher–Yates prefix: first `take` entries of a seeded permutation of [0, n). */
static void perm_prefix(uint64_t seed, uint64_t stream, uint64_t id, int32_t n, int32_t take, int32_t* out, int32_t* scratch) {
  for (int32_t i = 0; i < n; ++i) scratch[i] = i;
  for (int32_t i = 0; i < take; ++i) {
    int32_t j = i + (int32_t)(h4(seed, stream, id, (uint64_t)i) % (uint64_t)(n - i));
    int32_t t = scratch[i]; scratch[i] = scratch[j]; scratch[j] = t;
    out[i] = scratch[i];
  }
}

/*
 * Queries [first_q, first_q+count), layout [count][n][128].
 * Query q plants min(n_planted, n, kp(target)) noisy copies (sigma_p) of the
 * target reference's keypoints (target drawn from a set of R_total references
 * generated with (seed, K, sigma, m, kp_min)).  n_planted = 0 gives unrelated
 * queries.  targets_out (nullable) receives t(q) (or -1 when nothing planted).
 */
void tidgen_queries_t(uint64_t seed, int32_t K, double sigma, double sigma_p,
                      int64_t first_q, int64_t count, int32_t n, int32_t n_planted,
                      int64_t R_total, int32_t m, int32_t kp_min,
                      const int64_t* targets_in, uint8_t* out, int64_t* targets_out) {
  uint8_t* centres = (uint8_t*)malloc((size_t)K * 128);
  tidgen_centres(seed, K, centres);
#pragma omp parallel
  {
    int32_t* pos = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > m ? n : m));
    int32_t* src = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > m ? n : m));
    int32_t* scr = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > m ? n : m));
    uint8_t* planted_flag = (uint8_t*)malloc((size_t)n);
    int32_t* planted_src = (int32_t*)malloc(sizeof(int32_t) * (size_t)n);
    uint8_t tkp[128];
#pragma omp for schedule(dynamic, 1)
    for (int64_t jq = 0; jq < count; ++jq) {
      int64_t q = first_q + jq;
      uint8_t* o = out + (size_t)jq * n * 128;
      int64_t tgt = targets_in ? targets_in[jq]
                  : ((n_planted > 0 && R_total > 0) ? tidgen_target(seed, q, R_total) : -1);
      if (n_planted <= 0) tgt = -1;
      int32_t P = 0;
      memset(planted_flag, 0, (size_t)n);
      if (tgt >= 0) {
        int32_t mt = tidgen_ref_kp_count(seed, tgt, m, kp_min);
        P = n_planted; if (P > n) P = n; if (P > mt) P = mt;
        perm_prefix(seed, ST_Q_PERM, (uint64_t)q, n, P, pos, scr);
        perm_prefix(seed, ST_Q_SRC, (uint64_t)q, mt, P, src, scr);
        for (int32_t p = 0; p < P; ++p) { planted_flag[pos[p]] = 1; planted_src[pos[p]] = src[p]; }
      }
      for (int32_t j = 0; j < n; ++j) {
        uint8_t* row = o + (size_t)j * 128;
        uint64_t rid = ((uint64_t)q << 13) | (uint64_t)j;
        if (planted_flag[j]) {
          ref_keypoint(seed, centres, K, sigma, tgt, planted_src[j], tkp);
          for (int t = 0; t < 128; ++t)
            row[t] = sat_round((double)tkp[t] + sigma_p * gauss(h4(seed, ST_Q_NOISE, rid, (uint64_t)t)));
        } else {
          int k = (int)(h4(seed, ST_Q_K, (uint64_t)q, (uint64_t)j) % (uint64_t)K);
          const uint8_t* c = centres + (size_t)k * 128;
          for (int t = 0; t < 128; ++t)
            row[t] = sat_round((double)c[t] + sigma * gauss(h4(seed, ST_Q, rid, (uint64_t)t)));
        }
      }
      if (targets_out) targets_out[jq] = (P > 0) ? tgt : -1;
    }
    free(pos); free(src); free(scr); free(planted_flag); free(planted_src);
  }
  free(centres);
}

void tidgen_queries(uint64_t seed, int32_t K, double sigma, double sigma_p,
                    int64_t first_q, int64_t count, int32_t n, int32_t n_planted,
                    int64_t R_total, int32_t m, int32_t kp_min,
                    uint8_t* out, int64_t* targets_out) {
  tidgen_queries_t(seed, K, sigma, sigma_p, first_q, count, n, n_planted, R_total, m, kp_min,
                   NULL, out, targets_out);
}
