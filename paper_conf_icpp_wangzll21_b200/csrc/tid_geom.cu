// tid_geom.cu — SURVEY §8 row f4: post-match verification on the GPU (§3.1
// "the geometric verification is performed to remove the outliers that may be mismatched";
// §4.1 P:408-410 "ratio test and edge feature removing").  The paper names the steps without
// defining them; readings R14-R16 fix them:
//   R14 edge-feature removal: a good match (ratio test passed) is dropped when its query keypoint
//       or its nearest reference keypoint lies within `border` px of its image's edge;
//   R15 model: 2-D similarity X = a x - b y + tx, Y = b x + a y + ty fitted exactly to 2 matches;
//       inlier when the squared reprojection error is < thr^2;
//   R16 hypotheses: RANSAC, hypothesis t draws its 2 matches with a counter-based generator
//       (splitmix64 of seed, pair and t), or every pair u < v when iterations == 0; the best
//       hypothesis has the most inliers (ties: earliest t).
// One CTA per pair: the good matches are compacted in query-keypoint order into shared memory
// (block-wide ballot scan), then the CTA's threads evaluate hypotheses t = tid, tid + 256, ...
// and a block reduction picks the best.  All geometry in fp64 with explicitly rounded operations
// (no FMA contraction), in the order the readings write it, so every inlier decision is the same
// IEEE computation the CPU oracle makes.
#include "tid_kernels.cuh"

namespace tid {
namespace geom {

constexpr int kThreads = 256;

__device__ __forceinline__ uint64_t mix64(uint64_t z) {  // splitmix64 finaliser
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__device__ __forceinline__ double mul(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double add(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ double sub(double a, double b) { return __dsub_rn(a, b); }

// Similarity through (p1 -> q1, p2 -> q2); false when p1 == p2 (no hypothesis).
__device__ bool fit(float2 p1, float2 p2, float2 q1, float2 q2, double (&md)[4]) {
  const double dpx = sub(p2.x, p1.x), dpy = sub(p2.y, p1.y);
  const double dqx = sub(q2.x, q1.x), dqy = sub(q2.y, q1.y);
  const double den = add(mul(dpx, dpx), mul(dpy, dpy));
  if (den == 0.0) return false;
  const double a = __ddiv_rn(add(mul(dpx, dqx), mul(dpy, dqy)), den);
  const double b = __ddiv_rn(sub(mul(dpx, dqy), mul(dpy, dqx)), den);
  md[0] = a;
  md[1] = b;
  md[2] = sub(q1.x, sub(mul(a, p1.x), mul(b, p1.y)));
  md[3] = sub(q1.y, add(mul(b, p1.x), mul(a, p1.y)));
  return true;
}

__device__ int inliers(const float2* P, const float2* Q, int M, const double (&md)[4], double thr2) {
  int c = 0;
  for (int k = 0; k < M; ++k) {
    const double x = P[k].x, y = P[k].y;
    const double ex = sub(add(sub(mul(md[0], x), mul(md[1], y)), md[2]), static_cast<double>(Q[k].x));
    const double ey = sub(add(add(mul(md[1], x), mul(md[0], y)), md[3]), static_cast<double>(Q[k].y));
    c += add(mul(ex, ex), mul(ey, ey)) < thr2;
  }
  return c;
}

// Match pair of hypothesis t among M (M >= 2).
__device__ __forceinline__ void draw(uint64_t h0, int64_t t, int M, bool exhaustive, int& u, int& v) {
  if (!exhaustive) {
    const uint64_t h = mix64(h0 ^ static_cast<uint64_t>(t));
    u = static_cast<int>(h % static_cast<uint64_t>(M));
    v = static_cast<int>((h >> 32) % static_cast<uint64_t>(M - 1));
    v += v >= u;
  } else {  // t-th pair of (0,1), (0,2), ..., (0,M-1), (1,2), ...: row u starts at u*M - u*(u+1)/2
    int lo = 0, hi = M - 2;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      const int64_t start = static_cast<int64_t>(mid) * M - static_cast<int64_t>(mid) * (mid + 1) / 2;
      if (start <= t) lo = mid; else hi = mid - 1;
    }
    u = lo;
    v = u + 1 + static_cast<int>(t - (static_cast<int64_t>(u) * M - static_cast<int64_t>(u) * (u + 1) / 2));
  }
}

__global__ void __launch_bounds__(kThreads) geom_kernel(const int32_t* __restrict__ nn, int32_t n, int32_t m,
                                                         const int32_t* __restrict__ n_q,
                                                         const int32_t* __restrict__ m_r,
                                                         const float2* __restrict__ q_xy,
                                                         const float2* __restrict__ r_xy, GeomParams g,
                                                         uint32_t* __restrict__ good_out,
                                                         uint32_t* __restrict__ inl_out, double* __restrict__ model_out) {
  extern __shared__ float2 gsm[];
  float2* P = gsm;      // [n] query coordinates of the good matches, in query-keypoint order
  float2* Q = gsm + n;  // [n] their nearest reference keypoints
  __shared__ int warp_cnt[kThreads / 32];
  __shared__ int base_s;
  __shared__ long long best_key[kThreads / 32];
  const int64_t p = blockIdx.x;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int nq = n_q ? n_q[p] : n, mr = m_r ? m_r[p] : m;
  if (tid == 0) base_s = 0;
  __syncthreads();
  // ---- compaction: ratio test (readings R1 / R3) + edge-feature removal (R14)
  for (int j0 = 0; j0 < nq; j0 += kThreads) {
    const int j = j0 + tid;
    bool keep = false;
    float2 a = make_float2(0.f, 0.f), b = a;
    if (j < nq && mr >= 2) {
      const int4 o = reinterpret_cast<const int4*>(nn)[p * n + j];  // (d1, i1, d2, i2)
      keep = o.z >= 0 && uint64_t(g.den2) * uint64_t(o.x) < uint64_t(g.num2) * uint64_t(o.z);
      if (keep) {
        a = q_xy[p * n + j];
        b = r_xy[p * m + o.y];
        keep = !(a.x < g.border || a.y < g.border || a.x >= g.qw - g.border || a.y >= g.qh - g.border) &&
               !(b.x < g.border || b.y < g.border || b.x >= g.rw - g.border || b.y >= g.rh - g.border);
      }
    }
    const unsigned bal = __ballot_sync(0xffffffffu, keep);
    if (lane == 0) warp_cnt[wid] = __popc(bal);
    __syncthreads();
    int off = base_s;
    for (int w = 0; w < wid; ++w) off += warp_cnt[w];
    if (keep) {
      const int pos = off + __popc(bal & ((1u << lane) - 1u));
      P[pos] = a;
      Q[pos] = b;
    }
    __syncthreads();
    if (tid == 0) {
      int tot = 0;
      for (int w = 0; w < kThreads / 32; ++w) tot += warp_cnt[w];
      base_s += tot;
    }
    __syncthreads();
  }
  const int M = base_s;
  // ---- hypotheses (R15, R16): best = most inliers, ties to the earliest t
  const double thr2 = mul(static_cast<double>(g.thr), static_cast<double>(g.thr));
  const bool exhaustive = g.iters <= 0;
  const int64_t H = M < 2 ? 0 : (exhaustive ? static_cast<int64_t>(M) * (M - 1) / 2 : g.iters);
  const uint64_t h0 = mix64((g.seed << 32) + static_cast<uint64_t>(p));
  long long key = -1;  // inliers << 40 | (2^40 - 1 - t): larger = better
  for (int64_t t = tid; t < H; t += kThreads) {
    int u, v;
    draw(h0, t, M, exhaustive, u, v);
    double md[4];
    if (!fit(P[u], P[v], Q[u], Q[v], md)) continue;
    const long long k = (static_cast<long long>(inliers(P, Q, M, md, thr2)) << 40) | ((1ll << 40) - 1 - t);
    key = k > key ? k : key;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const long long w = __shfl_xor_sync(0xffffffffu, key, o);
    key = w > key ? w : key;
  }
  if (lane == 0) best_key[wid] = key;
  __syncthreads();
  if (tid == 0) {
    long long bk = -1;
    for (int w = 0; w < kThreads / 32; ++w) bk = best_key[w] > bk ? best_key[w] : bk;
    double md[4] = {0.0, 0.0, 0.0, 0.0};
    int cnt = 0;
    if (bk >= 0) {
      const int64_t t = (1ll << 40) - 1 - (bk & ((1ll << 40) - 1));
      int u, v;
      draw(h0, t, M, exhaustive, u, v);
      fit(P[u], P[v], Q[u], Q[v], md);
      cnt = static_cast<int>(bk >> 40);
    }
    good_out[p] = static_cast<uint32_t>(M);
    inl_out[p] = static_cast<uint32_t>(cnt);
    if (model_out)
      for (int i = 0; i < 4; ++i) model_out[p * 4 + i] = md[i];
  }
}

}  // namespace geom

cudaError_t launch_geometric(const int32_t* nn, int32_t n, int32_t m, int64_t P, const int32_t* n_q,
                             const int32_t* m_r, const float* q_xy, const float* r_xy, const GeomParams& g,
                             uint32_t* good, uint32_t* inl, double* model, cudaStream_t s) {
  if (P <= 0) return cudaSuccess;
  const size_t smem = static_cast<size_t>(n) * 2 * sizeof(float2);
  cudaError_t e = cudaFuncSetAttribute(geom::geom_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  geom::geom_kernel<<<static_cast<unsigned>(P), geom::kThreads, smem, s>>>(
      nn, n, m, n_q, m_r, reinterpret_cast<const float2*>(q_xy), reinterpret_cast<const float2*>(r_xy), g, good, inl,
      model);
  return cudaGetLastError();
}

}  // namespace tid
