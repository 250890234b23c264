// Step kernels of the seed-parallel SmoothE gradient step (sm_100a).
//
//   theta init (Philox4x32-10, reading S9)
//   segmented softmax + argmax + decode selection masks
//   linear / quadratic cost + backward initialisation     PAPER.md:101, 156; reading S24
//   softmax backward fused with Adam                      PAPER.md:275-277; reading S10
//
// All per-seed arrays are [row][Bp] fp32 (seed innermost): every gather of a
// parent/child row is a contiguous 16-byte-per-lane access (kcommon.cuh).
// The two propagation sweeps live in kernels_sweep.cu.
#include <algorithm>
#include <cfloat>

#include "kcommon.cuh"

namespace smoothe {

// ---------------------------------------------------------------------------
// theta = (x >> 8) * 2^-23 - 1, x = Philox4x32-10(key, ctr = (node, seed))[0]
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t philox_x0(uint64_t key, uint64_t node, uint64_t seed) {
  uint32_t c0 = (uint32_t)node, c1 = (uint32_t)(node >> 32);
  uint32_t c2 = (uint32_t)seed, c3 = (uint32_t)(seed >> 32);
  uint32_t k0 = (uint32_t)key, k1 = (uint32_t)(key >> 32);
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    if (r) {
      k0 += 0x9E3779B9u;
      k1 += 0xBB67AE85u;
    }
    const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
    const uint32_t n0 = hi1 ^ c1 ^ k0, n2 = hi0 ^ c3 ^ k1;
    c0 = n0;
    c1 = lo1;
    c2 = n2;
    c3 = lo0;
  }
  return c0;
}

__global__ void k_theta_init(int64_t total, int Bp, int B, uint64_t key, int64_t seed_begin,
                             float* __restrict__ theta, float* __restrict__ m, float* __restrict__ v) {
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int b = (int)(idx % Bp);
    const int64_t node = idx / Bp;
    float t = 0.f;
    if (b < B) {
      const uint32_t x = philox_x0(key, (uint64_t)node, (uint64_t)(seed_begin + b));
      t = (float)(x >> 8) * 0x1p-23f - 1.0f;  // exact: 24-bit grid
    }
    theta[idx] = t;
    m[idx] = 0.f;
    v[idx] = 0.f;
  }
}

void launch_theta_init(cudaStream_t s, const Shape& sh, uint64_t key, int64_t seed_begin,
                       float* theta, float* m, float* v) {
  const int64_t total = (int64_t)sh.N * sh.Bp;
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 16);
  k_theta_init<<<grid, 256, 0, s>>>(total, sh.Bp, sh.B, key, seed_begin, theta, m, v);
  SM_LAUNCH_CHECK();
}

// ---------------------------------------------------------------------------
// Segmented softmax within each e-class (Eq. 3b), the decode choice
// c_j = argmax_{k in m_j} theta_k (lowest id on ties, reading S17) and the
// selection masks sel[k][w] (bit l = seed 32w+l chose e-node k).
// One warp per (class, <=4 words of 32 seeds); lane l owns seed 32w+l so a
// ballot yields the mask word directly.  Classes with more than kBigClass
// e-nodes get a block of 8 warps striding over the e-nodes (max / arg-max and
// sum combined through shared memory in warp order).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(kBlock) k_softmax_argmax(int M, int Bp, int W, int nw,
                                                           const int32_t* __restrict__ class_ptr,
                                                           const int32_t* __restrict__ big,
                                                           int nbig,
                                                           const float* __restrict__ theta,
                                                           float* __restrict__ cp,
                                                           int32_t* __restrict__ choice,
                                                           uint32_t* __restrict__ sel) {
  constexpr int NWARP = kBlock / 32;
  __shared__ float smx[NWARP][4][32];
  __shared__ int sam[NWARP][4][32];
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  const int nwc = W / nw;
  int j, w0, kstart, kstep;
  const bool is_big = blockIdx.x < nbig * nwc;
  if (is_big) {
    j = big[blockIdx.x / nwc];
    w0 = (blockIdx.x % nwc) * nw;
    kstart = wi;
    kstep = NWARP;
  } else {
    const int warp = (blockIdx.x - nbig * nwc) * NWARP + wi;
    j = warp / nwc;
    if (j >= M) return;
    if (class_ptr[j + 1] - class_ptr[j] > kBigClass) return;  // a big-class block does it
    w0 = (warp % nwc) * nw;
    kstart = 0;
    kstep = 1;
  }
  const int k0 = class_ptr[j], k1 = class_ptr[j + 1];
  float mx[4], sum[4];
  int am[4];
#pragma unroll
  for (int s = 0; s < 4; ++s) {
    mx[s] = -FLT_MAX;
    sum[s] = 0.f;
    am[s] = k1;
  }
  for (int k = k0 + kstart; k < k1; k += kstep) {
#pragma unroll
    for (int s = 0; s < 4; ++s) {
      if (s < nw) {
        const float t = theta[(size_t)k * Bp + 32 * (w0 + s) + lane];
        if (t > mx[s] || am[s] == k1) {
          mx[s] = t;
          am[s] = k;
        }
      }
    }
  }
  if (is_big) {  // combine the warps' (max, lowest arg-max)
#pragma unroll
    for (int s = 0; s < 4; ++s) {
      smx[wi][s][lane] = mx[s];
      sam[wi][s][lane] = am[s];
    }
    __syncthreads();
#pragma unroll
    for (int s = 0; s < 4; ++s) {
      float m = smx[0][s][lane];
      int a = sam[0][s][lane];
      for (int w = 1; w < NWARP; ++w) {
        const float m2 = smx[w][s][lane];
        const int a2 = sam[w][s][lane];
        if (a2 < k1 && (a == k1 || m2 > m || (m2 == m && a2 < a))) {
          m = m2;
          a = a2;
        }
      }
      mx[s] = m;
      am[s] = a;
    }
    __syncthreads();
  }
  for (int k = k0 + kstart; k < k1; k += kstep) {
#pragma unroll
    for (int s = 0; s < 4; ++s)
      if (s < nw) sum[s] += expf(theta[(size_t)k * Bp + 32 * (w0 + s) + lane] - mx[s]);
  }
  if (is_big) {  // total in warp order
#pragma unroll
    for (int s = 0; s < 4; ++s) smx[wi][s][lane] = sum[s];
    __syncthreads();
#pragma unroll
    for (int s = 0; s < 4; ++s) {
      float t = smx[0][s][lane];
      for (int w = 1; w < NWARP; ++w) t += smx[w][s][lane];
      sum[s] = t;
    }
  }
  for (int k = k0 + kstart; k < k1; k += kstep) {
#pragma unroll
    for (int s = 0; s < 4; ++s) {
      if (s < nw) {
        const size_t idx = (size_t)k * Bp + 32 * (w0 + s) + lane;
        cp[idx] = expf(theta[idx] - mx[s]) / sum[s];
        const uint32_t bits = __ballot_sync(0xffffffffu, am[s] == k);
        if (lane == 0) sel[(size_t)k * W + w0 + s] = bits;
      }
    }
  }
  if (is_big && wi != 0) return;
#pragma unroll
  for (int s = 0; s < 4; ++s)
    if (s < nw) choice[(size_t)j * Bp + 32 * (w0 + s) + lane] = am[s];
}

void launch_softmax_argmax(cudaStream_t s, const Shape& sh, const DevGraph& g, const float* theta,
                           float* cp, int32_t* choice, uint32_t* sel) {
  const int nw = sh.W < 4 ? sh.W : 4;
  const int nwc = sh.W / nw;
  const int64_t warps = (int64_t)sh.M * nwc;
  const int grid = g.num_big * nwc + (int)((warps * 32 + kBlock - 1) / kBlock);
  k_softmax_argmax<<<grid, kBlock, 0, s>>>(sh.M, sh.Bp, sh.W, nw, g.class_ptr, g.big_class,
                                           g.num_big, theta, cp, choice, sel);
  SM_LAUNCH_CHECK();
}

// ---------------------------------------------------------------------------
// Linear cost f_b = sum_i u_i p_i with p = cp * q^K[ec] (P101), fused with the
// backward initialisation (App. C step 1-2): g_cp_i = u_i q^K_{ec(i)},
// g_q^K_j = sum_{i in m_j} u_i cp_i (0 at the root).  Per-block partial sums
// of f go to f_part[blockIdx.x][Bp] (reduced in fp64 by k_reduce_rows).
// ---------------------------------------------------------------------------
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_cost_linear(
    int M, int Bp, int root, const int32_t* __restrict__ class_ptr,
    const int32_t* __restrict__ big, int nbig, const float* __restrict__ u,
    const float* __restrict__ cp, const float* __restrict__ qK, float* __restrict__ gcp,
    float* __restrict__ gqK, float* __restrict__ f_part, float* __restrict__ p_out) {
  __shared__ float4 red[kBlock / LPR][LPR];
  constexpr int R = kBlock / LPR;
  const int lane = threadIdx.x % LPR, sub = threadIdx.x / LPR;
  const int s0 = blockIdx.y * (4 * LPR) + lane * 4;
  float4 facc = make_float4(0.f, 0.f, 0.f, 0.f);
  auto node = [&](int i, const float4& qv, float4& gq) {
    const float ui = __ldg(u + i);
    const size_t o = (size_t)i * Bp + s0;
    const float4 cv = ld4(cp + o);
    float4 p, gc;
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      comp(p, x) = __fmul_rn(comp(cv, x), comp(qv, x));
      comp(facc, x) += ui * comp(p, x);
      comp(gc, x) = ui * comp(qv, x);
      comp(gq, x) += ui * comp(cv, x);
    }
    st4(gcp + o, gc);
    if (p_out) st4(p_out + o, p);
  };
  if (blockIdx.x < nbig) {
    __shared__ float4 part[kClassParts][LPR];
    const int j = big[blockIdx.x];
    const float4 qv = ld4(qK + (size_t)j * Bp + s0);
    PartSums<LPR> ps;
    ps.run(class_ptr[j], class_ptr[j + 1], [&](int i, float4& gq) { node(i, qv, gq); });
    float4 gq = ps.total(part);
    if (j == root) gq = make_float4(0.f, 0.f, 0.f, 0.f);
    if (sub == 0) st4(gqK + (size_t)j * Bp + s0, gq);
  } else {
    const int j = (blockIdx.x - nbig) * R + sub;
    if (j < M && class_ptr[j + 1] - class_ptr[j] <= kBigClass) {
      const float4 qv = ld4(qK + (size_t)j * Bp + s0);
      float4 gq = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int i = class_ptr[j]; i < class_ptr[j + 1]; ++i) node(i, qv, gq);
      if (j == root) gq = make_float4(0.f, 0.f, 0.f, 0.f);
      st4(gqK + (size_t)j * Bp + s0, gq);
    }
  }
  const float4 ft = block_sum_rows<LPR>(red, facc);
  if (sub == 0) st4(f_part + (size_t)blockIdx.x * Bp + s0, ft);
}

void launch_cost_linear(cudaStream_t s, const Shape& sh, const DevGraph& g, const float* u,
                        const float* cp, const float* qK, float* gcp, float* gqK, float* f_part,
                        float* p_out, int32_t) {
  SM_DISPATCH_LPR(sh.Bp, {
    k_cost_linear<LPR><<<class_grid(sh.M, sh.Bp, LPR, g.num_big), kBlock, 0, s>>>(
        sh.M, sh.Bp, sh.root, g.class_ptr, g.big_class, g.num_big, u, cp, qK, gcp, gqK, f_part,
        p_out);
  });
  SM_LAUNCH_CHECK();
}

// p = cp * q^K[ec] materialised for the non-linear cost models; with u, also
// the per-block partial sums of the linear part u^T p (P409: f = f_lin + f_nl).
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_materialize_p(int M, int Bp,
                                                          const int32_t* __restrict__ class_ptr,
                                                          const int32_t* __restrict__ big, int nbig,
                                                          const float* __restrict__ u,
                                                          const float* __restrict__ cp,
                                                          const float* __restrict__ qK,
                                                          float* __restrict__ p,
                                                          float* __restrict__ f_part) {
  __shared__ float4 red[kBlock / LPR][LPR];
  constexpr int R = kBlock / LPR;
  const int lane = threadIdx.x % LPR, sub = threadIdx.x / LPR;
  const int s0 = blockIdx.y * (4 * LPR) + lane * 4;
  float4 facc = make_float4(0.f, 0.f, 0.f, 0.f);
  int j = -1, kstart = 0, kstep = 1;
  if (blockIdx.x < nbig) {
    j = big[blockIdx.x];
    kstart = sub;
    kstep = R;
  } else {
    const int row = (blockIdx.x - nbig) * R + sub;
    if (row < M && class_ptr[row + 1] - class_ptr[row] <= kBigClass) j = row;
  }
  if (j >= 0) {
    const float4 qv = ld4(qK + (size_t)j * Bp + s0);
    for (int i = class_ptr[j] + kstart; i < class_ptr[j + 1]; i += kstep) {
      const size_t o = (size_t)i * Bp + s0;
      const float4 cv = ld4(cp + o);
      const float ui = u ? __ldg(u + i) : 0.f;
      float4 pv;
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        comp(pv, x) = __fmul_rn(comp(cv, x), comp(qv, x));
        comp(facc, x) += ui * comp(pv, x);
      }
      st4(p + o, pv);
    }
  }
  if (!f_part) return;
  const float4 ft = block_sum_rows<LPR>(red, facc);
  if (sub == 0) st4(f_part + (size_t)blockIdx.x * Bp + s0, ft);
}

void launch_materialize_p_f(cudaStream_t s, const Shape& sh, const DevGraph& g, const float* u,
                            const float* cp, const float* qK, float* p, float* f_part) {
  SM_DISPATCH_LPR(sh.Bp, {
    k_materialize_p<LPR><<<class_grid(sh.M, sh.Bp, LPR, g.num_big), kBlock, 0, s>>>(
        sh.M, sh.Bp, g.class_ptr, g.big_class, g.num_big, u, cp, qK, p, f_part);
  });
  SM_LAUNCH_CHECK();
}

__global__ void k_fill_rows(float* base, int64_t stride, int count, int Bp, float value) {
  for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < count * Bp; idx += gridDim.x * blockDim.x)
    base[(size_t)(idx / Bp) * stride + idx % Bp] = value;
}

void launch_fill_rows(cudaStream_t s, float* base, int64_t stride, int count, int Bp, float value) {
  if (count <= 0) return;
  const int grid = std::min((count * Bp + 255) / 256, 1024);
  k_fill_rows<<<grid, 256, 0, s>>>(base, stride, count, Bp, value);
  SM_LAUNCH_CHECK();
}

// ftot[b] = f[b] + fextra[b];  L = sum_b ftot[b] + lambda * sum_g G h_g  (Eq. 10a; S12)
// L = sum_b f_b + lambda sum_g G h_g (reading S12); with a trace, row
// `step` (scal[2]) gets the relaxed side of the per-step record: min_b f(p_b)
// and mean_b f(p_b) (the decode writes the sampled side, k_best_update).
__global__ void k_loss(int B, int G, int ngroups, double lambda, const double* __restrict__ f,
                       const double* __restrict__ fextra, const double* __restrict__ h,
                       double* __restrict__ ftot, double* __restrict__ loss,
                       const double* __restrict__ scal, double* __restrict__ trace, int trace_cap) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  double L = 0.0, mn = INFINITY;
  for (int b = 0; b < B; ++b) {
    const double v = f[b] + (fextra ? fextra[b] : 0.0);
    ftot[b] = v;
    L += v;
    mn = fmin(mn, v);
  }
  const double fsum = L;
  if (h)
    for (int g = 0; g < ngroups; ++g) L += lambda * G * h[g];
  *loss = L;
  const int step = (int)scal[2];
  if (trace && step < trace_cap) {
    trace[4 * (size_t)step + 0] = mn;
    trace[4 * (size_t)step + 1] = fsum / B;
  }
}

void launch_loss(cudaStream_t s, int B, int G, int ngroups, double lambda, const double* f,
                 const double* fextra, const double* h, double* ftot, double* loss,
                 const double* scal, double* trace, int trace_cap) {
  k_loss<<<1, 32, 0, s>>>(B, G, ngroups, lambda, f, fextra, h, ftot, loss, scal, trace, trace_cap);
  SM_LAUNCH_CHECK();
}

// Backward initialisation from a general g_p = df/dp (quadratic / MLP).
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_cost_gp(int M, int Bp, int root,
                                                    const int32_t* __restrict__ class_ptr,
                                                    const int32_t* __restrict__ big, int nbig,
                                                    const float* __restrict__ gp,
                                                    const float* __restrict__ cp,
                                                    const float* __restrict__ qK,
                                                    float* __restrict__ gcp, float* __restrict__ gqK) {
  constexpr int R = kBlock / LPR;
  const int lane = threadIdx.x % LPR, sub = threadIdx.x / LPR;
  const int s0 = blockIdx.y * (4 * LPR) + lane * 4;
  auto node = [&](int i, const float4& qv, float4& gq) {
    const size_t o = (size_t)i * Bp + s0;
    const float4 gv = ld4(gp + o), cv = ld4(cp + o);
    float4 gc;
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      comp(gc, x) = comp(gv, x) * comp(qv, x);
      comp(gq, x) += comp(gv, x) * comp(cv, x);
    }
    st4(gcp + o, gc);
  };
  if (blockIdx.x < nbig) {
    __shared__ float4 part[kClassParts][LPR];
    const int j = big[blockIdx.x];
    const float4 qv = ld4(qK + (size_t)j * Bp + s0);
    PartSums<LPR> ps;
    ps.run(class_ptr[j], class_ptr[j + 1], [&](int i, float4& gq) { node(i, qv, gq); });
    float4 gq = ps.total(part);
    if (j == root) gq = make_float4(0.f, 0.f, 0.f, 0.f);
    if (sub == 0) st4(gqK + (size_t)j * Bp + s0, gq);
    return;
  }
  const int j = (blockIdx.x - nbig) * R + sub;
  if (j >= M || class_ptr[j + 1] - class_ptr[j] > kBigClass) return;
  const float4 qv = ld4(qK + (size_t)j * Bp + s0);
  float4 gq = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int i = class_ptr[j]; i < class_ptr[j + 1]; ++i) node(i, qv, gq);
  if (j == root) gq = make_float4(0.f, 0.f, 0.f, 0.f);
  st4(gqK + (size_t)j * Bp + s0, gq);
}

void launch_cost_gp(cudaStream_t s, const Shape& sh, const DevGraph& g, const float* gp,
                    const float* cp, const float* qK, float* gcp, float* gqK) {
  SM_DISPATCH_LPR(sh.Bp, {
    k_cost_gp<LPR><<<class_grid(sh.M, sh.Bp, LPR, g.num_big), kBlock, 0, s>>>(
        sh.M, sh.Bp, sh.root, g.class_ptr, g.big_class, g.num_big, gp, cp, qK, gcp, gqK);
  });
  SM_LAUNCH_CHECK();
}

// Quadratic cost (reading S24) over a symmetric neighbour list of the pairs:
//   f = sum_i p_i (u_i + 1/2 sum_{k in nbr(i)} w_ik p_k),   g_p_i = u_i + sum_k w_ik p_k.
// Rows are e-nodes.  Also used on the 0/1 decode vector s (exact for integer u, w).
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_cost_quadratic(int N, int Bp,
                                                           const int32_t* __restrict__ qptr,
                                                           const int32_t* __restrict__ qnbr,
                                                           const float* __restrict__ qw,
                                                           const float* __restrict__ u,
                                                           const float* __restrict__ p,
                                                           float* __restrict__ gp,
                                                           float* __restrict__ f_part) {
  __shared__ float4 red[kBlock / LPR][LPR];
  const RowGroup<LPR> rg;
  float4 facc = make_float4(0.f, 0.f, 0.f, 0.f);
  if (rg.row < N) {
    const int i = rg.row;
    const float ui = u ? u[i] : 0.f;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int e = qptr[i]; e < qptr[i + 1]; ++e) {
      const float w = __ldg(qw + e);
      const float4 pk = ld4(p + (size_t)__ldg(qnbr + e) * Bp + rg.s0);
#pragma unroll
      for (int x = 0; x < 4; ++x) comp(acc, x) += w * comp(pk, x);
    }
    const float4 pi = ld4(p + (size_t)i * Bp + rg.s0);
    float4 g;
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      comp(g, x) = ui + comp(acc, x);
      comp(facc, x) = comp(pi, x) * (ui + 0.5f * comp(acc, x));
    }
    if (gp) st4(gp + (size_t)i * Bp + rg.s0, g);
  }
  red[rg.sub][threadIdx.x % LPR] = facc;
  __syncthreads();
  if (threadIdx.x < LPR) {
    float4 acc = red[0][threadIdx.x];
    for (int r = 1; r < kBlock / LPR; ++r) {
      const float4 v = red[r][threadIdx.x];
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    st4(f_part + (size_t)blockIdx.x * Bp + rg.s0, acc);
  }
}

void launch_quadratic(cudaStream_t s, const Shape& sh, const int32_t* qptr, const int32_t* qnbr,
                      const float* qw, const float* u, const float* p, float* gp, float* f_part) {
  SM_DISPATCH_LPR(sh.Bp, {
    k_cost_quadratic<LPR><<<row_grid(sh.N, sh.Bp, LPR), kBlock, 0, s>>>(sh.N, sh.Bp, qptr, qnbr, qw,
                                                                       u, p, gp, f_part);
  });
  SM_LAUNCH_CHECK();
}

// out[b] = scale * sum_r part[r][b] in fp64, in a fixed order (deterministic,
// bit-identical run to run): stage 1 sums interleaved rows of each of S slices
// (32 seeds x 8 row strides per block, fixed-order smem combine), stage 2 sums
// the S slice totals in order.
constexpr int kRedSlices = 128;

template <typename T>
__global__ void __launch_bounds__(256) k_reduce_rows_s1(const T* __restrict__ part, int nrows, int Bp,
                                                        int per, double* __restrict__ scratch) {
  __shared__ double red[8][32];
  const int b = blockIdx.x * 32 + (threadIdx.x & 31);
  const int ty = threadIdx.x >> 5;
  const int r0 = blockIdx.y * per, r1 = min(nrows, r0 + per);
  double acc = 0.0;
  if (b < Bp)
    for (int r = r0 + ty; r < r1; r += 8) acc += (double)part[(size_t)r * Bp + b];
  red[ty][threadIdx.x & 31] = acc;
  __syncthreads();
  if (ty == 0 && b < Bp) {
    double t = red[0][threadIdx.x];
    for (int i = 1; i < 8; ++i) t += red[i][threadIdx.x];
    scratch[(size_t)blockIdx.y * Bp + b] = t;
  }
}

__global__ void k_reduce_rows_s2(const double* __restrict__ scratch, int S, int Bp,
                                 double* __restrict__ out, double scale) {
  const int b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= Bp) return;
  double acc = 0.0;
  for (int i = 0; i < S; ++i) acc += scratch[(size_t)i * Bp + b];
  out[b] = acc * scale;
}

template <typename T>
static void reduce_rows(cudaStream_t s, const T* part, int nrows, int Bp, double* out, double scale,
                        double* scratch) {
  const int S = std::max(1, std::min(kRedSlices, (nrows + 63) / 64));
  const int per = (nrows + S - 1) / S;
  k_reduce_rows_s1<T><<<dim3((Bp + 31) / 32, S), 256, 0, s>>>(part, nrows, Bp, per, scratch);
  SM_LAUNCH_CHECK();
  k_reduce_rows_s2<<<(Bp + 127) / 128, 128, 0, s>>>(scratch, S, Bp, out, scale);
  SM_LAUNCH_CHECK();
}

void launch_reduce_rows_f64(cudaStream_t s, const float* part, int32_t nrows, int32_t Bp,
                            double* out, double scale, double* scratch) {
  reduce_rows<float>(s, part, nrows, Bp, out, scale, scratch);
}

void launch_reduce_rows_f64d(cudaStream_t s, const double* part, int32_t nrows, int32_t Bp,
                             double* out, double* scratch) {
  reduce_rows<double>(s, part, nrows, Bp, out, 1.0, scratch);
}

// ---------------------------------------------------------------------------
// Step scalars: Adam bias corrections for step number t = counter + 1 (fp64).
// ---------------------------------------------------------------------------
__global__ void k_step_prologue(const int32_t* __restrict__ counter, double* __restrict__ scal,
                                double beta1, double beta2) {
  const double t = (double)(*counter + 1);
  scal[0] = 1.0 / (1.0 - pow(beta1, t));
  scal[1] = 1.0 / (1.0 - pow(beta2, t));
  scal[2] = (double)*counter;  // this step's index (k_loss's trace row)
}

void launch_step_prologue(cudaStream_t s, int32_t* step_counter, double* step_scalars,
                          double beta1, double beta2, const int32_t*) {
  k_step_prologue<<<1, 1, 0, s>>>(step_counter, step_scalars, beta1, beta2);
  SM_LAUNCH_CHECK();
}

// ---------------------------------------------------------------------------
// Softmax backward fused with the optimiser (P277; reading S10), per class:
//   g_tot_k = g_cp_k + pen_k(group)                      (App. B penalty term)
//   g_theta_k = cp_k (g_tot_k - sum_{k' in m_j} cp_k' g_tot_k')
//   Adam: m = b1 m + (1-b1) g; v = b2 v + (1-b2) g^2;
//         theta -= lr (m c1) / (sqrt(v c2) + eps),  c1,2 = 1/(1 - b1,2^t)
// ---------------------------------------------------------------------------
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_update(
    int M, int Bp, int G, int ngroups, const int32_t* __restrict__ class_ptr,
    const int32_t* __restrict__ big, int nbig, const int32_t* __restrict__ node_slot,
    const float* __restrict__ cp, const float* __restrict__ gcp, const float* __restrict__ pen,
    float* __restrict__ theta, float* __restrict__ m, float* __restrict__ v,
    const double* __restrict__ scal, int optimizer, float lr, float beta1, float beta2, float eps,
    float* __restrict__ gth_out, float* __restrict__ gcp_out, const int32_t* __restrict__ abort_flag) {
  // a step aborted by a full version pool is repeated: leave theta, m, v as they are
  if (abort_flag && *abort_flag) return;
  constexpr int R = kBlock / LPR;
  const int lane = threadIdx.x % LPR, sub = threadIdx.x / LPR;
  const int s0 = blockIdx.y * (4 * LPR) + lane * 4;
  int j, kstart, kstep;
  const bool is_big = blockIdx.x < nbig;
  if (is_big) {
    j = big[blockIdx.x];
    kstart = sub;
    kstep = R;
  } else {
    j = (blockIdx.x - nbig) * R + sub;
    if (j >= M || class_ptr[j + 1] - class_ptr[j] > kBigClass) return;
    kstart = 0;
    kstep = 1;
  }
  const int k0 = class_ptr[j] + kstart, k1 = class_ptr[j + 1];
  int grp[4];
#pragma unroll
  for (int x = 0; x < 4; ++x) grp[x] = min((s0 + x) / G, ngroups - 1);
  auto gtot = [&](int k, float4 gc) {
    const int slot = node_slot ? __ldg(node_slot + k) : -1;
    if (slot >= 0) {
#pragma unroll
      for (int x = 0; x < 4; ++x) comp(gc, x) += pen[(size_t)slot * ngroups + grp[x]];
    }
    return gc;
  };
  auto dot = [&](int k, float4& acc) {
    const size_t o = (size_t)k * Bp + s0;
    const float4 cv = ld4(cp + o);
    const float4 gt = gtot(k, ld4(gcp + o));
#pragma unroll
    for (int x = 0; x < 4; ++x) comp(acc, x) += comp(cv, x) * comp(gt, x);
  };
  float4 ssum = make_float4(0.f, 0.f, 0.f, 0.f);
  if (is_big) {
    __shared__ float4 part[kClassParts][LPR];
    PartSums<LPR> ps;
    ps.run(class_ptr[j], k1, dot);
    ssum = ps.total(part);
  } else {
    for (int k = k0; k < k1; ++k) dot(k, ssum);
  }
  const float c1 = (float)scal[0], c2 = (float)scal[1];
  for (int k = k0; k < k1; k += kstep) {
    const size_t o = (size_t)k * Bp + s0;
    const float4 cv = ld4(cp + o);
    const float4 gt = gtot(k, ld4(gcp + o));
    float4 th = ld4(theta + o), mv = ld4(m + o), vv = ld4(v + o), gth;
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      const float g = comp(cv, x) * (comp(gt, x) - comp(ssum, x));
      comp(gth, x) = g;
      if (optimizer == 0) {
        const float mn = beta1 * comp(mv, x) + (1.f - beta1) * g;
        const float vn = beta2 * comp(vv, x) + (1.f - beta2) * (g * g);
        comp(mv, x) = mn;
        comp(vv, x) = vn;
        comp(th, x) = comp(th, x) - lr * (mn * c1) / (sqrtf(vn * c2) + eps);
      } else {
        comp(th, x) = comp(th, x) - lr * g;
      }
    }
    st4(theta + o, th);
    st4(m + o, mv);
    st4(v + o, vv);
    if (gth_out) st4(gth_out + o, gth);
    if (gcp_out) st4(gcp_out + o, gt);
  }
}

void launch_update(cudaStream_t s, const Shape& sh, const DevGraph& g, int32_t G, const float* cp,
                   const float* gcp, const float* pen, float* theta, float* m, float* v,
                   const double* step_scalars, int32_t optimizer, float lr, float beta1,
                   float beta2, float eps, float* grad_theta_out, float* grad_cp_out,
                   const int32_t* abort_flag) {
  const int ngroups = (sh.B + G - 1) / G;
  SM_DISPATCH_LPR(sh.Bp, {
    k_update<LPR><<<class_grid(sh.M, sh.Bp, LPR, g.num_big), kBlock, 0, s>>>(
        sh.M, sh.Bp, G, ngroups, g.class_ptr, g.big_class, g.num_big, pen ? g.node_slot : nullptr,
        cp, gcp, pen, theta, m,
        v, step_scalars, optimizer, lr, beta1, beta2, eps, grad_theta_out, grad_cp_out, abort_flag);
  });
  SM_LAUNCH_CHECK();
}

}  // namespace smoothe
