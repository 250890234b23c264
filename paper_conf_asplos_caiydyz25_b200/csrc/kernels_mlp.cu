// MLP cost model f_mlp(p) = W3 relu(W2 relu(W1 p + b1) + b2) + b3 (
// reading S22: N -> 64 -> 8 -> 1) and its gradient, CUDA-core version.
//
// Layer 1 is the only large contraction: z1[h][b] = sum_k W1[h][k] p[k][b]
// (2*H1*N*B flop) and g_p[k][b] += sum_h W1[h][k] gz1[h][b] (same).  Split-K
// partial sums are reduced in a fixed order, so results are deterministic.
#include "kcommon.cuh"

namespace smoothe {

constexpr int kMlpTK = 32;     // nodes per tile
constexpr int kMlpMaxH1 = 64;
constexpr int kMlpMaxH2 = 16;

// z1_part[split][h][b] over the split's node range; block = 256 threads,
// seed chunk Bc = min(Bp, 128), each thread owns one seed and H1*Bc/256 hidden units.
__global__ void __launch_bounds__(256) k_mlp_l1(int N, int Bp, int H1, int nsplit,
                                                const float* __restrict__ W1,
                                                const float* __restrict__ p,
                                                float* __restrict__ z1_part) {
  __shared__ float sW[kMlpMaxH1][kMlpTK + 1];
  __shared__ float sP[kMlpTK][128];
  const int Bc = Bp < 128 ? Bp : 128;
  const int b = threadIdx.x % Bc;
  const int hg = threadIdx.x / Bc;
  const int ngroups = 256 / Bc;
  const int hper = (H1 + ngroups - 1) / ngroups;
  const int h0 = hg * hper;
  const int seed0 = blockIdx.y * Bc;
  const int split = blockIdx.x;
  const int64_t per = ((int64_t)N + nsplit - 1) / nsplit;
  const int64_t kb = (int64_t)split * per, ke = (int64_t)(split + 1) * per;
  const int k_begin = (int)(kb < N ? kb : N);
  const int k_end = (int)(ke < N ? ke : N);
  float acc[kMlpMaxH1];
#pragma unroll
  for (int h = 0; h < kMlpMaxH1; ++h) acc[h] = 0.f;
  for (int kt = k_begin; kt < k_end; kt += kMlpTK) {
    const int nk = min(kMlpTK, k_end - kt);
    for (int idx = threadIdx.x; idx < H1 * kMlpTK; idx += 256) {
      const int h = idx / kMlpTK, kk = idx % kMlpTK;
      sW[h][kk] = kk < nk ? W1[(size_t)h * N + kt + kk] : 0.f;
    }
    for (int idx = threadIdx.x; idx < kMlpTK * Bc; idx += 256) {
      const int kk = idx / Bc, bb = idx % Bc;
      sP[kk][bb] = kk < nk ? p[(size_t)(kt + kk) * Bp + seed0 + bb] : 0.f;
    }
    __syncthreads();
    for (int kk = 0; kk < kMlpTK; ++kk) {
      const float pv = sP[kk][b];
#pragma unroll
      for (int h = 0; h < kMlpMaxH1; ++h)
        if (h < hper && h0 + h < H1) acc[h] += sW[h0 + h][kk] * pv;
    }
    __syncthreads();
  }
#pragma unroll
  for (int h = 0; h < kMlpMaxH1; ++h)
    if (h < hper && h0 + h < H1)
      z1_part[((size_t)split * H1 + h0 + h) * Bp + seed0 + b] = acc[h];
}

// Per seed: reduce splits, layers 2-3, f_mlp, and gz1 = d f_mlp / d z1.
__global__ void k_mlp_head(int Bp, int H1, int H2, int nsplit, const float* __restrict__ b1,
                           const float* __restrict__ W2, const float* __restrict__ b2,
                           const float* __restrict__ W3, const float* __restrict__ b3,
                           const float* __restrict__ z1_part, double* __restrict__ f_mlp,
                           float* __restrict__ gz1) {
  const int b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= Bp) return;
  float z1[kMlpMaxH1], z2[kMlpMaxH2];
  for (int h = 0; h < H1; ++h) {
    float acc = b1[h];
    for (int sp = 0; sp < nsplit; ++sp) acc += z1_part[((size_t)sp * H1 + h) * Bp + b];
    z1[h] = acc;
  }
  float y = b3[0];
  for (int h2 = 0; h2 < H2; ++h2) {
    float acc = b2[h2];
    for (int h = 0; h < H1; ++h) acc += W2[h2 * H1 + h] * fmaxf(z1[h], 0.f);
    z2[h2] = acc;
    y += W3[h2] * fmaxf(acc, 0.f);
  }
  f_mlp[b] = (double)y;
  if (gz1) {
    for (int h = 0; h < H1; ++h) {
      float acc = 0.f;
      for (int h2 = 0; h2 < H2; ++h2)
        if (z2[h2] > 0.f) acc += W2[h2 * H1 + h] * W3[h2];
      gz1[(size_t)h * Bp + b] = z1[h] > 0.f ? acc : 0.f;  // ReLU'(0) = 0 (S25)
    }
  }
}

// gp[k][b] = u[k] + sum_h W1[h][k] gz1[h][b]
__global__ void __launch_bounds__(256) k_mlp_l1_back(int N, int Bp, int H1,
                                                     const float* __restrict__ W1,
                                                     const float* __restrict__ u,
                                                     const float* __restrict__ gz1,
                                                     float* __restrict__ gp) {
  __shared__ float sG[kMlpMaxH1][128];
  __shared__ float sW[kMlpMaxH1][kMlpTK + 1];
  const int Bc = Bp < 128 ? Bp : 128;
  const int seed0 = blockIdx.y * Bc;
  for (int idx = threadIdx.x; idx < H1 * Bc; idx += 256)
    sG[idx / Bc][idx % Bc] = gz1[(size_t)(idx / Bc) * Bp + seed0 + idx % Bc];
  const int kt = blockIdx.x * kMlpTK;
  const int nk = min(kMlpTK, N - kt);
  for (int idx = threadIdx.x; idx < H1 * kMlpTK; idx += 256) {
    const int h = idx / kMlpTK, kk = idx % kMlpTK;
    sW[h][kk] = kk < nk ? W1[(size_t)h * N + kt + kk] : 0.f;
  }
  __syncthreads();
  for (int idx = threadIdx.x; idx < nk * Bc; idx += 256) {
    const int kk = idx / Bc, b = idx % Bc;
    float acc = u[kt + kk];
    for (int h = 0; h < H1; ++h) acc += sW[h][kk] * sG[h][b];
    gp[(size_t)(kt + kk) * Bp + seed0 + b] = acc;
  }
}

void launch_mlp_fwd(cudaStream_t s, const Shape& sh, int32_t H1, int32_t H2, const float* W1,
                    const float* b1, const float* W2, const float* b2, const float* W3,
                    const float* b3, const float* p, float* z1_part, double* f_mlp, float* gz1,
                    int32_t nsplit) {
  const int Bc = sh.Bp < 128 ? sh.Bp : 128;
  k_mlp_l1<<<dim3(nsplit, sh.Bp / Bc), 256, 0, s>>>(sh.N, sh.Bp, H1, nsplit, W1, p, z1_part);
  SM_LAUNCH_CHECK();
  k_mlp_head<<<(sh.Bp + 127) / 128, 128, 0, s>>>(sh.Bp, H1, H2, nsplit, b1, W2, b2, W3, b3, z1_part,
                                                 f_mlp, gz1);
  SM_LAUNCH_CHECK();
}

void launch_mlp_bwd(cudaStream_t s, const Shape& sh, int32_t H1, const float* W1, const float* u,
                    const float* gz1, float* gp) {
  const int Bc = sh.Bp < 128 ? sh.Bp : 128;
  k_mlp_l1_back<<<dim3((sh.N + kMlpTK - 1) / kMlpTK, sh.Bp / Bc), 256, 0, s>>>(sh.N, sh.Bp, H1, W1,
                                                                              u, gz1, gp);
  SM_LAUNCH_CHECK();
}

}  // namespace smoothe
