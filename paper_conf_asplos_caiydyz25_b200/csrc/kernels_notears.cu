// NOTEARS acyclicity penalty per (penalty group, SCC) (sm_100a).
//
//   A_t[i][j] = sum_{k in m_i, m_j in ch_k} cp_k
//   h(A) = tr(e^A) - d, zero iff acyclic (Thm 3.1, Eqs. 8-9)
//   SCC decomposition: h = sum_S h(A_S)
//   batched approximation: exp of the seed-mean matrix (Eq. 11)  PAPER.md:320-325,
//     over groups of G seeds (reading S13)
//   gradient: dL/dcp_{k,b} += lambda * sum_{j in ch_k cap S} e^{Abar}[j][ec(k)]
//     (d tr e^A / dA = (e^A)^T)
//
// One CTA per (SCC, group).  Abar (|S| <= 64) lives in shared memory in fp64;
// e^A - I is formed directly (Horner form of the Taylor series of expm1 after
// scaling the inf-norm to <= 1/2, then Y <- Y^2 + 2Y per squaring), so
// h = tr(e^A - I) carries no cancellation.  The entry sums run over a fixed
// (entry, node, seed) order with a fixed warp-shuffle tree: h and the
// gradient are bit-identical at every GPU count.
#include "kcommon.cuh"

namespace smoothe {

constexpr int kNotearsMaxN = 64;
constexpr int kTaylorDeg = 16;

__device__ void smem_matmul(int n, const double* A, const double* B, double* C) {
  for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) {
    const int i = idx / n, j = idx % n;
    double acc = 0.0;
    for (int k = 0; k < n; ++k) acc += A[i * n + k] * B[k * n + j];
    C[idx] = acc;
  }
}

__global__ void __launch_bounds__(256) k_notears(
    int Bp, int G, int ngroups, double lambda, const int32_t* __restrict__ scc_class_ptr,
    const int32_t* __restrict__ ent_ptr, const int32_t* __restrict__ ent_i,
    const int32_t* __restrict__ ent_j, const int32_t* __restrict__ ent_node_ptr,
    const int32_t* __restrict__ ent_node, const int32_t* __restrict__ slot_ptr,
    const int32_t* __restrict__ slot_iloc, const int32_t* __restrict__ slot_jptr,
    const int32_t* __restrict__ slot_jloc, const float* __restrict__ cp,
    double* __restrict__ h_part, float* __restrict__ pen) {
  extern __shared__ double smem[];
  __shared__ int s_sq;
  const int scc = blockIdx.x, grp = blockIdx.y;
  const int n = scc_class_ptr[scc + 1] - scc_class_ptr[scc];
  double* X = smem;
  double* T = X + n * n;
  double* U = T + n * n;
  for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) X[idx] = 0.0;
  __syncthreads();
  // Abar_S[i][j] = (1/G) sum_{b in group} sum_{k in m_i, j in ch_k} cp_{k,b}
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nwarps = blockDim.x >> 5;
  const int b0 = grp * G;
  for (int e = ent_ptr[scc] + warp; e < ent_ptr[scc + 1]; e += nwarps) {
    double acc = 0.0;
    for (int a = ent_node_ptr[e]; a < ent_node_ptr[e + 1]; ++a) {
      const float* row = cp + (size_t)ent_node[a] * Bp + b0;
      for (int b = lane; b < G; b += 32) acc += (double)row[b];
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
    if (lane == 0) X[ent_i[e] * n + ent_j[e]] = acc / G;
  }
  __syncthreads();
  // scaling: 2^-s with s = max(0, ceil(log2 ||A||_inf) + 1)  =>  ||X|| <= 1/2
  if (threadIdx.x == 0) {
    double nrm = 0.0;
    for (int i = 0; i < n; ++i) {
      double r = 0.0;
      for (int j = 0; j < n; ++j) r += fabs(X[i * n + j]);
      nrm = fmax(nrm, r);
    }
    s_sq = nrm > 0.0 ? max(0, (int)ceil(log2(nrm)) + 1) : 0;
  }
  __syncthreads();
  const int sq = s_sq;
  const double scale = ldexp(1.0, -sq);
  for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) {
    X[idx] *= scale;
    const int i = idx / n, j = idx % n;
    T[idx] = (i == j ? 1.0 : 0.0) + X[idx] / kTaylorDeg;
  }
  __syncthreads();
  // Horner: T_m = I + X T_{m+1} / m, m = deg-1 .. 2;  Y = X T_2 = e^X - I
  for (int mdeg = kTaylorDeg - 1; mdeg >= 2; --mdeg) {
    smem_matmul(n, X, T, U);
    __syncthreads();
    for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) {
      const int i = idx / n, j = idx % n;
      T[idx] = (i == j ? 1.0 : 0.0) + U[idx] / mdeg;
    }
    __syncthreads();
  }
  smem_matmul(n, X, T, U);  // U = Y
  __syncthreads();
  double* Y = U;
  double* Z = T;
  for (int r = 0; r < sq; ++r) {  // e^{2A} - I = Y^2 + 2Y
    smem_matmul(n, Y, Y, Z);
    __syncthreads();
    for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) Z[idx] += 2.0 * Y[idx];
    __syncthreads();
    double* tmp = Y;
    Y = Z;
    Z = tmp;
  }
  if (threadIdx.x == 0) {
    double tr = 0.0;
    for (int i = 0; i < n; ++i) tr += Y[i * n + i];
    h_part[(size_t)scc * ngroups + grp] = tr;
  }
  // penalty gradient per e-node slot of this SCC (same for every seed of the group)
  for (int l = slot_ptr[scc] + threadIdx.x; l < slot_ptr[scc + 1]; l += blockDim.x) {
    const int il = slot_iloc[l];
    double acc = 0.0;
    for (int q = slot_jptr[l]; q < slot_jptr[l + 1]; ++q) {
      const int jl = slot_jloc[q];
      acc += Y[jl * n + il] + (jl == il ? 1.0 : 0.0);
    }
    pen[(size_t)l * ngroups + grp] = (float)(lambda * acc);
  }
}

void launch_notears(cudaStream_t s, const Shape& sh, const HostGraph& hg, const DevGraph& g,
                    int32_t G, double lambda, const float* cp, double* h_part, float* pen) {
  if (hg.num_scc == 0) return;
  const int ngroups = sh.B / G;
  const int n = hg.scc_max;
  const size_t smem = 3 * sizeof(double) * (size_t)n * n;
  static bool attr_set = false;
  if (!attr_set) {
    SM_CUDA(cudaFuncSetAttribute(k_notears, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 3 * sizeof(double) * kNotearsMaxN * kNotearsMaxN));
    attr_set = true;
  }
  k_notears<<<dim3(hg.num_scc, ngroups), 256, smem, s>>>(
      sh.Bp, G, ngroups, lambda, g.scc_class_ptr, g.ent_ptr, g.ent_i, g.ent_j, g.ent_node_ptr,
      g.ent_node, g.slot_ptr, g.slot_iloc, g.slot_jptr, g.slot_jloc, cp, h_part, pen);
  SM_LAUNCH_CHECK();
}

}  // namespace smoothe
