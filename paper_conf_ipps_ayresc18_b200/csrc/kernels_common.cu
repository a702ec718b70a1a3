// K1 transition matrices, K4 root integration, K5 scale accumulation and
// K6 edge integration (sm_100a).
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {

int device_slot() {
  int d = 0;
  cudaGetDevice(&d);
  return d < 0 ? 0 : (d < kMaxDevices ? d : kMaxDevices - 1);
}
namespace {

constexpr double kLn2 = 0.693147180559945309417232121458176568;
constexpr int kS61Row = 61;  // P^T row of the missing codon state (row sums)

// ---------------------------------------------------------------------- K1
// P_{m,c}[z][x] = sum_k V[z][k] exp(lambda_k r_c t_m) Vinv[k][x]  (fp64),
// Eq. (1)'s Pr(x | z, t) for a reversible Q = V diag(lambda) Vinv.  One block
// per (listed matrix, category); stored in the instance precision, padded to
// s_pad x s_pad (padding stays zero).
template <typename T>
__global__ void k_transition(int s, int s_pad, int C, const double *__restrict__ eig,
                             const double *__restrict__ rates, const int32_t *__restrict__ idx,
                             const double *__restrict__ tlen, T *__restrict__ P) {
  extern __shared__ double sm[];
  double *V = sm;
  double *Vi = sm + s * s;
  double *ex = sm + 2 * s * s;
  const int m = blockIdx.x, c = blockIdx.y;
  const double *lam = eig + 2 * s * s;
  for (int i = threadIdx.x; i < s * s; i += blockDim.x) {
    V[i] = eig[i];
    Vi[i] = eig[s * s + i];
  }
  const double rt = rates[c] * tlen[m];
  for (int k = threadIdx.x; k < s; k += blockDim.x) ex[k] = exp(lam[k] * rt);
  __syncthreads();
  T *out = P + ((size_t)idx[m] * C + c) * (size_t)s_pad * s_pad;
  for (int e = threadIdx.x; e < s * s; e += blockDim.x) {
    const int z = e / s, x = e % s;
    double acc = 0.0;
    for (int k = 0; k < s; ++k) acc = fma(V[z * s + k] * ex[k], Vi[k * s + x], acc);
    out[z * s_pad + x] = (T)acc;
  }
}

// K1 for 4 states: one thread per (listed matrix, category, row z), its four
// outputs P[z][0..3] stored as one vector -- the same sums in the same order
// as k_transition (bit-identical), without a block (and its 32 KB of shared
// staging and barrier) per (matrix, category): configs[1] lists 254 matrices
// x 4 categories, 1,016 blocks of 16 busy threads before.
template <typename T>
__global__ void __launch_bounds__(128)
k_transition4(int C, int items, const double *__restrict__ eig, const double *__restrict__ rates,
              const int32_t *__restrict__ idx, const double *__restrict__ tlen, T *__restrict__ P) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;  // ((m * C) + c) * 4 + z
  if (t >= items * C * 4) return;
  const int z = t & 3, mc = t >> 2, m = mc / C, c = mc % C;
  const double *V = eig, *Vi = eig + 16, *lam = eig + 32;
  const double rt = __ldg(rates + c) * __ldg(tlen + m);
  double ex[4], vz[4];
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    ex[k] = exp(__ldg(lam + k) * rt);
    vz[k] = __ldg(V + z * 4 + k);
  }
  T o[4];
#pragma unroll
  for (int x = 0; x < 4; ++x) {
    double acc = 0.0;
#pragma unroll
    for (int k = 0; k < 4; ++k) acc = fma(vz[k] * ex[k], __ldg(Vi + k * 4 + x), acc);
    o[x] = (T)acc;
  }
  T *out = P + ((size_t)__ldg(idx + m) * C + c) * 16 + z * 4;
#pragma unroll
  for (int x = 0; x < 4; ++x) out[x] = o[x];
}

// K1 for the codon state space (s_pad = 64): one block per (listed matrix,
// category).  The same sum as above, register-tiled: thread (ty, tx) of a
// 16 x 16 block owns the 4 x 4 outputs z in [4ty, 4ty+4), x in [4tx, 4tx+4),
// and per k reads 4 consecutive V^T[k][z] and 4 consecutive Vinv[k][x]
// (two 16-byte shared loads each) for 16 fp64 FMAs -- 4 loads per 16 FMAs
// instead of 2 per FMA.  V, Vinv are zero-padded to 64 x 64 in shared memory,
// so padding outputs come out exactly zero.  With Plo (fp32 codon instances
// feeding the tcgen05 kernel) the tf32 low part of every stored entry is
// written beside it, once per matrix instead of once per pattern tile.
__device__ inline float tf32_lo(float x) {  // rn_tf32(x - trunc_tf32(x)), the 3xTF32 low part
  const float hi = __uint_as_float(__float_as_uint(x) & 0xffffe000u);
  return __uint_as_float((__float_as_uint(x - hi) + 0x1000u) & 0xffffe000u);
}

template <typename T>
__global__ void __launch_bounds__(256)
k_transition64(int s, int C, int items, const double *__restrict__ eig, const double *__restrict__ rates,
               const int32_t *__restrict__ idx, const double *__restrict__ tlen, T *__restrict__ P,
               float *__restrict__ Plo, T *__restrict__ PT) {
  // Persistent: V and V^-1 (the same for every matrix) are staged in shared
  // memory once per block, which then walks (matrix, category) items.
  extern __shared__ double sm[];
  double *Vt = sm;              // [64 k][64 z]
  double *Vi = sm + 64 * 64;    // [64 k][64 x]
  double *ex = sm + 2 * 64 * 64;  // [64]
  const int tid = threadIdx.x;
  const double *lam = eig + 2 * s * s;
  for (int i = tid; i < 64 * 64; i += 256) {
    const int k = i >> 6, q = i & 63;  // consecutive threads: consecutive shared-memory words
    Vt[i] = (k < s && q < s) ? eig[q * s + k] : 0.0;          // V[z=q][k] -> Vt[k][z]
    Vi[i] = (k < s && q < s) ? eig[s * s + k * s + q] : 0.0;  // Vinv[k][x=q]
  }
  // thread: rows z0..z0+3, columns {2l, 2l+1, 32+2l, 33+2l} (l = tid & 15), so a
  // half-warp's column pairs are contiguous (conflict-free double2 loads)
  const int z0 = (tid >> 4) * 4, x0 = (tid & 15) * 2;
  for (int it = blockIdx.x; it < items; it += gridDim.x) {
    const int m = it / C, c = it - m * C;
    __syncthreads();  // V staged / the previous item's ex consumed
    if (tid < 64) ex[tid] = tid < s ? exp(lam[tid] * (rates[c] * tlen[m])) : 0.0;
    __syncthreads();
    double acc[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = 0.0;
#pragma unroll 4
    for (int k = 0; k < s; ++k) {
      const double2 va = *reinterpret_cast<const double2 *>(Vt + k * 64 + z0);
      const double2 vb = *reinterpret_cast<const double2 *>(Vt + k * 64 + z0 + 2);
      const double2 wa = *reinterpret_cast<const double2 *>(Vi + k * 64 + x0);
      const double2 wb = *reinterpret_cast<const double2 *>(Vi + k * 64 + 32 + x0);
      const double ek = ex[k];
      const double a[4] = {va.x * ek, va.y * ek, vb.x * ek, vb.y * ek};
      const double b[4] = {wa.x, wa.y, wb.x, wb.y};
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fma(a[i], b[j], acc[i][j]);
    }
    const size_t off = ((size_t)idx[m] * C + c) * 64 * 64;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      T *row = P + off + (z0 + i) * 64 + x0;
      if constexpr (sizeof(T) == 4) {
        const float2 va = make_float2((float)acc[i][0], (float)acc[i][1]);
        const float2 vb = make_float2((float)acc[i][2], (float)acc[i][3]);
        *reinterpret_cast<float2 *>(row) = va;
        *reinterpret_cast<float2 *>(row + 32) = vb;
        if (Plo != nullptr) {
          float *lo = Plo + off + (z0 + i) * 64 + x0;
          *reinterpret_cast<float2 *>(lo) = make_float2(tf32_lo(va.x), tf32_lo(va.y));
          *reinterpret_cast<float2 *>(lo + 32) = make_float2(tf32_lo(vb.x), tf32_lo(vb.y));
        }
      } else {
        *reinterpret_cast<double2 *>(row) = make_double2(acc[i][0], acc[i][1]);
        *reinterpret_cast<double2 *>(row + 32) = make_double2(acc[i][2], acc[i][3]);
      }
    }
    if (PT != nullptr) {
      // P^T for the tip-tip gather kernel: row x < 61 = column x of P (four
      // consecutive z per 16-byte store), row 61 = the row sums sum_x P[z][x]
      // (the all-ones partials of a missing state, reading A23; summed in fp64
      // over the 16 lanes sharing z0), rows 62-63 stay zero
      const int xs[4] = {x0, x0 + 1, 32 + x0, 33 + x0};
#pragma unroll
      for (int j = 0; j < 4; ++j)
        if (xs[j] < s) {
          T *dst = PT + off + xs[j] * 64 + z0;
#pragma unroll
          for (int i = 0; i < 4; ++i) dst[i] = (T)acc[i][j];
        }
      double rs[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        rs[i] = (acc[i][0] + acc[i][1]) + (acc[i][2] + acc[i][3]);
#pragma unroll
        for (int o = 1; o < 16; o <<= 1) rs[i] += __shfl_xor_sync(0xffffffffu, rs[i], o);
      }
      if ((tid & 15) == 0) {
        T *dst = PT + off + kS61Row * 64 + z0;
#pragma unroll
        for (int i = 0; i < 4; ++i) dst[i] = (T)rs[i];
      }
    }
  }
}

// P^T of one stored codon matrix set (rrl_set_transition_matrix): same layout
// and row-61 sums as K1 writes (sums in fp64 of the stored values).
template <typename T>
__global__ void k_codon_pt(const T *__restrict__ P, T *__restrict__ PT, int C) {
  const int c = blockIdx.x, z = threadIdx.x;  // 64 threads
  const T *row = P + ((size_t)c * 64 + z) * 64;
  T *pt = PT + (size_t)c * 64 * 64;
  double sum = 0.0;
  for (int x = 0; x < 64; ++x) {
    const T v = x < kS61Row ? row[x] : T(0);
    sum += (double)v;
    if (x != kS61Row) pt[x * 64 + z] = v;
  }
  pt[kS61Row * 64 + z] = (T)sum;
}

__global__ void k_split_tf32(const float *__restrict__ x, float *__restrict__ lo, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    lo[i] = tf32_lo(x[i]);
}

// ---------------------------------------------------------------------- K5
__global__ void k_accumulate(const int32_t *__restrict__ scale, int p_pad,
                             const int32_t *__restrict__ idx, int count, int32_t *__restrict__ cum,
                             int p) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < p; i += gridDim.x * blockDim.x) {
    int acc = cum[i];
    for (int k = 0; k < count; ++k) acc += __ldg(scale + (size_t)__ldg(idx + k) * p_pad + i);
    cum[i] = acc;
  }
}

// Fixed-order block reduction (deterministic for a fixed grid).
__device__ double block_sum(double v, double *red) {
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  if (l == 0) red[w] = v;
  __syncthreads();
  double r = 0.0;
  if (w == 0) {
    r = (l < (int)(blockDim.x >> 5)) ? red[l] : 0.0;
    for (int o = 16; o > 0; o >>= 1) r += __shfl_xor_sync(0xffffffffu, r, o);
  }
  return r;  // valid in thread 0
}

// Each block publishes its partial sum; the last block to finish (ticket)
// adds all of them in block order, so the result is deterministic for a
// fixed grid, with a single launch (no separate final-reduction kernel).
__device__ void finish_sum(double part, double *red, double *blocks, unsigned *count, double *out) {
  __shared__ bool last;
  const double r = block_sum(part, red);
  if (threadIdx.x == 0) {
    blocks[blockIdx.x] = r;
    __threadfence();
    last = atomicAdd(count, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!last) return;
  __threadfence();
  double v = 0.0;
  for (int i = threadIdx.x; i < (int)gridDim.x; i += blockDim.x) v += ((volatile double *)blocks)[i];
  __syncthreads();
  const double tot = block_sum(v, red);
  if (threadIdx.x == 0) {
    *out = tot;
    *count = 0u;
  }
}

template <typename T>
__device__ inline double site_root(const T *L, int s, int s_pad, int C, int i, int p_pad,
                                   const double *w, const double *pi) {
  double acc = 0.0;
  for (int c = 0; c < C; ++c) {
    const T *row = (s == 4) ? (L + ((size_t)i * C + c) * 4) : (L + ((size_t)c * p_pad + i) * s_pad);
    double sc = 0.0;
    for (int z = 0; z < s; ++z) sc = fma(pi[z], (double)row[z], sc);
    acc = fma(w[c], sc, acc);
  }
  return acc;
}

// ---------------------------------------------------------------------- K4
// lnL_i = ln(sum_c w_c sum_z pi_z L_root[i][c][z]) + E_i ln 2; block sums of
// wt_i lnL_i go to `blocks`, k_final adds them in a fixed order.
template <typename T>
__global__ void __launch_bounds__(256)
k_root(const T *__restrict__ L, int s, int s_pad, int C, const double *__restrict__ w,
       const double *__restrict__ pi, const int32_t *__restrict__ cum,
       const double *__restrict__ pw, int p, int p_pad, double *__restrict__ site,
       double *__restrict__ blocks, unsigned *__restrict__ count, double *__restrict__ out) {
  __shared__ double red[32];
  double part = 0.0;
  if (s_pad == 64) {
    // 61 states ([c][p_pad][64] rows of 256 B): one warp per pattern, lanes over
    // states (coalesced row reads), a fixed-order shuffle reduction
    const int lane = threadIdx.x & 31;
    const int nw = (gridDim.x * blockDim.x) >> 5;
    for (int i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < p; i += nw) {
      double a = 0.0;
      for (int c = 0; c < C; ++c) {
        const T *row = L + ((size_t)c * p_pad + i) * 64;
        double sc = lane < s ? pi[lane] * (double)row[lane] : 0.0;
        if (lane + 32 < s) sc = fma(pi[lane + 32], (double)row[lane + 32], sc);
        a = fma(w[c], sc, a);
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
      if (lane == 0) {
        double l = log(a);
        if (cum != nullptr) l += (double)cum[i] * kLn2;
        site[i] = l;
        part += pw[i] * l;
      }
    }
    finish_sum(part, red, blocks, count, out);
    return;
  }
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < p; i += gridDim.x * blockDim.x) {
    const double a = site_root(L, s, s_pad, C, i, p_pad, w, pi);
    double l = log(a);
    if (cum != nullptr) l += (double)cum[i] * kLn2;
    site[i] = l;
    part += pw[i] * l;
  }
  finish_sum(part, red, blocks, count, out);
}

// K4 for 4 states: C threads per pattern, thread c reads the pattern's
// category-c vector (16 / 32 contiguous bytes: a warp reads 512 / 1,024
// contiguous bytes per load) and forms sum_z pi_z L[z]; the category sum is
// gathered by shuffles in category order, so every site lnL is the same fp64
// value as site_root's.
template <typename T, int C>
__global__ void __launch_bounds__(256)
k_root4(const T *__restrict__ L, const double *__restrict__ w, const double *__restrict__ pi,
        const int32_t *__restrict__ cum, const double *__restrict__ pw, int p, double *__restrict__ site,
        double *__restrict__ blocks, unsigned *__restrict__ count, double *__restrict__ out) {
  __shared__ double red[32];
  double part = 0.0;
  const int lane = threadIdx.x & 31, c = lane % C;
  const double p0 = pi[0], p1 = pi[1], p2 = pi[2], p3 = pi[3];
  const int stride = (gridDim.x * blockDim.x) / C;
  for (int i0 = (blockIdx.x * blockDim.x + (threadIdx.x & ~31)) / C; i0 < p; i0 += stride) {
    const int i = i0 + lane / C;
    const bool valid = i < p;
    double sc = 0.0;
    if (valid) {
      const T *row = L + ((size_t)i * C + c) * 4;
      sc = fma(p0, (double)row[0], sc);
      sc = fma(p1, (double)row[1], sc);
      sc = fma(p2, (double)row[2], sc);
      sc = fma(p3, (double)row[3], sc);
    }
    double acc = 0.0;
#pragma unroll
    for (int k = 0; k < C; ++k) acc = fma(w[k], __shfl_sync(0xffffffffu, sc, (lane - c) + k), acc);
    if (valid && c == 0) {
      double l = log(acc);
      if (cum != nullptr) l += (double)cum[i] * kLn2;
      site[i] = l;
      part += pw[i] * l;
    }
  }
  finish_sum(part, red, blocks, count, out);
}

// ---------------------------------------------------------------------- K6
template <typename T>
__global__ void __launch_bounds__(256)
k_edge(const T *__restrict__ Lp, const void *__restrict__ child, int child_is_tip,
       const T *__restrict__ P, int s, int s_pad, int C, const double *__restrict__ w,
       const double *__restrict__ pi, const int32_t *__restrict__ cum_p,
       const int32_t *__restrict__ cum_c, const double *__restrict__ pw, int p, int p_pad,
       double *__restrict__ site, double *__restrict__ blocks, unsigned *__restrict__ count,
       double *__restrict__ out) {
  __shared__ double red[32];
  double part = 0.0;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < p; i += gridDim.x * blockDim.x) {
    double acc = 0.0;
    const unsigned st = child_is_tip ? (unsigned)static_cast<const uint8_t *>(child)[i] : 0u;
    for (int c = 0; c < C; ++c) {
      const size_t off = (s == 4) ? ((size_t)i * C + c) * 4 : ((size_t)c * p_pad + i) * s_pad;
      const T *lp = Lp + off;
      const T *lc = child_is_tip ? nullptr : static_cast<const T *>(child) + off;
      const T *Pc = P + (size_t)c * s_pad * s_pad;
      double sc = 0.0;
      for (int z = 0; z < s; ++z) {
        double v = 0.0;
        if (child_is_tip) {
          if (st < (unsigned)s) {
            v = (double)Pc[z * s_pad + st];
          } else {
            for (int x = 0; x < s; ++x) v += (double)Pc[z * s_pad + x];
          }
        } else {
          for (int x = 0; x < s; ++x) v = fma((double)Pc[z * s_pad + x], (double)lc[x], v);
        }
        sc = fma(pi[z] * (double)lp[z], v, sc);
      }
      acc = fma(w[c], sc, acc);
    }
    double l = log(acc);
    if (cum_p != nullptr) l += (double)cum_p[i] * kLn2;
    if (cum_c != nullptr) l += (double)cum_c[i] * kLn2;
    site[i] = l;
    part += pw[i] * l;
  }
  finish_sum(part, red, blocks, count, out);
}

}  // namespace

int launch_transition_matrices(int prec, int s, int s_pad, int c, const double *d_eig,
                               const double *d_rates, const int32_t *d_idx, const double *d_t,
                               int count, void *d_P, void *d_Plo, void *d_PT, void *stream) {
  if (count <= 0) return 0;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (s_pad == 64) {  // codon: register-tiled, persistent blocks over (matrix, category) items
    const size_t smem64 = sizeof(double) * (2 * 64 * 64 + 64);
    const int items = count * c;
    static int grid_caps[kMaxDevices] = {};
    int &grid_cap = grid_caps[device_slot()];
    if (grid_cap == 0) {
      int dev = 0, nsm = 0, per = 0;
      cudaGetDevice(&dev);
      cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
      cudaFuncSetAttribute(k_transition64<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem64);
      cudaFuncSetAttribute(k_transition64<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem64);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_transition64<double>, 256, smem64);
      grid_cap = nsm * (per > 0 ? per : 1);
    }
    const int grid = items < grid_cap ? items : grid_cap;
    if (prec == 32)
      k_transition64<float><<<grid, 256, smem64, st>>>(s, c, items, d_eig, d_rates, d_idx, d_t,
                                                       static_cast<float *>(d_P), static_cast<float *>(d_Plo),
                                                       static_cast<float *>(d_PT));
    else
      k_transition64<double><<<grid, 256, smem64, st>>>(s, c, items, d_eig, d_rates, d_idx, d_t,
                                                        static_cast<double *>(d_P), nullptr,
                                                        static_cast<double *>(d_PT));
    return (int)cudaGetLastError();
  }
  if (s == 4 && s_pad == 4) {
    const long long th = 4LL * count * c;
    const int blocks = (int)((th + 127) / 128);
    if (prec == 32)
      k_transition4<float><<<blocks, 128, 0, st>>>(c, count, d_eig, d_rates, d_idx, d_t, static_cast<float *>(d_P));
    else
      k_transition4<double><<<blocks, 128, 0, st>>>(c, count, d_eig, d_rates, d_idx, d_t, static_cast<double *>(d_P));
    return (int)cudaGetLastError();
  }
  const size_t smem = sizeof(double) * (2 * s * s + s);
  const int threads = (s <= 4) ? 32 : 256;
  for (int o = 0; o < count; o += 65535) {
    const int n = (count - o) < 65535 ? (count - o) : 65535;
    if (prec == 32) {
      if (smem > 48 * 1024)
        cudaFuncSetAttribute(k_transition<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      k_transition<float><<<dim3(n, c), threads, smem, st>>>(s, s_pad, c, d_eig, d_rates, d_idx + o,
                                                             d_t + o, static_cast<float *>(d_P));
    } else {
      if (smem > 48 * 1024)
        cudaFuncSetAttribute(k_transition<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      k_transition<double><<<dim3(n, c), threads, smem, st>>>(s, s_pad, c, d_eig, d_rates, d_idx + o,
                                                              d_t + o, static_cast<double *>(d_P));
    }
  }
  return (int)cudaGetLastError();
}

int launch_accumulate_scale(const int32_t *d_scale, int p_pad, const int32_t *d_idx, int count,
                            int32_t *d_cum, int p, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  int blocks = (p + 255) / 256;
  if (blocks > 148 * 8) blocks = 148 * 8;
  k_accumulate<<<blocks, 256, 0, st>>>(d_scale, p_pad, d_idx, count, d_cum, p);
  return (int)cudaGetLastError();
}

int launch_root_lnl(int prec, int s, int s_pad, int c, const void *root, const double *d_w,
                    const double *d_pi, const int32_t *cum, const double *d_pw, int p, int p_pad,
                    double *d_site, double *d_block, unsigned *d_count, int nblocks, double *d_out,
                    void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (s == 4 && s_pad == 4 && (c == 1 || c == 2 || c == 4 || c == 8)) {
#define RRL_ROOT4(T, CC)                                                                                 \
  k_root4<T, CC><<<nblocks, 256, 0, st>>>(static_cast<const T *>(root), d_w, d_pi, cum, d_pw, p, d_site, \
                                          d_block, d_count, d_out)
    if (prec == 32) {
      if (c == 1) RRL_ROOT4(float, 1); else if (c == 2) RRL_ROOT4(float, 2);
      else if (c == 4) RRL_ROOT4(float, 4); else RRL_ROOT4(float, 8);
    } else {
      if (c == 1) RRL_ROOT4(double, 1); else if (c == 2) RRL_ROOT4(double, 2);
      else if (c == 4) RRL_ROOT4(double, 4); else RRL_ROOT4(double, 8);
    }
#undef RRL_ROOT4
    return (int)cudaGetLastError();
  }
  if (prec == 32)
    k_root<float><<<nblocks, 256, 0, st>>>(static_cast<const float *>(root), s, s_pad, c, d_w, d_pi,
                                           cum, d_pw, p, p_pad, d_site, d_block, d_count, d_out);
  else
    k_root<double><<<nblocks, 256, 0, st>>>(static_cast<const double *>(root), s, s_pad, c, d_w, d_pi,
                                            cum, d_pw, p, p_pad, d_site, d_block, d_count, d_out);
  return (int)cudaGetLastError();
}

int launch_edge_lnl(int prec, int s, int s_pad, int c, const void *par, const void *child,
                    int child_is_tip, const void *P, const double *d_w, const double *d_pi,
                    const int32_t *cum_p, const int32_t *cum_c, const double *d_pw, int p, int p_pad,
                    double *d_site, double *d_block, unsigned *d_count, int nblocks, double *d_out,
                    void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (prec == 32)
    k_edge<float><<<nblocks, 256, 0, st>>>(static_cast<const float *>(par), child, child_is_tip,
                                           static_cast<const float *>(P), s, s_pad, c, d_w, d_pi,
                                           cum_p, cum_c, d_pw, p, p_pad, d_site, d_block, d_count, d_out);
  else
    k_edge<double><<<nblocks, 256, 0, st>>>(static_cast<const double *>(par), child, child_is_tip,
                                            static_cast<const double *>(P), s, s_pad, c, d_w, d_pi,
                                            cum_p, cum_c, d_pw, p, p_pad, d_site, d_block, d_count, d_out);
  return (int)cudaGetLastError();
}

int launch_codon_pt(int prec, const void *P, void *PT, int c, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (prec == 32)
    k_codon_pt<float><<<c, 64, 0, st>>>(static_cast<const float *>(P), static_cast<float *>(PT), c);
  else
    k_codon_pt<double><<<c, 64, 0, st>>>(static_cast<const double *>(P), static_cast<double *>(PT), c);
  return (int)cudaGetLastError();
}

int launch_split_tf32(const float *x, float *lo, size_t n, void *stream) {
  if (n == 0) return 0;
  const size_t blocks = (n + 255) / 256;
  k_split_tf32<<<(unsigned)(blocks < 4096 ? blocks : 4096), 256, 0, static_cast<cudaStream_t>(stream)>>>(x, lo, n);
  return (int)cudaGetLastError();
}

// Tip-state validation on the device (rrl_set_tip_states_u8): any code > s in
// `bytes` bytes (a multiple of 16: whole p_pad rows) sets *flag.  The padding
// columns hold s (missing), which passes.
__global__ void k_check_states(const uint4 *__restrict__ d, size_t n16, unsigned s, unsigned *__restrict__ flag) {
  unsigned bad = 0;
  const unsigned lim = s * 0x01010101u;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x) {
    const uint4 v = __ldg(d + i);
    // per-byte unsigned compare: __vcmpgtu4 gives 0xff in every byte where v > s
    bad |= __vcmpgtu4(v.x, lim) | __vcmpgtu4(v.y, lim) | __vcmpgtu4(v.z, lim) | __vcmpgtu4(v.w, lim);
  }
  if (__any_sync(0xffffffffu, bad != 0) && (threadIdx.x & 31) == 0) atomicOr(flag, 1u);
}

int launch_check_states(const uint8_t *d, size_t bytes, int s, unsigned *flag, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaMemsetAsync(flag, 0, sizeof(unsigned), st);
  if (e != cudaSuccess || bytes == 0) return (int)e;
  const size_t n16 = bytes / 16, blocks = (n16 + 255) / 256;
  k_check_states<<<(unsigned)(blocks < 2368 ? blocks : 2368), 256, 0, st>>>(reinterpret_cast<const uint4 *>(d),
                                                                           n16, (unsigned)s, flag);
  return (int)cudaGetLastError();
}

}  // namespace rrl
