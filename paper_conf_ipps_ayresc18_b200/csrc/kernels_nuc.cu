// K2: level-set updatePartials for 4-state models (sm_100a).
//
// Eq. (1) (§II-A) for every operation of one concurrent set in a
// single launch (§VI-A multi-operation kernel): grid.y indexes
// the operation, grid.x the pattern block.  Device layout [p][c][4]: one
// thread owns one (pattern, category) pair, i.e. one 16-byte (fp32) or 32-byte
// (fp64) state vector per child, so a warp moves 512 contiguous bytes per
// child per item with 128-bit loads.  The four transition matrices a thread
// needs (its category, both branches) live in registers; tip children are
// uint8 state codes resolved by selecting a column of P (code 4 = missing ->
// the row sum, i.e. an all-ones partial vector).
//
// Rescaling (reading A5) is fused: the C lanes of a pattern
// reduce max over (c, z) with warp shuffles, the frexp exponent e is taken,
// the outputs are multiplied by 2^-e (exact) and e (own, or own + children's
// cumulative) is stored as int32.
//
// HBM-bound: per (pattern, op) 2 x c x 4 x sizeof(T) child bytes (tips: 1 B)
// + c x 4 x sizeof(T) out + 4 B exponent; 1.8 flop/B in fp32.
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int kThreads = 256;

template <typename T> struct V4;
template <> struct V4<float> {
  __device__ static inline void ld(const float *p, float (&v)[4]) {
    const float4 x = __ldg(reinterpret_cast<const float4 *>(p));
    v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
  }
  __device__ static inline void st(float *p, const float (&v)[4]) {
    *reinterpret_cast<float4 *>(p) = make_float4(v[0], v[1], v[2], v[3]);
  }
};
template <> struct V4<double> {
  __device__ static inline void ld(const double *p, double (&v)[4]) {
    const double2 a = __ldg(reinterpret_cast<const double2 *>(p));
    const double2 b = __ldg(reinterpret_cast<const double2 *>(p) + 1);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
  __device__ static inline void st(double *p, const double (&v)[4]) {
    reinterpret_cast<double2 *>(p)[0] = make_double2(v[0], v[1]);
    reinterpret_cast<double2 *>(p)[1] = make_double2(v[2], v[3]);
  }
};

__device__ inline float frexp_t(float m, int *e) { return frexpf(m, e); }
__device__ inline double frexp_t(double m, int *e) { return frexp(m, e); }
__device__ inline float ldexp_t(float x, int e) { return ldexpf(x, e); }
__device__ inline double ldexp_t(double x, int e) { return ldexp(x, e); }

template <typename T>
__device__ inline void tip_column(const T (&P)[16], const T (&rs)[4], unsigned st, T (&v)[4]) {
#pragma unroll
  for (int z = 0; z < 4; ++z) {
    T a = P[z * 4 + 0];
    a = (st == 1u) ? P[z * 4 + 1] : a;
    a = (st == 2u) ? P[z * 4 + 2] : a;
    a = (st == 3u) ? P[z * 4 + 3] : a;
    v[z] = (st >= 4u) ? rs[z] : a;
  }
}

template <typename T>
__device__ inline void matvec(const T (&P)[16], const T (&L)[4], T (&v)[4]) {
#pragma unroll
  for (int z = 0; z < 4; ++z)
    v[z] = P[z * 4 + 0] * L[0] + P[z * 4 + 1] * L[1] + P[z * 4 + 2] * L[2] + P[z * 4 + 3] * L[3];
}

template <typename T, int C, int ITEMS>
__global__ void __launch_bounds__(kThreads)
k_partials_nuc(const DevOp *__restrict__ ops, int p) {
  const DevOp *opp = ops + blockIdx.y;
  const int flags = opp->flags;
  const void *in1 = opp->in1;
  const void *in2 = opp->in2;
  T *__restrict__ out = static_cast<T *>(opp->out);
  int32_t *__restrict__ scale_out = opp->scale_out;
  const int32_t *__restrict__ scale_in = opp->scale_in;
  const int32_t *__restrict__ cum1 = opp->cum1;
  const int32_t *__restrict__ cum2 = opp->cum2;

  const int cat = threadIdx.x % C;  // kThreads is a multiple of C
  T P1[16], P2[16], rs1[4], rs2[4];
  {
    const T *a = static_cast<const T *>(opp->P1) + cat * 16;
    const T *b = static_cast<const T *>(opp->P2) + cat * 16;
#pragma unroll
    for (int k = 0; k < 16; ++k) { P1[k] = __ldg(a + k); P2[k] = __ldg(b + k); }
#pragma unroll
    for (int z = 0; z < 4; ++z) {
      rs1[z] = P1[z * 4] + P1[z * 4 + 1] + P1[z * 4 + 2] + P1[z * 4 + 3];
      rs2[z] = P2[z * 4] + P2[z * 4 + 1] + P2[z * 4 + 2] + P2[z * 4 + 3];
    }
  }

  const long long base = (long long)blockIdx.x * (kThreads * ITEMS) + threadIdx.x;
  T L1[ITEMS][4], L2[ITEMS][4];
  unsigned s1[ITEMS], s2[ITEMS];
  // ---- load phase: all child reads of this thread in flight together
#pragma unroll
  for (int j = 0; j < ITEMS; ++j) {
    const long long item = base + j * kThreads;
    const int pat = (int)(item / C);
    const bool valid = pat < p;
    if (flags & OP_TIP1) {
      s1[j] = valid ? (unsigned)__ldg(static_cast<const uint8_t *>(in1) + pat) : 4u;
    } else if (valid) {
      V4<T>::ld(static_cast<const T *>(in1) + item * 4, L1[j]);
    } else {
#pragma unroll
      for (int z = 0; z < 4; ++z) L1[j][z] = T(0);
    }
    if (flags & OP_TIP2) {
      s2[j] = valid ? (unsigned)__ldg(static_cast<const uint8_t *>(in2) + pat) : 4u;
    } else if (valid) {
      V4<T>::ld(static_cast<const T *>(in2) + item * 4, L2[j]);
    } else {
#pragma unroll
      for (int z = 0; z < 4; ++z) L2[j][z] = T(0);
    }
  }
  // ---- compute + store phase
#pragma unroll
  for (int j = 0; j < ITEMS; ++j) {
    const long long item = base + j * kThreads;
    const int pat = (int)(item / C);
    const bool valid = pat < p;
    T v1[4], v2[4], r[4];
    if (flags & OP_TIP1) tip_column(P1, rs1, s1[j], v1); else matvec(P1, L1[j], v1);
    if (flags & OP_TIP2) tip_column(P2, rs2, s2[j], v2); else matvec(P2, L2[j], v2);
#pragma unroll
    for (int z = 0; z < 4; ++z) r[z] = v1[z] * v2[z];
    if (scale_out != nullptr) {
      T m = valid ? fmax(fmax(r[0], r[1]), fmax(r[2], r[3])) : T(0);
#pragma unroll
      for (int o = 1; o < C; o <<= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
      int e = 0;
      frexp_t(m, &e);
      if (m == T(0)) e = 0;
      if (e != 0) {
        if (e > -120 && e < 120) {
          const T f = ldexp_t(T(1), -e);
#pragma unroll
          for (int z = 0; z < 4; ++z) r[z] *= f;
        } else {
#pragma unroll
          for (int z = 0; z < 4; ++z) r[z] = ldexp_t(r[z], -e);
        }
      }
      if (valid && cat == 0) {
        int tot = e;
        if (cum1 != nullptr) tot += __ldg(cum1 + pat);
        if (cum2 != nullptr) tot += __ldg(cum2 + pat);
        scale_out[pat] = tot;
      }
    } else if (scale_in != nullptr) {
      const int e = valid ? __ldg(scale_in + pat) : 0;
#pragma unroll
      for (int z = 0; z < 4; ++z) r[z] = ldexp_t(r[z], -e);
    }
    if (valid) V4<T>::st(out + item * 4, r);
  }
}

template <typename T, int C>
int launch_t(const DevOp *ops, int nops, int p, cudaStream_t st) {
  constexpr int ITEMS = (sizeof(T) == 4) ? 2 : 2;
  const long long items = (long long)p * C;
  const int gx = (int)((items + kThreads * ITEMS - 1) / (kThreads * ITEMS));
  for (int o = 0; o < nops; o += 65535) {
    const int ny = (nops - o) < 65535 ? (nops - o) : 65535;
    k_partials_nuc<T, C, ITEMS><<<dim3(gx, ny), kThreads, 0, st>>>(ops + o, p);
  }
  return (int)cudaGetLastError();
}

template <typename T>
int dispatch_c(int c, const DevOp *ops, int nops, int p, cudaStream_t st) {
  switch (c) {
    case 1: return launch_t<T, 1>(ops, nops, p, st);
    case 2: return launch_t<T, 2>(ops, nops, p, st);
    case 4: return launch_t<T, 4>(ops, nops, p, st);
    case 8: return launch_t<T, 8>(ops, nops, p, st);
    default: return (int)cudaErrorInvalidValue;
  }
}

}  // namespace

int launch_update_partials_nuc(int prec, int c, const DevOp *ops, int nops, int p, int /*p_pad*/,
                               void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  return prec == 32 ? dispatch_c<float>(c, ops, nops, p, st) : dispatch_c<double>(c, ops, nops, p, st);
}

}  // namespace rrl
