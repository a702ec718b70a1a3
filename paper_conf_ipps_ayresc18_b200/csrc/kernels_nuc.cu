// K2: level-set updatePartials for 4-state models (sm_100a).
//
// Eq. (1) (§II-A) for every operation of one concurrent set in a
// single launch (§VI-A multi-operation kernel): grid.y indexes
// the operation, grid.x strides over pattern chunks.  Device layout [p][c][4]:
// one thread owns one (pattern, category) pair, i.e. one 16-byte (fp32) or
// 32-byte (fp64) state vector per child, so a warp moves 512 contiguous bytes
// per child per item with 128-bit loads; U items per thread are loaded before
// any is consumed.  The two 4x4 transition matrices of the thread's category
// live in registers (loaded once per block); tip children are uint8 state
// codes resolved by selecting a column of P (code 4 = missing -> the row sum,
// i.e. an all-ones partial vector).
//
// Rescaling (reading A5) is fused: the C lanes of a pattern
// reduce max over (c, z) with warp shuffles, the frexp exponent e is read from
// the float's exponent bits, the outputs are multiplied by 2^-e (exact) and e
// (own, or own + children's cumulative) is stored as int32.
//
// Launch-latency path (narrow sets, e.g. 2 ops per set for a rerooted
// pectinate tree): operation descriptors for sets of <= kInline ops travel in
// the kernel parameters (no dependent descriptor load), and launches use
// programmatic dependent launch: a block resolves its descriptor, then waits
// (griddepcontrol.wait) for the previous level set before touching P or any
// partials, then lets the next set's grid start launching.
//
// HBM-bound for wide sets: per (pattern, op) 2 x c x 4 x sizeof(T) child bytes
// (tips: 1 B) + c x 4 x sizeof(T) out + exponents; 1.8 flop/B in fp32.
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int kThreads = 256;
constexpr int kInline = 8;

struct OpPack {
  const DevOp *ops;  // used when n > kInline
  int n;
  DevOp inl[kInline];
};

template <typename T> struct V4;
template <> struct V4<float> {
  __device__ static inline void ld(const float *p, float (&v)[4]) {
    const float4 x = __ldg(reinterpret_cast<const float4 *>(p));
    v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
  }
  __device__ static inline void st(float *p, const float (&v)[4]) {
    *reinterpret_cast<float4 *>(p) = make_float4(v[0], v[1], v[2], v[3]);
  }
  __device__ static inline void lds(const float *p, float (&v)[4]) {
    const float4 x = *reinterpret_cast<const float4 *>(p);
    v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
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
  __device__ static inline void lds(const double *p, double (&v)[4]) {
    const double2 a = reinterpret_cast<const double2 *>(p)[0];
    const double2 b = reinterpret_cast<const double2 *>(p)[1];
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
};

// frexp exponent e (m = f 2^e, f in [0.5,1)) and the exact factor 2^-e.
// Fast path from the exponent bits for normal m; library fallback otherwise.
__device__ inline int frexp_exp(float m) {
  const unsigned b = __float_as_uint(m);
  const int eb = (int)((b >> 23) & 0xffu);
  if (eb != 0 && eb != 0xff) return eb - 126;
  if (m == 0.f) return 0;
  int e;
  frexpf(m, &e);
  return e;
}
__device__ inline int frexp_exp(double m) {
  const unsigned long long b = (unsigned long long)__double_as_longlong(m);
  const int eb = (int)((b >> 52) & 0x7ffull);
  if (eb != 0 && eb != 0x7ff) return eb - 1022;
  if (m == 0.0) return 0;
  int e;
  frexp(m, &e);
  return e;
}
__device__ inline void scale_pow2(float (&r)[4], int e) {
  if (e > -126 && e < 126) {
    const float f = __uint_as_float((unsigned)(127 - e) << 23);
#pragma unroll
    for (int z = 0; z < 4; ++z) r[z] *= f;
  } else {
#pragma unroll
    for (int z = 0; z < 4; ++z) r[z] = ldexpf(r[z], -e);
  }
}
__device__ inline void scale_pow2(double (&r)[4], int e) {
  if (e > -1022 && e < 1022) {
    const double f = __longlong_as_double((long long)(1023 - e) << 52);
#pragma unroll
    for (int z = 0; z < 4; ++z) r[z] *= f;
  } else {
#pragma unroll
    for (int z = 0; z < 4; ++z) r[z] = ldexp(r[z], -e);
  }
}

// P rows of one (branch, category) in shared memory: 16 entries P[z][x] then
// the 4 row sums (the tip lookup of a missing state).  Stride 20 keeps the
// LDS.128 rows of the C categories a warp touches in distinct banks.
constexpr int kPStride = 20;

template <typename T>
__device__ inline void tip_column(const T *P, unsigned st, T (&v)[4]) {
#pragma unroll
  for (int z = 0; z < 4; ++z) v[z] = P[st < 4u ? z * 4 + (int)st : 16 + z];
}

template <typename T>
__device__ inline void matvec(const T *P, const T (&L)[4], T (&v)[4]) {
#pragma unroll
  for (int z = 0; z < 4; ++z) {
    T row[4];
    V4<T>::lds(P + z * 4, row);
    v[z] = fma(row[3], L[3], fma(row[2], L[2], fma(row[1], L[1], row[0] * L[0])));
  }
}

__device__ inline void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ inline void pdl_launch() { asm volatile("griddepcontrol.launch_dependents;" :::); }

template <typename T, int C, int U>
__global__ void __launch_bounds__(kThreads)
k_partials_nuc(const __grid_constant__ OpPack pack, int p, int nchunks) {
  __shared__ __align__(16) T sP[2][C][kPStride];
  const DevOp &op = (pack.n <= kInline) ? pack.inl[blockIdx.y] : pack.ops[blockIdx.y];
  const int flags = op.flags;
  const bool tip1 = flags & OP_TIP1, tip2 = flags & OP_TIP2;

  // Everything above overlaps the previous level set; below reads its outputs.
  pdl_wait();
  pdl_launch();

  if (threadIdx.x < 2 * C * 16) {
    const int b = threadIdx.x / (C * 16), r = threadIdx.x % (C * 16);
    const T *src = static_cast<const T *>(b == 0 ? op.P1 : op.P2);
    sP[b][r / 16][r % 16] = src[r];
  }
  __syncthreads();
  if (threadIdx.x < 2 * C * 4) {
    const int b = threadIdx.x / (C * 4), r = threadIdx.x % (C * 4), c = r / 4, z = r % 4;
    const T *row = &sP[b][c][z * 4];
    sP[b][c][16 + z] = row[0] + row[1] + row[2] + row[3];
  }
  __syncthreads();

  const int cat = threadIdx.x % C;  // kThreads is a multiple of C
  const T *P1 = &sP[0][cat][0];
  const T *P2 = &sP[1][cat][0];
  const T *__restrict__ L1g = static_cast<const T *>(op.in1);
  const T *__restrict__ L2g = static_cast<const T *>(op.in2);
  const uint8_t *__restrict__ S1g = static_cast<const uint8_t *>(op.in1);
  const uint8_t *__restrict__ S2g = static_cast<const uint8_t *>(op.in2);
  T *__restrict__ out = static_cast<T *>(op.out);
  const unsigned nitems = (unsigned)p * C;

  for (int chunk = blockIdx.x; chunk < nchunks; chunk += gridDim.x) {
    const unsigned base = (unsigned)chunk * (kThreads * U) + threadIdx.x;
    T L1[U][4], L2[U][4];
    unsigned s1[U], s2[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {  // ---- all child reads of this thread in flight together
      const unsigned item = base + j * kThreads;
      const bool valid = item < nitems;
      const unsigned pat = item / C;
      if (tip1) {
        s1[j] = valid ? (unsigned)__ldg(S1g + pat) : 4u;
      } else if (valid) {
        V4<T>::ld(L1g + (size_t)item * 4, L1[j]);
      } else {
#pragma unroll
        for (int z = 0; z < 4; ++z) L1[j][z] = T(0);
      }
      if (tip2) {
        s2[j] = valid ? (unsigned)__ldg(S2g + pat) : 4u;
      } else if (valid) {
        V4<T>::ld(L2g + (size_t)item * 4, L2[j]);
      } else {
#pragma unroll
        for (int z = 0; z < 4; ++z) L2[j][z] = T(0);
      }
    }
#pragma unroll
    for (int j = 0; j < U; ++j) {  // ---- compute + store
      const unsigned item = base + j * kThreads;
      const bool valid = item < nitems;
      const unsigned pat = item / C;
      T v1[4], v2[4], r[4];
      if (tip1) tip_column(P1, s1[j], v1); else matvec(P1, L1[j], v1);
      if (tip2) tip_column(P2, s2[j], v2); else matvec(P2, L2[j], v2);
#pragma unroll
      for (int z = 0; z < 4; ++z) r[z] = v1[z] * v2[z];
      if (op.scale_out != nullptr) {
        T m = valid ? fmax(fmax(r[0], r[1]), fmax(r[2], r[3])) : T(0);
#pragma unroll
        for (int o = 1; o < C; o <<= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
        const int e = frexp_exp(m);
        if (e != 0) scale_pow2(r, e);
        if (valid && cat == 0) {
          int tot = e;
          if (op.cum1 != nullptr) tot += __ldg(op.cum1 + pat);
          if (op.cum2 != nullptr) tot += __ldg(op.cum2 + pat);
          op.scale_out[pat] = tot;
        }
      } else if (op.scale_in != nullptr) {
        const int e = valid ? __ldg(op.scale_in + pat) : 0;
        if (e != 0) scale_pow2(r, e);
      }
      if (valid) V4<T>::st(out + (size_t)item * 4, r);
    }
  }
}

template <typename T, int C>
int launch_t(const DevOp *d_ops, const DevOp *h_ops, int nops, int p, cudaStream_t st) {
  constexpr int U = 2;
  const long long items = (long long)p * C;
  const int nchunks = (int)((items + kThreads * U - 1) / (kThreads * U));
  // ~8 resident blocks' worth of waves over 148 SMs, at least one chunk per block
  const int target = 148 * 4 * 4;
  int gx = (target + nops - 1) / nops;
  if (gx > nchunks) gx = nchunks;
  if (gx < 1) gx = 1;
  for (int o = 0; o < nops; o += 65535) {
    const int ny = (nops - o) < 65535 ? (nops - o) : 65535;
    OpPack pack{};
    pack.n = ny;
    pack.ops = d_ops + o;
    if (ny <= kInline && h_ops != nullptr)
      for (int i = 0; i < ny; ++i) pack.inl[i] = h_ops[o + i];
    if (ny <= kInline && h_ops == nullptr) pack.n = kInline + 1;  // force pointer path
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(gx, ny);
    cfg.blockDim = dim3(kThreads);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, k_partials_nuc<T, C, U>, pack, p, nchunks);
    if (e != cudaSuccess) return (int)e;
  }
  return (int)cudaGetLastError();
}

template <typename T>
int dispatch_c(int c, const DevOp *d_ops, const DevOp *h_ops, int nops, int p, cudaStream_t st) {
  switch (c) {
    case 1: return launch_t<T, 1>(d_ops, h_ops, nops, p, st);
    case 2: return launch_t<T, 2>(d_ops, h_ops, nops, p, st);
    case 4: return launch_t<T, 4>(d_ops, h_ops, nops, p, st);
    case 8: return launch_t<T, 8>(d_ops, h_ops, nops, p, st);
    default: return (int)cudaErrorInvalidValue;
  }
}

}  // namespace

int launch_update_partials_nuc(int prec, int c, const DevOp *d_ops, const DevOp *h_ops, int nops,
                               int p, int /*p_pad*/, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  return prec == 32 ? dispatch_c<float>(c, d_ops, h_ops, nops, p, st)
                    : dispatch_c<double>(c, d_ops, h_ops, nops, p, st);
}

}  // namespace rrl
