// K3: level-set updatePartials for the 61-state codon model (sm_100a, SIMT).
//
// Eq. (1) (§II-A) with s = 61 ("61 for a codon model",
// PAPER.md:58): per operation, category c and pattern tile,
//     out[p][z] = (sum_x P1[c][z][x] A1[c][p][x]) * (sum_y P2[c][z][y] A2[c][p][y])
// i.e. two [patterns x 64] x [64 x 64] products multiplied elementwise, for an
// internal child; a tip child contributes the gathered column P[c][z][state]
// (missing state -> row sums).  Device layout [c][p_pad][64] (61 states padded
// to 64 with zeros, so every row is 256 B); padded states stay exactly zero
// because the padded rows/columns of P are zero.
//
// One CTA = one (operation, 64-pattern tile) for ALL categories, because the
// per-pattern rescale (reading A5) takes the max over
// (c, z).  256 threads: thread (pg, zg) owns patterns 4pg..4pg+3 and states
// {2zg, 2zg+1, 32+2zg, 33+2zg}, a 4x4 register tile; one child at a time sits in shared memory
// (per k step: 4 child values, padded rows, conflict-free, and a row of P^T
// for 16 FMAs).  Each category's unscaled product is stored at once and a
// running max over (c, z) kept; when the max is known (16-lane shuffle) the
// thread scales the values it stored by the exact power of two.
//
// This is the FP64 (and RRL_FLAG_CODON_SIMT fp32) path, ALU-bound: ~15 k
// flop per pattern-op at c = 4.  fp32 runs on the tcgen05 kernels
// (kernels_codon_tc5.cu, kernels_codon_tc.cu).
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int kS = 61;        // sense codons
constexpr int kSP = 64;       // padded states
constexpr int kTP = 64;       // patterns per CTA tile
constexpr int kThreads3 = 256;
constexpr int kAStride = 65;  // padded smem row (pattern-major A tile)
constexpr int kPRows = 65;    // P^T rows: x = 0..63, row 64 = row sums
constexpr int kPS = 68;       // P^T row stride (keeps 16-byte rows, 4-way staging conflicts)

__device__ inline int frexp_exp3(float m) {
  const unsigned b = __float_as_uint(m);
  const int eb = (int)((b >> 23) & 0xffu);
  if (eb != 0 && eb != 0xff) return eb - 126;
  if (m == 0.f) return 0;
  int e;
  frexpf(m, &e);
  return e;
}
__device__ inline int frexp_exp3(double m) {
  const unsigned long long b = (unsigned long long)__double_as_longlong(m);
  const int eb = (int)((b >> 52) & 0x7ffull);
  if (eb != 0 && eb != 0x7ff) return eb - 1022;
  if (m == 0.0) return 0;
  int e;
  frexp(m, &e);
  return e;
}
__device__ inline float pow2_neg(float, int e) {
  return (e > -126 && e < 126) ? __uint_as_float((unsigned)(127 - e) << 23) : ldexpf(1.f, -e);
}
__device__ inline double pow2_neg(double, int e) {
  return (e > -1022 && e < 1022) ? __longlong_as_double((long long)(1023 - e) << 52) : ldexp(1.0, -e);
}

template <typename T>
struct CodonSmem {
  T A[kTP * kAStride];   // one child tile, pattern-major, padded rows
  T Pt[kPRows * kPS];    // that child's P^T: Pt[x][z] = P[z][x]; row 64 = row sums
  uint8_t st[2][kTP];    // tip states
};

// State j (0..3) of thread group zg: {2zg, 2zg+1, 32+2zg, 33+2zg}, so that the
// 16 groups' pairs are contiguous (conflict-free 2-element shared loads,
// coalesced stores).
__device__ inline int zcol(int zg, int j) { return (j < 2 ? 0 : 32) + 2 * zg + (j & 1); }

template <typename T> struct Pair;
template <> struct Pair<float> {
  __device__ static inline void ld(const float *p, float &a, float &b) {
    const float2 v = *reinterpret_cast<const float2 *>(p);
    a = v.x; b = v.y;
  }
};
template <> struct Pair<double> {
  __device__ static inline void ld(const double *p, double &a, double &b) {
    const double2 v = *reinterpret_cast<const double2 *>(p);
    a = v.x; b = v.y;
  }
};

// One child (b) of category c for this thread's 4x4 (pattern, state) tile.
template <typename T>
__device__ inline void codon_child(CodonSmem<T> &sm, bool tip, int b, int pg, int zg, T (&acc)[4][4]) {
  if (tip) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const unsigned s = sm.st[b][pg * 4 + i];
      const int row = s < (unsigned)kS ? (int)s : 64;
      Pair<T>::ld(&sm.Pt[row * kPS + 2 * zg], acc[i][0], acc[i][1]);
      Pair<T>::ld(&sm.Pt[row * kPS + 32 + 2 * zg], acc[i][2], acc[i][3]);
    }
    return;
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = T(0);
  const T *Ab = &sm.A[(pg * 4) * kAStride];
  const T *Pb = &sm.Pt[2 * zg];
#pragma unroll 4
  for (int x = 0; x < kS; ++x) {
    T a[4], w[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) a[i] = Ab[i * kAStride + x];
    Pair<T>::ld(Pb + x * kPS, w[0], w[1]);
    Pair<T>::ld(Pb + x * kPS + 32, w[2], w[3]);
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = fma(a[i], w[j], acc[i][j]);
  }
}

// One child at a time in shared memory (68 KB in fp64, so two or three CTAs
// share an SM); each category's unscaled product goes straight to the output
// buffer while a running max over (c, z) is kept, and once the pattern's
// exponent is known the thread re-reads (L1/L2) and scales the values it wrote
// itself -- no per-category register file, no cross-thread hazard.
template <typename T, int C>
__global__ void __launch_bounds__(kThreads3, sizeof(T) == 8 ? 2 : 3)
k_partials_codon(const DevOp *__restrict__ ops, int p, int p_pad) {
  extern __shared__ __align__(16) unsigned char smem_raw3[];
  CodonSmem<T> &sm = *reinterpret_cast<CodonSmem<T> *>(smem_raw3);
  const DevOp &op = ops[blockIdx.y];
  p = op.p;  // this operation's pattern range (the grid covers the widest of the set)
  if ((int)blockIdx.x * kTP >= p) return;
  const bool tip[2] = {(op.flags & OP_TIP1) != 0, (op.flags & OP_TIP2) != 0};
  const void *in[2] = {op.in1, op.in2};
  const T *Pg[2] = {static_cast<const T *>(op.P1), static_cast<const T *>(op.P2)};
  const int p0 = blockIdx.x * kTP;
  const int tid = threadIdx.x;
  const int pg = tid >> 4, zg = tid & 15;  // 16 pattern groups x 16 state groups

  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" :::);

  for (int b = 0; b < 2; ++b)
    if (tip[b] && tid < kTP) {
      const int pp = p0 + tid;
      sm.st[b][tid] = pp < p ? static_cast<const uint8_t *>(in[b])[pp] : (uint8_t)kS;
    }

  // exponents known up front (stored factors) are applied in the first pass
  const bool two_pass = op.scale_out != nullptr;
  T f_in[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int pp = p0 + pg * 4 + i;
    f_in[i] = (!two_pass && op.scale_in != nullptr && pp < p) ? pow2_neg(T(0), op.scale_in[pp]) : T(1);
  }
  T *out = static_cast<T *>(op.out);
  T m[4] = {T(0), T(0), T(0), T(0)};
  for (int c = 0; c < C; ++c) {
    T prod[4][4];
    for (int b = 0; b < 2; ++b) {
      __syncthreads();  // the previous child's tiles are no longer read
      const T *P = Pg[b] + (size_t)c * kSP * kSP;
      for (int i = tid; i < kSP * kSP; i += kThreads3) {  // consecutive threads: consecutive z (conflict-free)
        const int z = i % kSP, x = i / kSP;
        sm.Pt[x * kPS + z] = __ldg(P + z * kSP + x);
      }
      if (!tip[b]) {
        const T *A = static_cast<const T *>(in[b]) + ((size_t)c * p_pad + p0) * kSP;
        for (int i = tid; i < kTP * kSP; i += kThreads3) {
          const int pp = i / kSP, x = i % kSP;
          sm.A[pp * kAStride + x] = A[i];  // rows beyond p exist (p_pad) and are never stored
        }
      }
      __syncthreads();
      if (tip[b]) {  // row sums (tip code >= 61 = missing)
        if (tid < kSP) {
          T acc = T(0);
          for (int x = 0; x < kSP; ++x) acc += sm.Pt[x * kPS + tid];
          sm.Pt[64 * kPS + tid] = acc;
        }
        __syncthreads();
      }
      T acc[4][4];
      codon_child(sm, tip[b], b, pg, zg, acc);
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) prod[i][j] = b == 0 ? acc[i][j] : prod[i][j] * acc[i][j];
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int pp = p0 + pg * 4 + i;
#pragma unroll
      for (int j = 0; j < 4; ++j) m[i] = fmax(m[i], prod[i][j]);
      if (pp < p) {
        T *dst = out + ((size_t)c * p_pad + pp) * kSP;
#pragma unroll
        for (int j = 0; j < 4; ++j) dst[zcol(zg, j)] = prod[i][j] * f_in[i];
      }
    }
  }
  if (!two_pass) return;

  // ---- rescale: max over (c, z) per pattern across the 16 zg lanes, then the
  // thread scales the values it stored above by the exact power of two
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int pp = p0 + pg * 4 + i;
    const bool valid = pp < p;
    T mm = m[i];
#pragma unroll
    for (int o = 1; o < 16; o <<= 1) mm = fmax(mm, __shfl_xor_sync(0xffffffffu, mm, o));
    const int e = frexp_exp3(mm);
    if (valid && zg == 0) {
      int tot = e;
      if (op.cum1 != nullptr) tot += op.cum1[pp];
      if (op.cum2 != nullptr) tot += op.cum2[pp];
      op.scale_out[pp] = tot;
    }
    const T f = pow2_neg(T(0), e);
    if (valid) {
#pragma unroll
      for (int c = 0; c < C; ++c) {
        T *dst = out + ((size_t)c * p_pad + pp) * kSP;
#pragma unroll
        for (int j = 0; j < 4; ++j) dst[zcol(zg, j)] = dst[zcol(zg, j)] * f;
      }
    }
  }
}

template <typename T, int C>
int launch_codon_t(const DevOp *d_ops, int nops, int p, int p_pad, cudaStream_t st) {
  const size_t smem = sizeof(CodonSmem<T>);
  static bool configured_dev[kMaxDevices] = {};
  bool &configured = configured_dev[device_slot()];
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(k_partials_codon<T, C>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return (int)e;
    configured = true;
  }
  const int gx = (p + kTP - 1) / kTP;
  for (int o = 0; o < nops; o += 65535) {
    const int ny = (nops - o) < 65535 ? (nops - o) : 65535;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(gx, ny);
    cfg.blockDim = dim3(kThreads3);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, k_partials_codon<T, C>, d_ops + o, p, p_pad);
    if (e != cudaSuccess) return (int)e;
  }
  return 0;
}

template <typename T>
int dispatch_codon(int c, const DevOp *d_ops, int nops, int p, int p_pad, cudaStream_t st) {
  switch (c) {
    case 1: return launch_codon_t<T, 1>(d_ops, nops, p, p_pad, st);
    case 2: return launch_codon_t<T, 2>(d_ops, nops, p, p_pad, st);
    case 4: return launch_codon_t<T, 4>(d_ops, nops, p, p_pad, st);
    case 8: return launch_codon_t<T, 8>(d_ops, nops, p, p_pad, st);
    default: return (int)cudaErrorInvalidValue;
  }
}

}  // namespace

int launch_update_partials_codon(int prec, int c, const DevOp *d_ops, const DevOp * /*h_ops*/, int nops,
                                 int p, int p_pad, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  return prec == 32 ? dispatch_codon<float>(c, d_ops, nops, p, p_pad, st)
                    : dispatch_codon<double>(c, d_ops, nops, p, p_pad, st);
}

}  // namespace rrl
