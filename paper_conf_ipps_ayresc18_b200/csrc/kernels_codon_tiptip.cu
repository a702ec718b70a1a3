// K3-TT: 61-state codon operations whose two children are tips (fp32, fp64).
//
// Eq. (1) (§II-A) with one-hot children is a gather, not a
// contraction: sum_x P1[z][x] [x = s1] = P1[z][s1], so
//     dest[c][p][z] = P1[c][z][s1(p)] * P2[c][z][s2(p)]
// (a missing state, code >= 61, is the row sum: the all-ones partials of
// reading A23).  These are exactly the cherries, i.e. the first level set of
// every tree: at configs[3] about 65 operations writing 10 MB each, so the
// launch is bound by its HBM stores (1 KB per pattern at c = 4) and the
// tensor-core kernel, which would land a P tile per (tile, category, child),
// is the wrong tool.  K1 writes P^T once per matrix (row x = column x of P,
// row 61 = the row sums), so a pattern's category row is one 256-byte
// coalesced read of an L1/L2-resident table per child.
//
// Mapping: a half-warp owns one pattern (lane q holds states 4q..4q+3 of every
// category), a warp two adjacent patterns, so every store instruction writes
// 512 contiguous bytes of the [c][p_pad][64] layout.  Rescaling (reading A5):
// m = max over (c, z) by four xor-shuffles inside the half-warp, e = frexp
// exponent, multiply by 2^-e (exact), int32 e stored (children are tips: no
// cumulative exponents to add).  Pattern-padding rows up to the next 128-row
// tile are written as zeros (the tensor-core kernel reads whole tiles).
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int kThrTT = 256;
constexpr int kChunkTT = 128;  // patterns per work item (one tensor-core tile)
constexpr int kMissing = 61;

__device__ inline int frexp_e_tt(float m) {
  const unsigned b = __float_as_uint(m);
  const int eb = (int)((b >> 23) & 0xffu);
  if (eb != 0 && eb != 0xff) return eb - 126;
  if (m == 0.f) return 0;
  int e;
  frexpf(m, &e);
  return e;
}
__device__ inline int frexp_e_tt(double m) {
  const unsigned long long b = (unsigned long long)__double_as_longlong(m);
  const int eb = (int)((b >> 52) & 0x7ffull);
  if (eb != 0 && eb != 0x7ff) return eb - 1022;
  if (m == 0.0) return 0;
  int e;
  frexp(m, &e);
  return e;
}
__device__ inline float pow2_neg_tt(float, int e) {
  return (e > -126 && e < 126) ? __uint_as_float((unsigned)(127 - e) << 23) : ldexpf(1.f, -e);
}
__device__ inline double pow2_neg_tt(double, int e) {
  return (e > -1022 && e < 1022) ? __longlong_as_double((long long)(1023 - e) << 52) : ldexp(1.0, -e);
}

// Four consecutive states of one row (16 bytes fp32, 32 bytes fp64).
template <typename T> struct Q4;
template <> struct Q4<float> {
  float v[4];
  __device__ void ld(const float *p) {
    const float4 x = __ldg(reinterpret_cast<const float4 *>(p));
    v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
  }
  __device__ void st(float *p) const { *reinterpret_cast<float4 *>(p) = make_float4(v[0], v[1], v[2], v[3]); }
};
template <> struct Q4<double> {
  double v[4];
  __device__ void ld(const double *p) {
    const double2 a = __ldg(reinterpret_cast<const double2 *>(p)), b = __ldg(reinterpret_cast<const double2 *>(p) + 1);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
  __device__ void st(double *p) const {
    reinterpret_cast<double2 *>(p)[0] = make_double2(v[0], v[1]);
    reinterpret_cast<double2 *>(p)[1] = make_double2(v[2], v[3]);
  }
};

template <typename T, int C>
__global__ void __launch_bounds__(kThrTT)
k_partials_codon_tiptip(const DevOp *__restrict__ ops, int nchunks, int total, int p_pad,
                        const T *__restrict__ PT) {
  asm volatile("griddepcontrol.wait;" ::: "memory");  // K1 / host uploads precede this launch
  asm volatile("griddepcontrol.launch_dependents;" :::);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int half = lane >> 4, q = lane & 15;
  constexpr size_t kMat = (size_t)C * 64 * 64;
  for (int item = blockIdx.x; item < total; item += gridDim.x) {
    const DevOp &op = ops[item / nchunks];
    const int p0 = (item % nchunks) * kChunkTT;
    const int p = op.p;
    if (p0 >= p) continue;  // a shorter pattern range of a partitioned call: not this op's rows
    const uint8_t *s1g = static_cast<const uint8_t *>(op.in1);
    const uint8_t *s2g = static_cast<const uint8_t *>(op.in2);
    const T *T1 = PT + (size_t)op.mat1 * kMat;
    const T *T2 = PT + (size_t)op.mat2 * kMat;
    T *out = static_cast<T *>(op.out);
#pragma unroll 2
    for (int k = warp * 2 + half; k < kChunkTT; k += 2 * (kThrTT / 32)) {
      const int pp = p0 + k;  // < p_tile: chunks are whole tiles
      const bool valid = pp < p;
      unsigned s1 = valid ? (unsigned)__ldg(s1g + pp) : 0u, s2 = valid ? (unsigned)__ldg(s2g + pp) : 0u;
      s1 = s1 < (unsigned)kMissing ? s1 : (unsigned)kMissing;
      s2 = s2 < (unsigned)kMissing ? s2 : (unsigned)kMissing;
      Q4<T> v[C];
      T m = T(0);
#pragma unroll
      for (int c = 0; c < C; ++c) {
        Q4<T> a, b;
        a.ld(T1 + (size_t)c * 4096 + s1 * 64 + 4 * q);
        b.ld(T2 + (size_t)c * 4096 + s2 * 64 + 4 * q);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          v[c].v[i] = a.v[i] * b.v[i];
          m = fmax(m, v[c].v[i]);
        }
      }
#pragma unroll
      for (int o = 1; o < 16; o <<= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
      int e = 0;
      if (op.scale_out != nullptr) e = frexp_e_tt(m);
      else if (op.scale_in != nullptr) e = valid ? __ldg(op.scale_in + pp) : 0;
      const T f = !valid ? T(0) : pow2_neg_tt(T(0), e);
#pragma unroll
      for (int c = 0; c < C; ++c) {
#pragma unroll
        for (int i = 0; i < 4; ++i) v[c].v[i] *= f;
        v[c].st(out + ((size_t)c * p_pad + pp) * 64 + 4 * q);
      }
      if (valid && q == 0 && op.scale_out != nullptr) op.scale_out[pp] = e;
    }
  }
}

template <typename T, int C>
int launch_tt(const DevOp *d_ops, int nops, int p, int p_pad, const T *PT, cudaStream_t st) {
  static int grid_dev[kMaxDevices] = {};
  int &grid_cap = grid_dev[device_slot()];
  if (grid_cap == 0) {
    int dev = 0, nsm = 148, per = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_partials_codon_tiptip<T, C>, kThrTT, 0);
    grid_cap = nsm * (per > 0 ? per : 1);
  }
  const int nchunks = (p + kChunkTT - 1) / kChunkTT;
  const long long total = (long long)nchunks * nops;
  if (total > 0x7fffffffLL) return (int)cudaErrorInvalidValue;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)(total < grid_cap ? total : grid_cap));
  cfg.blockDim = dim3(kThrTT);
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return (int)cudaLaunchKernelEx(&cfg, k_partials_codon_tiptip<T, C>, d_ops, nchunks, (int)total, p_pad, PT);
}

template <typename T>
int dispatch_tt(int c, const DevOp *d_ops, int nops, int p, int p_pad, const T *PT, cudaStream_t st) {
  switch (c) {
    case 1: return launch_tt<T, 1>(d_ops, nops, p, p_pad, PT, st);
    case 2: return launch_tt<T, 2>(d_ops, nops, p, p_pad, PT, st);
    case 4: return launch_tt<T, 4>(d_ops, nops, p, p_pad, PT, st);
    case 8: return launch_tt<T, 8>(d_ops, nops, p, p_pad, PT, st);
    default: return (int)cudaErrorNotSupported;
  }
}

}  // namespace

int launch_update_partials_codon_tiptip(int prec, int c, const DevOp *d_ops, int nops, int p, int p_pad,
                                        const void *d_PT, void *stream) {
  if (nops <= 0 || p <= 0) return 0;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  return prec == 32 ? dispatch_tt<float>(c, d_ops, nops, p, p_pad, static_cast<const float *>(d_PT), st)
                    : dispatch_tt<double>(c, d_ops, nops, p, p_pad, static_cast<const double *>(d_PT), st);
}

}  // namespace rrl
