// K3-D: 61-state codon updatePartials in fp64 on the FP64 tensor cores (DMMA).
//
// Eq. (1) (§II-A) for s = 61: per operation, category c and
// 64-pattern tile, D_b = A_b . P_b^T for an internal child b (A_b [64 x 64]
// child partials, P_b [64 x 64] transition matrix), a gather P_b[z][state]
// for a tip child (missing state -> row sums, reading A23); out = D_1 .* D_2,
// rescaled per pattern by the exact power of two of max over (c, z)
// (reading A5).  tcgen05 has no fp64 kind, so the contraction is issued as
// mma.sync.m8n8k4.f64 (DMMA): exact fp64 products, fp64 accumulation --
// the same arithmetic class as the SIMT fp64 kernel, with one instruction per
// 8 x 8 x 4 block instead of 256 FMAs and one shared-memory operand load per
// 32 FMAs instead of per 8.
//
// One CTA = one (operation, 64-pattern tile), all categories (the rescale
// needs max over (c, z)).  8 warps; warp w owns patterns 8w..8w+7 and all 64
// states: per K-step of 4, one A fragment (its pattern row, 4 consecutive x)
// and 8 B fragments (one per 8-state block) -> 8 DMMAs into 8 accumulator
// pairs.  DMMA fragment layout (m8n8k4, f64): lane = 4 g + t; A[g][t],
// B[t][g] (= P[8j + g][4k + t]), D[g][2t + i].  So a thread owns ONE pattern
// (8w + g) and the 16 states 8j + 2t + i -- the tip gather and the per-pattern
// max are per-thread work plus two xor-shuffles over the 4 lanes of a pattern.
// Both operand tiles sit in shared memory with a 68-double row stride (a
// warp's 32 LDS.64 of a fragment are two conflict-free wavefronts).  Each
// category's unscaled product is stored at once with a running max kept; when
// the max is known the thread rescales what it stored (L1/L2 hits).
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int kS = 61, kSP = 64, kTPD = 64, kThrD = 256;
constexpr int kRow = 68;  // shared-memory row stride (doubles); column 64 of the P tile = row sums

struct DmmaSmem {
  double A[kTPD * kRow];  // child tile [pattern][x]
  double P[kSP * kRow];   // the child's P [z][x], column 64 = sum_x P[z][x]
  uint8_t st[2][kTPD];    // tip states of both children
};

__device__ inline void dmma(double (&d)[2], double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
               : "+d"(d[0]), "+d"(d[1])
               : "d"(a), "d"(b));
}
__device__ inline int frexp_e64(double m) {
  const unsigned long long b = (unsigned long long)__double_as_longlong(m);
  const int eb = (int)((b >> 52) & 0x7ffull);
  if (eb != 0 && eb != 0x7ff) return eb - 1022;
  if (m == 0.0) return 0;
  int e;
  frexp(m, &e);
  return e;
}
__device__ inline double pow2_neg64(int e) {
  return (e > -1022 && e < 1022) ? __longlong_as_double((long long)(1023 - e) << 52) : ldexp(1.0, -e);
}

template <int C>
__global__ void __launch_bounds__(kThrD, 2)
k_partials_codon_dmma(const DevOp *__restrict__ ops, int p_pad) {
  extern __shared__ __align__(16) unsigned char smem_d[];
  DmmaSmem &sm = *reinterpret_cast<DmmaSmem *>(smem_d);
  const DevOp &op = ops[blockIdx.y];
  const int p = op.p;  // this operation's pattern range (the grid covers the widest of the set)
  const int p0 = blockIdx.x * kTPD;
  if (p0 >= p) return;
  const bool tip[2] = {(op.flags & OP_TIP1) != 0, (op.flags & OP_TIP2) != 0};
  const void *in[2] = {op.in1, op.in2};
  const double *Pg[2] = {static_cast<const double *>(op.P1), static_cast<const double *>(op.P2)};
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, g = lane >> 2, t = lane & 3;
  const int prow = warp * 8 + g;  // this thread's pattern in the tile
  const int pp = p0 + prow;
  const bool valid = pp < p;

  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" :::);
  for (int b = 0; b < 2; ++b)
    if (tip[b] && tid < kTPD) {
      const int q = p0 + tid;
      sm.st[b][tid] = q < p ? static_cast<const uint8_t *>(in[b])[q] : (uint8_t)kS;
    }
  const bool two_pass = op.scale_out != nullptr;
  const double f_in = (!two_pass && op.scale_in != nullptr && valid) ? pow2_neg64(op.scale_in[pp]) : 1.0;
  double *out = static_cast<double *>(op.out);
  double m = 0.0;
  for (int c = 0; c < C; ++c) {
    double d1[16];
    for (int b = 0; b < 2; ++b) {
      __syncthreads();  // the previous child's tiles are no longer read
      const double *P = Pg[b] + (size_t)c * kSP * kSP;
      for (int i = tid; i < kSP * kSP / 2; i += kThrD) {  // 16-byte chunks, coalesced
        const int z = i / 32, x2 = (i % 32) * 2;
        *reinterpret_cast<double2 *>(&sm.P[z * kRow + x2]) = __ldg(reinterpret_cast<const double2 *>(P) + i);
      }
      if (!tip[b]) {
        const double *A = static_cast<const double *>(in[b]) + ((size_t)c * p_pad + p0) * kSP;
        for (int i = tid; i < kTPD * kSP / 2; i += kThrD) {  // rows beyond p exist (p_pad)
          const int r = i / 32, x2 = (i % 32) * 2;
          *reinterpret_cast<double2 *>(&sm.A[r * kRow + x2]) = reinterpret_cast<const double2 *>(A)[i];
        }
      }
      __syncthreads();
      double v[16];
      if (tip[b]) {
        if (tid < kSP) {  // row sums: the all-ones partials of a missing state
          double s = 0.0;
          for (int x = 0; x < kS; ++x) s += sm.P[tid * kRow + x];
          sm.P[tid * kRow + kSP] = s;
        }
        __syncthreads();
        const unsigned s = sm.st[b][prow];
        const int col = s < (unsigned)kS ? (int)s : kSP;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          v[2 * j] = sm.P[(8 * j + 2 * t) * kRow + col];
          v[2 * j + 1] = sm.P[(8 * j + 2 * t + 1) * kRow + col];
        }
      } else {
        double acc[8][2];
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[j][0] = acc[j][1] = 0.0;
        const double *Ar = &sm.A[prow * kRow + t];
        const double *Pr = &sm.P[g * kRow + t];
#pragma unroll 4
        for (int k = 0; k < kSP / 4; ++k) {
          const double a = Ar[4 * k];
#pragma unroll
          for (int j = 0; j < 8; ++j) dmma(acc[j], a, Pr[(8 * j) * kRow + 4 * k]);
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          v[2 * j] = acc[j][0];
          v[2 * j + 1] = acc[j][1];
        }
      }
      if (b == 0) {
#pragma unroll
        for (int i = 0; i < 16; ++i) d1[i] = v[i];
      } else {
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          d1[i] *= v[i];
          m = fmax(m, d1[i]);
        }
      }
    }
    if (valid) {  // this category's unscaled (or stored-factor) product, states 8j + 2t + {0, 1}
      double *dst = out + ((size_t)c * p_pad + pp) * kSP + 2 * t;
#pragma unroll
      for (int j = 0; j < 8; ++j)
        *reinterpret_cast<double2 *>(dst + 8 * j) = make_double2(d1[2 * j] * f_in, d1[2 * j + 1] * f_in);
    }
  }
  if (!two_pass) return;
  // ---- rescale: max over (c, z) of the pattern across its 4 lanes, then each
  // thread scales the values it stored above by the exact power of two
  m = fmax(m, __shfl_xor_sync(0xffffffffu, m, 1));
  m = fmax(m, __shfl_xor_sync(0xffffffffu, m, 2));
  const int e = frexp_e64(m);
  if (!valid) return;
  if (t == 0) {
    int tot = e;
    if (op.cum1 != nullptr) tot += op.cum1[pp];
    if (op.cum2 != nullptr) tot += op.cum2[pp];
    op.scale_out[pp] = tot;
  }
  const double f = pow2_neg64(e);
#pragma unroll
  for (int c = 0; c < C; ++c) {
    double2 *dst = reinterpret_cast<double2 *>(out + ((size_t)c * p_pad + pp) * kSP + 2 * t);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const double2 x = dst[4 * j];
      dst[4 * j] = make_double2(x.x * f, x.y * f);
    }
  }
}

template <int C>
int launch_dmma(const DevOp *d_ops, int nops, int p, int p_pad, cudaStream_t st) {
  const size_t smem = sizeof(DmmaSmem);
  static bool configured_dev[kMaxDevices] = {};
  bool &configured = configured_dev[device_slot()];
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(k_partials_codon_dmma<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)smem);
    if (e != cudaSuccess) return (int)e;
    configured = true;
  }
  const int gx = (p + kTPD - 1) / kTPD;
  for (int o = 0; o < nops; o += 65535) {
    const int ny = (nops - o) < 65535 ? (nops - o) : 65535;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(gx, ny);
    cfg.blockDim = dim3(kThrD);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, k_partials_codon_dmma<C>, d_ops + o, p_pad);
    if (e != cudaSuccess) return (int)e;
  }
  return 0;
}

}  // namespace

int launch_update_partials_codon_dmma(int c, const DevOp *d_ops, int nops, int p, int p_pad, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  switch (c) {
    case 1: return launch_dmma<1>(d_ops, nops, p, p_pad, st);
    case 2: return launch_dmma<2>(d_ops, nops, p, p_pad, st);
    case 4: return launch_dmma<4>(d_ops, nops, p, p_pad, st);
    case 8: return launch_dmma<8>(d_ops, nops, p, p_pad, st);
    default: return (int)cudaErrorNotSupported;
  }
}

}  // namespace rrl
