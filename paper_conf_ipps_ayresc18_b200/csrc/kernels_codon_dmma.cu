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
// needs max over (c, z)), 8 warps of 32 x 16 (pattern x state) tiles.  DMMA
// fragment layout (m8n8k4, f64): lane = 4 g + t; A[g][t], B[t][g] (= P[z][x]),
// D[g][2t + i].  The child tile of an internal child sits in shared memory
// (68-double rows: a warp's 32 LDS.64 of a fragment are two conflict-free
// wavefronts), double-buffered: the next internal stage is copied with
// cp.async while the current stage's DMMAs run.  B fragments come straight
// from the 32 KB P tile (L1-resident: every warp of the CTA reads it), and a
// tip child reads the thread's entries from row `state` of K1's P^T slab --
// no staging, no barrier.  Each category's unscaled product is stored at once
// with a running max kept; when the max is known the thread rescales what it
// stored.
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int kS = 61, kSP = 64, kTPD = 64, kThrD = 256;
constexpr int kRow = 68;  // shared-memory row stride of the A tile (doubles)

struct DmmaSmem {
  double A[2][kTPD * kRow];  // double-buffered child tiles [pattern][x]
  double mx[4][kTPD];        // per-pattern maxima of the 4 state-quarter warps
  uint8_t st[2][kTPD];       // tip states of both children
};

__device__ inline void dmma(double (&d)[2], double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
               : "+d"(d[0]), "+d"(d[1])
               : "d"(a), "d"(b));
}
__device__ inline void cp_async16(void *smem, const void *gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(smem))),
               "l"(gmem)
               : "memory");
}
__device__ inline void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ inline void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }
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

// Stage (c, b) of a CTA = category c, child b; only internal children stage an
// A tile.  The next internal stage's tile is copied (cp.async) into the other
// buffer while the current stage's DMMAs run.
//
// Warp tile 32 patterns x 16 states (wr = warp & 1, wc = warp >> 1): per
// K-step 4 A fragments (shared memory) and 2 B fragments (the 32 KB P tile,
// L1-resident) feed 8 DMMAs, so the L1 carries a quarter of the B traffic of
// an 8 x 64 warp tile (which measured 91 % L1 throughput, the limit).  A
// thread owns patterns 32 wr + 8 rb + g (rb < 4) and states 16 wc + 8 cb +
// 2 t + i (cb, i < 2); the per-pattern max over (c, z) is reduced over the 4
// lanes t by shuffles and over the 4 warps wc through shared memory.
// (Measured on configs[3] fp64: 8 x 64 warp tiles with B from L1 were L1-bound
// at 91 %, 7.75 ms per pass; these 32 x 16 tiles 5.17 ms; 16 warps over 128
// patterns with the P tile staged in shared memory too: 5.68 ms.)
template <int C>
__global__ void __launch_bounds__(kThrD, 2)
k_partials_codon_dmma(const DevOp *__restrict__ ops, int p_pad, const double *__restrict__ PT) {
  extern __shared__ __align__(16) unsigned char smem_d[];
  DmmaSmem &sm = *reinterpret_cast<DmmaSmem *>(smem_d);
  const DevOp &op = ops[blockIdx.y];
  const int p = op.p;  // this operation's pattern range (the grid covers the widest of the set)
  const int p0 = blockIdx.x * kTPD;
  if (p0 >= p) return;
  const bool tip[2] = {(op.flags & OP_TIP1) != 0, (op.flags & OP_TIP2) != 0};
  const void *in[2] = {op.in1, op.in2};
  const double *Pg[2] = {static_cast<const double *>(op.P1), static_cast<const double *>(op.P2)};
  const int mat[2] = {op.mat1, op.mat2};
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, g = lane >> 2, t = lane & 3;
  const int wr = warp & 1, wc = warp >> 1;
  const int zbase = 16 * wc + 2 * t;  // + 8 cb + i

  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" :::);
  auto stage_A = [&](int c, int b, int buf) {  // 64 rows x 512 B, 16-byte chunks; rows beyond p exist (p_pad)
    const double *A = static_cast<const double *>(in[b]) + ((size_t)c * p_pad + p0) * kSP;
    for (int i = tid; i < kTPD * kSP / 2; i += kThrD) {
      const int r = i / 32, x2 = (i % 32) * 2;
      cp_async16(&sm.A[buf][r * kRow + x2], A + 2 * i);
    }
    cp_async_commit();
  };
  const int nint = (tip[0] ? 0 : 1) + (tip[1] ? 0 : 1);
  int si = 0;  // internal stages consumed so far
  if (nint > 0) stage_A(0, tip[0] ? 1 : 0, 0);
  for (int b = 0; b < 2; ++b)
    if (tip[b] && tid < kTPD) {
      const int q = p0 + tid;
      sm.st[b][tid] = q < p ? static_cast<const uint8_t *>(in[b])[q] : (uint8_t)kS;
    }
  const bool two_pass = op.scale_out != nullptr;
  int prow[4];
  bool valid[4];
  double f_in[4], m[4];
#pragma unroll
  for (int rb = 0; rb < 4; ++rb) {
    prow[rb] = 32 * wr + 8 * rb + g;
    valid[rb] = p0 + prow[rb] < p;
    f_in[rb] = (!two_pass && op.scale_in != nullptr && valid[rb]) ? pow2_neg64(op.scale_in[p0 + prow[rb]]) : 1.0;
    m[rb] = 0.0;
  }
  double *out = static_cast<double *>(op.out);
  __syncthreads();  // tip states
  for (int c = 0; c < C; ++c) {
    double d1[4][4];  // [rb][2 cb + i]
#pragma unroll
    for (int b = 0; b < 2; ++b) {
      double v[4][4];
      if (tip[b]) {
        // P[z][s] for the thread's states: row s of P^T (K1; row 61 = row sums for
        // a missing state), two 16-byte pairs per pattern, L1/L2-resident
        const double *base = PT + ((size_t)mat[b] * C + c) * kSP * kSP + zbase;
#pragma unroll
        for (int rb = 0; rb < 4; ++rb) {
          const unsigned s = sm.st[b][prow[rb]];
          const double *row = base + (s < (unsigned)kS ? s : kS) * kSP;
#pragma unroll
          for (int cb = 0; cb < 2; ++cb) {
            const double2 x = __ldg(reinterpret_cast<const double2 *>(row + 8 * cb));
            v[rb][2 * cb] = x.x;
            v[rb][2 * cb + 1] = x.y;
          }
        }
      } else {
        const int buf = si & 1;
        cp_async_wait_all();
        __syncthreads();  // this stage's tile landed for every thread; the other buffer is free
        ++si;
        if (si < nint * C) {  // prefetch the next internal stage
          const int nb = (nint == 2) ? (b ^ 1) : b;
          const int nc = (nint == 2) ? (b == 1 ? c + 1 : c) : c + 1;
          stage_A(nc, nb, buf ^ 1);
        }
        double acc[4][2][2];
#pragma unroll
        for (int rb = 0; rb < 4; ++rb)
#pragma unroll
          for (int cb = 0; cb < 2; ++cb) acc[rb][cb][0] = acc[rb][cb][1] = 0.0;
        const double *Ar = &sm.A[buf][(32 * wr + g) * kRow + t];
        // B fragment B[x][z] = P[z][x], z = 16 wc + 8 cb + g, x = 4k + t
        const double *Pr = Pg[b] + (size_t)c * kSP * kSP + (16 * wc + g) * kSP + t;
#pragma unroll 4
        for (int k = 0; k < kSP / 4; ++k) {
          const double b0 = __ldg(Pr + 4 * k), b1 = __ldg(Pr + 8 * kSP + 4 * k);
#pragma unroll
          for (int rb = 0; rb < 4; ++rb) {
            const double a = Ar[(8 * rb) * kRow + 4 * k];
            dmma(acc[rb][0], a, b0);
            dmma(acc[rb][1], a, b1);
          }
        }
#pragma unroll
        for (int rb = 0; rb < 4; ++rb)
#pragma unroll
          for (int cb = 0; cb < 2; ++cb) {
            v[rb][2 * cb] = acc[rb][cb][0];
            v[rb][2 * cb + 1] = acc[rb][cb][1];
          }
      }
#pragma unroll
      for (int rb = 0; rb < 4; ++rb)
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          if (b == 0) {
            d1[rb][i] = v[rb][i];
          } else {
            d1[rb][i] *= v[rb][i];
            m[rb] = fmax(m[rb], d1[rb][i]);
          }
        }
    }
#pragma unroll
    for (int rb = 0; rb < 4; ++rb)  // this category's unscaled (or stored-factor) product
      if (valid[rb]) {
        double *dst = out + ((size_t)c * p_pad + p0 + prow[rb]) * kSP + zbase;
#pragma unroll
        for (int cb = 0; cb < 2; ++cb)
          *reinterpret_cast<double2 *>(dst + 8 * cb) =
              make_double2(d1[rb][2 * cb] * f_in[rb], d1[rb][2 * cb + 1] * f_in[rb]);
      }
  }
  if (!two_pass) return;
  // ---- rescale: max over (c, z) of each pattern: over the 4 lanes t, then over
  // the 4 warps wc sharing the pattern (shared memory), then each thread scales
  // the values it stored above by the exact power of two
#pragma unroll
  for (int rb = 0; rb < 4; ++rb) {
    m[rb] = fmax(m[rb], __shfl_xor_sync(0xffffffffu, m[rb], 1));
    m[rb] = fmax(m[rb], __shfl_xor_sync(0xffffffffu, m[rb], 2));
    if (t == 0) sm.mx[wc][prow[rb]] = m[rb];
  }
  __syncthreads();
#pragma unroll
  for (int rb = 0; rb < 4; ++rb) {
    if (!valid[rb]) continue;
    const double mm = fmax(fmax(sm.mx[0][prow[rb]], sm.mx[1][prow[rb]]), fmax(sm.mx[2][prow[rb]], sm.mx[3][prow[rb]]));
    const int e = frexp_e64(mm);
    const int pp = p0 + prow[rb];
    if (wc == 0 && t == 0) {
      int tot = e;
      if (op.cum1 != nullptr) tot += op.cum1[pp];
      if (op.cum2 != nullptr) tot += op.cum2[pp];
      op.scale_out[pp] = tot;
    }
    const double f = pow2_neg64(e);
#pragma unroll
    for (int c = 0; c < C; ++c) {
      double2 *dst = reinterpret_cast<double2 *>(out + ((size_t)c * p_pad + pp) * kSP + zbase);
#pragma unroll
      for (int cb = 0; cb < 2; ++cb) {
        const double2 x = dst[4 * cb];
        dst[4 * cb] = make_double2(x.x * f, x.y * f);
      }
    }
  }
}

template <int C>
int launch_dmma(const DevOp *d_ops, int nops, int p, int p_pad, const double *PT, cudaStream_t st) {
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
    cudaError_t e = cudaLaunchKernelEx(&cfg, k_partials_codon_dmma<C>, d_ops + o, p_pad, PT);
    if (e != cudaSuccess) return (int)e;
  }
  return 0;
}

}  // namespace

int launch_update_partials_codon_dmma(int c, const DevOp *d_ops, int nops, int p, int p_pad, const void *d_PT,
                                      void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const double *PT = static_cast<const double *>(d_PT);
  switch (c) {
    case 1: return launch_dmma<1>(d_ops, nops, p, p_pad, PT, st);
    case 2: return launch_dmma<2>(d_ops, nops, p, p_pad, PT, st);
    case 4: return launch_dmma<4>(d_ops, nops, p, p_pad, PT, st);
    case 8: return launch_dmma<8>(d_ops, nops, p, p_pad, PT, st);
    default: return (int)cudaErrorNotSupported;
  }
}

}  // namespace rrl
