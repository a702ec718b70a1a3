// K3-TC: 61-state codon updatePartials on the 5th-generation tensor cores
// (tcgen05.mma kind::tf32, accumulators in TMEM), fp32 instances with c <= 4.
//
// Eq. (1) (§II-A) for s = 61 is, per operation, category c and
// 128-pattern tile, two dense products
//     D_b[p][z] = sum_x A_b[p][x] P_b[c][z][x]      (b = child 1, 2)
// followed by out = D_1 .* D_2 and the per-pattern rescale (max over (c, z)).
// This is the one place on the hot path that really is a dense contraction
// (BASELINE north star), so it runs on tcgen05:
//  * M = 128 patterns (TMEM lanes), N = 64 states (61 padded), K = 64 child
//    states in 8 steps of K = 8 (tf32).
//  * fp32 accuracy with 3xTF32: x = hi + lo, hi = x with the low 13 mantissa
//    bits cleared (exact), lo = x - hi rounded to the nearest tf32 (the tensor
//    core truncates operands to tf32; truncating lo would bias every
//    correction by up to 2^-22 in one direction).  The MMA aligns the addends of
//    an accumulation to the accumulator with ~20 bits and truncates, which
//    costs ~0.5 ulp of bias per accumulation step (tools/diag_codon_tc.py:
//    9e-7 for a 64-term sum in one accumulator vs 6e-7 on SIMT FP32).  So the
//    hi*hi terms go to four accumulators (two K steps each) and the
//    ~2^-11-smaller hi*lo + lo*hi corrections to a fifth; the five meet in
//    fp32 in the epilogue.  A tip child's A tile is one-hot (all ones for a
//    missing state -> row sums), exact in tf32, so its lo*hi is skipped.
//  * Work is a pipeline of phases (tile, category, child): while the MMAs of
//    phase k run, all 256 threads build phase k+1's operands (global loads,
//    hi/lo split) into the other half of a double-buffered shared-memory ring,
//    directly in the canonical no-swizzle K-major UMMA layout (8-row x 16-byte
//    core matrices; LBO = 128 B between the two K halves, SBO = 256 B between
//    8-row groups), published to the async proxy with fence.proxy.async; one
//    thread issues the MMAs and tcgen05.commit's them to an mbarrier.
//  * Epilogue of a phase: all 8 warps (warp w: TMEM lane quarter w%4, column
//    half w/4) sum the five accumulators (tcgen05.ld 32x32b.x16).  Child 1's
//    result is parked in shared memory; child 2's is multiplied with it,
//    stored unscaled and folded into the running max over (c, z).  After the
//    last category the two column halves exchange their maxima, and every
//    thread rescales its own rows by the exact 2^-e (an L2-resident re-read).
// Persistent CTAs (one per SM: 320 TMEM columns, ~225 KB of shared memory)
// walk the flattened (operation, tile) space of the level set.
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int TM = 128;  // patterns per tile = MMA M = TMEM lanes
constexpr int TS = 64;   // padded states: MMA N and K
constexpr int kS61 = 61;
constexpr int kThr = 256;
constexpr int A_BYTES = TM * TS * 4;  // 32 KB per operand tile
constexpr int B_BYTES = TS * TS * 4;  // 16 KB
constexpr int BUF_BYTES = 2 * A_BYTES + 2 * B_BYTES;  // A hi/lo + B hi/lo of one phase
constexpr int S1_STRIDE = TS;  // rows of 16 x 16-byte chunks, chunk k stored at k ^ (row & 15)
// smem: 2 operand buffers, child-1 result, tip states [tile parity][child][128],
// row maxima [2 halves][128], mbarrier, TMEM base address
constexpr int SMEM_BUF = 0;
constexpr int SMEM_S1 = 2 * BUF_BYTES;
constexpr int SMEM_ST = SMEM_S1 + TM * S1_STRIDE * 4;
constexpr int SMEM_MX = SMEM_ST + 2 * 2 * TM;
constexpr int SMEM_BAR = SMEM_MX + 2 * TM * 4;
constexpr int SMEM_TMEM = SMEM_BAR + 8;
constexpr int SMEM_TOTAL = SMEM_TMEM + 8;
constexpr int kTmemCols = 512;  // 5 x 64 accumulator columns (4 main + 1 correction) ...
constexpr int kProdCol = 5 * TS;  // ... then the parked unscaled products of categories 0..C-2

__device__ inline uint32_t smem_addr(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
// byte offset of the 16-byte chunk (row r, k-chunk j) in a K-major no-swizzle
// UMMA tile: [kb = j/2][row group r/8][k half j%2][row r%8][16 B]
__device__ inline uint32_t umma_off(int r, int j, int rows) {
  return (uint32_t)((j >> 1) * (rows * 32) + (r >> 3) * 256 + (j & 1) * 128 + (r & 7) * 16);
}
__device__ inline uint64_t umma_desc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)(128 >> 4) << 16) |
         ((uint64_t)(256 >> 4) << 32) | ((uint64_t)1 << 46);
}
// kind::tf32, D f32, A/B tf32 K-major, N = 64, M = 128
constexpr uint32_t kIdesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(TS >> 3) << 17) |
                            ((uint32_t)(TM >> 4) << 24);

__device__ inline void mma_tf32(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(kIdesc), "r"(acc));
}
__device__ inline void mma_commit(uint64_t *bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_addr(bar))
               : "memory");
}
__device__ inline void bar_wait(uint64_t *bar, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred P1;\nW_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra W_%=;\n}\n" ::"r"(smem_addr(bar)),
      "r"(parity)
      : "memory");
}
__device__ inline void tmem_ld16(uint32_t taddr, float (&v)[16]) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ inline void tmem_st16(uint32_t taddr, const float *v) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
      "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])), "r"(__float_as_uint(v[3])),
      "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])), "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7])),
      "r"(__float_as_uint(v[8])), "r"(__float_as_uint(v[9])), "r"(__float_as_uint(v[10])), "r"(__float_as_uint(v[11])),
      "r"(__float_as_uint(v[12])), "r"(__float_as_uint(v[13])), "r"(__float_as_uint(v[14])), "r"(__float_as_uint(v[15]))
      : "memory");
}
__device__ inline void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ inline void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ inline void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ inline void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ inline float tf32_hi(float x) { return __uint_as_float(__float_as_uint(x) & 0xffffe000u); }
// lo part rounded to the nearest tf32 (the tensor core would truncate it,
// a one-sided 2^-22 relative bias per correction term)
__device__ inline float tf32_rn(float x) { return __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xffffe000u); }

__device__ inline void sts128(uint32_t addr, float a, float b, float c, float d) {
  asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "f"(a), "f"(b), "f"(c), "f"(d)
               : "memory");
}

#ifdef RRL_TC_TRACE
// dev-only phase timeline of CTA 0, thread 0 (tools/microbench/codon_tc_trace.cu)
__device__ long long g_tc_trace[256][5];
#define TC_TRACE(g, k)                                                      \
  do {                                                                      \
    if (blockIdx.x == 0 && threadIdx.x == 0 && (g) < 256) g_tc_trace[g][k] = clock64(); \
  } while (0)
#else
#define TC_TRACE(g, k) \
  do {                 \
  } while (0)
#endif

__device__ inline int frexp_e(float m) {
  const unsigned b = __float_as_uint(m);
  const int eb = (int)((b >> 23) & 0xffu);
  if (eb != 0 && eb != 0xff) return eb - 126;
  if (m == 0.f) return 0;
  int e;
  frexpf(m, &e);
  return e;
}

template <int C>
__global__ void __launch_bounds__(kThr, 1)
k_partials_codon_tc(const DevOp *__restrict__ ops, int p, int p_pad, int ntiles, int total) {
  // categories 0..C-2 wait in TMEM for the tile's exponent when they fit
  constexpr bool kProdInTmem = kProdCol + (C - 1) * TS <= kTmemCols;
  extern __shared__ __align__(1024) unsigned char sm[];
  uint64_t *bar = reinterpret_cast<uint64_t *>(sm + SMEM_BAR);
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(sm + SMEM_TMEM);
  uint8_t *st_s = sm + SMEM_ST;
  float *S1 = reinterpret_cast<float *>(sm + SMEM_S1);
  float *mx = reinterpret_cast<float *>(sm + SMEM_MX);
  const uint32_t sbase = smem_addr(sm);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tmem_slot)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" :::);

  const int my_tiles = total > (int)blockIdx.x ? (total - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
  const int nphase = my_tiles * C * 2;  // phases (tile, category, child)

  // tip states of local tile lt (parity lt & 1)
  auto load_states = [&](int lt) {
    const int f = blockIdx.x + lt * gridDim.x;
    const DevOp &op = ops[f / ntiles];
    const int p0 = (f % ntiles) * TM;
    const void *in[2] = {op.in1, op.in2};
    const int fl[2] = {op.flags & OP_TIP1, op.flags & OP_TIP2};
    for (int b = 0; b < 2; ++b)
      if (fl[b] && tid < TM) {
        const int pp = p0 + tid;
        st_s[((lt & 1) * 2 + b) * TM + tid] = pp < op.p ? static_cast<const uint8_t *>(in[b])[pp] : (uint8_t)kS61;
      }
  };

  // Operands of phase g: fetch(g) issues every global load of the phase into
  // registers (fa / fb); stage(g) converts them (hi/lo split, or the one-hot
  // rows of a tip child) into buffer g & 1 in the UMMA layout.  fetch runs a
  // phase ahead of stage, so each phase's load latency hides behind the
  // previous phase's conversion, MMA wait and epilogue.
  constexpr int NA = TM * 16 / kThr, NB = TS * 16 / kThr;  // 16-byte chunks per thread
  float4 fa[NA], fb[NB];
  auto fetch = [&](int g) {
    const int lt = g / (2 * C), c = (g / 2) % C, b = g & 1;
    const int f = blockIdx.x + lt * gridDim.x;
    const DevOp &op = ops[f / ntiles];
    const int p0 = (f % ntiles) * TM;
    const bool tip = (op.flags & (b == 0 ? OP_TIP1 : OP_TIP2)) != 0;
    if (!tip) {
      const float *A = static_cast<const float *>(b == 0 ? op.in1 : op.in2) + ((size_t)c * p_pad + p0) * TS;
#pragma unroll
      for (int u = 0; u < NA; ++u) {
        const int i = tid + u * kThr;
        const int kh = i & 1, rr = (i >> 1) & (TM - 1), kb = i >> 8;
        fa[u] = (p0 + rr < op.p) ? __ldg(reinterpret_cast<const float4 *>(A + (size_t)rr * TS + (kb * 2 + kh) * 4))
                              : make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
    const float *P = static_cast<const float *>(b == 0 ? op.P1 : op.P2) + (size_t)c * TS * TS;
#pragma unroll
    for (int u = 0; u < NB; ++u) {  // natural [z][x] layout = K-major B
      const int i = tid + u * kThr;
      const int kh = i & 1, z = (i >> 1) & (TS - 1), kb = i >> 7;
      fb[u] = __ldg(reinterpret_cast<const float4 *>(P + z * TS + (kb * 2 + kh) * 4));
    }
  };
  auto stage = [&](int g) {
    const int lt = g / (2 * C), b = g & 1;
    const int f = blockIdx.x + lt * gridDim.x;
    const DevOp &op = ops[f / ntiles];
    const bool tip = (op.flags & (b == 0 ? OP_TIP1 : OP_TIP2)) != 0;
    const uint32_t a_hi = sbase + SMEM_BUF + (g & 1) * BUF_BYTES, a_lo = a_hi + A_BYTES;
    const uint32_t b_hi = a_hi + 2 * A_BYTES, b_lo = b_hi + B_BYTES;
    if (!tip) {
#pragma unroll
      for (int u = 0; u < NA; ++u) {
        const int i = tid + u * kThr;
        const int kh = i & 1, rr = (i >> 1) & (TM - 1), kb = i >> 8;
        const uint32_t o = umma_off(rr, kb * 2 + kh, TM);
        const float4 v = fa[u];
        const float h0 = tf32_hi(v.x), h1 = tf32_hi(v.y), h2 = tf32_hi(v.z), h3 = tf32_hi(v.w);
        sts128(a_hi + o, h0, h1, h2, h3);
        sts128(a_lo + o, tf32_rn(v.x - h0), tf32_rn(v.y - h1), tf32_rn(v.z - h2), tf32_rn(v.w - h3));
      }
    } else {
      const uint8_t *sts = st_s + ((lt & 1) * 2 + b) * TM;
#pragma unroll
      for (int u = 0; u < NA; ++u) {
        const int i = tid + u * kThr;
        const int kh = i & 1, rr = (i >> 1) & (TM - 1), kb = i >> 8;
        const int j = kb * 2 + kh;
        const unsigned sv = sts[rr];
        float v[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const unsigned k = (unsigned)(j * 4 + q);
          v[q] = (sv < (unsigned)kS61) ? (k == sv ? 1.f : 0.f) : (k < (unsigned)kS61 ? 1.f : 0.f);
        }
        sts128(a_hi + umma_off(rr, j, TM), v[0], v[1], v[2], v[3]);
      }
    }
#pragma unroll
    for (int u = 0; u < NB; ++u) {
      const int i = tid + u * kThr;
      const int kh = i & 1, z = (i >> 1) & (TS - 1), kb = i >> 7;
      const uint32_t o = umma_off(z, kb * 2 + kh, TS);
      const float4 v = fb[u];
      const float h0 = tf32_hi(v.x), h1 = tf32_hi(v.y), h2 = tf32_hi(v.z), h3 = tf32_hi(v.w);
      sts128(b_hi + o, h0, h1, h2, h3);
      sts128(b_lo + o, tf32_rn(v.x - h0), tf32_rn(v.y - h1), tf32_rn(v.z - h2), tf32_rn(v.w - h3));
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> async proxy
  };

  // single thread: the MMAs of phase g (operands in buffer g & 1)
  auto issue = [&](int g) {
    const int lt = g / (2 * C), b = g & 1;
    const int f = blockIdx.x + lt * gridDim.x;
    const bool tip = (ops[f / ntiles].flags & (b == 0 ? OP_TIP1 : OP_TIP2)) != 0;
    const uint32_t a_hi = sbase + SMEM_BUF + (g & 1) * BUF_BYTES, a_lo = a_hi + A_BYTES;
    const uint32_t b_hi = a_hi + 2 * A_BYTES, b_lo = b_hi + B_BYTES;
#pragma unroll
    for (int kb = 0; kb < TS / 8; ++kb) {
      const uint64_t ah = umma_desc(a_hi + kb * (TM * 32)), al = umma_desc(a_lo + kb * (TM * 32));
      const uint64_t bh = umma_desc(b_hi + kb * (TS * 32)), bl = umma_desc(b_lo + kb * (TS * 32));
      const uint32_t dmain = tmem + (uint32_t)((kb >> 1) * TS), dcorr = tmem + (uint32_t)(4 * TS);
      mma_tf32(dmain, ah, bh, (kb & 1) ? 1u : 0u);
      mma_tf32(dcorr, ah, bl, kb > 0 ? 1u : 0u);
      if (!tip) mma_tf32(dcorr, al, bh, 1u);
    }
    mma_commit(bar);
  };

  const int q = warp & 3, h = warp >> 2;  // TMEM lane quarter, column half
  const int r = q * 32 + lane;            // this thread's row (pattern) in the tile
  const uint32_t tl = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(h * 32);
  float m = 0.f;
  uint32_t phase = 0;

  if (nphase > 0) {
    load_states(0);
    fetch(0);
    __syncthreads();
    stage(0);
    if (nphase > 1) fetch(1);
    fence_before();
    __syncthreads();
    if (tid == 0) {
      fence_after();
      issue(0);
    }
  }
  for (int g = 0; g < nphase; ++g) {
    const int lt = g / (2 * C), c = (g / 2) % C, b = g & 1;
    TC_TRACE(g, 0);
    if (g + 1 < nphase) {
      if ((g + 1) % (2 * C) == 0) {  // next phase starts a new tile: its tip states
        load_states(lt + 1);
        __syncthreads();
      }
      stage(g + 1);                    // overlaps the MMAs of phase g
      if (g + 2 < nphase) fetch(g + 2);  // in flight through the epilogue of phase g
    }
    TC_TRACE(g, 1);
    bar_wait(bar, phase);
    phase ^= 1u;
    fence_after();
    TC_TRACE(g, 2);
    // ---- epilogue of phase g
    const int f = blockIdx.x + lt * gridDim.x;
    const DevOp &op = ops[f / ntiles];
    const int p0 = (f % ntiles) * TM;
    const int pp = p0 + r;
    const bool valid = pp < op.p;
    float d[32];
#pragma unroll
    for (int half = 0; half < 2; ++half) {
      float a0[16], a1[16], a2[16], a3[16], cc[16];
      tmem_ld16(tl + 0 * TS + half * 16, a0);
      tmem_ld16(tl + 1 * TS + half * 16, a1);
      tmem_ld16(tl + 2 * TS + half * 16, a2);
      tmem_ld16(tl + 3 * TS + half * 16, a3);
      tmem_ld16(tl + 4 * TS + half * 16, cc);
      tmem_wait_ld();
#pragma unroll
      for (int i = 0; i < 16; ++i) d[half * 16 + i] = ((a0[i] + a1[i]) + (a2[i] + a3[i])) + cc[i];
    }
    // S1 chunk (row, k) lives at S1 + row*64 + 4*(k ^ (row & 15)): the 32 lanes
    // (32 rows) of a row-per-lane access hit different banks
    auto s1 = [&](int row, int k) -> float4 * {
      return reinterpret_cast<float4 *>(S1 + row * S1_STRIDE + 4 * (k ^ (row & 15)));
    };
    if (b == 0) {
#pragma unroll
      for (int i = 0; i < 8; ++i) *s1(r, h * 8 + i) = make_float4(d[4 * i], d[4 * i + 1], d[4 * i + 2], d[4 * i + 3]);
    } else {
      float *out = static_cast<float *>(op.out);
#pragma unroll
      for (int i = 0; i < 8; ++i) {  // product, running max over (c, z)
        const float4 v = *s1(r, h * 8 + i);
        d[4 * i] *= v.x; d[4 * i + 1] *= v.y; d[4 * i + 2] *= v.z; d[4 * i + 3] *= v.w;
        m = fmaxf(m, fmaxf(fmaxf(d[4 * i], d[4 * i + 1]), fmaxf(d[4 * i + 2], d[4 * i + 3])));
      }
      if constexpr (kProdInTmem) {
        if (c < C - 1) {  // park the unscaled product in TMEM until the exponent is known
          tmem_st16(tl + (uint32_t)(kProdCol + c * TS), d);
          tmem_st16(tl + (uint32_t)(kProdCol + c * TS + 16), d + 16);
          tmem_wait_st();
        }
      } else {
        __syncthreads();  // S1 no longer read as child 1: stage the product for a coalesced store
#pragma unroll
        for (int i = 0; i < 8; ++i) *s1(r, h * 8 + i) = make_float4(d[4 * i], d[4 * i + 1], d[4 * i + 2], d[4 * i + 3]);
        __syncthreads();
#pragma unroll
        for (int u = 0; u < TM * 16 / kThr; ++u) {
          const int i = tid + u * kThr, row = i >> 4, ch = i & 15;
          if (p0 + row < op.p)
            *reinterpret_cast<float4 *>(out + ((size_t)c * p_pad + p0 + row) * TS + ch * 4) = *s1(row, ch);
        }
      }
      if (c == C - 1) {  // ---- tile done: exponent from max over (c, z)
        mx[h * TM + r] = m;
        __syncthreads();
        if (h == 0) {
          const float mm = fmaxf(mx[r], mx[TM + r]);
          int e = 0;
          if (op.scale_out != nullptr) {
            e = frexp_e(mm);
            if (valid) {
              int tot = e;
              if (op.cum1 != nullptr) tot += op.cum1[pp];
              if (op.cum2 != nullptr) tot += op.cum2[pp];
              op.scale_out[pp] = tot;
            }
          } else if (op.scale_in != nullptr) {
            e = valid ? op.scale_in[pp] : 0;
          }
          mx[r] = (e > -126 && e < 126) ? __uint_as_float((unsigned)(127 - e) << 23) : ldexpf(1.f, -e);
        }
        __syncthreads();
        if constexpr (kProdInTmem) {
          // scaled categories staged all at once -- slot 0..2 in the operand
          // buffer MMA(g) has finished with, slot C-1 in S1 -- then coalesced
          // stores: one barrier for the tile instead of two per category
          const float sc = mx[r];
          float *slot_base = reinterpret_cast<float *>(sm + SMEM_BUF + (g & 1) * BUF_BYTES);
          auto slot = [&](int cat, int row, int k) -> float4 * {
            float *bse = (cat == C - 1) ? S1 : slot_base + cat * TM * TS;
            return reinterpret_cast<float4 *>(bse + row * S1_STRIDE + 4 * (k ^ (row & 15)));
          };
          for (int cat = 0; cat < C; ++cat) {
            float v[32];
            if (cat < C - 1) {
              float lo16[16], hi16[16];
              tmem_ld16(tl + (uint32_t)(kProdCol + cat * TS), lo16);
              tmem_ld16(tl + (uint32_t)(kProdCol + cat * TS + 16), hi16);
              tmem_wait_ld();
#pragma unroll
              for (int i = 0; i < 16; ++i) { v[i] = lo16[i]; v[16 + i] = hi16[i]; }
            } else {
#pragma unroll
              for (int i = 0; i < 32; ++i) v[i] = d[i];
            }
#pragma unroll
            for (int i = 0; i < 8; ++i)
              *slot(cat, r, h * 8 + i) = make_float4(v[4 * i] * sc, v[4 * i + 1] * sc, v[4 * i + 2] * sc, v[4 * i + 3] * sc);
          }
          __syncthreads();
          for (int cat = 0; cat < C; ++cat)
#pragma unroll
            for (int u = 0; u < TM * 16 / kThr; ++u) {
              const int i = tid + u * kThr, row = i >> 4, ch = i & 15;
              if (p0 + row < op.p)
                *reinterpret_cast<float4 *>(out + ((size_t)cat * p_pad + p0 + row) * TS + ch * 4) = *slot(cat, row, ch);
            }
        } else {
          // products already stored unscaled: coalesced in-place rescale (L2-resident)
          for (int cat = 0; cat < C; ++cat) {
            float4 v[TM * 16 / kThr];
#pragma unroll
            for (int u = 0; u < TM * 16 / kThr; ++u) {  // all loads first
              const int i = tid + u * kThr, row = i >> 4, ch = i & 15;
              v[u] = (p0 + row < op.p)
                         ? *reinterpret_cast<const float4 *>(out + ((size_t)cat * p_pad + p0 + row) * TS + ch * 4)
                         : make_float4(0.f, 0.f, 0.f, 0.f);
            }
#pragma unroll
            for (int u = 0; u < TM * 16 / kThr; ++u) {
              const int i = tid + u * kThr, row = i >> 4, ch = i & 15;
              const float sc = mx[row];
              if (p0 + row < op.p && sc != 1.f)
                *reinterpret_cast<float4 *>(out + ((size_t)cat * p_pad + p0 + row) * TS + ch * 4) =
                    make_float4(v[u].x * sc, v[u].y * sc, v[u].z * sc, v[u].w * sc);
            }
          }
        }
        m = 0.f;
      }
    }
    TC_TRACE(g, 3);
    fence_before();
    __syncthreads();  // TMEM accumulators read, S1 / maxima settled, phase g+1 operands visible
    TC_TRACE(g, 4);
    if (g + 1 < nphase && tid == 0) {
      fence_after();
      issue(g + 1);
    }
  }
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
}

template <int C>
int launch_tc(const DevOp *d_ops, int nops, int p, int p_pad, cudaStream_t st) {
  static int nsm_dev[kMaxDevices] = {};
  int &nsm = nsm_dev[device_slot()];
  if (nsm == 0) {
    cudaError_t e = cudaFuncSetAttribute(k_partials_codon_tc<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         SMEM_TOTAL);
    if (e != cudaSuccess) return (int)e;
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  }
  const int ntiles = (p + TM - 1) / TM;
  const long long total = (long long)ntiles * nops;
  if (total > 0x7fffffffLL) return (int)cudaErrorInvalidValue;
  const int grid = (int)(total < nsm ? total : nsm);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThr);
  cfg.dynamicSmemBytes = SMEM_TOTAL;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return (int)cudaLaunchKernelEx(&cfg, k_partials_codon_tc<C>, d_ops, p, p_pad, ntiles, (int)total);
}

}  // namespace

// fp32 codon instances, c in {1, 2, 4, 8}; cudaErrorNotSupported otherwise
// (the caller then uses the SIMT kernel).
int launch_update_partials_codon_tc(int c, const DevOp *d_ops, int nops, int p, int p_pad, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  switch (c) {
    case 1: return launch_tc<1>(d_ops, nops, p, p_pad, st);
    case 2: return launch_tc<2>(d_ops, nops, p, p_pad, st);
    case 4: return launch_tc<4>(d_ops, nops, p, p_pad, st);
    case 8: return launch_tc<8>(d_ops, nops, p, p_pad, st);
    default: return (int)cudaErrorNotSupported;
  }
}

}  // namespace rrl
