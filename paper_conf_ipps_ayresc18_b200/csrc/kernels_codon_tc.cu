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
//  * Warp specialisation (one 288-thread CTA per SM, it owns all of TMEM):
//    phases (tile, category, child) flow from 4 producer warps (global loads,
//    hi/lo split straight into the canonical no-swizzle K-major UMMA layout
//    -- 8-row x 16-byte core matrices, LBO = 128 B, SBO = 256 B -- in a
//    2-stage shared-memory ring, fence.proxy.async) through one MMA-issuing
//    lane (tcgen05.mma + tcgen05.commit) to 4 epilogue warps, connected only
//    by mbarriers (full/empty per stage, acc_full/acc_empty for TMEM), so
//    loads, conversions, MMAs and epilogues of consecutive phases overlap.
//  * Epilogue (one pattern row per thread, tcgen05.ld 32x32b.x16): child 1
//    stays in registers, child 2 forms the product, which is parked in TMEM
//    for categories < C-1 (C <= 4 fits); after the last category the row's
//    exponent is known (max over (c, z) is thread-local), every category is
//    scaled and written once, coalesced, through a swizzled shared tile.
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
constexpr int kEpi = 256;             // warps 0-7: epilogue (TMEM lane quarter x column half)
constexpr int kProd = 128;            // warps 8-11: operand producers
constexpr int kThr = kEpi + kProd + 32;  // + warp 12: MMA issuer
constexpr int A_BYTES = TM * TS * 4;  // 32 KB per operand tile
constexpr int B_BYTES = TS * TS * 4;  // 16 KB
constexpr int BUF_BYTES = 2 * A_BYTES + 2 * B_BYTES;  // A hi/lo + B hi/lo of one phase
constexpr int S1_STRIDE = TS;  // rows of 16 x 16-byte chunks, chunk k stored at k ^ (row & 15)
// smem: 2-stage operand ring, epilogue staging tile, producer tip states
// [child][128], mbarriers full[2] empty[2] acc_full acc_empty, TMEM address
constexpr int SMEM_BUF = 0;
constexpr int SMEM_S1 = 2 * BUF_BYTES;
constexpr int SMEM_ST = SMEM_S1 + TM * S1_STRIDE * 4;
constexpr int SMEM_MX = SMEM_ST + 2 * TM;       // row maxima / scale factors [2][128]
constexpr int SMEM_BAR = SMEM_MX + 2 * TM * 4;
constexpr int SMEM_TMEM = SMEM_BAR + 6 * 8;
constexpr int SMEM_TOTAL = SMEM_TMEM + 8;
constexpr int kTmemCols = 512;    // 5 x 64 accumulator columns (4 main + 1 correction) ...
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

__device__ inline int frexp_e(float m) {
  const unsigned b = __float_as_uint(m);
  const int eb = (int)((b >> 23) & 0xffu);
  if (eb != 0 && eb != 0xff) return eb - 126;
  if (m == 0.f) return 0;
  int e;
  frexpf(m, &e);
  return e;
}

__device__ inline void mbar_init1(uint64_t *bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count));
}
__device__ inline void mbar_arrive1(uint64_t *bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
__device__ inline void named_sync(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

// Warp-specialised tcgen05 codon kernel.  Phases g = (local tile, category c,
// child b) flow through three roles connected by mbarriers:
//   producers (warps 4-7): wait empty[g&1]; load child tile + P rows; split
//     hi/lo into the UMMA layout of stage g&1; fence.proxy.async; arrive full[g&1]
//   MMA issuer (warp 8, one lane): wait full[g&1] and acc_empty; 8 K-steps of
//     main (4 accumulators) + correction MMAs; commit -> empty[g&1], acc_full
//   epilogue (warps 0-3, one pattern row per thread): wait acc_full; sum the
//     five accumulators; release acc_empty; child 1 -> registers, child 2 ->
//     product (parked in TMEM for categories < C-1); after the last category:
//     exponent of the row, scale, coalesced stores through a swizzled tile.
template <int C>
__global__ void __launch_bounds__(kThr, 1)
k_partials_codon_tc(const DevOp *__restrict__ ops, int p, int p_pad, int ntiles, int total) {
  static_assert(kProdCol + (C - 1) * TS <= kTmemCols, "parked products must fit TMEM");
  extern __shared__ __align__(1024) unsigned char sm[];
  uint64_t *full = reinterpret_cast<uint64_t *>(sm + SMEM_BAR);
  uint64_t *empty = full + 2;
  uint64_t *acc_full = full + 4;
  uint64_t *acc_empty = full + 5;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(sm + SMEM_TMEM);
  uint8_t *st_p = sm + SMEM_ST;
  float *S1 = reinterpret_cast<float *>(sm + SMEM_S1);
  const uint32_t sbase = smem_addr(sm);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tmem_slot)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == kEpi + kProd) {
    mbar_init1(&full[0], kProd / 32);
    mbar_init1(&full[1], kProd / 32);
    mbar_init1(&empty[0], 1);
    mbar_init1(&empty[1], 1);
    mbar_init1(acc_full, 1);
    mbar_init1(acc_empty, kEpi / 32);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" :::);

  const int my_tiles = total > (int)blockIdx.x ? (total - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
  const int nphase = my_tiles * C * 2;

  if (warp >= (kEpi + kProd) / 32) {
    // =============================================================== MMA issuer
    if (lane == 0) {
      for (int g = 0; g < nphase; ++g) {
        const int lt = g / (2 * C), b = g & 1;
        const int f = blockIdx.x + lt * gridDim.x;
        const bool tip = (ops[f / ntiles].flags & (b == 0 ? OP_TIP1 : OP_TIP2)) != 0;
        bar_wait(&full[g & 1], (uint32_t)(g >> 1) & 1u);
        bar_wait(acc_empty, (uint32_t)(g & 1) ^ 1u);
        fence_after();
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
        mma_commit(&empty[g & 1]);  // operand stage free once these MMAs completed
        mma_commit(acc_full);       // accumulators ready for the epilogue
      }
    }
  } else if (warp >= kEpi / 32) {
    // =============================================================== producers
    const int pt = tid - kEpi;
    int cur_tile = -1;
    for (int g = 0; g < nphase; ++g) {
      const int lt = g / (2 * C), c = (g / 2) % C, b = g & 1;
      const int f = blockIdx.x + lt * gridDim.x;
      const DevOp &op = ops[f / ntiles];
      const int p0 = (f % ntiles) * TM;
      if (lt != cur_tile) {  // the tile's tip states (both children)
        named_sync(2, kProd);  // every producer is done with the previous tile's states
        const uint8_t *s1p = static_cast<const uint8_t *>(op.in1), *s2p = static_cast<const uint8_t *>(op.in2);
        const int pp = p0 + pt;
        st_p[pt] = ((op.flags & OP_TIP1) && pp < p) ? s1p[pp] : (uint8_t)kS61;
        st_p[TM + pt] = ((op.flags & OP_TIP2) && pp < p) ? s2p[pp] : (uint8_t)kS61;
        named_sync(2, kProd);
        cur_tile = lt;
      }
      const bool tip = (op.flags & (b == 0 ? OP_TIP1 : OP_TIP2)) != 0;
      constexpr int NA = TM * 16 / kProd, NB = TS * 16 / kProd;  // 16-byte chunks per thread
      float4 fa[NA], fb[NB];
      // all global loads of the phase first (they overlap the wait for the stage)
      if (!tip) {
        const float *A = static_cast<const float *>(b == 0 ? op.in1 : op.in2) + ((size_t)c * p_pad + p0) * TS;
#pragma unroll
        for (int u = 0; u < NA; ++u) {
          const int i = pt + u * kProd;
          const int kh = i & 1, rr = (i >> 1) & (TM - 1), kb = i >> 8;
          fa[u] = (p0 + rr < p) ? __ldg(reinterpret_cast<const float4 *>(A + (size_t)rr * TS + (kb * 2 + kh) * 4))
                                : make_float4(0.f, 0.f, 0.f, 0.f);
        }
      }
      const float *P = static_cast<const float *>(b == 0 ? op.P1 : op.P2) + (size_t)c * TS * TS;
#pragma unroll
      for (int u = 0; u < NB; ++u) {  // natural [z][x] layout = K-major B
        const int i = pt + u * kProd;
        const int kh = i & 1, z = (i >> 1) & (TS - 1), kb = i >> 7;
        fb[u] = __ldg(reinterpret_cast<const float4 *>(P + z * TS + (kb * 2 + kh) * 4));
      }
      bar_wait(&empty[g & 1], ((uint32_t)(g >> 1) & 1u) ^ 1u);  // MMAs of phase g-2 done
      const uint32_t a_hi = sbase + SMEM_BUF + (g & 1) * BUF_BYTES, a_lo = a_hi + A_BYTES;
      const uint32_t b_hi = a_hi + 2 * A_BYTES, b_lo = b_hi + B_BYTES;
      if (!tip) {
#pragma unroll
        for (int u = 0; u < NA; ++u) {
          const int i = pt + u * kProd;
          const int kh = i & 1, rr = (i >> 1) & (TM - 1), kb = i >> 8;
          const uint32_t o = umma_off(rr, kb * 2 + kh, TM);
          const float4 v = fa[u];
          const float h0 = tf32_hi(v.x), h1 = tf32_hi(v.y), h2 = tf32_hi(v.z), h3 = tf32_hi(v.w);
          sts128(a_hi + o, h0, h1, h2, h3);
          sts128(a_lo + o, tf32_rn(v.x - h0), tf32_rn(v.y - h1), tf32_rn(v.z - h2), tf32_rn(v.w - h3));
        }
      } else {
        const uint8_t *sts = st_p + b * TM;
#pragma unroll
        for (int u = 0; u < NA; ++u) {
          const int i = pt + u * kProd;
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
        const int i = pt + u * kProd;
        const int kh = i & 1, z = (i >> 1) & (TS - 1), kb = i >> 7;
        const uint32_t o = umma_off(z, kb * 2 + kh, TS);
        const float4 v = fb[u];
        const float h0 = tf32_hi(v.x), h1 = tf32_hi(v.y), h2 = tf32_hi(v.z), h3 = tf32_hi(v.w);
        sts128(b_hi + o, h0, h1, h2, h3);
        sts128(b_lo + o, tf32_rn(v.x - h0), tf32_rn(v.y - h1), tf32_rn(v.z - h2), tf32_rn(v.w - h3));
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> async proxy
      __syncwarp();
      if (lane == 0) mbar_arrive1(&full[g & 1]);
    }
  } else {
    // =============================================================== epilogue
    // warp w: TMEM lane quarter w & 3 (one pattern row per thread), column
    // half h = w >> 2 (32 of the 64 states): two warps per lane quarter
    // double the tcgen05.ld throughput that paces the accumulator turnaround.
    const int h = warp >> 2;
    const int r = (warp & 3) * 32 + lane;
    const uint32_t tl = tmem + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)(h * 32);
    float *mx = reinterpret_cast<float *>(sm + SMEM_MX);
    auto s1 = [&](int row, int k) -> float4 * {
      return reinterpret_cast<float4 *>(S1 + row * S1_STRIDE + 4 * (k ^ (row & 15)));
    };
    float m = 0.f;  // child 1 of the current category waits in this thread's own S1 half-row
    for (int g = 0; g < nphase; ++g) {
      const int lt = g / (2 * C), c = (g / 2) % C, b = g & 1;
      const int f = blockIdx.x + lt * gridDim.x;
      const DevOp &op = ops[f / ntiles];
      const int p0 = (f % ntiles) * TM;
      const int pp = p0 + r;
      const bool valid = pp < p;
      bar_wait(acc_full, (uint32_t)g & 1u);
      fence_after();
      float dv[32];
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        float a0[16], a1[16], a2[16], a3[16], cc[16];
        tmem_ld16(tl + 0 * TS + q * 16, a0);
        tmem_ld16(tl + 1 * TS + q * 16, a1);
        tmem_ld16(tl + 2 * TS + q * 16, a2);
        tmem_ld16(tl + 3 * TS + q * 16, a3);
        tmem_ld16(tl + 4 * TS + q * 16, cc);
        tmem_wait_ld();
#pragma unroll
        for (int i = 0; i < 16; ++i) dv[q * 16 + i] = ((a0[i] + a1[i]) + (a2[i] + a3[i])) + cc[i];
      }
      fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive1(acc_empty);  // the MMAs of phase g+1 may overwrite them
      if (b == 0) {
#pragma unroll
        for (int k = 0; k < 8; ++k)
          *s1(r, h * 8 + k) = make_float4(dv[4 * k], dv[4 * k + 1], dv[4 * k + 2], dv[4 * k + 3]);
        continue;
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const float4 w = *s1(r, h * 8 + k);
        dv[4 * k] *= w.x; dv[4 * k + 1] *= w.y; dv[4 * k + 2] *= w.z; dv[4 * k + 3] *= w.w;
        m = fmaxf(m, fmaxf(fmaxf(dv[4 * k], dv[4 * k + 1]), fmaxf(dv[4 * k + 2], dv[4 * k + 3])));
      }
      if (c < C - 1) {  // park the unscaled product in TMEM until the exponent is known
        tmem_st16(tl + (uint32_t)(kProdCol + c * TS), dv);
        tmem_st16(tl + (uint32_t)(kProdCol + c * TS + 16), dv + 16);
        tmem_wait_st();
        continue;
      }
      // ---- tile done: row exponent from max over (c, z) of both halves
      mx[h * TM + r] = m;
      named_sync(1, kEpi);
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
      named_sync(1, kEpi);
      const float sc = mx[r];
      float *out = static_cast<float *>(op.out);
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
          for (int i = 0; i < 32; ++i) v[i] = dv[i];
        }
        named_sync(1, kEpi);  // staging tile free
#pragma unroll
        for (int k = 0; k < 8; ++k)
          *s1(r, h * 8 + k) = make_float4(v[4 * k] * sc, v[4 * k + 1] * sc, v[4 * k + 2] * sc, v[4 * k + 3] * sc);
        named_sync(1, kEpi);
        const int et = tid;  // 0..255
#pragma unroll
        for (int u = 0; u < TM * 16 / kEpi; ++u) {  // coalesced: a warp writes 2 rows
          const int i = et + u * kEpi, row = i >> 4, ch = i & 15;
          if (p0 + row < p)
            *reinterpret_cast<float4 *>(out + ((size_t)cat * p_pad + p0 + row) * TS + ch * 4) = *s1(row, ch);
        }
      }
      named_sync(1, kEpi);  // staging reads done before rows are reused for child 1
      m = 0.f;
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
}

template <int C>
int launch_tc(const DevOp *d_ops, int nops, int p, int p_pad, cudaStream_t st) {
  static int nsm = 0;
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

// fp32 codon instances, c in {1, 2, 4}; cudaErrorNotSupported otherwise
// (the caller then uses the SIMT kernel).
int launch_update_partials_codon_tc(int c, const DevOp *d_ops, int nops, int p, int p_pad, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  switch (c) {
    case 1: return launch_tc<1>(d_ops, nops, p, p_pad, st);
    case 2: return launch_tc<2>(d_ops, nops, p, p_pad, st);
    case 4: return launch_tc<4>(d_ops, nops, p, p_pad, st);
    default: return (int)cudaErrorNotSupported;  // c = 8: products do not fit TMEM -> SIMT
  }
}

}  // namespace rrl
