// K3-TC5: 61-state codon updatePartials, TMA-fed tcgen05 pipeline (fp32, c <= 4).
//
// Eq. (1) (§II-A) for s = 61: per operation, category c and
// 128-pattern tile, D_b = A_b . P_b^T for both children (A_b: [128 x 64]
// child partials, P_b: [64 x 64] transition matrix, K-major = its natural
// row-major layout), out = D_1 .* D_2, rescaled per pattern by the exact
// power of two of max over (c, z).
//
// Pipeline of phases (tile, category, child) through four warp roles, joined
// only by mbarriers (no block-wide barrier in steady state):
//  * producer (warp 12, one lane): TMA (cp.async.bulk.tensor.4d) of the
//    child tile straight from the [buffer][c][p_pad][64] partials slab and of
//    the P tile from the [matrix][c][64][64] slab into one of two 96 KB
//    stages, 128-byte swizzled -- the canonical SWIZZLE_128B K-major UMMA
//    layout, so the raw fp32 tile IS the tf32 "hi" operand (the tensor core
//    reads the top 19 bits of each 32-bit element);
//  * converters (warps 8-11): the tf32 "lo" parts of the child tile,
//    lo = rn_tf32(x - hi(x)), elementwise in place of layout (same swizzled
//    offsets); P's lo parts come precomputed from K1 (a second slab, TMA'd);
//  * a tip child (uint8 states) is no contraction at all: sum_x P[z][x] [x = obs]
//    = P[z][obs], so its phase lands only the raw P tile and the epilogue
//    gathers the column from shared memory (row sums for a missing state) --
//    no conversion, no MMA, no TMEM traffic;
//  * MMA issuer (warp 13, one lane): per K-step of 8, one N = 128 MMA
//    A_hi.[P_hi|P_lo]^T into [main_h | corr_h] and one N = 64 MMA A_lo.P_hi^T
//    into corr_h (h = K-half: two main accumulators, never mixed with the
//    corrections -- the accumulation-precision reading in DESIGN.md),
//    tcgen05.commit to the stage's `empty` and to `acc_full`;
//  * epilogue (warps 0-7: TMEM lane quarter w%4, column half w/4): sums the
//    four accumulators (tcgen05.ld 32x32b.x16), releases `acc_empty`, parks
//    child 1 in the category's TMEM slot, forms the product with child 2, parks
//    it in the same slot until the tile's last category, then scales by 2^-e
//    and writes every category once through a swizzled staging tile that a TMA
//    bulk tensor store drains asynchronously (padding rows as zeros).
// Compared with K3-TC (kernels_codon_tc.cu) the SM no longer moves the child
// tile through registers: per phase it only writes the lo halves.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "rrl_internal.h"

namespace rrl {

#ifdef RRL_TC5_TRACE  // dev build only (tools/trace_tc5.py): clock64 timeline of CTA 0
__device__ long long g_tc5_trace[18][4096];
__device__ int g_tc5_kind[4096];
#define TR(ev, g)                                                            \
  do {                                                                       \
    if (blockIdx.x == 0 && (g) < 4096) g_tc5_trace[ev][g] = clock64();      \
  } while (0)
#else
#define TR(ev, g) \
  do {            \
  } while (0)
#endif

namespace {

constexpr int TM = 128;  // patterns per tile = MMA M = TMEM lanes
constexpr int TS = 64;   // padded states: MMA N and K
constexpr int kS61 = 61;
constexpr int kEpiThr = 256;                 // warps 0-7
constexpr int kConvThr = 128;                // warps 8-11
constexpr int kProdA = 12, kMmaWarp = 13, kProdB = 14;
constexpr int kThr = 15 * 32;
// Shared memory: a ring of NA raw child tiles (TMA; the tf32 hi operand, two
// 16 KB K-halves each), one tile of lo parts, a ring of two matrix tiles (per
// K-half h: [P hi rows 0-63 | P lo rows 0-63], 16 KB, so one N = 128 MMA reads
// A hi once for hi.hi and hi.lo), the output staging tile.
#ifndef RRL_TC5_ALO_TMEM
#define RRL_TC5_ALO_TMEM 1
#endif
#ifndef RRL_TC5_NLO
#define RRL_TC5_NLO 1
#endif
#ifndef RRL_TC5_NB
#define RRL_TC5_NB (RRL_TC5_TIP_PT ? 2 : 3)
#endif
// Build knobs, all measured on configs[3] fp32 (updatePartials per pass):
//  * RRL_TC5_DIRECT_STORE=1: write-back by direct 16-byte stores from the
//    epilogue (a thread's row is 128 contiguous bytes, a warp instruction
//    touches 32 rows) instead of the swizzled staging tile drained by TMA
//    stores, freeing 32 KB for a fourth child tile in flight: 2.03 ms vs
//    1.535 -- the uncoalesced stores cost far more than the deeper ring wins;
//  * RRL_TC5_NLO=2 (a second lo tile, so the converters run under the
//    previous phase's MMAs), RRL_TC5_NB=3 (a third matrix slot), RRL_TC5_ACC4=1
//    (round 1's [main_h | corr_h] accumulators: per K-step one N = 128 + one
//    N = 64 MMA instead of K-half 1's three N = 64): 1.536-1.543 ms, no change.
// The phase timeline (tools/trace_tc5.py) puts the MMAs of an internal phase
// at ~1,350 cycles (24 tf32 MMAs) and a child tile's TMA load from HBM at
// ~2.5 K cycles; the period stays ~2.4 K cycles per phase whichever ring
// is deepened.
// Round 2 (configs[3] updatePartials per pass, interleaved A/B): A_lo in TMEM
// (RRL_TC5_ALO_TMEM) 1.535 -> 1.501 ms; the previous tile's write-back after
// the accumulators are released (RRL_TC5_LATE_DRAIN) -> 1.458; a third matrix
// slot (RRL_TC5_NB=3, the MMA issuer's longest wait was its P tile) -> 1.431.
// No gain: the lo hand-over per K-half (RRL_TC5_LOSPLIT, 1.550 / 1.530 with
// smem / TMEM lo), two TMEM lo slots with the last category kept in registers
// (RRL_TC5_NLO=2, 1.475-1.518), tip columns from P^T (RRL_TC5_TIP_PT, 1.734),
// a fourth matrix slot instead of the third child tile (1.442), tip phases'
// P tiles released per epilogue warp instead of behind a 256-thread barrier
// (1.4315 vs 1.4321, backed out).
// RRL_TC5_LOSPLIT=1: the lo tile is handed over per K-half (two full / empty
// barrier pairs per lo slot): the MMAs of K-half 0 start once the converters
// finished that half, and the converters start the next phase's K-half 0 as
// soon as this phase's K-half-0 MMAs completed (the phase chain was converter
// then MMAs, serial, ~1.1 K + 1.3 K cycles).
#ifndef RRL_TC5_LOSPLIT
#define RRL_TC5_LOSPLIT 0
#endif
constexpr int LOH = RRL_TC5_LOSPLIT ? 2 : 1;  // lo hand-over parts per slot
#ifndef RRL_TC5_LATE_DRAIN
#define RRL_TC5_LATE_DRAIN 1
#endif
#ifndef RRL_TC5_DIRECT_STORE
#define RRL_TC5_DIRECT_STORE 0
#endif
// RRL_TC5_ALO_TMEM=1: the converters write the child's tf32 lo parts into TMEM
// (tcgen05.st, one 64-column slot) and the A_lo.P_hi MMAs read A from TMEM, so
// the lo tile never passes through shared memory (its write and its MMA reads,
// 64 KB of shared-memory traffic per phase, and 32 KB of ring space given to a
// fourth child tile); K-half 1 runs as N = 128 MMAs A_hi.[P_lo | P_hi] into
// [corr | main_1] after its first K-step (the matrix producer lands K-half 1
// of an internal phase's P tile as [lo | hi]), so A_hi is read 9 instead of 12
// times per phase.
constexpr bool kAloTmem = RRL_TC5_ALO_TMEM != 0;
// RRL_TC5_TIP_PT=1: a tip child's column P[.][obs] comes from K1's P^T slab in
// global memory (row obs = column obs of P, row 61 = row sums), copied into a
// per-thread shared-memory slot (cp.async) one phase ahead, so tip phases take
// no matrix-ring slot, no TMA and no shared-memory gather.  Measured slower:
// 1.734 vs 1.431 ms per configs[3] pass (the slot costs a child tile of the
// ring; round 1 saw global P^T gathers lose too).  Off.
#ifndef RRL_TC5_TIP_PT
#define RRL_TC5_TIP_PT 0
#endif
constexpr bool kTipPT = RRL_TC5_TIP_PT != 0;

constexpr int NLO = RRL_TC5_NLO;  // lo tiles (2: the converters run under the previous phase's MMAs)
constexpr int NB = RRL_TC5_NB;    // matrix tiles (3: a tip phase's P tile lands while the previous one is read)
constexpr int NLO_SM = kAloTmem ? 0 : NLO;                          // lo tiles in shared memory
constexpr int NPF = kTipPT ? 1 : 0;  // 32 KB: the epilogue threads' prefetched tip columns
constexpr int NA = (RRL_TC5_DIRECT_STORE ? 7 : 6) - NLO_SM - NB - NPF;  // child tiles: 7 x 32 KB of rings fit 227 KB
constexpr int SM_A = 0, SM_ALO = NA * 32768, SM_B = SM_ALO + NLO_SM * 32768, SM_PF = SM_B + NB * 32768,
              SM_S1 = SM_PF + NPF * 32768;
// Two TMEM lo slots (the converters write phase g+1's lo parts while phase g's
// MMAs read phase g's): the budget (512 columns) then holds only C - 1 parked
// products, so the tile's last category is written back from registers at the
// tile's end instead of being parked.
constexpr bool kLastInRegs = kAloTmem && NLO == 2;
static_assert(!kAloTmem || NLO <= 2, "TMEM lo slots");
constexpr int kBars = 24;
static_assert(NA >= 1 && 2 * (NA + NB + NLO * LOH) + 2 <= kBars, "ring sizes / mbarrier slots");
constexpr int SMEM_MX = SM_S1 + (RRL_TC5_DIRECT_STORE ? 0 : TM * TS * 4);  // row maxima / scale [2][128]
constexpr int SMEM_BAR = SMEM_MX + 2 * TM * 4;         // kBars mbarriers
constexpr int SMEM_TMEM = SMEM_BAR + kBars * 8;
constexpr int SMEM_TOTAL = SMEM_TMEM + 16;
#ifndef RRL_TC5_ACC4
#define RRL_TC5_ACC4 0
#endif
constexpr int kTmemCols = 512;
// accumulators: ACC4 [main_0 | corr_0 | main_1 | corr_1] (4 x 64: per K-half one
// N = 128 MMA A_hi.[P_hi|P_lo] + one N = 64 A_lo.P_hi), else [main_0 | corr |
// main_1] (3 x 64: K-half 1 as three N = 64 MMAs); then one 64-column slot per
// category (the unscaled product)
constexpr int kAloCol = (RRL_TC5_ACC4 ? 4 : 3) * TS;     // TMEM lo slot (kAloTmem)
constexpr int kProdCol = kAloCol + (kAloTmem ? NLO * TS : 0);
static_assert(!(kAloTmem && RRL_TC5_ACC4), "ALO_TMEM uses the 3-accumulator layout");

__device__ inline uint32_t sa(const void *p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ inline uint64_t desc_sw128(uint32_t saddr) {  // K-major, 128-byte swizzle, 8-row atoms of 1 KB
  return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__host__ __device__ constexpr uint32_t idesc_tf32(int n) {  // kind::tf32, D f32, K-major A/B, M 128, N n
  return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(TM >> 4) << 24);
}

__device__ inline void mma_tf32(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ inline void mma_tf32_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(d),
      "r"(a_tmem), "l"(b), "r"(idesc), "r"(acc));
}
__device__ inline void commit(uint64_t *bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sa(bar))
               : "memory");
}
__device__ inline void bar_init(uint64_t *bar, unsigned n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(bar)), "r"(n));
}
__device__ inline void bar_arrive(uint64_t *bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(bar)) : "memory");
}
__device__ inline void bar_expect(uint64_t *bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(bar)), "r"(bytes) : "memory");
}
__device__ inline void bar_wait(uint64_t *bar, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred P1;\nW_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra W_%=;\n}\n" ::"r"(sa(bar)),
      "r"(parity)
      : "memory");
}
__device__ inline void tma4(uint32_t dst, const void *tmap, int x, int y, int z, int w, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];" ::"r"(
          dst),
      "l"(tmap), "r"(x), "r"(y), "r"(z), "r"(w), "r"(sa(bar))
      : "memory");
}
__device__ inline void tma_store4(const void *tmap, int x, int y, int z, int w, uint32_t src) {
  asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%1, %2, %3, %4}], [%5];" ::"l"(tmap),
               "r"(x), "r"(y), "r"(z), "r"(w), "r"(src)
               : "memory");
}
__device__ inline void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ inline void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ inline void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
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
__device__ inline void tmem_st32(uint32_t taddr, const float *v) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])), "r"(__float_as_uint(v[3])),
      "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])), "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7])),
      "r"(__float_as_uint(v[8])), "r"(__float_as_uint(v[9])), "r"(__float_as_uint(v[10])), "r"(__float_as_uint(v[11])),
      "r"(__float_as_uint(v[12])), "r"(__float_as_uint(v[13])), "r"(__float_as_uint(v[14])), "r"(__float_as_uint(v[15])),
      "r"(__float_as_uint(v[16])), "r"(__float_as_uint(v[17])), "r"(__float_as_uint(v[18])), "r"(__float_as_uint(v[19])),
      "r"(__float_as_uint(v[20])), "r"(__float_as_uint(v[21])), "r"(__float_as_uint(v[22])), "r"(__float_as_uint(v[23])),
      "r"(__float_as_uint(v[24])), "r"(__float_as_uint(v[25])), "r"(__float_as_uint(v[26])), "r"(__float_as_uint(v[27])),
      "r"(__float_as_uint(v[28])), "r"(__float_as_uint(v[29])), "r"(__float_as_uint(v[30])), "r"(__float_as_uint(v[31]))
      : "memory");
}
__device__ inline void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ inline void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ inline void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ inline void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ inline void named_sync(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

__device__ inline float lo_tf32(float x) {  // rn_tf32(x - trunc_tf32(x))
  const float hi = __uint_as_float(__float_as_uint(x) & 0xffffe000u);
  return __uint_as_float((__float_as_uint(x - hi) + 0x1000u) & 0xffffe000u);
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

template <int C>
__global__ void __launch_bounds__(kThr, 1)
k_partials_codon_tc5(const DevOp *__restrict__ ops, int ntiles, int total, int p_pad,
                     const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmP,
                     const __grid_constant__ CUtensorMap tmPlo, const float *__restrict__ PT) {
  static_assert(kProdCol + (C - (kLastInRegs ? 1 : 0)) * TS <= kTmemCols, "category slots must fit TMEM");
  extern __shared__ __align__(1024) unsigned char sm[];
  uint64_t *a_full = reinterpret_cast<uint64_t *>(sm + SMEM_BAR);  // [NA] child tile landed
  uint64_t *a_empty = a_full + NA;                                  // [NA] its MMAs completed
  uint64_t *b_full = a_full + 2 * NA;                               // [NB] matrix tile landed
  uint64_t *b_empty = b_full + NB;                                  // [NB] MMAs / tip gather done
  uint64_t *lo_full = b_full + 2 * NB;                              // [NLO][LOH] converters wrote the lo tile (part)
  uint64_t *lo_empty = lo_full + NLO * LOH;                         // [NLO][LOH] its MMAs completed
  uint64_t *acc_full = lo_full + 2 * NLO * LOH;
  uint64_t *acc_empty = acc_full + 1;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(sm + SMEM_TMEM);
  float *S1 = reinterpret_cast<float *>(sm + SM_S1);
  float *mx = reinterpret_cast<float *>(sm + SMEM_MX);
  const uint32_t sbase = sa(sm);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if ((sbase & 1023u) != 0u) __trap();  // swizzled stages need 1 KB alignment

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(sa(tmem_slot)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == kProdA * 32) {
    for (int i = 0; i < NA; ++i) {
      bar_init(&a_full[i], 1);
      bar_init(&a_empty[i], 1);
    }
    for (int i = 0; i < NB; ++i) {
      bar_init(&b_full[i], 1);
      bar_init(&b_empty[i], 1);
    }
    for (int i = 0; i < NLO * LOH; ++i) {
      bar_init(&lo_full[i], kConvThr / 32);
      bar_init(&lo_empty[i], 1);
    }
    bar_init(acc_full, 1);
    bar_init(acc_empty, kEpiThr / 32);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmP) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmPlo) : "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;
  asm volatile("griddepcontrol.wait;" ::: "memory");  // everything above overlaps the previous level set
  asm volatile("griddepcontrol.launch_dependents;" :::);

  const int my_tiles = total > (int)blockIdx.x ? (total - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
  const int nphase = my_tiles * C * 2;  // (tile, category, child)

  // phase g = (local tile lt, category c, child b); internal-child phases are
  // counted separately (ia): only they use the child-tile ring and the lo tile.
  auto phase_op = [&](int g, int &c, int &b, int &p0) -> const DevOp & {
    const int lt = g / (2 * C), f = blockIdx.x + lt * gridDim.x;
    c = (g / 2) % C;
    b = g & 1;
    p0 = (f % ntiles) * TM;
    return ops[f / ntiles];
  };
  auto is_tip = [](const DevOp &op, int b) { return (op.flags & (b == 0 ? OP_TIP1 : OP_TIP2)) != 0; };

  if (warp == kProdA) {
    // ================================================================ child-tile producer
    if (lane == 0) {
      uint32_t ia = 0;
      for (int g = 0; g < nphase; ++g) {
        int c, b, p0;
        const DevOp &op = phase_op(g, c, b, p0);
        if (is_tip(op, b) || p0 >= op.p) continue;
        const uint32_t sl = ia % NA, use = ia / NA;
        ++ia;
        bar_wait(&a_empty[sl], (use & 1u) ^ 1u);  // the MMAs NA internal phases back are done
        TR(0, g);
        const uint32_t dst = sbase + SM_A + sl * 32768;
        bar_expect(&a_full[sl], 32768u);
        const int buf = b == 0 ? op.buf1 : op.buf2;
        tma4(dst, &tmA, 0, op.pat0 + p0, c, buf, &a_full[sl]);
        tma4(dst + 16384, &tmA, 32, op.pat0 + p0, c, buf, &a_full[sl]);
      }
    }
  } else if (warp == kProdB) {
    // ================================================================ matrix producer
    if (lane == 0) {
      uint32_t gb = 0;  // phases processed (tiles past an op's own range are skipped)
      for (int g = 0; g < nphase; ++g) {
        int c, b, p0;
        const DevOp &op = phase_op(g, c, b, p0);
        if (p0 >= op.p) continue;
        const bool tip = is_tip(op, b);
        if (kTipPT && tip) continue;  // the epilogue reads the column from P^T
        const uint32_t sl = gb % NB, use = gb / NB;
        ++gb;
        bar_wait(&b_empty[sl], (use & 1u) ^ 1u);
        TR(16, g);  // matrix tile issued
#ifdef RRL_TC5_TRACE
        if (blockIdx.x == 0 && g < 4096) g_tc5_kind[g] = tip ? 1 : 0;
#endif
        const uint32_t dst = sbase + SM_B + sl * 32768;
        const int mat = b == 0 ? op.mat1 : op.mat2;
        bar_expect(&b_full[sl], tip ? 16384u : 32768u);
        // K-half h at h * 16 KB: [P hi | P lo] (8 KB each); K-half 1 of an internal phase
        // as [P lo | P hi] with ALO_TMEM (its N = 128 MMAs write [corr | main_1])
        const uint32_t h1hi = (!tip && kAloTmem) ? 8192u : 0u;
        tma4(dst, &tmP, 0, 0, c, mat, &b_full[sl]);
        tma4(dst + 16384 + h1hi, &tmP, 32, 0, c, mat, &b_full[sl]);
        if (!tip) {  // the matrix's tf32 low parts, precomputed by K1
          tma4(dst + 8192, &tmPlo, 0, 0, c, mat, &b_full[sl]);
          tma4(dst + 16384 + (8192u - h1hi), &tmPlo, 32, 0, c, mat, &b_full[sl]);
        }
      }
    }
  } else if (warp == kMmaWarp) {
    // ================================================================ MMA issuer
    if (lane == 0) {
      uint32_t ia = 0;
      uint32_t gb = 0;
      for (int g = 0; g < nphase; ++g) {
        int c, b, p0;
        const DevOp &op = phase_op(g, c, b, p0);
        if (p0 >= op.p) continue;
        if (kTipPT && is_tip(op, b)) continue;  // no matrix slot, no MMA
        const uint32_t bs = gb % NB;
        bar_wait(&b_full[bs], (uint32_t)(gb / NB) & 1u);
        TR(12, g);
        ++gb;
        if (is_tip(op, b)) continue;  // a tip child is a P-column gather in the epilogue: no MMA
        const uint32_t sl = ia % NA, use = ia / NA;
        bar_wait(&a_full[sl], use & 1u);
        TR(13, g);
        const uint32_t ls = ia % NLO, lpar = (ia / NLO) & 1u;
        if (LOH == 1) bar_wait(&lo_full[ls], lpar);
        TR(14, g);
        bar_wait(acc_empty, (ia & 1u) ^ 1u);  // the epilogue drained the previous accumulators
        TR(15, g);
        ++ia;
        fence_after();
        TR(3, g);
        // Accumulators [main_0 | corr | main_1]: K-half 0 as A_hi . [P_hi | P_lo]^T (N = 128)
        // -> [main_0 | corr] plus A_lo . P_hi^T -> corr; K-half 1 as three N = 64 MMAs
        // (A_hi P_hi -> main_1, A_hi P_lo and A_lo P_hi -> corr; same tensor time).  The
        // hi.hi sums of the two K-halves and the ~2^-11-smaller corrections never share
        // an accumulator (tf32 accumulation reading); one shared correction
        // accumulator saves a quarter of the epilogue's TMEM reads.  (Issuing the A_hi
        // MMAs before waiting for the lo tile, to overlap the converters, measured no
        // faster: 1.557 vs 1.533 ms per configs[3] pass.)
#pragma unroll
        for (int kk = 0; kk < TS / 8; ++kk) {
          const int h = kk >> 2, kin = kk & 3;
          if (LOH == 2 && kin == 0) {  // this K-half's lo part written by the converters
            bar_wait(&lo_full[ls * LOH + h], lpar);
            fence_after();
          }
          const uint64_t ah = desc_sw128(sbase + SM_A + sl * 32768 + h * 16384 + kin * 32);
          const uint64_t al = desc_sw128(sbase + SM_ALO + ls * 32768 + h * 16384 + kin * 32);
          const uint64_t bb = desc_sw128(sbase + SM_B + bs * 32768 + h * 16384 + kin * 32);
          if (kAloTmem) {
            const uint32_t at = tmem + (uint32_t)(kAloCol + ls * TS + kk * 8);  // A_lo columns of this K-step
            if (h == 0) {  // B = [P hi | P lo]
              mma_tf32(tmem, ah, bb, idesc_tf32(2 * TS), kin > 0 ? 1u : 0u);  // [main_0 | corr]
              mma_tf32_ts(tmem + TS, at, bb, idesc_tf32(TS), 1u);             // corr += A_lo P_hi
            } else {       // B = [P lo | P hi]
              const uint64_t bh = desc_sw128(sbase + SM_B + bs * 32768 + h * 16384 + 8192 + kin * 32);
              if (kin == 0) {  // main_1 starts here, corr accumulates: two N = 64
                mma_tf32(tmem + 2 * TS, ah, bh, idesc_tf32(TS), 0u);
                mma_tf32(tmem + TS, ah, bb, idesc_tf32(TS), 1u);
              } else {
                mma_tf32(tmem + TS, ah, bb, idesc_tf32(2 * TS), 1u);  // [corr | main_1]
              }
              mma_tf32_ts(tmem + TS, at, bh, idesc_tf32(TS), 1u);
            }
          } else if (RRL_TC5_ACC4) {
            const uint32_t d = tmem + (uint32_t)(h * 2 * TS);
            mma_tf32(d, ah, bb, idesc_tf32(2 * TS), kin > 0 ? 1u : 0u);  // [main_h | corr_h]
            mma_tf32(d + TS, al, bb, idesc_tf32(TS), 1u);                // corr_h += A_lo P_hi
          } else if (h == 0) {
            mma_tf32(tmem, ah, bb, idesc_tf32(2 * TS), kin > 0 ? 1u : 0u);
            mma_tf32(tmem + TS, al, bb, idesc_tf32(TS), 1u);
          } else {
            const uint64_t bl = desc_sw128(sbase + SM_B + bs * 32768 + h * 16384 + 8192 + kin * 32);
            mma_tf32(tmem + 2 * TS, ah, bb, idesc_tf32(TS), kin > 0 ? 1u : 0u);
            mma_tf32(tmem + TS, ah, bl, idesc_tf32(TS), 1u);
            mma_tf32(tmem + TS, al, bb, idesc_tf32(TS), 1u);
          }
          if (LOH == 2 && kin == 3) commit(&lo_empty[ls * LOH + h]);  // this K-half's lo part is free
        }
        commit(&a_empty[sl]);  // child tile, lo tile and matrix tile free once these MMAs completed
        if (LOH == 1) commit(&lo_empty[ls]);
        commit(&b_empty[bs]);
        commit(acc_full);  // accumulators ready for the epilogue
        TR(4, g);
      }
    }
  } else if (warp >= kEpiThr / 32 && warp < kEpiThr / 32 + kConvThr / 32) {
    // ================================================================ converters
    const int ct = tid - kEpiThr;
    uint32_t ia = 0;
    for (int g = 0; g < nphase; ++g) {
      int c, b, p0;
      const DevOp &op = phase_op(g, c, b, p0);
      if (is_tip(op, b) || p0 >= op.p) continue;
      const uint32_t sl = ia % NA, use = ia / NA;
      bar_wait(&a_full[sl], use & 1u);
      const uint32_t ls = ia % NLO, lpar = ((ia / NLO) & 1u) ^ 1u;
      ++ia;
      const unsigned char *src = sm + SM_A + sl * 32768;
      unsigned char *dst = sm + SM_ALO + ls * 32768;
      if constexpr (kAloTmem) {
        // thread = tile row (TMEM lane) r of this warp's lane quarter; per K-half its 8
        // swizzled 16-byte chunks (states 4j..4j+3 at chunk j ^ (r & 7)) -> 32 lo parts
        // -> TMEM columns kAloCol + 32 h + (0..31)
        const int wq = warp & 3, r = wq * 32 + lane;
        const uint32_t trow = tmem + ((uint32_t)(wq * 32) << 16) + (uint32_t)(kAloCol + ls * TS);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          if (h == 0 || LOH == 2) {  // the MMAs of the previous internal phase read this slot (part)
            bar_wait(&lo_empty[ls * LOH + (LOH == 2 ? h : 0)], lpar);
            fence_after();
            if (ct == 0 && h == 0) TR(1, g);
          }
          float lo[32];
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const float4 v = *reinterpret_cast<const float4 *>(src + h * 16384 + r * 128 + ((j ^ (r & 7)) << 4));
            lo[4 * j] = lo_tf32(v.x);
            lo[4 * j + 1] = lo_tf32(v.y);
            lo[4 * j + 2] = lo_tf32(v.z);
            lo[4 * j + 3] = lo_tf32(v.w);
          }
          tmem_st32(trow + (uint32_t)(h * 32), lo);
          if (LOH == 2 || h == 1) {
            tmem_wait_st();
            fence_before();
            __syncwarp();
            if (lane == 0) bar_arrive(&lo_full[ls * LOH + (LOH == 2 ? h : 0)]);
          }
        }
        if (ct == 0) TR(2, g);
        continue;
      }
      // chunk u * kConvThr + ct of the 2,048 16-byte chunks: u < 8 is K-half 0, u >= 8 K-half 1
#pragma unroll
      for (int u = 0; u < TM * 16 / kConvThr; u += 8) {  // lo of every 16-byte chunk, same swizzled offset
        const int part = LOH == 2 ? u / 8 : 0;
        if (u == 0 || LOH == 2) {  // the MMAs NLO internal phases back read this lo tile (part)
          bar_wait(&lo_empty[ls * LOH + part], lpar);
          if (ct == 0 && u == 0) TR(1, g);
        }
        float4 v[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) v[q] = *reinterpret_cast<const float4 *>(src + (ct + (u + q) * kConvThr) * 16);
#pragma unroll
        for (int q = 0; q < 8; ++q)
          *reinterpret_cast<float4 *>(dst + (ct + (u + q) * kConvThr) * 16) =
              make_float4(lo_tf32(v[q].x), lo_tf32(v[q].y), lo_tf32(v[q].z), lo_tf32(v[q].w));
        if (LOH == 2 || u + 8 >= TM * 16 / kConvThr) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> async proxy
          __syncwarp();
          if (lane == 0) bar_arrive(&lo_full[ls * LOH + part]);
        }
      }
      if (ct == 0) TR(2, g);
    }
  } else {
    // ================================================================ epilogue
    const int h = warp >> 2;               // column half
    const int r = (warp & 3) * 32 + lane;  // TMEM lane = pattern row of the tile
    const uint32_t tl = tmem + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)(h * 32);
    // output staging in the TMA store's SWIZZLE_128B layout: column half hh is a
    // 16 KB box of 128 rows x 128 B, 16-byte chunk j of row `row` at j ^ (row & 7)
    auto s1 = [&](int row, int hh, int j) -> float4 * {
      return reinterpret_cast<float4 *>(S1 + hh * (TM * 32) + row * 32 + 4 * (j ^ (row & 7)));
    };
    // Row metadata of a tile (tip states of both children, the children's summed
    // cumulative exponents or the stored factor to apply), loaded one tile ahead so
    // the global-memory latency hides behind the current tile's phases.
    auto load_meta = [&](int lt, uint32_t &sv, int &ex) {
      const int f = blockIdx.x + lt * gridDim.x;
      const DevOp &op = ops[f / ntiles];
      const int pp = (f % ntiles) * TM + r;
      const bool valid = pp < op.p;
      const uint32_t s1v = (valid && (op.flags & OP_TIP1)) ? static_cast<const uint8_t *>(op.in1)[pp] : 0u;
      const uint32_t s2v = (valid && (op.flags & OP_TIP2)) ? static_cast<const uint8_t *>(op.in2)[pp] : 0u;
      sv = s1v | (s2v << 8);
      ex = 0;
      if (valid && op.scale_out != nullptr) {
        if (op.cum1 != nullptr) ex += op.cum1[pp];
        if (op.cum2 != nullptr) ex += op.cum2[pp];
      } else if (valid && op.scale_in != nullptr) {
        ex = op.scale_in[pp];
      }
    };
    uint32_t sv_cur = 0, sv_nxt = 0;
    int ex_cur = 0, ex_nxt = 0;
    // write-back of the previous tile: scale slot `cat` by 2^-e, stage it in the
    // swizzled layout, and hand it to an asynchronous TMA bulk tensor store
    float sc_prev = 0.f;
    int prev_y = 0, prev_buf = 0;
    float *prev_dst = nullptr;  // direct write-back: row p0 of category 0 of the previous tile's output
    bool have_prev = false;
    // scale the 32 values of this thread's row half of category `cat` of the
    // previous tile by 2^-e, stage them, and hand the tile to a TMA store
    auto stage_store = [&](int cat, const float (&w)[32]) {
      if (RRL_TC5_DIRECT_STORE) {
        float4 *dst = reinterpret_cast<float4 *>(prev_dst + ((size_t)cat * p_pad + r) * TS + h * 32);
#pragma unroll
        for (int k = 0; k < 8; ++k)
          dst[k] = make_float4(w[4 * k] * sc_prev, w[4 * k + 1] * sc_prev, w[4 * k + 2] * sc_prev,
                               w[4 * k + 3] * sc_prev);
        return;
      }
      if (tid == 0) bulk_wait_read0();  // the previous store has read the staging tile
      named_sync(1, kEpiThr);
#pragma unroll
      for (int k = 0; k < 8; ++k)
        *s1(r, h, k) = make_float4(w[4 * k] * sc_prev, w[4 * k + 1] * sc_prev, w[4 * k + 2] * sc_prev,
                                   w[4 * k + 3] * sc_prev);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> TMA store
      named_sync(1, kEpiThr);
      if (tid == 0) {
        tma_store4(&tmA, 0, prev_y, cat, prev_buf, sa(S1));
        tma_store4(&tmA, 32, prev_y, cat, prev_buf, sa(S1) + TM * 128);
        bulk_commit();
      }
    };
    auto drain = [&](int cat) {  // a parked category of the previous tile
      float w[32];
      tmem_ld16(tl + (uint32_t)(kProdCol + cat * TS), *reinterpret_cast<float(*)[16]>(w));
      tmem_ld16(tl + (uint32_t)(kProdCol + cat * TS + 16), *reinterpret_cast<float(*)[16]>(w + 16));
      tmem_wait_ld();
      stage_store(cat, w);
    };
    constexpr int kParked = C - (kLastInRegs ? 1 : 0);  // categories written back during the next tile
    // tip column of the next phase (kTipPT): 128 bytes of P^T copied by cp.async
    // into this thread's slot one phase ahead ([k][thread] float4 layout: a warp's
    // k-th float4s are 512 contiguous bytes)
    const uint32_t pf_s = sbase + SM_PF + (uint32_t)tid * 16;
    int lt_cur = 0;
    auto issue_pf = [&](int g2) {
      if (!kTipPT || g2 >= nphase) return;
      const int lt2 = g2 / (2 * C), c2 = (g2 / 2) % C, b2 = g2 & 1;
      const int f2 = blockIdx.x + lt2 * gridDim.x;
      const DevOp &op2 = ops[f2 / ntiles];
      if (!(op2.flags & (b2 == 0 ? OP_TIP1 : OP_TIP2)) || (f2 % ntiles) * TM >= op2.p) return;
      const uint32_t svw = lt2 == lt_cur ? sv_cur : sv_nxt;
      unsigned sv = (svw >> (8 * b2)) & 0xffu;
      sv = sv < (unsigned)kS61 ? sv : (unsigned)kS61;  // row 61 = row sums (missing state)
      const float *src = PT + ((size_t)(b2 == 0 ? op2.mat1 : op2.mat2) * C + c2) * (TS * TS) + sv * TS + h * 32;
#pragma unroll
      for (int k = 0; k < 8; ++k)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(pf_s + (uint32_t)(k * kEpiThr * 16)),
                     "l"(src + 4 * k)
                     : "memory");
      asm volatile("cp.async.commit_group;" ::: "memory");
    };
    float m = 0.f;  // running max over (c, z) of this thread's row half
    float d1[32];     // child 1's contraction of the current category
    uint32_t ni = 0;  // internal-child phases consumed (accumulator barrier parity)
    uint32_t gb = 0;  // phases processed (matrix ring parity)
    for (int g = 0; g < nphase; ++g) {
      const int lt = g / (2 * C), c = (g / 2) % C, b = g & 1;
      const int f = blockIdx.x + lt * gridDim.x;
      const DevOp &op = ops[f / ntiles];
      const int p0 = (f % ntiles) * TM;
      const int pp = p0 + r;
      const bool valid = pp < op.p;
      if (c == 0 && b == 0) {  // tile start: rotate the prefetched metadata
        if (lt == 0) load_meta(0, sv_nxt, ex_nxt);
        sv_cur = sv_nxt;
        ex_cur = ex_nxt;
        lt_cur = lt;
        if (lt + 1 < my_tiles) load_meta(lt + 1, sv_nxt, ex_nxt);
        if (lt == 0) issue_pf(0);
      }
      const bool tip_ph = (op.flags & (b == 0 ? OP_TIP1 : OP_TIP2)) != 0;
      float dv[32];
      if (kTipPT && tip_ph) {  // this phase's column, copied during the previous phase
        asm volatile("cp.async.wait_group 0;" ::: "memory");
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const float4 v = *reinterpret_cast<const float4 *>(sm + SM_PF + (k * kEpiThr + tid) * 16);
          dv[4 * k] = v.x;
          dv[4 * k + 1] = v.y;
          dv[4 * k + 2] = v.z;
          dv[4 * k + 3] = v.w;
        }
      }
      issue_pf(g + 1);
      if (p0 >= op.p) continue;  // past this op's own range (a shorter partition): another op's rows
      const uint32_t gcur = (kTipPT && tip_ph) ? 0u : gb++;
      // Write-back of the previous tile's category c (slot c is reused by this tile's
      // product of category c): RRL_TC5_LATE_DRAIN=1 after this phase's accumulators
      // are read and released, so the staging / TMA-store round trip is off the MMAs' path.
      if (!RRL_TC5_LATE_DRAIN && b == 0 && have_prev && c < kParked) {
        drain(c);
        if (tid == 0) TR(9, g);
      }
      if (kTipPT && tip_ph) {
        if (tid == 0) TR(7, g);
        if (tid == 0) TR(5, g);
      } else if (tip_ph) {
        // Tip child: sum_x P[z][x] [x == obs] = P[z][obs], read from the raw fp32 P tile the
        // producer landed in stage g&1 (swizzled K-major: row z, 16-byte chunk (x&31)/4 at
        // position chunk ^ (z&7) of half x>>5). A missing state (code >= 61) is the row sum.
        const int s = gcur % NB;
        bar_wait(&b_full[s], (uint32_t)(gcur / NB) & 1u);
        if (tid == 0) TR(7, g);
        const unsigned char *pt = sm + SM_B + s * 32768;  // P hi of K-half h at h * 16 KB
        const unsigned sv = (sv_cur >> (8 * b)) & 0xffu;  // prefetched (0 for padding rows)
        if (sv < (unsigned)kS61) {
          const unsigned char *base = pt + (sv >> 5) * 16384 + (sv & 3) * 4;
          const unsigned j = (sv & 31) >> 2;
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const int z = h * 32 + i;
            dv[i] = *reinterpret_cast<const float *>(base + z * 128 + ((j ^ (unsigned)(z & 7)) << 4));
          }
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i) dv[i] = 0.f;
#pragma unroll 1
          for (int x = 0; x < kS61; ++x) {
            const unsigned char *base = pt + (x >> 5) * 16384 + (x & 3) * 4;
            const unsigned j = (unsigned)(x & 31) >> 2;
#pragma unroll
            for (int i = 0; i < 32; ++i) {
              const int z = h * 32 + i;
              dv[i] += *reinterpret_cast<const float *>(base + z * 128 + ((j ^ (unsigned)(z & 7)) << 4));
            }
          }
        }
        named_sync(1, kEpiThr);  // every epilogue thread has read the P tile
        if (tid == 0) bar_arrive(&b_empty[s]);
        if (tid == 0) TR(5, g);
      } else {
        if (tid == 0) TR(11, g);
        bar_wait(acc_full, ni & 1u);
        ++ni;
        fence_after();
        if (tid == 0) TR(7, g);
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          float m0[16], cc[16], m1[16];  // main_0 (columns 0-63), a correction (64-127), main_1 (128-191)
          tmem_ld16(tl + 0 * TS + q * 16, m0);
          tmem_ld16(tl + 1 * TS + q * 16, cc);
          tmem_ld16(tl + 2 * TS + q * 16, m1);
          if (RRL_TC5_ACC4) {  // + corr_1 (192-255)
            float c1[16];
            tmem_ld16(tl + 3 * TS + q * 16, c1);
            tmem_wait_ld();
#pragma unroll
            for (int i = 0; i < 16; ++i) dv[q * 16 + i] = (m0[i] + m1[i]) + (cc[i] + c1[i]);
          } else {
            tmem_wait_ld();
#pragma unroll
            for (int i = 0; i < 16; ++i) dv[q * 16 + i] = (m0[i] + m1[i]) + cc[i];
          }
        }
        fence_before();
        __syncwarp();
        if (lane == 0) bar_arrive(acc_empty);  // the MMAs of the next internal phase may overwrite them
        if (tid == 0) TR(5, g);
      }
      const uint32_t slot = tl + (uint32_t)(kProdCol + c * TS);  // this category's TMEM slot
      if (b == 0) {  // child 1 waits in registers: child 2's phase of the same category is next
#pragma unroll
        for (int i = 0; i < 32; ++i) d1[i] = dv[i];
        if (RRL_TC5_LATE_DRAIN && have_prev && c < kParked) {
          drain(c);
          if (tid == 0) TR(9, g);
        }
        if (tid == 0) TR(6, g);
        continue;
      }
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        dv[i] *= d1[i];
        m = fmaxf(m, dv[i]);
      }
      if (c < kParked) {
        tmem_st16(slot, dv);  // park the unscaled product until written back
        tmem_st16(slot + 16, dv + 16);
        tmem_wait_st();
      }
      if (c < C - 1) {
        if (tid == 0) TR(6, g);
        continue;
      }
      // ---- tile done: row exponent from max over (c, z) of both column halves
      mx[h * TM + r] = m;
      named_sync(1, kEpiThr);
      if (h == 0) {
        const float mm = fmaxf(mx[r], mx[TM + r]);
        int e = 0;
        if (op.scale_out != nullptr) {
          e = frexp_e(mm);
          if (valid) op.scale_out[pp] = e + ex_cur;  // + the children's cumulative exponents
        } else if (op.scale_in != nullptr) {
          e = ex_cur;  // stored factor (0 for padding rows)
        }
        mx[r] = (e > -126 && e < 126) ? __uint_as_float((unsigned)(127 - e) << 23) : ldexpf(1.f, -e);
      }
      named_sync(1, kEpiThr);
      if (tid == 0) TR(8, g);
      // the products wait in their slots; tile t's category c is written back during
      // tile t+1's phase (c, child 1), so the TMA stores overlap the next tile's work
      sc_prev = valid ? mx[r] : 0.f;  // padding rows of the tile are written as zeros
      prev_y = op.pat0 + p0;
      prev_buf = op.bufd;
      prev_dst = static_cast<float *>(op.out) + (size_t)p0 * TS;
      have_prev = true;
      if (kLastInRegs) stage_store(C - 1, dv);  // the last category, straight from registers
      if (tid == 0) TR(6, g);
      m = 0.f;
    }
    if (have_prev)  // the CTA's last tile
      for (int cat = 0; cat < kParked; ++cat) drain(cat);
  }
  if (tid == 0) bulk_wait0();  // output stores complete before the grid does
  fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
}

template <int C>
int launch_tc5(const DevOp *d_ops, int nops, int p, int p_pad, const CUtensorMap *tA, const CUtensorMap *tP,
               const CUtensorMap *tPlo, const float *PT, cudaStream_t st) {
  static int nsm_dev[kMaxDevices] = {};
  int &nsm = nsm_dev[device_slot()];
  if (nsm == 0) {
    cudaError_t e = cudaFuncSetAttribute(k_partials_codon_tc5<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
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
  return (int)cudaLaunchKernelEx(&cfg, k_partials_codon_tc5<C>, d_ops, ntiles, (int)total, p_pad, *tA, *tP,
                                 *tPlo, PT);
}

}  // namespace

int launch_update_partials_codon_tc5(int c, const DevOp *d_ops, const DevOp *h_ops, int nops, int p,
                                     int p_pad, const void *tmap_partials, const void *tmap_P,
                                     const void *tmap_Plo, const void *d_PT, void *stream) {
  // every child must live in the tensor-mapped slab (internal buffers) or be tip states; the
  // destination is always in the slab (its tile is written back by TMA store)
  for (int i = 0; i < nops; ++i)
    if ((!(h_ops[i].flags & OP_TIP1) && h_ops[i].buf1 < 0) || (!(h_ops[i].flags & OP_TIP2) && h_ops[i].buf2 < 0) ||
        h_ops[i].bufd < 0)
      return (int)cudaErrorNotSupported;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const CUtensorMap *tA = static_cast<const CUtensorMap *>(tmap_partials);
  const CUtensorMap *tP = static_cast<const CUtensorMap *>(tmap_P);
  const CUtensorMap *tPlo = static_cast<const CUtensorMap *>(tmap_Plo);
  switch (c) {
    case 1: return launch_tc5<1>(d_ops, nops, p, p_pad, tA, tP, tPlo, static_cast<const float *>(d_PT), st);
    case 2: return launch_tc5<2>(d_ops, nops, p, p_pad, tA, tP, tPlo, static_cast<const float *>(d_PT), st);
    case 4: return launch_tc5<4>(d_ops, nops, p, p_pad, tA, tP, tPlo, static_cast<const float *>(d_PT), st);
    default: return (int)cudaErrorNotSupported;
  }
}

}  // namespace rrl

#ifdef RRL_TC5_TRACE
extern "C" int rrl_debug_tc5_trace(long long *ev /*[18*4096]*/, int *kind /*[4096]*/) {
  if (cudaMemcpyFromSymbol(ev, rrl::g_tc5_trace, sizeof(rrl::g_tc5_trace)) != cudaSuccess) return -1;
  if (cudaMemcpyFromSymbol(kind, rrl::g_tc5_kind, sizeof(rrl::g_tc5_kind)) != cudaSuccess) return -1;
  return 0;
}
#endif
