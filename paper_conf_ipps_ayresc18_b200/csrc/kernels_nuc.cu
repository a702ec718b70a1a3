// K2: level-set updatePartials for 4-state models (sm_100a).
//
// Eq. (1) (§II-A) for every operation of one concurrent set in a
// single launch (§VI-A multi-operation kernel).  Device layout
// [p][c][4]: one thread owns one (pattern, category) item, i.e. one 16-byte
// (fp32) or 32-byte (fp64) state vector per child.  The two 4x4 transition
// matrices of an operation sit in shared memory twice: row-major for the
// internal-child mat-vec and column-major (plus the row-sum column) so that a
// tip child's contribution P[.][state] is a single 128-bit LDS (state code 4 =
// missing -> the row sums, i.e. an all-ones partial vector).
//
// Rescaling (reading A5) is fused: the C lanes of a pattern
// reduce max over (c, z) with warp shuffles, the frexp exponent e is read from
// the float's exponent bits, the outputs are multiplied by 2^-e (exact) and e
// (own, or own + children's cumulative) is stored as int32.
//
// Two variants, chosen per launch by the host:
//  * k_partials_nuc (latency path, narrow sets / few patterns): grid
//    (pattern chunks x ops); descriptors of sets of <= kInline ops travel in
//    the kernel parameters; child vectors are loaded straight into registers.
//  * k_partials_nuc_bulk (bandwidth path, many patterns): persistent blocks
//    walk a contiguous range of the flattened (op, chunk) space; one thread
//    streams each chunk's child partials / tip states / child exponents into
//    a kStages-deep shared-memory ring with cp.async.bulk (TMA bulk copies,
//    mbarrier completion) while all threads compute the previous stage, so
//    bytes in flight no longer depend on registers per thread.
// Both use programmatic dependent launch: the prologue overlaps the previous
// level set; griddepcontrol.wait precedes every read of P or partials.
//
// HBM-bound: per (pattern, op) 2 x c x 4 x sizeof(T) child bytes (tips: 1 B)
// + c x 4 x sizeof(T) out + exponents; 1.8 flop/B in fp32.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "rrl_internal.h"

namespace rrl {
namespace {

constexpr int kThreads = 256;
#ifndef RRL_LAT_INLINE
#define RRL_LAT_INLINE 8
#endif
constexpr int kInline = RRL_LAT_INLINE;
// Latency path: the transition tables live in shared memory (staged before
// griddepcontrol.wait when K1 is not the immediate predecessor) instead of 32
// registers per thread, and the CTA is held to 12 resident per SM (42
// registers, no spills), so the next level set's CTAs (2.1 per SM at
// configs[1]) are resident beside the current set's under programmatic
// dependent launch and finish their whole prologue before its wait.
// Measured on configs[1] (updatePartials per pass, fp32; round 1): rows in
// registers, 80 registers 0.173 ms; tables in shared memory, 256-thread CTAs
// at 3 / 4 / 5 / 6 per SM 0.163 / 0.178 (spills) / 0.145 / 0.169 ms;
// 128-thread CTAs at 10 per SM 0.143 ms; 512-thread CTAs 0.176-0.183 ms.
// Round 2 (after the descriptor and table-staging fixes, 0.117-0.119 ms):
// 8 / 10 / 12 / 14 / 16 CTAs per SM 0.145 / 0.119 / 0.117 / 0.119 / 0.119 ms;
// 2 items per thread 0.153; 64- or 256-thread CTAs 0.162 / 0.132;
// launch_dependents at the top of the kernel 0.145; an L2 prefetch of the
// children's pages before the wait 0.163; tip states read after the wait
// 0.151; the tip-state array bulk-prefetched into L2 by the first set 0.157
// (one SM's bulk engine streams 1.3 MB while that CTA cannot retire); 2 or 4
// inline descriptors instead of 8 0.117 / 0.118 (the pointer path for a
// 2-operation set: 0.147); children read with ld.global.cg instead of .nc
// (RRL_LAT_CG) 0.1174 vs 0.1173.  The trigger position is a balance: the
// next set's launch fires once every CTA of this one has run its prologue,
// and the HBM round trip of the tip-state loads in that prologue paces it --
// without those loads (a timing-only build that skipped them) or with the tip states
// prefetched into L2 the pass is slower (0.152 / 0.128 ms: the set after next
// starts its prologue inside this set's critical section); triggering only
// after the tip states arrived (RRL_LAT_TRIG_AFTER_TIP) 0.120, after the wait
// 0.118, at the top 0.145.  fp64 (configs[1] fp64, updatePartials): 4 / 5 /
// 6 / 8 / 10 / 12 CTAs per SM 0.155 / 0.155 / 0.172 / 0.194 / 0.222 / 0.280
// ms (5: one level set's 626 CTAs resident at a time); fp32 at 4-6: 0.136.  fp64 (tables in shared memory already) keeps 3
// CTAs per SM: at 5 it spills and is no faster.
#ifndef RRL_LAT_MINB
#define RRL_LAT_MINB 12
#endif
#ifndef RRL_LAT_PSMEM
#define RRL_LAT_PSMEM 1
#endif
constexpr int kLatencyMinBlocks = RRL_LAT_MINB;
// griddepcontrol.launch_dependents before the wait: the next level set's
// grid is launched as soon as every CTA of this one has started, not after
// this one's wait (configs[1]: 0.1396 vs 0.1411 ms per pass, two runs).
#ifndef RRL_LAT_PDL_EARLY
#define RRL_LAT_PDL_EARLY 1
#endif
#ifndef RRL_LAT_U  // items per thread on the latency path
#define RRL_LAT_U 1
#endif
#ifndef RRL_LAT_CG  // children and their exponents read with ld.global.cg (L2 only) instead of ld.global.nc
#define RRL_LAT_CG 0
#endif
#ifndef RRL_LAT_TRIG_AFTER_TIP
#define RRL_LAT_TRIG_AFTER_TIP 0
#endif
#ifndef RRL_LAT_PIN
#define RRL_LAT_PIN 0
#endif
#ifndef RRL_LAT_PDL_TOP
#define RRL_LAT_PDL_TOP 0
#endif
#ifndef RRL_LAT_TLB_PREFETCH
#define RRL_LAT_TLB_PREFETCH 0
#endif
#ifndef RRL_LAT_THREADS
#define RRL_LAT_THREADS 128
#endif
constexpr int kLatThreads = RRL_LAT_THREADS;  // latency-path CTA size
#ifndef RRL_LAT_MINB64
#define RRL_LAT_MINB64 5  // fp64: 640 resident threads per SM (measured best, 4-12)
#endif
constexpr int kLatencyMinBlocks64 = RRL_LAT_MINB64;
constexpr int kChunkItems = 512;  // items (pattern x category) per bulk chunk
constexpr int kPTab = 36;         // per (branch, cat): 16 rows P[z][x] + 5 columns x 4

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
  __device__ static inline void ldcg(const float *p, float (&v)[4]) {  // L2 only (no L1 allocation)
    const float4 x = __ldcg(reinterpret_cast<const float4 *>(p));
    v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
  }
  __device__ static inline void lds(const float *p, float (&v)[4]) {
    const float4 x = *reinterpret_cast<const float4 *>(p);
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
  __device__ static inline void ldcg(const double *p, double (&v)[4]) {
    const double2 a = __ldcg(reinterpret_cast<const double2 *>(p));
    const double2 b = __ldcg(reinterpret_cast<const double2 *>(p) + 1);
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
  __device__ static inline void lds(const double *p, double (&v)[4]) {
    const double2 a = reinterpret_cast<const double2 *>(p)[0];
    const double2 b = reinterpret_cast<const double2 *>(p)[1];
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
  }
  __device__ static inline void st(double *p, const double (&v)[4]) {
    reinterpret_cast<double2 *>(p)[0] = make_double2(v[0], v[1]);
    reinterpret_cast<double2 *>(p)[1] = make_double2(v[2], v[3]);
  }
};

// frexp exponent e (m = f 2^e, f in [0.5,1)), fast path from the exponent bits.
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
// r *= 2^-e, exactly.
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

// Shared-memory transition tables of one operation: [branch][cat][kPTab].
template <typename T, int C, int NT>  // NT = blockDim.x (compile-time: no runtime trip-count division)
__device__ inline void load_ptables(T (*sP)[C][kPTab], const DevOp &op) {
  // one thread per row P[c][z][.] of either branch: one vector load, the row,
  // its 4 column entries and its sum written straight away, one barrier
#pragma unroll
  for (int t0 = 0; t0 < 2 * C * 4; t0 += NT) {
    const int t = t0 + threadIdx.x;
    if (t < 2 * C * 4) {
      const int b = t / (C * 4), r = t % (C * 4), c = r / 4, z = r % 4;
      T row[4];
      V4<T>::ld(static_cast<const T *>(b == 0 ? op.P1 : op.P2) + r * 4, row);
      T *tab = &sP[b][c][0];
      V4<T>::st(tab + z * 4, row);                        // row-major P[z][x]
#pragma unroll
      for (int x = 0; x < 4; ++x) tab[16 + x * 4 + z] = row[x];  // column x at 16 + 4x
      tab[32 + z] = row[0] + row[1] + row[2] + row[3];    // "column 4" = row sums
    }
  }
  __syncthreads();
}

template <typename T>
__device__ inline void tip_column(const T *P, unsigned st, T (&v)[4]) {
  V4<T>::lds(P + 16 + 4 * (st < 4u ? st : 4u), v);
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

// Rescale + store of one item (pattern `pat`, category `cat`).  All lanes of
// the warp must call it (shuffles).  `cum_a`, `cum_b`: children's cumulative
// exponents (already fetched), 0 when absent.
template <typename T, int C>
__device__ inline void finish_item(const DevOp &op, T (&r)[4], bool valid, unsigned pat, int cat,
                                   int cum_a, int cum_b, T *out_item) {
  if (op.scale_out != nullptr) {
    T m = valid ? fmax(fmax(r[0], r[1]), fmax(r[2], r[3])) : T(0);
#pragma unroll
    for (int o = 1; o < C; o <<= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
    const int e = frexp_exp(m);
    if (e != 0) scale_pow2(r, e);
    if (valid && cat == 0) op.scale_out[pat] = e + cum_a + cum_b;
  } else if (op.scale_in != nullptr) {
    const int e = valid ? __ldg(op.scale_in + pat) : 0;
    if (e != 0) scale_pow2(r, e);
  }
  if (valid) V4<T>::st(out_item, r);
}

__device__ inline void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ inline void prefetch_l2(const void *p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }
#ifdef RRL_LAT_TRACE  // dev build only (tools/trace_latency.py): per-CTA globaltimer stamps
// per-SM slots (no single contended counter): record k of SM s at [s * kLatSlots + k]
constexpr unsigned kLatSlots = 1024;
__device__ unsigned long long g_lat_trace[160 * kLatSlots][4];
__device__ unsigned int g_lat_n[160];
__device__ inline unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)::"memory");
  return t;
}
// stamp issued after x is available (in-order issue: the add waits for x)
__device__ inline unsigned long long gtime_after(float x) {
  unsigned long long t;
  asm volatile("{.reg .f32 d; add.f32 d, %1, 0f00000000; mov.u64 %0, %%globaltimer;}" : "=l"(t) : "f"(x) : "memory");
  return t;
}
#endif
__device__ inline void pdl_launch() { asm volatile("griddepcontrol.launch_dependents;" :::); }

// ============================================================ latency path
// One dependent memory round trip per launch: after griddepcontrol.wait every
// thread issues its transition-matrix rows (L2-resident), its child vectors
// and its children's exponents together, then computes and stores.
template <typename T>
__device__ inline void tip_select(const T (&P)[16], unsigned st, T (&v)[4]) {
#pragma unroll
  for (int z = 0; z < 4; ++z) {
    const T rs = P[z * 4] + P[z * 4 + 1] + P[z * 4 + 2] + P[z * 4 + 3];
    T a = (st == 0u) ? P[z * 4] : rs;
    a = (st == 1u) ? P[z * 4 + 1] : a;
    a = (st == 2u) ? P[z * 4 + 2] : a;
    a = (st == 3u) ? P[z * 4 + 3] : a;
    v[z] = a;
  }
}

template <typename T>
__device__ inline void matvec_r(const T (&P)[16], const T (&L)[4], T (&v)[4]) {
#pragma unroll
  for (int z = 0; z < 4; ++z)
    v[z] = fma(P[z * 4 + 3], L[3], fma(P[z * 4 + 2], L[2], fma(P[z * 4 + 1], L[1], P[z * 4] * L[0])));
}

// `early` (host-decided): bit 0 -- tip states may be read before griddepcontrol.wait
// (only host copies write them); bit 1 -- so may the transition matrices (K1 is
// not this launch's immediate predecessor, so it completed before the previous
// level set passed its own wait).  Only the previous level set's partials and
// exponents must wait.
template <typename T, int C, int U, bool INL>
__global__ void __launch_bounds__(kLatThreads, sizeof(T) == 4 ? kLatencyMinBlocks : kLatencyMinBlocks64)
k_partials_nuc(const __grid_constant__ OpPack pack, int p, int nchunks, int early) {
#if RRL_LAT_PDL_TOP
  pdl_launch();
#endif
  // The descriptor by value: inline descriptors are read from the parameter
  // bank (LDC, register-indexed); a reference selecting between the bank and
  // global memory would turn every field into a generic load, and the ones
  // first used after griddepcontrol.wait (cumulative-exponent pointers) into
  // an extra dependent round trip.
  // INL is a separate kernel: with a runtime branch the compiler loads both
  // sources and selects, i.e. every warp also reads the global copy.
  DevOp op;
  if constexpr (INL) op = pack.inl[blockIdx.y];
  else op = pack.ops[blockIdx.y];
#if RRL_LAT_PIN
  {  // the pointers used after the wait held in registers from here on (not re-read from the bank)
    const void *a = op.in1, *b = op.in2, *c1 = op.cum1, *c2 = op.cum2, *si = op.scale_in;
    void *o = op.out, *so = op.scale_out;
    asm volatile("" : "+l"(a), "+l"(b), "+l"(c1), "+l"(c2), "+l"(si), "+l"(o), "+l"(so));
    op.in1 = a; op.in2 = b; op.out = o;
    op.cum1 = static_cast<const int32_t *>(c1); op.cum2 = static_cast<const int32_t *>(c2);
    op.scale_in = static_cast<const int32_t *>(si); op.scale_out = static_cast<int32_t *>(so);
  }
#endif
  const bool tip1 = op.flags & OP_TIP1, tip2 = op.flags & OP_TIP2;
  const int cat = threadIdx.x % C;  // kLatThreads is a multiple of C
  const T *__restrict__ P1g = static_cast<const T *>(op.P1) + cat * 16;
  const T *__restrict__ P2g = static_cast<const T *>(op.P2) + cat * 16;
  const T *__restrict__ L1g = static_cast<const T *>(op.in1);
  const T *__restrict__ L2g = static_cast<const T *>(op.in2);
  const uint8_t *__restrict__ S1g = static_cast<const uint8_t *>(op.in1);
  const uint8_t *__restrict__ S2g = static_cast<const uint8_t *>(op.in2);
  T *__restrict__ out = static_cast<T *>(op.out);
  const bool scale_w = op.scale_out != nullptr;
  const unsigned nitems = (unsigned)op.p * C;  // this operation's pattern range
  (void)p;
#ifdef RRL_LAT_TRACE
  const unsigned long long t_entry = gtime();
  unsigned long long t_ld = 0;
  // slot claimed at entry (its round trip overlaps the prologue), per-SM counter
  unsigned tr_smid, tr_k = kLatSlots;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(tr_smid));
  if (threadIdx.x == 0 && tr_smid < 160) tr_k = atomicAdd(&g_lat_n[tr_smid], 1u);
#endif

  // fp32: each thread holds its category's rows in registers.  fp64: the rows
  // would cost 64 registers, so the block stages the tables in shared memory
  // (issued after this thread's first child loads, see below).
  constexpr bool kRegP = sizeof(T) == 4 && !RRL_LAT_PSMEM;
  __shared__ __align__(16) T sP[kRegP ? 1 : 2][kRegP ? 1 : C][kRegP ? 4 : kPTab];
  T P1[kRegP ? 16 : 1], P2[kRegP ? 16 : 1];
  auto load_rows = [&]() {
    if constexpr (kRegP) {
#pragma unroll
      for (int k = 0; k < 16; k += 4) {
        V4<T>::ld(P1g + k, *reinterpret_cast<T(*)[4]>(&P1[k]));
        V4<T>::ld(P2g + k, *reinterpret_cast<T(*)[4]>(&P2[k]));
      }
    }
  };
  // first chunk's tip states (and rows) in flight while the previous level set finishes
  unsigned s1p[U], s2p[U];
  if (early & 1) {
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const unsigned item = (unsigned)blockIdx.x * (kLatThreads * U) + threadIdx.x + j * kLatThreads;
      const bool valid = item < nitems && (int)blockIdx.x < nchunks;
      s1p[j] = (tip1 && valid) ? (unsigned)__ldg(S1g + item / C) : 4u;
      s2p[j] = (tip2 && valid) ? (unsigned)__ldg(S2g + item / C) : 4u;
    }
  }
  if (early & 2) load_rows();
  bool tables = kRegP;
  if constexpr (!kRegP) {
    if (early & 2) {  // K1 completed before the previous set: the tables can be staged before the wait
      load_ptables<T, C, kLatThreads>(sP, op);
      tables = true;
    }
  }

#if RRL_LAT_TLB_PREFETCH
  // Address-translation warm-up before the wait: one L2 prefetch per warp into
  // each page this warp will touch.  No value is read (a prefetch only moves
  // a line into L2, the coherence point, so a later write by the previous set
  // still lands there); the children are consumed after griddepcontrol.wait.
  if ((threadIdx.x & 31) == 0 && (int)blockIdx.x < nchunks) {
    const unsigned item = (unsigned)blockIdx.x * (kLatThreads * U) + threadIdx.x;
    if (item < nitems) {
      if (!tip1) prefetch_l2(L1g + (size_t)item * 4);
      if (!tip2) prefetch_l2(L2g + (size_t)item * 4);
      prefetch_l2(out + (size_t)item * 4);
      if (scale_w) {
        prefetch_l2(op.scale_out + item / C);
        if (op.cum1 != nullptr) prefetch_l2(op.cum1 + item / C);
        if (op.cum2 != nullptr) prefetch_l2(op.cum2 + item / C);
      }
    }
  }
#endif
#if RRL_LAT_PDL_TOP
  pdl_wait();  // everything above overlaps the previous level set
#elif RRL_LAT_PDL_EARLY
#if RRL_LAT_TRIG_AFTER_TIP
  // trigger the next level set's launch only once this thread's tip states have
  // arrived (the comparison waits on their scoreboard)
  if (early & 1) {
    unsigned acc = 0;
#pragma unroll
    for (int j = 0; j < U; ++j) acc |= s1p[j] | s2p[j];
    if (acc == 0xffffffffu) __nanosleep(1);
  }
#endif
  pdl_launch();
  pdl_wait();  // everything above overlaps the previous level set
#else
  pdl_wait();  // everything above overlaps the previous level set
  pdl_launch();
#endif
#ifdef RRL_LAT_TRACE
  const unsigned long long t_wait = gtime();
#endif

  if (!(early & 2)) load_rows();
  for (int chunk = blockIdx.x; chunk < nchunks; chunk += gridDim.x) {
    const bool pre = (early & 1) && chunk == (int)blockIdx.x;
    const unsigned base = (unsigned)chunk * (kLatThreads * U) + threadIdx.x;
    T L1[U][4], L2[U][4];
    unsigned s1[U], s2[U];
    int ca[U], cb[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {  // ---- all reads of this thread in flight together
      const unsigned item = base + j * kLatThreads;
      const bool valid = item < nitems;
      const unsigned pat = item / C;
      if (tip1) {
        s1[j] = pre ? s1p[j] : valid ? (unsigned)__ldg(S1g + pat) : 4u;
      } else if (valid) {
        if (RRL_LAT_CG) V4<T>::ldcg(L1g + (size_t)item * 4, L1[j]);
        else V4<T>::ld(L1g + (size_t)item * 4, L1[j]);
      } else {
#pragma unroll
        for (int z = 0; z < 4; ++z) L1[j][z] = T(0);
      }
      if (tip2) {
        s2[j] = pre ? s2p[j] : valid ? (unsigned)__ldg(S2g + pat) : 4u;
      } else if (valid) {
        if (RRL_LAT_CG) V4<T>::ldcg(L2g + (size_t)item * 4, L2[j]);
        else V4<T>::ld(L2g + (size_t)item * 4, L2[j]);
      } else {
#pragma unroll
        for (int z = 0; z < 4; ++z) L2[j][z] = T(0);
      }
      ca[j] = (scale_w && valid && cat == 0 && op.cum1 != nullptr) ? (RRL_LAT_CG ? __ldcg(op.cum1 + pat) : __ldg(op.cum1 + pat)) : 0;
      cb[j] = (scale_w && valid && cat == 0 && op.cum2 != nullptr) ? (RRL_LAT_CG ? __ldcg(op.cum2 + pat) : __ldg(op.cum2 + pat)) : 0;
    }
    if constexpr (!kRegP) {
      if (!tables) {  // block-uniform, first chunk only
        load_ptables<T, C, kLatThreads>(sP, op);
        tables = true;
      }
    }
#pragma unroll
    for (int j = 0; j < U; ++j) {  // ---- compute + store
      const unsigned item = base + j * kLatThreads;
      const bool valid = item < nitems;
      const unsigned pat = item / C;
      T v1[4], v2[4], r[4];
      if constexpr (kRegP) {
        if (tip1) tip_select(P1, s1[j], v1); else matvec_r(P1, L1[j], v1);
        if (tip2) tip_select(P2, s2[j], v2); else matvec_r(P2, L2[j], v2);
      } else {
        const T *t1 = &sP[0][cat][0], *t2 = &sP[kRegP ? 0 : 1][cat][0];
        if (tip1) tip_column(t1, s1[j], v1); else matvec(t1, L1[j], v1);
        if (tip2) tip_column(t2, s2[j], v2); else matvec(t2, L2[j], v2);
      }
#pragma unroll
      for (int z = 0; z < 4; ++z) r[z] = v1[z] * v2[z];
#ifdef RRL_LAT_TRACE
      if (j == 0 && threadIdx.x == 0 && t_ld == 0) t_ld = gtime_after((float)r[0] + (float)ca[0] + (float)cb[0]);
#endif
      finish_item<T, C>(op, r, valid, pat, cat, ca[j], cb[j], out + (size_t)item * 4);
    }
  }
#ifdef RRL_LAT_TRACE
  // thread 0's stores issued (no barrier: the stamp must not delay the CTA's exit)
  if (threadIdx.x == 0) {
    const unsigned smid = tr_smid, k = tr_k;
    const unsigned long long t_end = gtime();
    if (k < kLatSlots) {
      const unsigned long long q = smid * kLatSlots + k;
      const DevOp &op0 = INL ? pack.inl[0] : pack.ops[0];  // identifies the level set
      g_lat_trace[q][0] = (unsigned long long)op0.out;
      g_lat_trace[q][1] = (unsigned long long)blockIdx.x | ((unsigned long long)blockIdx.y << 16) |
                          ((unsigned long long)smid << 32);
      g_lat_trace[q][2] = t_entry;
      g_lat_trace[q][3] = (t_wait - t_entry) | ((t_ld ? t_ld - t_entry : 0ull) << 21) | ((t_end - t_entry) << 42);
    }
  }
#endif
}

// ============================================================ fused pass
// RRL_FLAG_FUSED_PASS (beyond the paper): the whole operation
// list in ONE launch.  Eq. (1) couples a pattern's partials only to the same
// pattern of the children, and every operation maps item
// (pattern, category) to the same thread here, so each thread's inputs in
// level set k are its own outputs of earlier sets: program order replaces the
// launch boundary, no grid or block synchronisation is needed.  The G
// operations of a group (one set) issue all their reads together.  Measured
// (DESIGN.md §9 "Fused pass"): with ~8 warps per SM at configs[1] each warp's
// serial walk over all operations is instruction-latency bound, so this is
// slower than the per-set launches on a rerooted tree; opt-in only.  A child made
// by one of the previous W-1 operations comes from the thread's own slot of a
// shared-memory ring (host-resolved DevOp::ring1/ring2), so on a rerooted
// pectinate tree the chain never leaves the SM.  Other reads of
// partials / exponents written in this launch are plain coherent loads (no
// __ldg); transition matrices and tip states were written before it.
// Shared-memory layout of the fused kernel: the ring, then one window of
// descriptors, their transition matrices [op][branch][cat][16] and their tip
// codes [op][branch][pattern of the chunk].
template <typename T, int C, int W> struct FusedSmem {
  static constexpr int kPats = kThreads / C;  // patterns per chunk
  static constexpr size_t ring = (size_t)W * kThreads * (4 * sizeof(T) + sizeof(int));
  static constexpr size_t per_op = sizeof(DevOp) + 2 * C * 16 * sizeof(T) + 2 * kPats;
  static size_t bytes(int wops) { return ring + (size_t)wops * per_op; }
};

template <typename T, int C, int G, int W, int H>
__global__ void __launch_bounds__(kThreads * H)
k_partials_nuc_fused(const DevOp *__restrict__ ops, int nops, int p, int nchunks, int wops) {
  using S = FusedSmem<T, C, W>;
  extern __shared__ __align__(16) unsigned char fsm[];
  // H groups of kThreads threads share the chunk's items: the ops of one
  // level set are dealt round-robin (G at a time) to the groups, a barrier
  // closes each set.  Ring of the last W operations' outputs (and cumulative
  // exponents) per item: a child produced by a recent op is read back from
  // shared memory, off the L2 round trip (DevOp::ring1/ring2, host-resolved so
  // that no op running concurrently reuses the slot)
  T (*ringL)[kThreads][4] = reinterpret_cast<T (*)[kThreads][4]>(fsm);
  int (*ringE)[kThreads] = reinterpret_cast<int (*)[kThreads]>(fsm + (size_t)W * kThreads * 4 * sizeof(T));
  DevOp *sOps = reinterpret_cast<DevOp *>(fsm + S::ring);
  T *sP = reinterpret_cast<T *>(fsm + S::ring + (size_t)wops * sizeof(DevOp));
  uint8_t *sTip = reinterpret_cast<uint8_t *>(sP + (size_t)wops * 2 * C * 16);
  const int tid = threadIdx.x % kThreads, h = threadIdx.x / kThreads;
  const int cat = tid % C;
  const int lpat = tid / C;
  const unsigned nitems = (unsigned)p * C;
  pdl_wait();
  for (int chunk = blockIdx.x; chunk < nchunks; chunk += gridDim.x) {
    const unsigned item = (unsigned)chunk * kThreads + tid;
    const bool valid = item < nitems;
    const unsigned pat = valid ? item / C : 0u;
    for (int w0 = 0; w0 < nops; w0 += wops) {
      // ---- stage the window: descriptors, then (one round trip) every
      // matrix and tip code of its ops; none depends on partials
      const int nw = min(wops, nops - w0);
      __syncthreads();  // the previous window is consumed
      {
        const int4 *src = reinterpret_cast<const int4 *>(ops + w0);
        int4 *dst = reinterpret_cast<int4 *>(sOps);
        for (int t = threadIdx.x; t < nw * (int)(sizeof(DevOp) / 16); t += kThreads * H) dst[t] = __ldg(src + t);
      }
      __syncthreads();
      constexpr int kV = 16 / sizeof(T);              // elements per 16-byte vector
      constexpr int kPv = C * 16 / kV;                // vectors per branch
      for (int t = threadIdx.x; t < nw * 2 * kPv; t += kThreads * H) {
        const int o = t / (2 * kPv), r = t % (2 * kPv), br = r / kPv, v = r % kPv;
        const int4 *src = reinterpret_cast<const int4 *>(br == 0 ? sOps[o].P1 : sOps[o].P2);
        reinterpret_cast<int4 *>(sP)[t] = __ldg(src + v);
      }
      const unsigned pat0 = (unsigned)chunk * S::kPats;
      for (int t = threadIdx.x; t < nw * 2 * S::kPats; t += kThreads * H) {
        const int o = t / (2 * S::kPats), r = t % (2 * S::kPats), br = r / S::kPats, q = r % S::kPats;
        const DevOp &op = sOps[o];
        uint8_t code = 4u;
        if ((op.flags & (br == 0 ? OP_TIP1 : OP_TIP2)) && pat0 + q < (unsigned)p)
          code = __ldg(static_cast<const uint8_t *>(br == 0 ? op.in1 : op.in2) + pat0 + q);
        sTip[t] = code;
      }
      __syncthreads();
      for (int i0 = w0; i0 < w0 + nw;) {
        int se = i0;  // this level set's ops within the window: [i0, se)
        while (se < w0 + nw - 1 && !(sOps[se - w0].flags & OP_SET_END)) ++se;
        ++se;
        for (int base = i0; base < se; base += H * G) {
        const int i = base + h * G;
        const int ng = max(0, min(G, se - i));  // this group's ops (warp-uniform)
        T P1[G][16], P2[G][16], L1[G][4], L2[G][4];
        unsigned s1[G], s2[G];
        int ca[G], cb[G];
#pragma unroll
        for (int j = 0; j < G; ++j) {  // ---- every read of the group in flight together
          if (j < ng) {
            const int o = i + j - w0;
            const DevOp &op = sOps[o];
            const bool sw = op.scale_out != nullptr;
            const T *pt = sP + (size_t)o * 2 * C * 16 + cat * 16;
#pragma unroll
            for (int k = 0; k < 16; k += 4) {
              V4<T>::lds(pt + k, *reinterpret_cast<T(*)[4]>(&P1[j][k]));
              V4<T>::lds(pt + C * 16 + k, *reinterpret_cast<T(*)[4]>(&P2[j][k]));
            }
            s1[j] = sTip[(o * 2 + 0) * S::kPats + lpat];
            s2[j] = sTip[(o * 2 + 1) * S::kPats + lpat];
#pragma unroll
            for (int z = 0; z < 4; ++z) L1[j][z] = L2[j][z] = T(0);
            const int fl = op.flags, r1 = op.ring1, r2 = op.ring2;
            if (!(fl & OP_TIP1) && valid)
              V4<T>::lds(r1 >= 0 ? &ringL[r1][tid][0] : static_cast<const T *>(op.in1) + (size_t)item * 4,
                         L1[j]);
            if (!(fl & OP_TIP2) && valid)
              V4<T>::lds(r2 >= 0 ? &ringL[r2][tid][0] : static_cast<const T *>(op.in2) + (size_t)item * 4,
                         L2[j]);
            ca[j] = (sw && valid && cat == 0 && op.cum1 != nullptr)
                        ? ((fl & OP_RING_E1) ? ringE[r1][tid] : op.cum1[pat]) : 0;
            cb[j] = (sw && valid && cat == 0 && op.cum2 != nullptr)
                        ? ((fl & OP_RING_E2) ? ringE[r2][tid] : op.cum2[pat]) : 0;
          }
        }
#pragma unroll
        for (int j = 0; j < G; ++j) {  // ---- compute, rescale, store
          if (j < ng) {
            const DevOp &op = sOps[i + j - w0];
            T v1[4], v2[4], r[4];
            if (op.flags & OP_TIP1) tip_select(P1[j], s1[j], v1); else matvec_r(P1[j], L1[j], v1);
            if (op.flags & OP_TIP2) tip_select(P2[j], s2[j], v2); else matvec_r(P2[j], L2[j], v2);
#pragma unroll
            for (int z = 0; z < 4; ++z) r[z] = v1[z] * v2[z];
            const int slot = (i + j) % W;
            if (op.scale_out != nullptr) {
              T m = valid ? fmax(fmax(r[0], r[1]), fmax(r[2], r[3])) : T(0);
#pragma unroll
              for (int o = 1; o < C; o <<= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
              const int e = frexp_exp(m);
              if (e != 0) scale_pow2(r, e);
              const int et = e + ca[j] + cb[j];
              ringE[slot][tid] = et;
              if (valid && cat == 0) op.scale_out[pat] = et;
            } else if (op.scale_in != nullptr) {
              const int e = valid ? op.scale_in[pat] : 0;
              if (e != 0) scale_pow2(r, e);
            }
            V4<T>::st(&ringL[slot][tid][0], r);
            if (valid) V4<T>::st(static_cast<T *>(op.out) + (size_t)item * 4, r);
          }
        }
        }
        if (H > 1) __syncthreads();  // the set's outputs are visible to every group
        i0 = se;
      }
    }
  }
}

// ============================================================ bandwidth path
__device__ inline uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ inline void mbar_init(uint64_t *bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ inline void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ inline void mbar_wait(uint64_t *bar, unsigned parity) {
  asm volatile(
      "{\n.reg .pred P1;\nWAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ inline void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

template <typename T, int C>
struct BulkStage {
  static constexpr int kPat = kChunkItems / C;                      // patterns per chunk
  static constexpr int kPartBytes = kChunkItems * 4 * (int)sizeof(T);
  T c1[kChunkItems * 4];   // child-1 partials, or its tip states (kPat bytes)
  T c2[kChunkItems * 4];
  int32_t e1[kPat];        // child cumulative exponents (cumulative scaling)
  int32_t e2[kPat];
};

// Pair-table operations (two tip children, not applying stored factors) move
// only 1-byte tip codes, so one stage carries up to kTipGroup consecutive
// chunks of them (one copy per child instead of one per chunk): the producer
// and the consumers derive the same group sizes from the same arguments.
constexpr int kTipGroup = 16;
__device__ inline bool pair_table_op(const DevOp &op) {
  return (op.flags & (OP_TIP1 | OP_TIP2)) == (OP_TIP1 | OP_TIP2) &&
         (op.scale_out != nullptr || op.scale_in == nullptr);
}
template <int C>
__device__ inline int tip_group(const DevOp &op, int chunk, int chunk_end) {
  const int valid = (int)(((long long)op.p * C + kChunkItems - 1) / kChunkItems);  // chunks inside op.p
  if (chunk >= valid) return 1;
  return min(kTipGroup, min(chunk_end, valid) - chunk);
}

// Issue every bulk copy of chunk `chunk` of operation `oi` into `st`, arming `bar`.
template <typename T, int C>
__device__ inline void issue_chunk(const DevOp *ops, int oi, int chunk, int group, BulkStage<T, C> *st,
                                   uint64_t *bar) {
  using S = BulkStage<T, C>;
  const DevOp &op = ops[oi];
  if ((long long)chunk * kChunkItems >= (long long)op.p * C) {  // beyond this op's pattern range
    mbar_expect_tx(bar, 0u);
    return;
  }
  const bool t1 = op.flags & OP_TIP1, t2 = op.flags & OP_TIP2;
  if (pair_table_op(op)) {  // `group` chunks of tip codes
    const unsigned b = (unsigned)group * S::kPat;
    mbar_expect_tx(bar, 2 * b);
    const size_t pat0 = (size_t)chunk * S::kPat;
    bulk_g2s(st->c1, static_cast<const uint8_t *>(op.in1) + pat0, b, bar);
    bulk_g2s(st->c2, static_cast<const uint8_t *>(op.in2) + pat0, b, bar);
    return;
  }
  const bool cum = op.scale_out != nullptr;
  const bool e1 = cum && !t1 && op.cum1 != nullptr, e2 = cum && !t2 && op.cum2 != nullptr;
  const unsigned b1 = t1 ? S::kPat : S::kPartBytes, b2 = t2 ? S::kPat : S::kPartBytes;
  const unsigned be = S::kPat * 4;
  mbar_expect_tx(bar, b1 + b2 + (e1 ? be : 0u) + (e2 ? be : 0u));
  const size_t pat0 = (size_t)chunk * S::kPat;
  bulk_g2s(st->c1, t1 ? (const void *)(static_cast<const uint8_t *>(op.in1) + pat0)
                      : (const void *)(static_cast<const char *>(op.in1) + (size_t)chunk * S::kPartBytes),
           b1, bar);
  bulk_g2s(st->c2, t2 ? (const void *)(static_cast<const uint8_t *>(op.in2) + pat0)
                      : (const void *)(static_cast<const char *>(op.in2) + (size_t)chunk * S::kPartBytes),
           b2, bar);
  if (e1) bulk_g2s(st->e1, op.cum1 + pat0, be, bar);
  if (e2) bulk_g2s(st->e2, op.cum2 + pat0, be, bar);
}

__device__ inline void mbar_arrive(uint64_t *bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ inline void consumer_sync() {  // named barrier 1: the kThreads consumer threads only
  asm volatile("bar.sync 1, %0;" ::"n"(kThreads) : "memory");
}

// Transition tables for the consumers only (named barrier; the producer warp
// never touches them).
template <typename T, int C>
__device__ inline void load_ptables_consumers(T (*sP)[C][kPTab], const DevOp &op) {
  for (int t = threadIdx.x; t < 2 * C * 16; t += kThreads) {
    const int b = t / (C * 16), r = t % (C * 16), c = r / 16, zx = r % 16;
    const T v = __ldg(static_cast<const T *>(b == 0 ? op.P1 : op.P2) + r);
    sP[b][c][zx] = v;
    sP[b][c][16 + (zx % 4) * 4 + zx / 4] = v;
  }
  consumer_sync();
  for (int t = threadIdx.x; t < 2 * C * 4; t += kThreads) {
    const int b = t / (C * 4), r = t % (C * 4), c = r / 4, z = r % 4;
    const T *row = &sP[b][c][z * 4];
    sP[b][c][32 + z] = row[0] + row[1] + row[2] + row[3];
  }
  consumer_sync();
}

// Both children tips: a pattern's whole output (every category, scaled) and its
// exponent depend only on the pair of state codes, so the consumers evaluate
// the 5 x 5 pairs once per operation with exactly the per-item arithmetic
// (column lookups, product, max over (c, z), exact 2^-e) and each item becomes
// a table read.  tab: [25][C][4], tabe: [25].
template <typename T, int C, int SCALE>
__device__ inline void build_tiptip_table(T (*sP)[C][kPTab], T *tab, int *tabe) {
  const int t = threadIdx.x;
  if (t < ((25 * C + 31) / 32) * 32) {  // whole warps (the max is a C-lane shuffle)
    const int cat = t % C, combo = min(t / C, 24);
    const unsigned s1 = (unsigned)(combo / 5), s2 = (unsigned)(combo % 5);
    T v1[4], v2[4], r[4];
    tip_column(&sP[0][cat][0], s1, v1);
    tip_column(&sP[1][cat][0], s2, v2);
#pragma unroll
    for (int z = 0; z < 4; ++z) r[z] = v1[z] * v2[z];
    int e = 0;
    if (SCALE == 1) {
      T m = fmax(fmax(r[0], r[1]), fmax(r[2], r[3]));
#pragma unroll
      for (int o = 1; o < C; o <<= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
      e = frexp_exp(m);
      scale_pow2(r, e);
    }
    if (t / C < 25) {
      V4<T>::st(tab + (size_t)t * 4, r);
      if (cat == 0) tabe[combo] = e;
    }
  }
  consumer_sync();
}

// Consumer loop over chunks [c0, c1) of one operation, specialised on the
// operation's shape (tip / internal children, scaling) so the per-item body
// is branch-free: 2 LDS.128 (or 1 per tip child), the 4x4 mat-vecs from
// registers, the rescale and one STG.128.  Each warp releases a stage to the
// producer (empty barrier) as soon as it has read it.
template <typename T, int C, int kStages, bool TIP1, bool TIP2, int SCALE>
__device__ inline void bulk_chunks(const DevOp &op, const T (&P1)[16], const T (&P2)[16],
                                   const T *P1tab, const T *P2tab, BulkStage<T, C> *stages,
                                   uint64_t *full, uint64_t *empty, int c0, int c1, int &i,
                                   unsigned nitems, const T *tab, const int *tabe) {
  constexpr bool kTab = TIP1 && TIP2 && SCALE != 2;  // whole output from the pair table
  const int cat = threadIdx.x % C;
  T *__restrict__ out = static_cast<T *>(op.out);
  if constexpr (kTab) {
    for (int chunk = c0; chunk < c1; ++i) {
      const int g = tip_group<C>(op, chunk, c1);
      const int s = i % kStages;
      mbar_wait(&full[s], (unsigned)(i / kStages) & 1u);
      const BulkStage<T, C> &st = stages[s];
      const uint8_t *k1 = reinterpret_cast<const uint8_t *>(st.c1), *k2 = reinterpret_cast<const uint8_t *>(st.c2);
      for (int q = 0; q < g; ++q) {
#pragma unroll
        for (int j = 0; j < kChunkItems / kThreads; ++j) {
          const int li = threadIdx.x + j * kThreads;
          const int lp = q * (kChunkItems / C) + li / C;
          const unsigned item = (unsigned)(chunk + q) * kChunkItems + li;
          const unsigned combo = min((unsigned)k1[lp], 4u) * 5 + min((unsigned)k2[lp], 4u);
          T r[4];
          V4<T>::lds(tab + (combo * C + cat) * 4, r);
          if (item < nitems) {
            if (SCALE == 1 && cat == 0) op.scale_out[item / C] = tabe[combo];  // tips: no child exponents
            V4<T>::st(out + (size_t)item * 4, r);
          }
        }
      }
      __syncwarp();
      if ((threadIdx.x & 31) == 0) mbar_arrive(&empty[s]);
      chunk += g;
    }
  } else {
  for (int chunk = c0; chunk < c1; ++chunk, ++i) {
    const int s = i % kStages;
    mbar_wait(&full[s], (unsigned)(i / kStages) & 1u);
    const BulkStage<T, C> &st = stages[s];
    T r[kChunkItems / kThreads][4];
    int ex[kChunkItems / kThreads];
#pragma unroll
    for (int j = 0; j < kChunkItems / kThreads; ++j) {  // ---- read the stage
      const int li = threadIdx.x + j * kThreads;
      const int lp = li / C;
      T v1[4], v2[4];
      if (TIP1) {
        tip_column(P1tab, reinterpret_cast<const uint8_t *>(st.c1)[lp], v1);
      } else {
        T L[4];
        V4<T>::lds(st.c1 + li * 4, L);
        if constexpr (sizeof(T) == 8) {  // fp64: rows from shared memory (register budget)
          matvec(P1tab, L, v1);
        } else {
#pragma unroll
          for (int z = 0; z < 4; ++z)
            v1[z] = fma(P1[z * 4 + 3], L[3], fma(P1[z * 4 + 2], L[2], fma(P1[z * 4 + 1], L[1], P1[z * 4] * L[0])));
        }
      }
      if (TIP2) {
        tip_column(P2tab, reinterpret_cast<const uint8_t *>(st.c2)[lp], v2);
      } else {
        T L[4];
        V4<T>::lds(st.c2 + li * 4, L);
        if constexpr (sizeof(T) == 8) {  // fp64: rows from shared memory (register budget)
          matvec(P2tab, L, v2);
        } else {
#pragma unroll
          for (int z = 0; z < 4; ++z)
            v2[z] = fma(P2[z * 4 + 3], L[3], fma(P2[z * 4 + 2], L[2], fma(P2[z * 4 + 1], L[1], P2[z * 4] * L[0])));
        }
      }
#pragma unroll
      for (int z = 0; z < 4; ++z) r[j][z] = v1[z] * v2[z];
      ex[j] = 0;
      if (SCALE == 1 && cat == 0) {
        if (!TIP1 && op.cum1 != nullptr) ex[j] += st.e1[lp];
        if (!TIP2 && op.cum2 != nullptr) ex[j] += st.e2[lp];
      }
    }
    __syncwarp();
    if ((threadIdx.x & 31) == 0) mbar_arrive(&empty[s]);  // stage s free for the producer
#pragma unroll
    for (int j = 0; j < kChunkItems / kThreads; ++j) {  // ---- rescale + store
      const int li = threadIdx.x + j * kThreads;
      const unsigned item = (unsigned)chunk * kChunkItems + li;
      const bool valid = item < nitems;
      if (SCALE == 1) {
        T m = fmax(fmax(r[j][0], r[j][1]), fmax(r[j][2], r[j][3]));
#pragma unroll
        for (int o = 1; o < C; o <<= 1) m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
        const int e = frexp_exp(m);
        scale_pow2(r[j], e);
        if (valid && cat == 0) op.scale_out[item / C] = e + ex[j];
      } else if (SCALE == 2) {
        const int e = valid ? __ldg(op.scale_in + item / C) : 0;
        scale_pow2(r[j], e);
      }
      if (valid) V4<T>::st(out + (size_t)item * 4, r[j]);
    }
  }
  }
}

// Warp-specialised persistent kernel: warps 0..7 compute, warp 8 (one elected
// lane) streams chunks in with cp.async.bulk.  full[s]: bytes landed (tx
// count); empty[s]: all 8 consumer warps have read stage s.
template <typename T, int C, int kStages>
__global__ void __launch_bounds__(kThreads + 32, sizeof(T) == 4 ? 3 : 2)
k_partials_nuc_bulk(const DevOp *__restrict__ ops, int p, int nchunks, int total) {
  using S = BulkStage<T, C>;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  S *stages = reinterpret_cast<S *>(smem_raw);
  __shared__ __align__(16) T sP[2][C][kPTab];
  __shared__ __align__(16) T sTab[25 * C * 4];  // tip-tip pair table (build_tiptip_table)
  __shared__ int sTabE[25];
  __shared__ __align__(8) uint64_t full[kStages];
  __shared__ __align__(8) uint64_t empty[kStages];

  const int lo = (int)((long long)total * blockIdx.x / gridDim.x);
  const int hi = (int)((long long)total * (blockIdx.x + 1) / gridDim.x);
  if (lo >= hi) return;
  if (threadIdx.x == kThreads) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], kThreads / 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  pdl_wait();  // barrier setup overlaps the previous level set
  pdl_launch();

  if (threadIdx.x >= kThreads) {  // ------------------------------ producer warp
    if (threadIdx.x == kThreads) {
      int oi = lo / nchunks, chunk = lo % nchunks;
      for (int k = 0, f = lo; f < hi; ++k) {
        const int s = k % kStages;
        mbar_wait(&empty[s], ((unsigned)(k / kStages) & 1u) ^ 1u);
        // the consumers' chunk range of this op ends at min(nchunks, this CTA's end)
        const int g = pair_table_op(ops[oi]) ? tip_group<C>(ops[oi], chunk, min(nchunks, chunk + (hi - f))) : 1;
        issue_chunk<T, C>(ops, oi, chunk, g, &stages[s], &full[s]);
        f += g;
        chunk += g;
        if (chunk == nchunks) { chunk = 0; ++oi; }
      }
    }
    return;
  }

  // ------------------------------------------------------------------ consumers
  const int cat = threadIdx.x % C;
  (void)p;
  const int op_lo = lo / nchunks, op_hi = (hi - 1) / nchunks;
  int i = 0;
  for (int oi = op_lo; oi <= op_hi; ++oi) {
    const int c0 = (oi == op_lo) ? lo % nchunks : 0;
    const int c1 = (oi == op_hi) ? (hi - 1) % nchunks + 1 : nchunks;
    consumer_sync();  // previous op's tables no longer in use
    const DevOp op = ops[oi];
    const unsigned nitems = (unsigned)op.p * C;  // this operation's pattern range
    load_ptables_consumers<T, C>(sP, op);
    T P1[16], P2[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) { P1[k] = sP[0][cat][k]; P2[k] = sP[1][cat][k]; }
    const T *P1t = &sP[0][cat][0];
    const T *P2t = &sP[1][cat][0];
    const int scale = op.scale_out != nullptr ? 1 : (op.scale_in != nullptr ? 2 : 0);
    const int kind = (op.flags & 3) * 3 + scale;
    if (kind == 9) build_tiptip_table<T, C, 0>(sP, sTab, sTabE);
    if (kind == 10) build_tiptip_table<T, C, 1>(sP, sTab, sTabE);
#define RRL_BULK_CASE(K, T1, T2, SC)                                                               \
  case K:                                                                                         \
    bulk_chunks<T, C, kStages, T1, T2, SC>(op, P1, P2, P1t, P2t, stages, full, empty, c0, c1, i,   \
                                           nitems, sTab, sTabE);                                  \
    break;
    switch (kind) {
      RRL_BULK_CASE(0, false, false, 0)
      RRL_BULK_CASE(1, false, false, 1)
      RRL_BULK_CASE(2, false, false, 2)
      RRL_BULK_CASE(3, true, false, 0)
      RRL_BULK_CASE(4, true, false, 1)
      RRL_BULK_CASE(5, true, false, 2)
      RRL_BULK_CASE(6, false, true, 0)
      RRL_BULK_CASE(7, false, true, 1)
      RRL_BULK_CASE(8, false, true, 2)
      RRL_BULK_CASE(9, true, true, 0)
      RRL_BULK_CASE(10, true, true, 1)
      RRL_BULK_CASE(11, true, true, 2)
    }
#undef RRL_BULK_CASE
  }
}

// ============================================================ host launchers
template <typename T, int C, int U>
int launch_latency_u(const DevOp *d_ops, const DevOp *h_ops, int nops, int p, int gx_cap, int early,
                     cudaStream_t st) {
  const long long items = (long long)p * C;
  const int nchunks = (int)((items + kLatThreads * U - 1) / (kLatThreads * U));
  int gx = gx_cap / nops;
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
    cfg.blockDim = dim3(kLatThreads);
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
#ifdef RRL_LAT_NO_PRETIP
    early &= ~1;
#endif
    cudaError_t e = pack.n <= kInline ? cudaLaunchKernelEx(&cfg, k_partials_nuc<T, C, U, true>, pack, p, nchunks, early)
                                      : cudaLaunchKernelEx(&cfg, k_partials_nuc<T, C, U, false>, pack, p, nchunks, early);
    if (e != cudaSuccess) return (int)e;
  }
  return 0;
}

// One item per thread and at most one full wave of resident CTAs: measured on
// configs[1], fewer CTAs with more items per thread (leaving slots free for
// the next level set's early PDL launch) is slower (0.29-0.41 ms vs 0.236 ms
// per step): a launch this small is bound by its one dependent memory round
// trip, so the widest single round wins.
template <typename T, int C>
int launch_latency(const DevOp *d_ops, const DevOp *h_ops, int nops, int p, int early, cudaStream_t st) {
  static int resident_dev[kMaxDevices] = {};  // per template instance and device
  int &resident = resident_dev[device_slot()];
  if (resident <= 0) {
    int per_sm = 1, dev = 0, nsm = 148;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_partials_nuc<T, C, RRL_LAT_U, true>, kLatThreads, 0);
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    resident = (per_sm > 0 ? per_sm : 1) * nsm;
  }
  return launch_latency_u<T, C, RRL_LAT_U>(d_ops, h_ops, nops, p, resident, early, st);
}

template <typename T, int C>
int launch_bulk(const DevOp *d_ops, int nops, int p, cudaStream_t st) {
  constexpr int kStages = sizeof(T) == 4 ? 4 : 3;
  const int nchunks = (int)(((long long)p * C + kChunkItems - 1) / kChunkItems);
  const long long total = (long long)nops * nchunks;
  if (total > 0x7fffffffLL) return (int)cudaErrorInvalidValue;
  const size_t smem = sizeof(BulkStage<T, C>) * kStages;
  static int per_sm_dev[kMaxDevices] = {};  // per template instance and device
  static int nsm_dev[kMaxDevices] = {};
  const int slot = device_slot();
  int &per_sm = per_sm_dev[slot], &nsm = nsm_dev[slot];
  if (per_sm <= 0) {
    cudaError_t e = cudaFuncSetAttribute(k_partials_nuc_bulk<T, C, kStages>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return (int)e;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_partials_nuc_bulk<T, C, kStages>,
                                                      kThreads + 32, smem);
    if (e != cudaSuccess) return (int)e;
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (per_sm < 1) per_sm = 1;
  }
  long long blocks = (long long)nsm * per_sm;
  if (blocks > total) blocks = total;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)blocks);
  cfg.blockDim = dim3(kThreads + 32);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return (int)cudaLaunchKernelEx(&cfg, k_partials_nuc_bulk<T, C, kStages>, d_ops, p, nchunks, (int)total);
}

// Bandwidth path once an operation has enough patterns to keep a pipeline
// busy; the latency path for narrow work (few patterns) where a launch is
// dominated by its fixed cost.
constexpr long long kBulkMinItems = 64LL * 1024;

template <typename T, int C>
int launch_t(const DevOp *d_ops, const DevOp *h_ops, int nops, int p, int early, cudaStream_t st) {
  if ((long long)p * C >= kBulkMinItems) return launch_bulk<T, C>(d_ops, nops, p, st);
  return launch_latency<T, C>(d_ops, h_ops, nops, p, early, st);
}

template <typename T>
int dispatch_c(int c, const DevOp *d_ops, const DevOp *h_ops, int nops, int p, int early, cudaStream_t st) {
  switch (c) {
    case 1: return launch_t<T, 1>(d_ops, h_ops, nops, p, early, st);
    case 2: return launch_t<T, 2>(d_ops, h_ops, nops, p, early, st);
    case 4: return launch_t<T, 4>(d_ops, h_ops, nops, p, early, st);
    case 8: return launch_t<T, 8>(d_ops, h_ops, nops, p, early, st);
    default: return (int)cudaErrorInvalidValue;
  }
}

template <typename T, int C>
int launch_fused_t(const DevOp *d_ops, int nops, int p, cudaStream_t st) {
  constexpr int G = 2;
  constexpr int W = fused_ring(sizeof(T) == 4 ? 32 : 64);
  constexpr int H = 1;  // thread groups per CTA (H = 2 measured no faster)
  using S = FusedSmem<T, C, W>;
  constexpr size_t kBudget = 200 * 1024;
  constexpr int kMaxWin = (int)((kBudget - S::ring) / S::per_op);
  static_assert(kMaxWin >= 16, "fused window");
  static int nsm_dev[kMaxDevices] = {};
  int &nsm = nsm_dev[device_slot()];
  if (nsm == 0) {
    cudaError_t e = cudaFuncSetAttribute(k_partials_nuc_fused<T, C, G, W, H>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBudget);
    if (e != cudaSuccess) return (int)e;
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  }
  const long long items = (long long)p * C;
  const int nchunks = (int)((items + kThreads - 1) / kThreads);
  // a CTA walks the whole pass per chunk, so a second round of chunks doubles
  // the pass: shrink the window until every chunk has its own resident CTA
  int wops = std::min(nops, kMaxWin), per_sm = 1;
  for (;;) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_partials_nuc_fused<T, C, G, W, H>, kThreads * H,
                                                  S::bytes(wops));
    if ((long long)std::max(per_sm, 1) * nsm >= nchunks || wops <= 16) break;
    wops = std::max(16, wops / 2);
  }
  const size_t smem = S::bytes(wops);
  const int resident = std::max(per_sm, 1) * nsm;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)std::min(nchunks, resident));
  cfg.blockDim = dim3(kThreads * H);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return (int)cudaLaunchKernelEx(&cfg, k_partials_nuc_fused<T, C, G, W, H>, d_ops, nops, p, nchunks, wops);
}

template <typename T>
int dispatch_fused(int c, const DevOp *d_ops, int nops, int p, cudaStream_t st) {
  switch (c) {
    case 1: return launch_fused_t<T, 1>(d_ops, nops, p, st);
    case 2: return launch_fused_t<T, 2>(d_ops, nops, p, st);
    case 4: return launch_fused_t<T, 4>(d_ops, nops, p, st);
    case 8: return launch_fused_t<T, 8>(d_ops, nops, p, st);
    default: return (int)cudaErrorInvalidValue;
  }
}

}  // namespace

int launch_update_partials_nuc_fused(int prec, int c, const DevOp *d_ops, int nops, int p, void *stream) {
  if (nops <= 0 || p <= 0) return 0;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  return prec == 32 ? dispatch_fused<float>(c, d_ops, nops, p, st) : dispatch_fused<double>(c, d_ops, nops, p, st);
}

int launch_update_partials_nuc(int prec, int c, const DevOp *d_ops, const DevOp *h_ops, int nops,
                               int p, int /*p_pad*/, int early, void *stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  return prec == 32 ? dispatch_c<float>(c, d_ops, h_ops, nops, p, early, st)
                    : dispatch_c<double>(c, d_ops, h_ops, nops, p, early, st);
}

}  // namespace rrl

#ifdef RRL_LAT_TRACE
// Dev build only: copy out and reset the latency-path trace.  rec: [160 * 1024][4]
// (SM s's records at s * 1024, count cnt[s]); returns 0 or -1.
extern "C" int rrl_debug_lat_trace(unsigned long long *rec, unsigned *cnt /*[160]*/) {
  if (cudaDeviceSynchronize() != cudaSuccess) return -1;
  if (cudaMemcpyFromSymbol(cnt, rrl::g_lat_n, sizeof(rrl::g_lat_n)) != cudaSuccess) return -1;
  if (cudaMemcpyFromSymbol(rec, rrl::g_lat_trace, sizeof(rrl::g_lat_trace)) != cudaSuccess) return -1;
  static const unsigned z[160] = {};
  if (cudaMemcpyToSymbol(rrl::g_lat_n, z, sizeof(z)) != cudaSuccess) return -1;
  return 0;
}
#endif
