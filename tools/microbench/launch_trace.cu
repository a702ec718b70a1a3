// Microbenchmark (dev tool): globaltimer timeline of a CUDA-graph chain of
// dependent touch2 kernels (one float4 load of the previous launch's output
// after griddepcontrol.wait, a 4-lane shuffle max, one float4 store) -- the
// same stamps as tools/trace_latency.py takes inside the latency-path K2, for
// a kernel with nothing else in it.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o launch_trace launch_trace.cu
#include <algorithm>
#include <cstdio>
#include <vector>
#include <cuda_runtime.h>

__device__ inline unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)::"memory");
  return t;
}
__device__ inline unsigned long long gtime_after(float x) {
  unsigned long long t;
  asm volatile("{.reg .f32 d; add.f32 d, %1, 0f00000000; mov.u64 %0, %%globaltimer;}" : "=l"(t) : "f"(x) : "memory");
  return t;
}

// F (feature bits, to find what the latency-path K2 adds over touch2):
//  1: cat-0 threads also load a 4-byte exponent written by the previous launch
//     and store one (the cumulative exponents)
//  2: the child goes through a 4x4 mat-vec from shared-memory tables staged
//     before the wait, times a tip column (LDS)
//  4: rescale as K2 does (frexp exponent, power-of-two multiply, branches)
template <int F>
__global__ void k_t2(const float *__restrict__ in, float *__restrict__ out, const float *__restrict__ side, int n,
                     unsigned long long *rec, int launch, const int *__restrict__ ein, int *__restrict__ eout,
                     const float *__restrict__ P) {
  __shared__ __align__(16) float sP[4][36];
  const unsigned long long t0 = gtime();
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  float4 s = make_float4(1.f, 1.f, 1.f, 1.f);
  if (i < n) s = __ldg(reinterpret_cast<const float4 *>(side) + i);
  if (F & 2) {
    if (threadIdx.x < 16) {
      const float4 row = __ldg(reinterpret_cast<const float4 *>(P) + threadIdx.x);
      float *tab = &sP[threadIdx.x / 4][0];
      const int z = threadIdx.x % 4;
      reinterpret_cast<float4 *>(tab)[z] = row;
      tab[16 + z] = row.x; tab[20 + z] = row.y; tab[24 + z] = row.z; tab[28 + z] = row.w;
      tab[32 + z] = row.x + row.y + row.z + row.w;
    }
    __syncthreads();
  }
  asm volatile("griddepcontrol.launch_dependents;");
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const unsigned long long t1 = gtime();
  unsigned long long t2 = 0;
  const int cat = threadIdx.x & 3;
  if (i < n) {
    float4 v = reinterpret_cast<const float4 *>(in)[i];
    int ea = 0;
    if ((F & 1) && cat == 0) ea = __ldg(ein + i / 4);
    float4 r;
    if (F & 2) {
      const float *t = &sP[cat][0];
      const float4 tc = *reinterpret_cast<const float4 *>(t + 16 + 4 * (int)(s.x) % 5);
      float a[4];
#pragma unroll
      for (int z = 0; z < 4; ++z) {
        const float4 row = *reinterpret_cast<const float4 *>(t + 4 * z);
        a[z] = fmaf(row.w, v.w, fmaf(row.z, v.z, fmaf(row.y, v.y, row.x * v.x)));
      }
      r = make_float4(a[0] * tc.x, a[1] * tc.y, a[2] * tc.z, a[3] * tc.w);
    } else {
      r = make_float4(v.x * s.x + 1.f, v.y * s.y, v.z * s.z, v.w * s.w);
    }
    if (threadIdx.x == 0) t2 = gtime_after(r.x + (float)ea);
    float m = fmaxf(fmaxf(r.x, r.y), fmaxf(r.z, r.w));
    m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 1));
    m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 2));
    int e = 0;
    if (F & 4) {
      const unsigned b = __float_as_uint(m);
      const int eb = (int)((b >> 23) & 0xffu);
      if (eb != 0 && eb != 0xff) e = eb - 126;
      else if (m != 0.f) frexpf(m, &e);
      if (e != 0) {
        if (e > -126 && e < 126) {
          const float f = __uint_as_float((unsigned)(127 - e) << 23);
          r.x *= f; r.y *= f; r.z *= f; r.w *= f;
        } else {
          r.x = ldexpf(r.x, -e); r.y = ldexpf(r.y, -e); r.z = ldexpf(r.z, -e); r.w = ldexpf(r.w, -e);
        }
      }
    } else {
      const float f = 1.f / m;
      r.x *= f; r.y *= f; r.z *= f; r.w *= f;
    }
    reinterpret_cast<float4 *>(out)[i] = r;
    if ((F & 1) && cat == 0) eout[i / 4] = e + ea;
  }
  if (threadIdx.x == 0) {
    const unsigned long long t3 = gtime();
    unsigned long long *q = rec + ((size_t)launch * gridDim.x + blockIdx.x) * 4;
    q[0] = t0; q[1] = t1; q[2] = t2; q[3] = t3;
  }
}

// F8: the latency K2's addressing -- a 2-D grid (blockIdx.y = operation) and
// the per-operation pointers in a 912-byte by-value parameter struct (8 inline
// descriptors of 112 bytes), read after the wait like K2's exponent pointers.
struct Desc {
  const float *in;
  float *out;
  const float *side;
  const int *ein;
  int *eout;
  const float *P;
  long long pad[8];
};
struct Pack {
  const Desc *ops;
  int n;
  Desc inl[8];
};
__global__ void k_t2p(const __grid_constant__ Pack pack, int n, unsigned long long *rec, int launch) {
  __shared__ __align__(16) float sP[4][36];
  const unsigned long long t0 = gtime();
  Desc d = pack.inl[blockIdx.y];
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  float4 s = make_float4(1.f, 1.f, 1.f, 1.f);
  if (i < n) s = __ldg(reinterpret_cast<const float4 *>(d.side) + i);
  if (threadIdx.x < 16) {
    const float4 row = __ldg(reinterpret_cast<const float4 *>(d.P) + threadIdx.x);
    float *tab = &sP[threadIdx.x / 4][0];
    const int z = threadIdx.x % 4;
    reinterpret_cast<float4 *>(tab)[z] = row;
    tab[16 + z] = row.x; tab[20 + z] = row.y; tab[24 + z] = row.z; tab[28 + z] = row.w;
    tab[32 + z] = row.x + row.y + row.z + row.w;
  }
  __syncthreads();
  asm volatile("griddepcontrol.launch_dependents;");
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const unsigned long long t1 = gtime();
  unsigned long long t2 = 0;
  const int cat = threadIdx.x & 3;
  if (i < n) {
    float4 v = reinterpret_cast<const float4 *>(d.in)[i];
    int ea = 0;
    if (cat == 0) ea = __ldg(d.ein + i / 4);
    const float *t = &sP[cat][0];
    const float4 tc = *reinterpret_cast<const float4 *>(t + 16 + 4 * ((int)(s.x) % 5));
    float a[4];
#pragma unroll
    for (int z = 0; z < 4; ++z) {
      const float4 row = *reinterpret_cast<const float4 *>(t + 4 * z);
      a[z] = fmaf(row.w, v.w, fmaf(row.z, v.z, fmaf(row.y, v.y, row.x * v.x)));
    }
    float4 r = make_float4(a[0] * tc.x, a[1] * tc.y, a[2] * tc.z, a[3] * tc.w);
    if (threadIdx.x == 0) t2 = gtime_after(r.x + (float)ea);
    float m = fmaxf(fmaxf(r.x, r.y), fmaxf(r.z, r.w));
    m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 1));
    m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 2));
    const unsigned b = __float_as_uint(m);
    const int eb = (int)((b >> 23) & 0xffu);
    int e = (eb != 0 && eb != 0xff) ? eb - 126 : 0;
    const float f = __uint_as_float((unsigned)(127 - e) << 23);
    r.x *= f; r.y *= f; r.z *= f; r.w *= f;
    reinterpret_cast<float4 *>(d.out)[i] = r;
    if (cat == 0) d.eout[i / 4] = e + ea;
  }
  if (threadIdx.x == 0) {
    const unsigned long long t3 = gtime();
    unsigned long long *q = rec + ((size_t)launch * gridDim.x * gridDim.y + blockIdx.y * gridDim.x + blockIdx.x) * 4;
    q[0] = t0; q[1] = t1; q[2] = t2; q[3] = t3;
  }
}

static double med(std::vector<double> v) {
  std::sort(v.begin(), v.end());
  return v.empty() ? 0 : v[v.size() / 2];
}

int main() {
  const int chain = 64;
  // spread = 0: ping-pong between two buffers; 1: launch i reads buffer i and
  // writes buffer i + 1 (every launch touches new pages, like the level sets)
  for (int F : {7, 8})
  for (int spread = 0; spread < 2; ++spread)
  for (int threads : {128})
    for (int blocks : {313, 626}) {
      if (F != 0 && spread == 0) continue;
      float *x;
      const size_t stride = (size_t)blocks * threads * 4;  // floats per buffer
      const size_t bytes = spread ? (stride * (chain + 2) * 4 + (32 << 20)) : (96 << 20);
      cudaMalloc(&x, bytes);
      cudaMemset(x, 0, bytes);
      int *ex;
      cudaMalloc(&ex, (size_t)(chain + 2) * blocks * threads);
      cudaMemset(ex, 0, (size_t)(chain + 2) * blocks * threads);
      float *y = x + (16 << 20) / 4, *side = spread ? x + stride * (chain + 2) : x + (32 << 20) / 4;
      unsigned long long *rec;
      cudaMalloc(&rec, (size_t)chain * blocks * 4 * 8);
      cudaStream_t s;
      cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
      cudaGraph_t g;
      cudaGraphExec_t ge;
      cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
      const int n = blocks * threads;
      for (int i = 0; i < chain; ++i) {
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(blocks);
        cfg.blockDim = dim3(threads);
        cfg.stream = s;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        float *a = (i & 1) ? y : x, *b = (i & 1) ? x : y;
        if (spread) a = x + stride * i, b = x + stride * (i + 1);
        const int *ea = ex + (size_t)(i % 2) * blocks * threads / 4;
        int *eb = ex + (size_t)((i + 1) % 2) * blocks * threads / 4;
        if (spread) ea = ex + (size_t)i * blocks * threads / 4, eb = ex + (size_t)(i + 1) * blocks * threads / 4;
        const float *Pm = side + n * 4;
        if (F == 0) cudaLaunchKernelEx(&cfg, k_t2<0>, (const float *)a, b, (const float *)side, n, rec, i, ea, eb, Pm);
        if (F == 1) cudaLaunchKernelEx(&cfg, k_t2<1>, (const float *)a, b, (const float *)side, n, rec, i, ea, eb, Pm);
        if (F == 2) cudaLaunchKernelEx(&cfg, k_t2<2>, (const float *)a, b, (const float *)side, n, rec, i, ea, eb, Pm);
        if (F == 4) cudaLaunchKernelEx(&cfg, k_t2<4>, (const float *)a, b, (const float *)side, n, rec, i, ea, eb, Pm);
        if (F == 7) cudaLaunchKernelEx(&cfg, k_t2<7>, (const float *)a, b, (const float *)side, n, rec, i, ea, eb, Pm);
        if (F == 8) {  // the same work as two operations of half the CTAs each (gridDim.y = 2)
          Pack pk{};
          pk.n = 2;
          const int half = n / 2;
          for (int o = 0; o < 2; ++o) {
            pk.inl[o].in = a + (size_t)o * half * 4;
            pk.inl[o].out = b + (size_t)o * half * 4;
            pk.inl[o].side = side + (size_t)o * half * 4;
            pk.inl[o].ein = ea + (size_t)o * half / 4;
            pk.inl[o].eout = eb + (size_t)o * half / 4;
            pk.inl[o].P = Pm + o * 64;
          }
          cfg.gridDim = dim3(blocks / 2, 2);
          cudaLaunchKernelEx(&cfg, k_t2p, pk, half, rec, i);
        }
      }
      cudaStreamEndCapture(s, &g);
      cudaGraphInstantiate(&ge, g, 0);
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      for (int w = 0; w < 5; ++w) cudaGraphLaunch(ge, s);
      cudaEventRecord(e0, s);
      for (int r = 0; r < 20; ++r) cudaGraphLaunch(ge, s);
      cudaEventRecord(e1, s);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      std::vector<unsigned long long> h((size_t)chain * blocks * 4);
      cudaMemcpy(h.data(), rec, h.size() * 8, cudaMemcpyDeviceToHost);
      std::vector<double> body, rel, ldmed, ldmax, tail;
      unsigned long long prev_end = 0;
      for (int l = 0; l < chain; ++l) {
        unsigned long long wmin = ~0ull, emax = 0, lmax = 0;
        std::vector<double> lds, tails;
        for (int b = 0; b < blocks; ++b) {
          const unsigned long long *q = &h[((size_t)l * blocks + b) * 4];
          wmin = std::min(wmin, q[1]);
          emax = std::max(emax, q[3]);
          lmax = std::max(lmax, q[2]);
        }
        for (int b = 0; b < blocks; ++b) {
          const unsigned long long *q = &h[((size_t)l * blocks + b) * 4];
          lds.push_back((double)(q[2] - q[1]));
          tails.push_back((double)(q[3] - q[2]));
        }
        body.push_back((double)(emax - wmin));
        ldmed.push_back(med(lds));
        ldmax.push_back((double)(lmax - wmin));
        tail.push_back(med(tails));
        if (l > 0) rel.push_back((double)wmin - (double)prev_end);
        prev_end = emax;
      }
      printf("F%d %s touch2 %3d threads x %4d blocks: %.3f us per launch | body %.0f  release %.0f  wait->ld median CTA %.0f  "
             "first wait->last ld %.0f  ld->end %.0f ns\n",
             F, spread ? "spread  " : "pingpong", threads, blocks, ms * 1e3 / (20 * chain), med(body), med(rel), med(ldmed), med(ldmax), med(tail));
      cudaGraphExecDestroy(ge);
      cudaGraphDestroy(g);
      cudaStreamDestroy(s);
      cudaFree(rec);
      cudaFree(ex);
      cudaFree(x);
    }
  return 0;
}
