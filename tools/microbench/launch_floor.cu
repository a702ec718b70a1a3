// Microbenchmark (dev tool): per-launch time of a chain of dependent tiny
// kernels replayed from a CUDA graph, with and without programmatic dependent
// launch -- the floor under one level-set launch.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o launch_floor launch_floor.cu
//
// pdl: 0 = no PDL attribute, 1 = wait then launch_dependents, 2 = launch_dependents
// first (the latency K2's order).  kind: empty (one store), touch (one float4
// load + store per thread of the previous launch's data), touch2 (two float4
// loads of which one from the previous launch + a 4-lane shuffle max + store),
// i.e. the shape of one latency-path K2 item.
#include <cstdio>
#include <cuda_runtime.h>

template <int PDL>
__device__ inline void pdl_sync() {
  if (PDL == 1) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
  } else if (PDL == 2) {
    asm volatile("griddepcontrol.launch_dependents;");
    asm volatile("griddepcontrol.wait;" ::: "memory");
  }
}

template <int PDL>
__global__ void k_empty(float *x) {
  pdl_sync<PDL>();
  if (threadIdx.x == 0 && blockIdx.x == 0) x[0] += 1.f;
}

template <int PDL>
__global__ void k_touch(float *x, int n) {  // each thread 1 float4 load + store
  pdl_sync<PDL>();
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) {
    float4 v = reinterpret_cast<float4 *>(x)[i];
    v.x += 1.f;
    reinterpret_cast<float4 *>(x)[i] = v;
  }
}

template <int PDL>
__global__ void k_touch2(const float *__restrict__ in, float *__restrict__ out, const float *__restrict__ side,
                         int n) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
  if (i < n) s = __ldg(reinterpret_cast<const float4 *>(side) + i);  // "tip" data, before the wait
  pdl_sync<PDL>();
  if (i < n) {
    float4 v = reinterpret_cast<const float4 *>(in)[i];
    float4 r = make_float4(v.x * s.x, v.y * s.y, v.z * s.z, v.w * s.w);
    float m = fmaxf(fmaxf(r.x, r.y), fmaxf(r.z, r.w));
    m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 1));
    m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, 2));
    const float f = 1.f / m;
    reinterpret_cast<float4 *>(out)[i] = make_float4(r.x * f, r.y * f, r.z * f, r.w * f);
  }
}

float run(int kind, int pdl, int blocks, int threads, int chain) {
  float *x;
  cudaMalloc(&x, 64 << 20);
  cudaMemset(x, 0, 64 << 20);
  float *y = x + (16 << 20) / 4, *side = x + (32 << 20) / 4;
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
    at[0].val.programmaticStreamSerializationAllowed = pdl != 0;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    float *a = (i & 1) ? y : x, *b = (i & 1) ? x : y;
    if (kind == 0) {
      if (pdl == 0) cudaLaunchKernelEx(&cfg, k_empty<0>, x);
      if (pdl == 1) cudaLaunchKernelEx(&cfg, k_empty<1>, x);
      if (pdl == 2) cudaLaunchKernelEx(&cfg, k_empty<2>, x);
    } else if (kind == 1) {
      if (pdl == 0) cudaLaunchKernelEx(&cfg, k_touch<0>, x, n);
      if (pdl == 1) cudaLaunchKernelEx(&cfg, k_touch<1>, x, n);
      if (pdl == 2) cudaLaunchKernelEx(&cfg, k_touch<2>, x, n);
    } else {
      if (pdl == 0) cudaLaunchKernelEx(&cfg, k_touch2<0>, (const float *)a, b, (const float *)side, n);
      if (pdl == 1) cudaLaunchKernelEx(&cfg, k_touch2<1>, (const float *)a, b, (const float *)side, n);
      if (pdl == 2) cudaLaunchKernelEx(&cfg, k_touch2<2>, (const float *)a, b, (const float *)side, n);
    }
  }
  cudaStreamEndCapture(s, &g);
  cudaGraphInstantiate(&ge, g, 0);
  for (int w = 0; w < 5; ++w) cudaGraphLaunch(ge, s);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a, s);
  const int reps = 50;
  for (int r = 0; r < reps; ++r) cudaGraphLaunch(ge, s);
  cudaEventRecord(b, s);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  cudaGraphExecDestroy(ge);
  cudaGraphDestroy(g);
  cudaStreamDestroy(s);
  cudaFree(x);
  return ms * 1e3f / (reps * chain);
}

int main() {
  const char *names[] = {"empty", "touch", "touch2"};
  for (int kind = 0; kind < 3; ++kind)
    for (int threads : {128, 256})
      for (int blocks : {1, 148, 313, 626, 1252})
        for (int pdl = 0; pdl < 3; ++pdl)
          printf("%-6s threads %3d blocks %4d pdl %d: %.3f us per launch\n", names[kind], threads, blocks, pdl,
                 run(kind, pdl, blocks, threads, 64));
  return 0;
}
