// Microbenchmark (dev tool): per-launch time of a chain of dependent tiny
// kernels replayed from a CUDA graph, with and without programmatic dependent
// launch -- the floor under one level-set launch.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_empty(float *x, int pdl) {
  if (pdl) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
  }
  if (threadIdx.x == 0 && blockIdx.x == 0) x[0] += 1.f;
}

__global__ void k_touch(float *x, int n, int pdl) {  // each thread 1 float4 load + store
  if (pdl) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
  }
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) {
    float4 v = reinterpret_cast<float4 *>(x)[i];
    v.x += 1.f;
    reinterpret_cast<float4 *>(x)[i] = v;
  }
}

float run(int kind, int pdl, int blocks, int chain) {
  float *x;
  cudaMalloc(&x, 64 << 20);
  cudaMemset(x, 0, 64 << 20);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
  for (int i = 0; i < chain; ++i) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(blocks);
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = pdl;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    if (kind == 0) cudaLaunchKernelEx(&cfg, k_empty, x, pdl);
    else cudaLaunchKernelEx(&cfg, k_touch, x, blocks * 256, pdl);
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
  cudaFree(x);
  return ms * 1e3f / (reps * chain);
}

int main() {
  for (int kind = 0; kind < 2; ++kind)
    for (int blocks : {1, 148, 314, 888})
      for (int pdl = 0; pdl < 2; ++pdl)
        printf("%-6s blocks %4d pdl %d: %.2f us per launch\n", kind ? "touch" : "empty", blocks, pdl,
               run(kind, pdl, blocks, 64));
  return 0;
}
