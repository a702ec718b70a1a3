// Dev tool: phase timeline of the tcgen05 codon kernel (CTA 0, thread 0).
// Builds one level set of `nops` internal-internal operations on random
// buffers (c = 4, p patterns) and prints per-phase cycle splits:
//   stage(g+1)+fetch | wait MMA(g) | epilogue(g) | end-of-phase barrier
#define RRL_TC_TRACE 1
#include "../../paper_conf_ipps_ayresc18_b200/csrc/kernels_codon_tc.cu"

#include <cstdio>
#include <vector>

int main(int argc, char **argv) {
  using namespace rrl;
  const int p = 10240, p_pad = 10240, C = 4, nops = argc > 1 ? atoi(argv[1]) : 64;
  const size_t buf = (size_t)C * p_pad * 64;
  float *d_in, *d_out, *d_P;
  int32_t *d_sc;
  cudaMalloc(&d_in, buf * 4 * 2);
  cudaMalloc(&d_out, buf * 4 * nops);
  cudaMalloc(&d_P, (size_t)C * 64 * 64 * 4);
  cudaMalloc(&d_sc, (size_t)p_pad * 4 * nops);
  std::vector<float> h(buf * 2);
  for (size_t i = 0; i < h.size(); ++i) h[i] = (float)((i * 2654435761u) % 1000) / 1000.f;
  cudaMemcpy(d_in, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  std::vector<float> hp((size_t)C * 64 * 64, 0.f);
  for (int c = 0; c < C; ++c)
    for (int z = 0; z < 61; ++z)
      for (int x = 0; x < 61; ++x) hp[((size_t)c * 64 + z) * 64 + x] = (z == x ? 0.9f : 0.1f / 60);
  cudaMemcpy(d_P, hp.data(), hp.size() * 4, cudaMemcpyHostToDevice);
  std::vector<DevOp> ops(nops);
  for (int i = 0; i < nops; ++i) {
    DevOp d{};
    d.in1 = d_in;
    d.in2 = d_in + buf;
    d.out = d_out + buf * i;
    d.P1 = d_P;
    d.P2 = d_P;
    d.scale_out = d_sc + (size_t)p_pad * i;
    ops[i] = d;
  }
  DevOp *d_ops;
  cudaMalloc(&d_ops, sizeof(DevOp) * nops);
  cudaMemcpy(d_ops, ops.data(), sizeof(DevOp) * nops, cudaMemcpyHostToDevice);
  for (int rep = 0; rep < 3; ++rep) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    int e = launch_update_partials_codon_tc(C, d_ops, nops, p, p_pad, 0);
    cudaEventRecord(b);
    cudaDeviceSynchronize();
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    printf("rep %d: err %d (%s) %.3f ms for %d ops x %d tiles -> %.2f us per tile per SM\n", rep, e,
           cudaGetErrorString(cudaGetLastError()), ms, nops, p / 128, ms * 1e3 * 148 / (nops * (p / 128.0)));
  }
  long long tr[256][5];
  cudaMemcpyFromSymbol(tr, g_tc_trace, sizeof(tr));
  printf("phase  stage+fetch  waitMMA  epilogue  barrier  (cycles)\n");
  for (int g = 0; g < 24; ++g)
    printf("%4d %10lld %9lld %9lld %8lld\n", g, tr[g][1] - tr[g][0], tr[g][2] - tr[g][1], tr[g][3] - tr[g][2],
           tr[g][4] - tr[g][3]);
  long long tot[4] = {0, 0, 0, 0};
  for (int g = 8; g < 200; ++g)
    for (int k = 0; k < 4; ++k) tot[k] += tr[g][k + 1] - tr[g][k];
  printf("avg over phases 8..199: stage %.0f  waitMMA %.0f  epilogue %.0f  barrier %.0f\n", tot[0] / 192.0,
         tot[1] / 192.0, tot[2] / 192.0, tot[3] / 192.0);
  return 0;
}
