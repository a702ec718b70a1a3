// Instance management and the host side of the C ABI in include/rrl.h.
//
// One instance = one device + one stream + device-resident buffers sized for
// 180 GB of HBM: internal partials in one slab, tip states as uint8 (1 B per
// pattern instead of s x c x 4 B of partials), transition matrices, scale
// exponents.  rrl_update_partials resolves the caller's operations into
// device descriptors (DevOp) once per distinct operation list, then issues
// ONE kernel launch per concurrent operation set, optionally
// captured into a CUDA graph and replayed.
#include <cuda.h>  // CUtensorMap (encoded through the runtime's driver entry point)
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "rrl.h"
#include "rrl_internal.h"

namespace rrl {

thread_local std::string g_last_error;

int fail(int code, const std::string &msg) {
  g_last_error = msg;
  return code;
}

namespace {

struct EvPair {
  cudaEvent_t a, b;
  int kind;  // 0 partials, 1 matrices, 2 root, 3 scale
};

struct Instance {
  int device = 0;
  cudaStream_t own_stream = nullptr, stream = nullptr;
  int n_tips = 0, n_buf = 0, s = 0, s_pad = 0, p = 0, p_pad = 0, c = 0;
  int n_mat = 0, n_eig = 0, n_scale = 0, prec = 32;
  uint32_t flags = 0;
  size_t elt = 4, buf_elems = 0, buf_bytes = 0, mat_elems = 0;

  char *d_partials = nullptr;            // internal buffers
  std::vector<void *> tip_partials;      // lazily allocated
  std::vector<char> has_states;
  uint8_t *d_states = nullptr;           // [n_tips][p_pad]
  char *d_P = nullptr;                   // [n_mat][c][s_pad][s_pad]
  float *d_Plo = nullptr;                // fp32 codon: tf32 low parts of d_P (3xTF32 operand), same layout
  char *d_PT = nullptr;                  // codon: P^T per (matrix, category), row 61 = row sums (K3-TT)
  int32_t *d_scale = nullptr;            // [n_scale][p_pad]
  double *d_eig = nullptr;               // [n_eig][2 s^2 + s]
  double *d_rates = nullptr;             // [n_eig][c] (per model / partition)
  double *d_catw = nullptr;              // [n_eig][c]
  double *d_freqs = nullptr;             // [n_eig][s]
  double *d_pw = nullptr;                // [p]
  double *d_site = nullptr;              // [p_pad]
  double *d_block = nullptr;             // [nblocks]
  double *d_out = nullptr;               // scalar
  unsigned *d_count = nullptr;           // last-block-done ticket of K4/K6
  unsigned *d_flag = nullptr;            // tip-state validation result
  double *h_out = nullptr;               // pinned scalar
  int nblocks = 0;

  // transition-matrix call staging
  double *d_t = nullptr;       // [t_cap] branch lengths, then d_midx [t_cap] (one allocation)
  int32_t *d_midx = nullptr;
  std::vector<char> h_tstage;  // host staging of the same layout: one H2D copy per call
  int t_cap = 0;
  int t_count = -1;            // entries of h_tstage that mirror d_t (-1: none)
  // accumulate-scale index list
  int32_t *d_sidx = nullptr;
  int sidx_cap = 0;

  // operation descriptors
  DevOp *d_ops = nullptr;
  DevOp *h_ops = nullptr;  // pinned staging
  int ops_cap = 0;
  cudaEvent_t staging_ev = nullptr;
  std::vector<rrl_op> last_ops;
  std::vector<int32_t> last_offs;
  std::vector<int32_t> last_ranges;
  std::vector<int> set_tt;               // 61-state fp32: tip-tip ops at the front of each set
  bool ops_valid = false;
  cudaGraphExec_t graph = nullptr;       // replay of the set launches
  cudaStream_t graph_stream = nullptr;
  int graph_kernels = 0;
  // K1 deferred into the level-set graph (RRL_FLAG_CUDA_GRAPH, profiling off):
  // rrl_update_transition_matrices records it, the next rrl_update_partials
  // replays it as the graph's first node; any other call launches it first.
  bool k1_pending = false;
  int k1_eig = 0, k1_count = 0;
  // The level-set graph's launch deferred to the next call (graph mode,
  // profiling off): rrl_calculate_root_log_likelihoods_device replays it and
  // K4 as one graph (child graph + K4 node), any other call launches it first.
  bool pass_pending = false;
  cudaGraph_t graph_tmpl = nullptr;        // the captured level-set graph (child of root_graph)
  unsigned graph_gen = 0;                  // bumped at every (re)capture
  cudaGraphExec_t root_graph = nullptr;    // [level-set graph] -> K4
  unsigned root_gen = ~0u;
  int root_key[4] = {-2, -2, -2, -2};
  double *root_out = nullptr;
  bool graph_has_k1 = false;               // the captured graph starts with K1 for:
  int graph_k1_eig = -1, graph_k1_count = -1;
  const double *graph_k1_t = nullptr;

  bool profiling = false;
  std::vector<EvPair> events;
  std::vector<cudaEvent_t> ev_pool;
  rrl_profile prof{};

  // TMA descriptors of the internal-partials and matrix slabs (61-state fp32, K3-TC5)
  CUtensorMap tmap_partials{}, tmap_P{}, tmap_Plo{};
  bool tmaps_ok = false;

};

std::mutex g_mu;
std::vector<Instance *> g_inst;

#define CK(x)                                                                        \
  do {                                                                               \
    cudaError_t e_ = (x);                                                            \
    if (e_ != cudaSuccess)                                                           \
      return fail(e_ == cudaErrorMemoryAllocation ? RRL_ERROR_OUT_OF_MEMORY : RRL_ERROR_CUDA, \
                  std::string(#x) + ": " + cudaGetErrorString(e_));                  \
  } while (0)

#define CKL(x)                                                                       \
  do {                                                                               \
    int e_ = (x);                                                                    \
    if (e_ != 0)                                                                     \
      return fail(RRL_ERROR_CUDA, std::string(#x) + ": " +                           \
                                      cudaGetErrorString(static_cast<cudaError_t>(e_))); \
  } while (0)

Instance *get(int id) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (id < 0 || id >= (int)g_inst.size()) return nullptr;
  return g_inst[id];
}

int use_device(Instance *I) {
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != I->device) CK(cudaSetDevice(I->device));
  return 0;
}

int launch_k1(Instance *I, int eigen_idx, int count);
int flush_pass(Instance *I);
// A deferred K1 (and a deferred level-set graph) go onto the stream before
// anything else the instance does.
int flush_k1(Instance *I) {
  int r = flush_pass(I);
  if (r < 0 || !I->k1_pending) return r;
  I->k1_pending = false;
  return launch_k1(I, I->k1_eig, I->k1_count);
}

#define GET_RAW(I, id)                                                              \
  Instance *I = get(id);                                                            \
  if (!I) return fail(RRL_ERROR_UNINITIALIZED_INSTANCE, "no such instance");        \
  {                                                                                 \
    int r_ = use_device(I);                                                         \
    if (r_ < 0) return r_;                                                          \
  }
#define GET(I, id)                                                                  \
  GET_RAW(I, id)                                                                    \
  {                                                                                 \
    int r_ = flush_k1(I);                                                           \
    if (r_ < 0) return r_;                                                          \
  }

cudaEvent_t take_event(Instance *I) {
  if (!I->ev_pool.empty()) {
    cudaEvent_t e = I->ev_pool.back();
    I->ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  cudaEventCreate(&e);
  return e;
}

struct Timed {  // brackets one launch with events when profiling
  Instance *I;
  EvPair ep{};
  bool on;
  Timed(Instance *in, int kind, bool enabled = true) : I(in), on(in->profiling && enabled) {
    if (on) {
      ep.a = take_event(I);
      ep.b = take_event(I);
      ep.kind = kind;
      cudaEventRecord(ep.a, I->stream);
    }
  }
  ~Timed() {
    if (on) {
      cudaEventRecord(ep.b, I->stream);
      I->events.push_back(ep);
    }
  }
};

void drain_events(Instance *I) {
  for (auto &ep : I->events) {
    cudaEventSynchronize(ep.b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ep.a, ep.b);
    switch (ep.kind) {
      case 0: I->prof.partials_ms += ms; break;
      case 1: I->prof.matrices_ms += ms; break;
      case 2: I->prof.root_ms += ms; break;
      default: I->prof.scale_ms += ms; break;
    }
    I->ev_pool.push_back(ep.a);
    I->ev_pool.push_back(ep.b);
  }
  I->events.clear();
}

int drop_graphs(Instance *I) {
  if (I->graph) cudaGraphExecDestroy(I->graph);
  I->graph = nullptr;
  if (I->graph_tmpl) cudaGraphDestroy(I->graph_tmpl);
  I->graph_tmpl = nullptr;
  if (I->root_graph) cudaGraphExecDestroy(I->root_graph);
  I->root_graph = nullptr;
  I->graph_gen += 1;
  return 0;
}

int flush_pass(Instance *I) {
  if (!I->pass_pending) return 0;
  I->pass_pending = false;
  Timed tm(I, 0);
  CK(cudaGraphLaunch(I->graph, I->stream));
  return 0;
}

// K1 on the instance stream (eagerly, or inside the level-set graph's capture).
int launch_k1(Instance *I, int eigen_idx, int count) {
  const size_t eig_sz = 2 * (size_t)I->s * I->s + I->s;
  {
    Timed tm(I, 1);
    CKL(launch_transition_matrices(I->prec, I->s, I->s_pad, I->c, I->d_eig + eig_sz * eigen_idx,
                                   I->d_rates + (size_t)eigen_idx * I->c, I->d_midx, I->d_t, count, I->d_P,
                                   I->d_Plo, I->d_PT, I->stream));
  }
  I->prof.matrices_launches += (count + 65534) / 65535;
  I->prof.kernel_launches += (count + 65534) / 65535;
  return RRL_SUCCESS;
}

void destroy(Instance *I) {
  cudaSetDevice(I->device);
  if (I->stream) cudaStreamSynchronize(I->stream);
  drop_graphs(I);
  for (void *t : I->tip_partials)
    if (t) cudaFree(t);
  void *ptrs[] = {I->d_partials, I->d_states, I->d_P,    I->d_scale, I->d_eig,  I->d_rates,
                  I->d_catw,     I->d_freqs,  I->d_pw,   I->d_site,  I->d_block, I->d_out, I->d_count,
                  I->d_t,      I->d_sidx, I->d_ops,  I->d_Plo,  I->d_flag, I->d_PT};
  for (void *q : ptrs)
    if (q) cudaFree(q);
  if (I->h_ops) cudaFreeHost(I->h_ops);
  if (I->h_out) cudaFreeHost(I->h_out);
  for (auto &ep : I->events) {
    cudaEventDestroy(ep.a);
    cudaEventDestroy(ep.b);
  }
  for (auto e : I->ev_pool) cudaEventDestroy(e);
  if (I->staging_ev) cudaEventDestroy(I->staging_ev);
  if (I->own_stream) cudaStreamDestroy(I->own_stream);
  delete I;
}

size_t pidx(const Instance *I, int pat, int cat, int z) {  // device element index
  if (I->s == 4) return ((size_t)pat * I->c + cat) * 4 + z;
  return ((size_t)cat * I->p_pad + pat) * I->s_pad + z;
}

void *buffer_ptr(Instance *I, int b) {
  if (b < I->n_tips) return I->tip_partials[b];
  return I->d_partials + (size_t)(b - I->n_tips) * I->buf_bytes;
}

int upload_partials(Instance *I, int b, const double *host_cps /*[c][p][s]*/, bool tip_pattern_major) {
  std::vector<char> h(I->buf_bytes, 0);
  for (int cat = 0; cat < I->c; ++cat)
    for (int pat = 0; pat < I->p; ++pat)
      for (int z = 0; z < I->s; ++z) {
        const double v = tip_pattern_major ? host_cps[(size_t)pat * I->s + z]
                                           : host_cps[((size_t)cat * I->p + pat) * I->s + z];
        const size_t k = pidx(I, pat, cat, z);
        if (I->prec == 32) reinterpret_cast<float *>(h.data())[k] = (float)v;
        else reinterpret_cast<double *>(h.data())[k] = v;
      }
  CK(cudaMemcpyAsync(buffer_ptr(I, b), h.data(), I->buf_bytes, cudaMemcpyHostToDevice, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int ensure_cap_ops(Instance *I, int n) {
  if (n <= I->ops_cap) return 0;
  if (I->staging_ev) CK(cudaEventSynchronize(I->staging_ev));
  CK(cudaStreamSynchronize(I->stream));
  if (I->d_ops) cudaFree(I->d_ops);
  if (I->h_ops) cudaFreeHost(I->h_ops);
  I->d_ops = nullptr;
  I->h_ops = nullptr;
  const int cap = std::max(n, 64);
  CK(cudaMalloc(&I->d_ops, sizeof(DevOp) * cap));
  CK(cudaMallocHost(&I->h_ops, sizeof(DevOp) * cap));
  I->ops_cap = cap;
  return 0;
}

}  // namespace
}  // namespace rrl

using namespace rrl;

extern "C" {

const char *rrl_version(void) { return "rrl 0.1.0 (sm_100a)"; }

const char *rrl_last_error_message(void) { return rrl::g_last_error.c_str(); }

const char *rrl_error_string(int code) {
  switch (code) {
    case RRL_SUCCESS: return "success";
    case RRL_ERROR_GENERAL: return "general error";
    case RRL_ERROR_OUT_OF_MEMORY: return "out of memory";
    case RRL_ERROR_UNIDENTIFIED_EXCEPTION: return "unidentified exception";
    case RRL_ERROR_UNINITIALIZED_INSTANCE: return "uninitialized instance";
    case RRL_ERROR_OUT_OF_RANGE: return "index out of range";
    case RRL_ERROR_NO_RESOURCE: return "no such resource (device)";
    case RRL_ERROR_NO_IMPLEMENTATION: return "no implementation for this configuration";
    case RRL_ERROR_FLOATING_POINT: return "non-finite log-likelihood";
    case RRL_ERROR_INVALID_TREE: return "invalid tree";
    case RRL_ERROR_CUDA: return "CUDA error";
    default: return "unknown error";
  }
}

int rrl_create_instance(int tip_count, int partials_buffer_count, int state_count,
                        int pattern_count, int category_count, int matrix_count, int eigen_count,
                        int scale_buffer_count, int device, int precision, uint32_t flags) {
  if (state_count != 4 && state_count != 61)
    return fail(RRL_ERROR_NO_IMPLEMENTATION, "state_count must be 4 or 61");
  if (category_count != 1 && category_count != 2 && category_count != 4 && category_count != 8)
    return fail(RRL_ERROR_NO_IMPLEMENTATION, "category_count must be 1, 2, 4 or 8");
  if (precision != 32 && precision != 64) return fail(RRL_ERROR_NO_IMPLEMENTATION, "precision 32|64");
  if (tip_count < 2 || partials_buffer_count < tip_count + 1 || pattern_count < 1 ||
      matrix_count < 1 || eigen_count < 1 || scale_buffer_count < 0)
    return fail(RRL_ERROR_GENERAL, "bad instance dimensions");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev)
    return fail(RRL_ERROR_NO_RESOURCE, "no such CUDA device");
  auto *I = new Instance();
  I->device = device;
  I->n_tips = tip_count;
  I->n_buf = partials_buffer_count;
  I->s = state_count;
  I->s_pad = state_count == 4 ? 4 : 64;
  I->p = pattern_count;
  I->p_pad = (pattern_count + 511) / 512 * 512;  // whole bulk-copy chunks (kernels_nuc.cu)
  I->c = category_count;
  I->n_mat = matrix_count;
  I->n_eig = eigen_count;
  I->n_scale = scale_buffer_count;
  I->prec = precision;
  I->flags = flags;
  I->elt = precision == 32 ? 4 : 8;
  I->buf_elems = (size_t)I->p_pad * I->c * I->s_pad;
  I->buf_bytes = I->buf_elems * I->elt;
  I->mat_elems = (size_t)I->c * I->s_pad * I->s_pad;
  I->tip_partials.assign(tip_count, nullptr);
  I->has_states.assign(tip_count, 0);
  // K4/K6 grid: c threads per pattern (4 states, K4; K6 takes a thread per pattern
  // within the same grid) or a warp per pattern (61 states)
  I->nblocks = std::min(148 * 4, state_count == 61 ? (pattern_count + 7) / 8
                                                   : (int)(((long long)pattern_count * category_count + 255) / 256));
  auto bail = [&](int code, const std::string &m) {
    destroy(I);
    return fail(code, m);
  };
#define CKC(x)                                                                         \
  do {                                                                                 \
    cudaError_t e_ = (x);                                                              \
    if (e_ != cudaSuccess)                                                             \
      return bail(e_ == cudaErrorMemoryAllocation ? RRL_ERROR_OUT_OF_MEMORY : RRL_ERROR_CUDA, \
                  std::string(#x) + ": " + cudaGetErrorString(e_));                    \
  } while (0)
  CKC(cudaSetDevice(device));
  CKC(cudaStreamCreateWithFlags(&I->own_stream, cudaStreamNonBlocking));
  I->stream = I->own_stream;
  CKC(cudaEventCreateWithFlags(&I->staging_ev, cudaEventDisableTiming));
  const size_t n_int = (size_t)(partials_buffer_count - tip_count);
  CKC(cudaMalloc(&I->d_partials, std::max<size_t>(n_int * I->buf_bytes, 256)));
  CKC(cudaMalloc(&I->d_states, (size_t)tip_count * I->p_pad));
  CKC(cudaMemset(I->d_states, state_count, (size_t)tip_count * I->p_pad));
  CKC(cudaMalloc(&I->d_P, (size_t)matrix_count * I->mat_elems * I->elt));
  CKC(cudaMemset(I->d_P, 0, (size_t)matrix_count * I->mat_elems * I->elt));
  CKC(cudaMalloc(&I->d_scale, std::max<size_t>((size_t)scale_buffer_count * I->p_pad * 4, 256)));
  CKC(cudaMemset(I->d_scale, 0, std::max<size_t>((size_t)scale_buffer_count * I->p_pad * 4, 256)));
  const size_t eig_sz = 2 * (size_t)state_count * state_count + state_count;
  CKC(cudaMalloc(&I->d_eig, sizeof(double) * eig_sz * eigen_count));
  CKC(cudaMalloc(&I->d_rates, sizeof(double) * category_count * eigen_count));
  CKC(cudaMalloc(&I->d_catw, sizeof(double) * category_count * eigen_count));
  CKC(cudaMalloc(&I->d_freqs, sizeof(double) * state_count * eigen_count));
  CKC(cudaMalloc(&I->d_pw, sizeof(double) * I->p_pad));
  CKC(cudaMalloc(&I->d_site, sizeof(double) * I->p_pad));
  CKC(cudaMalloc(&I->d_block, sizeof(double) * I->nblocks));
  CKC(cudaMalloc(&I->d_out, sizeof(double)));
  CKC(cudaMalloc(&I->d_count, sizeof(unsigned)));
  CKC(cudaMemset(I->d_count, 0, sizeof(unsigned)));
  if (state_count == 61 && precision == 32 && n_int > 0) {
    // 4-D maps, innermost first: internal partials {64 states, p_pad, c, buffer},
    // matrices {64 child states, 64 parent states, c, matrix}; boxes of 32 states
    // (one 128-byte swizzle row) x 128 patterns / 64 parent states.
    const char *env = std::getenv("RRL_CODON_TC5");
    PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (!(env && env[0] == '0') &&
        cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &q) == cudaSuccess &&
        enc != nullptr && n_int <= 0x7fffffff) {
      const cuuint64_t gA[4] = {64, (cuuint64_t)I->p_pad, (cuuint64_t)I->c, (cuuint64_t)n_int};
      const cuuint64_t sA[3] = {256, (cuuint64_t)I->p_pad * 256, (cuuint64_t)I->buf_bytes};
      const cuuint32_t bA[4] = {32, 128, 1, 1}, es[4] = {1, 1, 1, 1};
      const cuuint64_t gP[4] = {64, 64, (cuuint64_t)I->c, (cuuint64_t)matrix_count};
      const cuuint64_t sP[3] = {256, 64 * 256, (cuuint64_t)I->c * 64 * 256};
      const cuuint32_t bP[4] = {32, 64, 1, 1};
      const CUresult r1 = enc(&I->tmap_partials, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, I->d_partials, gA, sA, bA, es,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                              CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      const CUresult r2 = enc(&I->tmap_P, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, I->d_P, gP, sP, bP, es,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                              CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      const size_t pbytes = (size_t)matrix_count * I->mat_elems * I->elt;
      CKC(cudaMalloc(&I->d_Plo, pbytes));
      CKC(cudaMemset(I->d_Plo, 0, pbytes));
      const CUresult r3 = enc(&I->tmap_Plo, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, I->d_Plo, gP, sP, bP, es,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                              CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      I->tmaps_ok = (r1 == CUDA_SUCCESS && r2 == CUDA_SUCCESS && r3 == CUDA_SUCCESS);
    }
  }
  if (state_count == 61) {
    const size_t pbytes = (size_t)matrix_count * I->mat_elems * I->elt;
    CKC(cudaMalloc(&I->d_PT, pbytes));
    CKC(cudaMemset(I->d_PT, 0, pbytes));
  }
  CKC(cudaMallocHost(&I->h_out, sizeof(double)));
  CKC(cudaMalloc(&I->d_flag, sizeof(unsigned)));
  {
    std::vector<double> ones(I->p_pad, 1.0), r((size_t)category_count * eigen_count, 1.0),
        w((size_t)category_count * eigen_count, 1.0 / category_count),
        f((size_t)state_count * eigen_count, 1.0 / state_count);
    CKC(cudaMemcpy(I->d_pw, ones.data(), sizeof(double) * I->p, cudaMemcpyHostToDevice));
    CKC(cudaMemcpy(I->d_rates, r.data(), sizeof(double) * r.size(), cudaMemcpyHostToDevice));
    CKC(cudaMemcpy(I->d_catw, w.data(), sizeof(double) * w.size(), cudaMemcpyHostToDevice));
    CKC(cudaMemcpy(I->d_freqs, f.data(), sizeof(double) * f.size(), cudaMemcpyHostToDevice));
  }
#undef CKC
  std::lock_guard<std::mutex> lk(g_mu);
  g_inst.push_back(I);
  return (int)g_inst.size() - 1;
}

int rrl_finalize_instance(int inst) {
  Instance *I = nullptr;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    if (inst < 0 || inst >= (int)g_inst.size() || !g_inst[inst])
      return fail(RRL_ERROR_UNINITIALIZED_INSTANCE, "no such instance");
    I = g_inst[inst];
    g_inst[inst] = nullptr;
  }
  destroy(I);
  return RRL_SUCCESS;
}

int rrl_set_stream(int inst, void *cuda_stream) {
  GET(I, inst);
  cudaStream_t ns = static_cast<cudaStream_t>(cuda_stream);  // NULL = legacy default stream
  if (ns != I->stream) {
    CK(cudaStreamSynchronize(I->stream));
    I->stream = ns;
  }
  return RRL_SUCCESS;
}

int rrl_synchronize(int inst) {
  GET(I, inst);
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_set_tip_states(int inst, int tip, const int32_t *states) {
  GET(I, inst);
  if (tip < 0 || tip >= I->n_tips) return fail(RRL_ERROR_OUT_OF_RANGE, "tip index");
  if (!states) return fail(RRL_ERROR_GENERAL, "states NULL");
  std::vector<uint8_t> h(I->p);
  for (int i = 0; i < I->p; ++i)
    h[i] = (states[i] < 0 || states[i] >= I->s) ? (uint8_t)I->s : (uint8_t)states[i];
  CK(cudaMemcpyAsync(I->d_states + (size_t)tip * I->p_pad, h.data(), I->p, cudaMemcpyHostToDevice,
                     I->stream));
  CK(cudaStreamSynchronize(I->stream));
  if (!I->has_states[tip]) I->ops_valid = false;  // resolved descriptors name it as partials
  I->has_states[tip] = 1;
  return RRL_SUCCESS;
}

int rrl_set_tip_states_u8(int inst, int first_tip, int count, const uint8_t *states) {
  GET(I, inst);
  if (first_tip < 0 || count < 0 || first_tip + count > I->n_tips)
    return fail(RRL_ERROR_OUT_OF_RANGE, "tip range");
  if (!states) return fail(RRL_ERROR_GENERAL, "states NULL");
  if (count == 0) return RRL_SUCCESS;
  // the rows go straight to the device (one DMA from a pinned caller buffer);
  // the code range (<= s, s = missing) is checked there, not byte by byte on the host
  uint8_t *dst = I->d_states + (size_t)first_tip * I->p_pad;
  CK(cudaMemcpy2DAsync(dst, I->p_pad, states, I->p, I->p, count, cudaMemcpyHostToDevice, I->stream));
  CK(static_cast<cudaError_t>(launch_check_states(dst, (size_t)count * I->p_pad, I->s, I->d_flag, I->stream)));
  CK(cudaMemcpyAsync(I->h_out, I->d_flag, sizeof(unsigned), cudaMemcpyDeviceToHost, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  unsigned bad = 0;
  std::memcpy(&bad, I->h_out, sizeof(unsigned));
  for (int t = first_tip; t < first_tip + count; ++t) {
    if (!I->has_states[t]) I->ops_valid = false;  // resolved descriptors name it as partials
    I->has_states[t] = 1;
  }
  if (bad) {
    // the rows are left as "missing" (all-ones) rather than holding out-of-range codes
    CK(cudaMemset2DAsync(dst, I->p_pad, I->s, I->p, count, I->stream));
    CK(cudaStreamSynchronize(I->stream));
    return fail(RRL_ERROR_OUT_OF_RANGE, "state code > state_count");
  }
  return RRL_SUCCESS;
}

int rrl_set_tip_partials(int inst, int tip, const double *partials) {
  GET(I, inst);
  if (tip < 0 || tip >= I->n_tips) return fail(RRL_ERROR_OUT_OF_RANGE, "tip index");
  if (!partials) return fail(RRL_ERROR_GENERAL, "partials NULL");
  if (!I->tip_partials[tip]) {
    CK(cudaMalloc(&I->tip_partials[tip], I->buf_bytes));
    CK(cudaMemset(I->tip_partials[tip], 0, I->buf_bytes));
  }
  I->has_states[tip] = 0;
  I->ops_valid = false;
  return upload_partials(I, tip, partials, true);
}

int rrl_set_partials(int inst, int buffer, const double *partials) {
  GET(I, inst);
  if (buffer < 0 || buffer >= I->n_buf) return fail(RRL_ERROR_OUT_OF_RANGE, "buffer index");
  if (!partials) return fail(RRL_ERROR_GENERAL, "partials NULL");
  if (buffer < I->n_tips && !I->tip_partials[buffer]) {
    CK(cudaMalloc(&I->tip_partials[buffer], I->buf_bytes));
    CK(cudaMemset(I->tip_partials[buffer], 0, I->buf_bytes));
    I->has_states[buffer] = 0;
    I->ops_valid = false;
  }
  return upload_partials(I, buffer, partials, false);
}

int rrl_get_partials(int inst, int buffer, double *out) {
  GET(I, inst);
  if (buffer < 0 || buffer >= I->n_buf) return fail(RRL_ERROR_OUT_OF_RANGE, "buffer index");
  if (!out) return fail(RRL_ERROR_GENERAL, "out NULL");
  void *src = buffer_ptr(I, buffer);
  if (!src) return fail(RRL_ERROR_GENERAL, "tip buffer holds states, not partials");
  std::vector<char> h(I->buf_bytes);
  CK(cudaMemcpyAsync(h.data(), src, I->buf_bytes, cudaMemcpyDeviceToHost, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  for (int cat = 0; cat < I->c; ++cat)
    for (int pat = 0; pat < I->p; ++pat)
      for (int z = 0; z < I->s; ++z) {
        const size_t k = pidx(I, pat, cat, z);
        out[((size_t)cat * I->p + pat) * I->s + z] =
            I->prec == 32 ? (double)reinterpret_cast<float *>(h.data())[k]
                          : reinterpret_cast<double *>(h.data())[k];
      }
  return RRL_SUCCESS;
}

int rrl_set_pattern_weights(int inst, const double *w) {
  GET(I, inst);
  if (!w) return fail(RRL_ERROR_GENERAL, "weights NULL");
  CK(cudaMemcpyAsync(I->d_pw, w, sizeof(double) * I->p, cudaMemcpyHostToDevice, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_set_state_frequencies(int inst, int idx, const double *pi) {
  GET(I, inst);
  if (idx < 0 || idx >= I->n_eig) return fail(RRL_ERROR_OUT_OF_RANGE, "freqs index");
  if (!pi) return fail(RRL_ERROR_GENERAL, "pi NULL");
  CK(cudaMemcpyAsync(I->d_freqs + (size_t)idx * I->s, pi, sizeof(double) * I->s,
                     cudaMemcpyHostToDevice, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_set_category_rates(int inst, const double *r) {
  GET(I, inst);
  if (!r) return fail(RRL_ERROR_GENERAL, "rates NULL");
  for (int idx = 0; idx < I->n_eig; ++idx)  // every model slot
    CK(cudaMemcpyAsync(I->d_rates + (size_t)idx * I->c, r, sizeof(double) * I->c, cudaMemcpyHostToDevice,
                       I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_set_category_rates_idx(int inst, int idx, const double *r) {
  GET(I, inst);
  if (idx < 0 || idx >= I->n_eig) return fail(RRL_ERROR_OUT_OF_RANGE, "rates index");
  if (!r) return fail(RRL_ERROR_GENERAL, "rates NULL");
  CK(cudaMemcpyAsync(I->d_rates + (size_t)idx * I->c, r, sizeof(double) * I->c, cudaMemcpyHostToDevice,
                     I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_set_category_weights(int inst, int idx, const double *w) {
  GET(I, inst);
  if (idx < 0 || idx >= I->n_eig) return fail(RRL_ERROR_OUT_OF_RANGE, "weights index");
  if (!w) return fail(RRL_ERROR_GENERAL, "weights NULL");
  CK(cudaMemcpyAsync(I->d_catw + (size_t)idx * I->c, w, sizeof(double) * I->c,
                     cudaMemcpyHostToDevice, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_set_eigen_decomposition(int inst, int idx, const double *V, const double *Vinv,
                                const double *lambda) {
  GET(I, inst);
  if (idx < 0 || idx >= I->n_eig) return fail(RRL_ERROR_OUT_OF_RANGE, "eigen index");
  if (!V || !Vinv || !lambda) return fail(RRL_ERROR_GENERAL, "eigen NULL");
  const size_t ss = (size_t)I->s * I->s;
  std::vector<double> h(2 * ss + I->s);
  std::memcpy(h.data(), V, sizeof(double) * ss);
  std::memcpy(h.data() + ss, Vinv, sizeof(double) * ss);
  std::memcpy(h.data() + 2 * ss, lambda, sizeof(double) * I->s);
  CK(cudaMemcpyAsync(I->d_eig + (size_t)idx * h.size(), h.data(), sizeof(double) * h.size(),
                     cudaMemcpyHostToDevice, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_update_transition_matrices(int inst, int eigen_idx, const int32_t *matrix_idx,
                                   const double *t, int count) {
  GET(I, inst);
  if (eigen_idx < 0 || eigen_idx >= I->n_eig) return fail(RRL_ERROR_OUT_OF_RANGE, "eigen index");
  if (count < 0) return fail(RRL_ERROR_GENERAL, "count");
  if (count == 0) return RRL_SUCCESS;
  if (!matrix_idx || !t) return fail(RRL_ERROR_GENERAL, "NULL arrays");
  for (int i = 0; i < count; ++i)
    if (matrix_idx[i] < 0 || matrix_idx[i] >= I->n_mat) return fail(RRL_ERROR_OUT_OF_RANGE, "matrix index");
  if (count > I->t_cap) {
    CK(cudaStreamSynchronize(I->stream));
    if (I->d_t) cudaFree(I->d_t);
    I->d_t = nullptr;
    I->d_midx = nullptr;
    const size_t bytes = (sizeof(double) + sizeof(int32_t)) * (size_t)count;
    CK(cudaMalloc(&I->d_t, bytes));
    I->h_tstage.resize(bytes);
    I->t_count = -1;
    I->d_midx = reinterpret_cast<int32_t *>(I->d_t + count);
    I->t_cap = count;
  }
  // [t | matrix_idx] packed, one H2D copy.  A copy from pageable memory is
  // staged by the driver before cudaMemcpyAsync returns, so neither the
  // caller's arrays nor h_tstage are referenced after return.  The same
  // branch lengths and indices as the previous call are already resident on
  // the device (d_t is written only here): no copy.
  double *ht = reinterpret_cast<double *>(I->h_tstage.data());
  int32_t *hi = reinterpret_cast<int32_t *>(ht + I->t_cap);
  const bool resident = count == I->t_count && std::memcmp(ht, t, sizeof(double) * count) == 0 &&
                        std::memcmp(hi, matrix_idx, sizeof(int32_t) * count) == 0;
  if (!resident) {
    std::memcpy(ht, t, sizeof(double) * count);
    std::memcpy(hi, matrix_idx, sizeof(int32_t) * count);
    CK(cudaMemcpyAsync(I->d_t, ht, (sizeof(double) + sizeof(int32_t)) * (size_t)I->t_cap, cudaMemcpyHostToDevice,
                       I->stream));
    I->t_count = count;
  }
  if ((I->flags & RRL_FLAG_CUDA_GRAPH) && I->stream != nullptr && !I->profiling) {
    // deferred: the next level-set graph replays it as its first node
    I->k1_pending = true;
    I->k1_eig = eigen_idx;
    I->k1_count = count;
    return RRL_SUCCESS;
  }
  return launch_k1(I, eigen_idx, count);
}


int rrl_set_transition_matrix(int inst, int idx, const double *P) {
  GET(I, inst);
  if (idx < 0 || idx >= I->n_mat) return fail(RRL_ERROR_OUT_OF_RANGE, "matrix index");
  if (!P) return fail(RRL_ERROR_GENERAL, "P NULL");
  std::vector<char> h(I->mat_elems * I->elt, 0);
  for (int cat = 0; cat < I->c; ++cat)
    for (int z = 0; z < I->s; ++z)
      for (int x = 0; x < I->s; ++x) {
        const size_t k = ((size_t)cat * I->s_pad + z) * I->s_pad + x;
        const double v = P[((size_t)cat * I->s + z) * I->s + x];
        if (I->prec == 32) reinterpret_cast<float *>(h.data())[k] = (float)v;
        else reinterpret_cast<double *>(h.data())[k] = v;
      }
  CK(cudaMemcpyAsync(I->d_P + (size_t)idx * h.size(), h.data(), h.size(), cudaMemcpyHostToDevice,
                     I->stream));
  if (I->d_Plo)  // keep the 3xTF32 low parts of this matrix in step (device split, like K1's)
    CKL(launch_split_tf32(reinterpret_cast<const float *>(I->d_P + (size_t)idx * h.size()),
                         I->d_Plo + (size_t)idx * I->mat_elems, I->mat_elems, I->stream));
  if (I->d_PT)  // and its transpose for the tip-tip gathers
    CKL(launch_codon_pt(I->prec, I->d_P + (size_t)idx * h.size(), I->d_PT + (size_t)idx * h.size(), I->c,
                        I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_get_transition_matrix(int inst, int idx, double *out) {
  GET(I, inst);
  if (idx < 0 || idx >= I->n_mat) return fail(RRL_ERROR_OUT_OF_RANGE, "matrix index");
  if (!out) return fail(RRL_ERROR_GENERAL, "out NULL");
  std::vector<char> h(I->mat_elems * I->elt);
  CK(cudaMemcpyAsync(h.data(), I->d_P + (size_t)idx * h.size(), h.size(), cudaMemcpyDeviceToHost,
                     I->stream));
  CK(cudaStreamSynchronize(I->stream));
  for (int cat = 0; cat < I->c; ++cat)
    for (int z = 0; z < I->s; ++z)
      for (int x = 0; x < I->s; ++x) {
        const size_t k = ((size_t)cat * I->s_pad + z) * I->s_pad + x;
        out[((size_t)cat * I->s + z) * I->s + x] =
            I->prec == 32 ? (double)reinterpret_cast<float *>(h.data())[k]
                          : reinterpret_cast<double *>(h.data())[k];
      }
  return RRL_SUCCESS;
}

static int update_partials_impl(Instance *I, const rrl_op *ops, const int32_t *ranges, int op_count,
                                const int32_t *set_offsets, int set_count);

int rrl_update_partials(int inst, const rrl_op *ops, int op_count, const int32_t *set_offsets,
                        int set_count) {
  GET_RAW(I, inst);  // a deferred K1 becomes the first node of the level-set graph
  {
    int r = flush_pass(I);  // a previous deferred pass runs first
    if (r < 0) return r;
  }
  return update_partials_impl(I, ops, nullptr, op_count, set_offsets, set_count);
}

int rrl_update_partials_ranged(int inst, const rrl_op *ops, const int32_t *pattern_ranges, int op_count,
                               const int32_t *set_offsets, int set_count) {
  GET(I, inst);
  if (op_count > 0 && !pattern_ranges) return fail(RRL_ERROR_GENERAL, "pattern_ranges NULL");
  for (int i = 0; i < op_count; ++i) {
    const int b = pattern_ranges[2 * i], e = pattern_ranges[2 * i + 1];
    if (b < 0 || e > I->p || b >= e) return fail(RRL_ERROR_OUT_OF_RANGE, "pattern range");
    if (b % RRL_PATTERN_RANGE_ALIGN != 0)
      return fail(RRL_ERROR_GENERAL, "pattern range must start at a multiple of RRL_PATTERN_RANGE_ALIGN");
  }
  return update_partials_impl(I, ops, pattern_ranges, op_count, set_offsets, set_count);
}

static int update_partials_impl(Instance *I, const rrl_op *ops, const int32_t *ranges, int op_count,
                                const int32_t *set_offsets, int set_count) {
  if (op_count < 0 || (op_count > 0 && !ops)) return fail(RRL_ERROR_GENERAL, "ops");
  if (op_count == 0) return RRL_SUCCESS;
  const bool cumulative = (I->flags & RRL_FLAG_SCALE_CUMULATIVE) != 0;

  // --- sets: caller's offsets, or greedy batching in submission order
  std::vector<int32_t> offs;
  if (set_offsets) {
    if (set_count < 1) return fail(RRL_ERROR_GENERAL, "set_count");
    offs.assign(set_offsets, set_offsets + set_count + 1);
    if (offs.front() != 0 || offs.back() != op_count) return fail(RRL_ERROR_GENERAL, "set offsets must span ops");
    for (int k = 0; k < set_count; ++k)
      if (offs[k + 1] <= offs[k]) return fail(RRL_ERROR_GENERAL, "empty or decreasing set");
  } else {
    std::vector<int> stamp(I->n_buf, -1);
    offs.push_back(0);
    int cur = 0;
    for (int i = 0; i < op_count; ++i) {
      const rrl_op &o = ops[i];
      const bool dep = (o.child1 >= 0 && o.child1 < I->n_buf && stamp[o.child1] == cur) ||
                       (o.child2 >= 0 && o.child2 < I->n_buf && stamp[o.child2] == cur) ||
                       (o.dest >= 0 && o.dest < I->n_buf && stamp[o.dest] == cur);
      if (dep && i > offs.back()) {
        offs.push_back(i);
        ++cur;
      }
      if (o.dest >= 0 && o.dest < I->n_buf) stamp[o.dest] = cur;
    }
    offs.push_back(op_count);
  }
  const int nsets = (int)offs.size() - 1;

  std::vector<int32_t> rng;
  if (ranges) rng.assign(ranges, ranges + 2 * op_count);
  const bool same = I->ops_valid && I->last_ops.size() == (size_t)op_count &&
                    I->last_offs == offs && I->last_ranges == rng &&
                    std::memcmp(I->last_ops.data(), ops, sizeof(rrl_op) * op_count) == 0;
  if (!same) {
    // --- validate
    std::vector<int> stamp(I->n_buf, -1);
    // per-node (non-cumulative) exponents are only summed after the call (K5),
    // so two ops of one call writing the same scale buffer would lose the first
    // op's exponents: rejected (recycled buffers need RRL_FLAG_SCALE_CUMULATIVE)
    std::vector<int> scale_writer(cumulative ? 0 : I->n_scale, -1);
    // ranged calls: ops of one set writing the same buffer must cover disjoint
    // pattern ranges (different partitions of one node)
    std::vector<std::vector<std::pair<int, int>>> dest_ranges;
    if (ranges) dest_ranges.resize(I->n_buf);
    for (int k = 0; k < nsets; ++k) {
      for (int i = offs[k]; i < offs[k + 1]; ++i) {
        const rrl_op &o = ops[i];
        if (o.dest < I->n_tips || o.dest >= I->n_buf) return fail(RRL_ERROR_OUT_OF_RANGE, "dest buffer");
        if (o.child1 < 0 || o.child1 >= I->n_buf || o.child2 < 0 || o.child2 >= I->n_buf)
          return fail(RRL_ERROR_OUT_OF_RANGE, "child buffer");
        if (o.matrix1 < 0 || o.matrix1 >= I->n_mat || o.matrix2 < 0 || o.matrix2 >= I->n_mat)
          return fail(RRL_ERROR_OUT_OF_RANGE, "matrix index");
        if (o.dest_scale_write < RRL_NONE || o.dest_scale_write >= I->n_scale ||
            o.dest_scale_read < RRL_NONE || o.dest_scale_read >= I->n_scale)
          return fail(RRL_ERROR_OUT_OF_RANGE, "scale index");
        for (int ch : {o.child1, o.child2})
          if (ch < I->n_tips && !I->has_states[ch] && !I->tip_partials[ch])
            return fail(RRL_ERROR_GENERAL, "tip without data");
        if (stamp[o.dest] == k && !ranges) return fail(RRL_ERROR_GENERAL, "two ops write one buffer in a set");
        if (ranges) {
          auto &dr = dest_ranges[o.dest];
          if (stamp[o.dest] != k) dr.clear();
          const int b = ranges[2 * i], e = ranges[2 * i + 1];
          for (const auto &q : dr)
            if (b < q.second && q.first < e)
              return fail(RRL_ERROR_GENERAL, "two ops of a set write overlapping pattern ranges of one buffer");
          dr.push_back({b, e});
        }
        stamp[o.dest] = k;
        if (!cumulative && o.dest_scale_write >= 0) {
          const int prev = scale_writer[o.dest_scale_write];
          // (partition copies of one node: same dest in the same set, ranges checked disjoint above)
          if (prev >= 0 && !(ranges && ops[prev].dest == o.dest && prev >= offs[k]))
            return fail(RRL_ERROR_GENERAL,
                        "two ops write one scale buffer in one call (per-node exponents would be lost "
                        "before accumulation; use distinct scale buffers or RRL_FLAG_SCALE_CUMULATIVE)");
          scale_writer[o.dest_scale_write] = i;
        }
        if (cumulative && o.dest_scale_write >= 0) {
          if (o.dest_scale_write != o.dest - I->n_tips)
            return fail(RRL_ERROR_GENERAL, "cumulative scaling needs dest_scale_write = dest - tip_count");
          for (int ch : {o.child1, o.child2})
            if (ch >= I->n_tips && ch - I->n_tips >= I->n_scale)
              return fail(RRL_ERROR_OUT_OF_RANGE, "child scale buffer");
        }
      }
      for (int i = offs[k]; i < offs[k + 1]; ++i)
        if (stamp[ops[i].child1] == k || stamp[ops[i].child2] == k)
          return fail(RRL_ERROR_GENERAL, "operation depends on another op of the same set");
    }
    // --- resolve descriptors
    int r = ensure_cap_ops(I, op_count);
    if (r < 0) return r;
    CK(cudaEventSynchronize(I->staging_ev));  // previous upload has consumed the staging
    // 61-state fp32: inside each set (independent ops, any order) the ops whose
    // children are both tips go first; they run as the K3-TT gather kernel
    std::vector<int> perm(op_count);
    for (int i = 0; i < op_count; ++i) perm[i] = i;
    I->set_tt.assign(nsets, 0);
    if (I->s == 61 && I->d_PT) {
      auto tiptip = [&](int i) {
        const rrl_op &o = ops[i];
        return o.child1 < I->n_tips && I->has_states[o.child1] && o.child2 < I->n_tips && I->has_states[o.child2];
      };
      for (int k = 0; k < nsets; ++k) {
        auto b = perm.begin() + offs[k], e = perm.begin() + offs[k + 1];
        auto mid = std::stable_partition(b, e, tiptip);
        I->set_tt[k] = (int)(mid - b);
      }
    }
    for (int pi = 0; pi < op_count; ++pi) {
      const int i = perm[pi];
      const rrl_op &o = ops[i];
      DevOp d{};
      auto child = [&](int b, const void **in, const int32_t **cum, int tipflag) {
        if (b < I->n_tips && I->has_states[b]) {
          *in = I->d_states + (size_t)b * I->p_pad;
          d.flags |= tipflag;
        } else {
          *in = buffer_ptr(I, b);
        }
        *cum = (cumulative && b >= I->n_tips) ? I->d_scale + (size_t)(b - I->n_tips) * I->p_pad : nullptr;
      };
      child(o.child1, &d.in1, &d.cum1, OP_TIP1);
      child(o.child2, &d.in2, &d.cum2, OP_TIP2);
      d.out = buffer_ptr(I, o.dest);
      d.buf1 = (o.child1 >= I->n_tips) ? o.child1 - I->n_tips : -1;
      d.buf2 = (o.child2 >= I->n_tips) ? o.child2 - I->n_tips : -1;
      d.bufd = o.dest - I->n_tips;
      d.mat1 = o.matrix1;
      d.mat2 = o.matrix2;
      d.pat0 = ranges ? ranges[2 * i] : 0;
      d.P1 = I->d_P + (size_t)o.matrix1 * I->mat_elems * I->elt;
      d.P2 = I->d_P + (size_t)o.matrix2 * I->mat_elems * I->elt;
      d.scale_out = o.dest_scale_write >= 0 ? I->d_scale + (size_t)o.dest_scale_write * I->p_pad : nullptr;
      d.scale_in = (o.dest_scale_write < 0 && o.dest_scale_read >= 0)
                       ? I->d_scale + (size_t)o.dest_scale_read * I->p_pad
                       : nullptr;
      if (!d.scale_out) d.cum1 = d.cum2 = nullptr;
      // pattern range: every pointer is advanced to the range's first pattern
      // (the partials' pattern stride is c*s_pad elements for 4 states, s_pad
      // within each category plane for 61 states)
      const int pb = ranges ? ranges[2 * i] : 0;
      d.p = ranges ? ranges[2 * i + 1] - pb : I->p;
      if (pb > 0) {
        const size_t pel = (I->s == 4 ? (size_t)I->c * 4 : (size_t)I->s_pad) * pb * I->elt;
        auto adv = [&](const void *q, bool tip) -> const void * {
          return static_cast<const char *>(q) + (tip ? (size_t)pb : pel);
        };
        d.in1 = adv(d.in1, d.flags & OP_TIP1);
        d.in2 = adv(d.in2, d.flags & OP_TIP2);
        d.out = const_cast<void *>(adv(d.out, false));
        if (d.scale_out) d.scale_out += pb;
        if (d.scale_in) d.scale_in += pb;
        if (d.cum1) d.cum1 += pb;
        if (d.cum2) d.cum2 += pb;
      }
      I->h_ops[pi] = d;
    }
    for (int k = 0; k < nsets; ++k) I->h_ops[offs[k + 1] - 1].flags |= OP_SET_END;
    // fused pass: a child produced by op j is read from the CTA's
    // shared-memory ring (slot = j mod W) if no other op from the start of the
    // producer's set to the end of the consumer's set -- the ops of one set run
    // concurrently -- shares that slot: set_last(i) - set_first(j) < W
    const bool fused_desc = I->s == 4 && (I->flags & RRL_FLAG_FUSED_PASS) && !ranges;
    const int W = fused_ring(I->prec);
    std::vector<int> set_last(fused_desc ? op_count : 0), set_first(fused_desc ? op_count : 0);
    for (int k = 0; k < nsets && fused_desc; ++k)
      for (int i = offs[k]; i < offs[k + 1]; ++i) {
        set_last[i] = offs[k + 1] - 1;
        set_first[i] = offs[k];
      }
    for (int i = 0; i < op_count; ++i) {
      DevOp &d = I->h_ops[i];
      if (!fused_desc) {  // ring slots are read only by the fused-pass kernel
        d.ring1 = d.ring2 = -1;
        continue;
      }
      int32_t *ring[2] = {&d.ring1, &d.ring2};
      const int ch[2] = {ops[i].child1, ops[i].child2};
      const int32_t *cum[2] = {d.cum1, d.cum2};
      for (int b = 0; b < 2; ++b) {
        *ring[b] = -1;
        if (d.flags & (b == 0 ? OP_TIP1 : OP_TIP2)) continue;
        for (int j = i - 1; j >= 0 && j > set_last[i] - W; --j) {
          if (ops[j].dest != ch[b]) continue;
          if (set_last[i] - set_first[j] >= W) break;
          *ring[b] = j % W;
          if (cum[b] != nullptr && I->h_ops[j].scale_out == cum[b]) d.flags |= (b == 0 ? OP_RING_E1 : OP_RING_E2);
          break;
        }
      }
    }
    CK(cudaMemcpyAsync(I->d_ops, I->h_ops, sizeof(DevOp) * op_count, cudaMemcpyHostToDevice, I->stream));
    CK(cudaEventRecord(I->staging_ev, I->stream));
    I->last_ops.assign(ops, ops + op_count);
    I->last_offs = offs;
    I->last_ranges = rng;
    I->ops_valid = true;
    int rg = drop_graphs(I);
    if (rg < 0) return rg;
  }

  const bool fused = I->s == 4 && (I->flags & RRL_FLAG_FUSED_PASS) && !ranges;
  auto launch_all = [&](bool capturing) -> int {
    if (fused) {  // one launch for every set (RRL_FLAG_FUSED_PASS)
      Timed tm(I, 0, !capturing);
      const int e = launch_update_partials_nuc_fused(I->prec, I->c, I->d_ops, op_count, I->p, I->stream);
      if (e != 0) return fail(RRL_ERROR_CUDA, std::string("updatePartials fused launch: ") +
                                                  cudaGetErrorString(static_cast<cudaError_t>(e)));
      return 0;
    }
    for (int k = 0; k < nsets; ++k) {
      const int n = offs[k + 1] - offs[k];
      int pmax = I->p;  // widest pattern range of the set (grids are sized for it)
      if (ranges) {
        pmax = 0;
        for (int i = offs[k]; i < offs[k + 1]; ++i) pmax = std::max(pmax, ranges[2 * i + 1] - ranges[2 * i]);
      }
      Timed tm(I, 0, !capturing);  // eager profiling: one event pair per set launch
      int e;
      if (I->s == 4) {
        // tip states may be read before the PDL wait; the matrices too unless this
        // launch directly follows K1 (k = 0: K1 or a host update may be its predecessor)
        e = launch_update_partials_nuc(I->prec, I->c, I->d_ops + offs[k], I->h_ops + offs[k], n, pmax,
                                       I->p_pad, k > 0 ? 3 : 1, I->stream);
      } else {
        e = 0;
        int o0 = offs[k], nr = n;  // the ops left for the contraction kernels
        const bool tc = I->prec == 32 && !(I->flags & RRL_FLAG_CODON_SIMT);
        const bool simt = (I->flags & RRL_FLAG_CODON_SIMT) != 0;
        if (!simt && I->set_tt[k] > 0) {  // cherries: gathers from P^T, no contraction (K3-TT)
          e = launch_update_partials_codon_tiptip(I->prec, I->c, I->d_ops + o0, I->set_tt[k], pmax, I->p_pad,
                                                  I->d_PT, I->stream);
          o0 += I->set_tt[k];
          nr -= I->set_tt[k];
        }
        if (e == 0 && nr > 0) {
          e = (int)cudaErrorNotSupported;
          if (tc && I->tmaps_ok)  // TMA-fed tcgen05, one CTA per tile (c <= 4)
            e = launch_update_partials_codon_tc5(I->c, I->d_ops + o0, I->h_ops + o0, nr, pmax, I->p_pad,
                                                 &I->tmap_partials, &I->tmap_P, &I->tmap_Plo, I->d_PT, I->stream);
          if (e == (int)cudaErrorNotSupported && tc)
            e = launch_update_partials_codon_tc(I->c, I->d_ops + o0, nr, pmax, I->p_pad, I->stream);
          if (e == (int)cudaErrorNotSupported && I->prec == 64 && !(I->flags & RRL_FLAG_CODON_SIMT))
            e = launch_update_partials_codon_dmma(I->c, I->d_ops + o0, nr, pmax, I->p_pad, I->d_PT, I->stream);
          if (e == (int)cudaErrorNotSupported)
            e = launch_update_partials_codon(I->prec, I->c, I->d_ops + o0, I->h_ops + o0, nr, pmax, I->p_pad,
                                             I->stream);
        }
      }
      if (e == (int)cudaErrorNotSupported) return fail(RRL_ERROR_NO_IMPLEMENTATION, "kernel variant");
      if (e != 0) return fail(RRL_ERROR_CUDA, std::string("updatePartials launch: ") +
                                                  cudaGetErrorString(static_cast<cudaError_t>(e)));
    }
    return 0;
  };
  int kl = 0;
  if (fused) kl = 1;
  else
    for (int k = 0; k < nsets; ++k) {
      const int tt = (I->s == 61 && !(I->flags & RRL_FLAG_CODON_SIMT)) ? I->set_tt[k] : 0;
      const int n = offs[k + 1] - offs[k];
      kl += (tt > 0 ? 1 : 0) + (n - tt > 0 ? (n - tt + 65534) / 65535 : 0);
    }

  // (the legacy default stream cannot be captured: eager launches there)
  const bool use_graph = (I->flags & RRL_FLAG_CUDA_GRAPH) && I->stream != nullptr;
  const bool with_k1 = use_graph && I->k1_pending && !I->profiling;
  if (!with_k1) {
    int r = flush_k1(I);
    if (r < 0) return r;
  }
  if (use_graph) {
    if (I->graph && (I->graph_stream != I->stream || I->graph_has_k1 != with_k1 ||
                     (with_k1 && (I->graph_k1_eig != I->k1_eig || I->graph_k1_count != I->k1_count ||
                                  I->graph_k1_t != I->d_t)))) {
      int r = drop_graphs(I);
      if (r < 0) return r;
    }
    if (!I->graph) {
      cudaGraph_t g;
      CK(cudaStreamBeginCapture(I->stream, cudaStreamCaptureModeThreadLocal));
      int e = 0;
      if (with_k1) {  // K1 as the graph's first node (set 0 already waits for its predecessor)
        e = launch_transition_matrices(I->prec, I->s, I->s_pad, I->c,
                                       I->d_eig + (2 * (size_t)I->s * I->s + I->s) * I->k1_eig,
                                       I->d_rates + (size_t)I->k1_eig * I->c, I->d_midx, I->d_t, I->k1_count,
                                       I->d_P, I->d_Plo, I->d_PT, I->stream);
        if (e != 0) e = fail(RRL_ERROR_CUDA, std::string("K1 capture: ") +
                                                 cudaGetErrorString(static_cast<cudaError_t>(e)));
      }
      if (e == 0) e = launch_all(true);
      cudaError_t ce = cudaStreamEndCapture(I->stream, &g);
      if (e < 0) return e;
      CK(ce);
      cudaError_t ie = cudaGraphInstantiate(&I->graph, g, 0);
      if (ie != cudaSuccess) cudaGraphDestroy(g);
      CK(ie);
      I->graph_tmpl = g;  // kept: the child of the [level sets -> K4] graph
      I->graph_stream = I->stream;
      I->graph_kernels = kl;
      I->graph_has_k1 = with_k1;
      I->graph_k1_eig = with_k1 ? I->k1_eig : -1;
      I->graph_k1_count = with_k1 ? I->k1_count : -1;
      I->graph_k1_t = with_k1 ? I->d_t : nullptr;
    }
    if (with_k1) {  // replayed inside the graph
      I->k1_pending = false;
      I->prof.matrices_launches += (I->k1_count + 65534) / 65535;
      I->prof.kernel_launches += (I->k1_count + 65534) / 65535;
    }
    if (!I->profiling) {
      I->pass_pending = true;  // launched by the next call (with K4 by the device root call)
    } else {
      // profiling: one event pair around the whole replay on the launching
      // stream; per-launch duration = region time / launches (events inside
      // the graph would break the programmatic-dependent-launch overlap).
      Timed tm(I, 0);
      CK(cudaGraphLaunch(I->graph, I->stream));
    }
    I->prof.graph_launches += 1;
  } else {
    int e = launch_all(false);
    if (e < 0) return e;
  }
  I->prof.kernel_launches += kl;
  I->prof.partials_launches += kl;
  return RRL_SUCCESS;
}

int rrl_accumulate_scale_factors(int inst, const int32_t *scale_idx, int count, int cumulative_idx) {
  GET(I, inst);
  if (cumulative_idx < 0 || cumulative_idx >= I->n_scale) return fail(RRL_ERROR_OUT_OF_RANGE, "cumulative index");
  if (count <= 0) return RRL_SUCCESS;
  if (!scale_idx) return fail(RRL_ERROR_GENERAL, "scale_idx NULL");
  for (int i = 0; i < count; ++i)
    if (scale_idx[i] < 0 || scale_idx[i] >= I->n_scale) return fail(RRL_ERROR_OUT_OF_RANGE, "scale index");
  if (count > I->sidx_cap) {
    CK(cudaStreamSynchronize(I->stream));
    if (I->d_sidx) cudaFree(I->d_sidx);
    I->d_sidx = nullptr;
    CK(cudaMalloc(&I->d_sidx, sizeof(int32_t) * count));
    I->sidx_cap = count;
  }
  CK(cudaMemcpyAsync(I->d_sidx, scale_idx, sizeof(int32_t) * count, cudaMemcpyHostToDevice, I->stream));
  {
    Timed tm(I, 3);
    CKL(launch_accumulate_scale(I->d_scale, I->p_pad, I->d_sidx, count,
                                I->d_scale + (size_t)cumulative_idx * I->p_pad, I->p, I->stream));
  }
  I->prof.scale_launches += 1;
  I->prof.kernel_launches += 1;
  return RRL_SUCCESS;
}

int rrl_reset_scale_factors(int inst, int cumulative_idx) {
  GET(I, inst);
  if (cumulative_idx < 0 || cumulative_idx >= I->n_scale) return fail(RRL_ERROR_OUT_OF_RANGE, "cumulative index");
  CK(cudaMemsetAsync(I->d_scale + (size_t)cumulative_idx * I->p_pad, 0, sizeof(int32_t) * I->p_pad,
                     I->stream));
  return RRL_SUCCESS;
}

int rrl_get_scale_factors(int inst, int idx, int32_t *out) {
  GET(I, inst);
  if (idx < 0 || idx >= I->n_scale) return fail(RRL_ERROR_OUT_OF_RANGE, "scale index");
  if (!out) return fail(RRL_ERROR_GENERAL, "out NULL");
  CK(cudaMemcpyAsync(out, I->d_scale + (size_t)idx * I->p_pad, sizeof(int32_t) * I->p,
                     cudaMemcpyDeviceToHost, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

static int root_common(Instance *I, int root_buffer, int cat_weights_idx, int freqs_idx,
                       int cumulative_idx, double *d_out, int pb = 0, int pe = -1) {
  if (pe < 0) pe = I->p;
  if (pb < 0 || pe > I->p || pb >= pe) return fail(RRL_ERROR_OUT_OF_RANGE, "pattern range");
  if (root_buffer < 0 || root_buffer >= I->n_buf) return fail(RRL_ERROR_OUT_OF_RANGE, "root buffer");
  if (cat_weights_idx < 0 || cat_weights_idx >= I->n_eig || freqs_idx < 0 || freqs_idx >= I->n_eig)
    return fail(RRL_ERROR_OUT_OF_RANGE, "weights/freqs index");
  if (cumulative_idx < RRL_NONE || cumulative_idx >= I->n_scale)
    return fail(RRL_ERROR_OUT_OF_RANGE, "cumulative index");
  const void *root = buffer_ptr(I, root_buffer);
  if (!root) return fail(RRL_ERROR_GENERAL, "root buffer has no partials");
  const int32_t *cum = cumulative_idx >= 0 ? I->d_scale + (size_t)cumulative_idx * I->p_pad + pb : nullptr;
  const size_t pel = (I->s == 4 ? (size_t)I->c * 4 : (size_t)I->s_pad) * pb * I->elt;
  const int np = pe - pb;
  const int per_block = I->s == 61 ? 8 : std::max(1, 256 / I->c);  // patterns per K4 block
  const int nb = std::max(1, std::min(I->nblocks, (np + per_block - 1) / per_block));
  {
    Timed tm(I, 2);
    CKL(launch_root_lnl(I->prec, I->s, I->s_pad, I->c, static_cast<const char *>(root) + pel,
                        I->d_catw + (size_t)cat_weights_idx * I->c, I->d_freqs + (size_t)freqs_idx * I->s, cum,
                        I->d_pw + pb, np, I->p_pad, I->d_site + pb, I->d_block, I->d_count, nb, d_out,
                        I->stream));
  }
  I->prof.root_launches += 1;
  I->prof.kernel_launches += 1;
  return RRL_SUCCESS;
}

int rrl_calculate_root_log_likelihoods(int inst, int root_buffer, int cat_weights_idx, int freqs_idx,
                                       int cumulative_idx, double *out_sum) {
  GET(I, inst);
  if (!out_sum) return fail(RRL_ERROR_GENERAL, "out NULL");
  int r = root_common(I, root_buffer, cat_weights_idx, freqs_idx, cumulative_idx, I->d_out);
  if (r < 0) return r;
  CK(cudaMemcpyAsync(I->h_out, I->d_out, sizeof(double), cudaMemcpyDeviceToHost, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  *out_sum = *I->h_out;
  if (!std::isfinite(*out_sum)) return fail(RRL_ERROR_FLOATING_POINT, "non-finite log-likelihood");
  return RRL_SUCCESS;
}

int rrl_calculate_root_log_likelihoods_device(int inst, int root_buffer, int cat_weights_idx,
                                              int freqs_idx, int cumulative_idx, double *d_out) {
  GET_RAW(I, inst);
  if (!d_out) return fail(RRL_ERROR_GENERAL, "d_out NULL");
  if (!I->pass_pending || I->profiling || !I->graph_tmpl) {
    int r = flush_k1(I);
    if (r < 0) return r;
    return root_common(I, root_buffer, cat_weights_idx, freqs_idx, cumulative_idx, d_out);
  }
  // the deferred level-set graph and K4 as one graph
  const int key[4] = {root_buffer, cat_weights_idx, freqs_idx, cumulative_idx};
  if (!I->root_graph || I->root_gen != I->graph_gen || I->root_out != d_out ||
      std::memcmp(key, I->root_key, sizeof(key)) != 0) {
    if (I->root_graph) cudaGraphExecDestroy(I->root_graph);
    I->root_graph = nullptr;
    cudaGraph_t k4g = nullptr;
    CK(cudaStreamBeginCapture(I->stream, cudaStreamCaptureModeThreadLocal));
    const int r = root_common(I, root_buffer, cat_weights_idx, freqs_idx, cumulative_idx, d_out);
    const cudaError_t ce = cudaStreamEndCapture(I->stream, &k4g);
    if (r < 0) {
      if (k4g) cudaGraphDestroy(k4g);
      return r;
    }
    CK(ce);
    cudaGraph_t g = nullptr;
    cudaGraphNode_t pass = nullptr, k4 = nullptr;
    cudaError_t e = cudaGraphCreate(&g, 0);
    if (e == cudaSuccess) e = cudaGraphAddChildGraphNode(&pass, g, nullptr, 0, I->graph_tmpl);
    if (e == cudaSuccess) e = cudaGraphAddChildGraphNode(&k4, g, &pass, 1, k4g);
    if (e == cudaSuccess) e = cudaGraphInstantiate(&I->root_graph, g, 0);
    if (g) cudaGraphDestroy(g);
    cudaGraphDestroy(k4g);
    CK(e);
    I->root_gen = I->graph_gen;
    I->root_out = d_out;
    std::memcpy(I->root_key, key, sizeof(key));
  } else {
    I->prof.root_launches += 1;  // (root_common counted the captured launch)
    I->prof.kernel_launches += 1;
  }
  I->pass_pending = false;
  CK(cudaGraphLaunch(I->root_graph, I->stream));
  return RRL_SUCCESS;
}

int rrl_calculate_edge_log_likelihoods(int inst, int parent_buffer, int child_buffer, int matrix_idx,
                                       int cat_weights_idx, int freqs_idx, int parent_scale_idx,
                                       int child_scale_idx, double *out_sum) {
  GET(I, inst);
  if (!out_sum) return fail(RRL_ERROR_GENERAL, "out NULL");
  if (parent_buffer < 0 || parent_buffer >= I->n_buf || child_buffer < 0 || child_buffer >= I->n_buf)
    return fail(RRL_ERROR_OUT_OF_RANGE, "buffer index");
  if (matrix_idx < 0 || matrix_idx >= I->n_mat) return fail(RRL_ERROR_OUT_OF_RANGE, "matrix index");
  if (cat_weights_idx < 0 || cat_weights_idx >= I->n_eig || freqs_idx < 0 || freqs_idx >= I->n_eig)
    return fail(RRL_ERROR_OUT_OF_RANGE, "weights/freqs index");
  if (parent_scale_idx < RRL_NONE || parent_scale_idx >= I->n_scale || child_scale_idx < RRL_NONE ||
      child_scale_idx >= I->n_scale)
    return fail(RRL_ERROR_OUT_OF_RANGE, "scale index");
  const void *par = buffer_ptr(I, parent_buffer);
  if (!par) return fail(RRL_ERROR_GENERAL, "parent buffer has no partials");
  const bool tip = child_buffer < I->n_tips && I->has_states[child_buffer];
  const void *child = tip ? (const void *)(I->d_states + (size_t)child_buffer * I->p_pad)
                          : buffer_ptr(I, child_buffer);
  if (!child) return fail(RRL_ERROR_GENERAL, "child buffer has no data");
  const int32_t *cp = parent_scale_idx >= 0 ? I->d_scale + (size_t)parent_scale_idx * I->p_pad : nullptr;
  const int32_t *cc = child_scale_idx >= 0 ? I->d_scale + (size_t)child_scale_idx * I->p_pad : nullptr;
  {
    Timed tm(I, 2);
    CKL(launch_edge_lnl(I->prec, I->s, I->s_pad, I->c, par, child, tip ? 1 : 0,
                        I->d_P + (size_t)matrix_idx * I->mat_elems * I->elt,
                        I->d_catw + (size_t)cat_weights_idx * I->c, I->d_freqs + (size_t)freqs_idx * I->s,
                        cp, cc, I->d_pw, I->p, I->p_pad, I->d_site, I->d_block, I->d_count, I->nblocks, I->d_out,
                        I->stream));
  }
  I->prof.root_launches += 1;
  I->prof.kernel_launches += 1;
  CK(cudaMemcpyAsync(I->h_out, I->d_out, sizeof(double), cudaMemcpyDeviceToHost, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  *out_sum = *I->h_out;
  if (!std::isfinite(*out_sum)) return fail(RRL_ERROR_FLOATING_POINT, "non-finite log-likelihood");
  return RRL_SUCCESS;
}

int rrl_calculate_root_log_likelihoods_range(int inst, int root_buffer, int cat_weights_idx, int freqs_idx,
                                             int cumulative_idx, int pattern_begin, int pattern_end,
                                             double *out_sum) {
  GET(I, inst);
  if (!out_sum) return fail(RRL_ERROR_GENERAL, "out NULL");
  int r = root_common(I, root_buffer, cat_weights_idx, freqs_idx, cumulative_idx, I->d_out, pattern_begin,
                      pattern_end);
  if (r < 0) return r;
  CK(cudaMemcpyAsync(I->h_out, I->d_out, sizeof(double), cudaMemcpyDeviceToHost, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  *out_sum = *I->h_out;
  if (!std::isfinite(*out_sum)) return fail(RRL_ERROR_FLOATING_POINT, "non-finite log-likelihood");
  return RRL_SUCCESS;
}

int rrl_get_site_log_likelihoods(int inst, double *out) {
  GET(I, inst);
  if (!out) return fail(RRL_ERROR_GENERAL, "out NULL");
  CK(cudaMemcpyAsync(out, I->d_site, sizeof(double) * I->p, cudaMemcpyDeviceToHost, I->stream));
  CK(cudaStreamSynchronize(I->stream));
  return RRL_SUCCESS;
}

int rrl_set_profiling(int inst, int enable) {
  GET(I, inst);
  I->profiling = enable != 0;
  return RRL_SUCCESS;
}

int rrl_get_profile(int inst, rrl_profile *out) {
  GET(I, inst);
  if (!out) return fail(RRL_ERROR_GENERAL, "out NULL");
  CK(cudaStreamSynchronize(I->stream));
  drain_events(I);
  *out = I->prof;
  return RRL_SUCCESS;
}

int rrl_reset_profile(int inst) {
  GET(I, inst);
  CK(cudaStreamSynchronize(I->stream));
  drain_events(I);
  I->prof = rrl_profile{};
  return RRL_SUCCESS;
}

}  // extern "C"
