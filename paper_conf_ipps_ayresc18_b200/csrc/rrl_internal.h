// Internal declarations shared by the host C++ and the CUDA kernels.
#pragma once

#include <cstdint>
#include <string>

#include "rrl.h"

namespace rrl {

// Records a thread-local error message and returns `code`.
int fail(int code, const std::string &msg);

// Kernel attributes (dynamic shared-memory opt-in) and SM counts are per
// device context: launchers cache them per device slot (the current device,
// clamped to kMaxDevices - 1), so instances on different GPUs of one process
// each configure their own device.
constexpr int kMaxDevices = 64;
int device_slot();

// Resolved operation descriptor, one per rrl_op, resident in device memory.
// The multi-operation kernel reads its descriptor by blockIdx.y ("pointer
// arithmetic to allow different input and output arrays for different
// execution blocks", §VI-A).
struct DevOp {
  const void *in1;          // child 1: partials, or uint8 tip states
  const void *in2;          // child 2
  void *out;                // dest partials
  const void *P1;           // [c][s][s] transition matrices of branch 1
  const void *P2;           // branch 2
  int32_t *scale_out;       // own (or cumulative) exponent [p], or null
  const int32_t *scale_in;  // existing factors to apply [p], or null
  const int32_t *cum1;      // child 1 cumulative exponent (cumulative mode) or null
  const int32_t *cum2;      // child 2
  int32_t flags;            // bit0: child1 is tip states, bit1: child2 is tip states
  int32_t p;                // patterns of this operation (pointers are pre-offset to its range)
  // tensor-map coordinates for the TMA-fed codon kernel (K3-TC5)
  int32_t buf1, buf2;       // child internal-buffer index in the partials slab, -1 if not in it
  int32_t mat1, mat2;       // transition-matrix indices
  int32_t pat0;             // first pattern of the range
  int32_t bufd;             // dest internal-buffer index in the partials slab
  // fused pass (4 states): ring slot (op index mod fused_ring(prec)) holding the
  // child's partials in shared memory if its producer is one of the previous
  // fused_ring - 1 operations, else -1
  int32_t ring1, ring2;
};
static_assert(sizeof(DevOp) == 112, "DevOp layout");

// Fused-pass ring depth (operations whose outputs each thread keeps in shared memory).
constexpr int fused_ring(int prec) { return prec == 32 ? 8 : 4; }

// OP_SET_END marks the last operation of a level set (read by the fused-pass kernel).
// OP_RING_E1/2: the child's cumulative exponent is in the ring too (its
// producer wrote the scale buffer this op reads as cum1/cum2).
enum : int32_t { OP_TIP1 = 1, OP_TIP2 = 2, OP_SET_END = 4, OP_RING_E1 = 8, OP_RING_E2 = 16 };

// ---------------------------------------------------------------- launchers
// All launchers enqueue on `stream` and return cudaError_t as int.
// d_ops: descriptors in device memory; h_ops: the same descriptors on the host
// (small sets are passed by value in the kernel parameters), may be null.
int launch_update_partials_nuc(int prec, int c, const DevOp *d_ops, const DevOp *h_ops, int nops,
                               int p, int p_pad, int early, void *stream);
// RRL_FLAG_FUSED_PASS: the whole 4-state operation list (sets marked by
// OP_SET_END, no pattern ranges) as one launch.
int launch_update_partials_nuc_fused(int prec, int c, const DevOp *d_ops, int nops, int p, void *stream);
int launch_update_partials_codon(int prec, int c, const DevOp *d_ops, const DevOp *h_ops, int nops,
                                 int p, int p_pad, void *stream);
// tcgen05 (tf32, 3xTF32) codon kernel: fp32, c in {1,2,4,8}; cudaErrorNotSupported otherwise.
int launch_update_partials_codon_tc(int c, const DevOp *d_ops, int nops, int p, int p_pad, void *stream);
// TMA-fed tcgen05 codon kernel: A tiles and P tiles arrive by TMA from the
// partials slab / matrix slab tensor maps (opaque 128-byte CUtensorMap values
// passed as void*), converter warps derive the tf32 lo parts in shared memory.
// cudaErrorNotSupported when a child of the set is not in the slab.
// tf32 low parts lo = rn(x - trunc_tf32(x)) of n fp32 values (the 3xTF32 split of P).
int launch_split_tf32(const float *x, float *lo, size_t n, void *stream);
int launch_update_partials_codon_tc5(int c, const DevOp *d_ops, const DevOp *h_ops, int nops, int p,
                                     int p_pad, const void *tmap_partials, const void *tmap_P,
                                     const void *tmap_Plo, const void *d_PT, void *stream);
// fp64 codon operations on the FP64 tensor cores (mma.sync m8n8k4 f64), c in {1, 2, 4, 8}.
int launch_update_partials_codon_dmma(int c, const DevOp *d_ops, int nops, int p, int p_pad, const void *d_PT,
                                      void *stream);
// *flag = 1 if any of `bytes` (multiple of 16) uint8 tip codes exceeds s, else 0.
int launch_check_states(const uint8_t *d, size_t bytes, int s, unsigned *flag, void *stream);
int launch_transition_matrices(int prec, int s, int s_pad, int c, const double *d_eig,
                               const double *d_rates, const int32_t *d_idx, const double *d_t,
                               int count, void *d_P, void *d_Plo, void *d_PT, void *stream);
// P^T of one codon matrix set [c][64][64] (row 61 = row sums), as K1 writes it.
int launch_codon_pt(int prec, const void *P, void *PT, int c, void *stream);
// 61-state operations whose two children are tips (first level set), fp32 or
// fp64: dest[c][p][z] = P1[c][z][s1] P2[c][z][s2] from the P^T slab, rescaled.
int launch_update_partials_codon_tiptip(int prec, int c, const DevOp *d_ops, int nops, int p, int p_pad,
                                        const void *d_PT, void *stream);
int launch_accumulate_scale(const int32_t *d_scale, int p_pad, const int32_t *d_idx, int count,
                            int32_t *d_cum, int p, void *stream);
int launch_root_lnl(int prec, int s, int s_pad, int c, const void *root, const double *d_w,
                    const double *d_pi, const int32_t *cum, const double *d_pw, int p, int p_pad,
                    double *d_site, double *d_block, unsigned *d_count, int nblocks, double *d_out,
                    void *stream);
int launch_edge_lnl(int prec, int s, int s_pad, int c, const void *par, const void *child,
                    int child_is_tip, const void *P, const double *d_w, const double *d_pi,
                    const int32_t *cum_p, const int32_t *cum_c, const double *d_pw, int p, int p_pad,
                    double *d_site, double *d_block, unsigned *d_count, int nblocks, double *d_out,
                    void *stream);

}  // namespace rrl
