/*
 * rrl.h -- C ABI of the rerooted, level-batched phylogenetic partial-likelihood
 * library (B200 / sm_100a).  From-scratch implementation of the data-parallel
 * hot path of Ayres & Cummings, "Rerooting Trees Increases Opportunities for
 * Concurrent Computation ..." (IPDPSW 2018), cited as PAPER.md:<line> §<sec>.
 *
 * Hot path:
 *   reroot (host) -> schedule (host) -> transition matrices (K1)
 *   -> one updatePartials launch per level set (K2 4-state / K3 61-state)
 *   -> scale accumulation (K5, or fused) -> root / edge log-likelihood (K4/K6)
 *   -> [multi-GPU: all-reduce of the fp64 sum, done by the caller through
 *       torch.distributed -- not part of this ABI].
 *
 * ---------------------------------------------------------------------------
 * Conventions (apply to every function below)
 * ---------------------------------------------------------------------------
 * Return value: int.  >= 0 is success (create returns an instance id, the
 *   others 0).  < 0 is one of the RRL_ERROR_* codes.  rrl_error_string(code)
 *   returns static text; rrl_last_error_message() returns a thread-local,
 *   human-readable description of the last failure (e.g. the CUDA error).
 * Ownership: every pointer argument is caller-owned.  Host pointers are read
 *   (or written) only during the call; the library copies inputs and never
 *   retains caller pointers.  Functions whose name ends in _device take a
 *   DEVICE pointer on the instance's device, written asynchronously on the
 *   instance stream.  The instance owns its device memory until
 *   rrl_finalize_instance.  One instance = one CUDA device + one stream.
 *   Calls on one instance are not re-entrant; distinct instances may be used
 *   from distinct threads.
 * Indices: partials buffers 0..tip_count-1 are the tips (PAPER.md:83:
 *   n tips, n-1 internal "subtree operations"); buffers tip_count.. are
 *   internal.  RRL_NONE (-1) means "absent".
 * Layouts (row-major, host side):
 *   transition matrix  P[c][z][x] = Pr(child state x | parent state z, r_c t)
 *                      (Eq. (1) PAPER.md:55 §II-A; reading A2);
 *   partials (get/set) L[c][p][s]  (category, pattern, state);
 *   tip states         uint8/int32 [p], 0..s-1, code s (or any value >= s,
 *                      or < 0) = missing -> all-ones partials (reading A23);
 *   eigensystem        V[s][s], Vinv[s][s], lambda[s] with
 *                      Q = V diag(lambda) Vinv.
 * Device layouts (for readers of DESIGN.md; not part of the ABI):
 *   4-state partials [p][c][4]; 61-state partials [c][p][64] (padded).
 * Precision: 32 or 64 (partials, matrices and kernel arithmetic); transition
 *   matrices are always computed in fp64 and rounded on store; root/edge
 *   integration always accumulates in fp64.
 * Errors: invalid arguments return RRL_ERROR_OUT_OF_RANGE (indices) or
 *   RRL_ERROR_GENERAL without touching state; CUDA failures return
 *   RRL_ERROR_CUDA.  A non-finite log-likelihood returns
 *   RRL_ERROR_FLOATING_POINT with the value still written.
 */
#ifndef RRL_H
#define RRL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define RRL_SUCCESS 0
#define RRL_ERROR_GENERAL (-1)
#define RRL_ERROR_OUT_OF_MEMORY (-2)
#define RRL_ERROR_UNIDENTIFIED_EXCEPTION (-3)
#define RRL_ERROR_UNINITIALIZED_INSTANCE (-4)
#define RRL_ERROR_OUT_OF_RANGE (-5)
#define RRL_ERROR_NO_RESOURCE (-6)
#define RRL_ERROR_NO_IMPLEMENTATION (-7)
#define RRL_ERROR_FLOATING_POINT (-8)
#define RRL_ERROR_INVALID_TREE (-9)
#define RRL_ERROR_CUDA (-10)

#define RRL_NONE (-1)

/* Pattern ranges of rrl_update_partials_ranged start at multiples of this
 * (whole bulk-copy chunks); pad partitions with zero-weight patterns. */
#define RRL_PATTERN_RANGE_ALIGN 512

/* Instance flags (rrl_create_instance). */
#define RRL_FLAG_SCALE_CUMULATIVE 0x1u /* dest scale = own exponent + children's
                                          (child scale buffer = child - tip_count);
                                          no separate accumulation pass needed */
#define RRL_FLAG_CUDA_GRAPH 0x2u       /* capture each distinct operation list's
                                          level-set launches in a CUDA graph and
                                          replay it on later identical calls */
#define RRL_FLAG_CODON_SIMT 0x4u       /* 61 states: use the SIMT kernel (FFMA /
                                          DFMA) instead of the tensor-core one
                                          (tcgen05 3xTF32 for fp32, DMMA for fp64) */
#define RRL_FLAG_FUSED_PASS 0x8u       /* 4 states, no pattern ranges: run a whole
                                          rrl_update_partials call as ONE launch in
                                          which every thread owns the same (pattern,
                                          category) items in every operation and
                                          walks the level sets in order (Eq. (1)
                                          couples only equal patterns).
                                          Beyond the paper's one launch per set
                                          (PAPER.md:116,128); same arithmetic,
                                          bit-identical results. */

/* Schedule flags (rrl_reroot_and_schedule). Low byte = mode. */
#define RRL_SCHED_SEQUENTIAL 1u  /* post-order, one op per set (Fig.2 upper) */
#define RRL_SCHED_LEVEL 2u       /* level sets on the given rooting */
#define RRL_SCHED_REROOT 3u      /* optimal reroot + level sets */
#define RRL_SCHED_REUSE_BUFFERS 0x100u /* liveness-based internal buffer reuse */

/* One subtree operation = Eq. (1) for one internal node (PAPER.md:53-55,
 * Fig. 1):  dest(z) = (sum_x P_matrix1[z][x] child1(x)) *
 *                     (sum_y P_matrix2[z][y] child2(y))
 * for every pattern, category and parent state z.
 * dest_scale_write >= 0: per pattern, m = max over (c, z) of dest; e = the
 *   frexp exponent of m (m = f 2^e, f in [0.5, 1)); dest *= 2^-e (exact);
 *   scale buffer dest_scale_write[p] = e  (plus the children's cumulative
 *   exponents under RRL_FLAG_SCALE_CUMULATIVE)  (reading A5).
 * dest_scale_read >= 0 (and no write): dest *= 2^-scale[dest_scale_read][p]
 *   (reuse of existing factors, the paper's rescale-frequency regime A6).
 * Both RRL_NONE: no rescaling. */
typedef struct rrl_op {
  int32_t dest;
  int32_t dest_scale_write;
  int32_t dest_scale_read;
  int32_t child1;
  int32_t matrix1;
  int32_t child2;
  int32_t matrix2;
} rrl_op;

/* Kernel timing collected when profiling is enabled: CUDA events on the
 * instance stream around every eager launch, or around each CUDA-graph replay
 * of a whole updatePartials call (RRL_FLAG_CUDA_GRAPH), whose time is then
 * attributed to its partials_launches. */
typedef struct rrl_profile {
  double partials_ms;          /* sum of updatePartials set-launch durations */
  int64_t partials_launches;   /* number of updatePartials launches */
  double matrices_ms;          /* K1 */
  int64_t matrices_launches;
  double root_ms;              /* K4/K6 (+ final reduction) */
  int64_t root_launches;
  double scale_ms;             /* K5 */
  int64_t scale_launches;
  int64_t kernel_launches;     /* all kernels launched by this instance
                                  since the last reset (counted always) */
  int64_t graph_launches;      /* CUDA graph replays (each = many kernels) */
} rrl_profile;

const char *rrl_error_string(int code);
const char *rrl_last_error_message(void);
const char *rrl_version(void);

/* ------------------------------------------------------------------ instance
 * Create an instance on CUDA device `device` (PAPER.md:167 --rsrc).
 * tip_count >= 2; partials_buffer_count >= 2*tip_count-1 for a full tree
 *   (fewer when the caller reuses buffers); state_count in {4, 61}
 *   (otherwise RRL_ERROR_NO_IMPLEMENTATION); pattern_count >= 1;
 *   category_count in {1, 2, 4, 8}; precision in {32, 64}.
 * Returns the instance id (>= 0) or an error. */
int rrl_create_instance(int tip_count, int partials_buffer_count, int state_count,
                        int pattern_count, int category_count, int matrix_count,
                        int eigen_count, int scale_buffer_count, int device,
                        int precision, uint32_t flags);
int rrl_finalize_instance(int inst);

/* Enqueue all later work on the caller's CUDA stream (e.g.
 * torch.cuda.current_stream().cuda_stream).  The stream is used as given:
 * NULL is the legacy default stream (RRL_FLAG_CUDA_GRAPH then launches
 * eagerly, since the legacy stream cannot be captured).  Until this is
 * called the instance uses its own non-blocking stream. */
int rrl_set_stream(int inst, void *cuda_stream);
int rrl_synchronize(int inst);

/* --------------------------------------------------------------------- data
 * Tip data (reading A23).  Tip partials are category-independent [p][s]. */
int rrl_set_tip_states(int inst, int tip, const int32_t *states /*[p]*/);
/* Tips first_tip..first_tip+count-1 as uint8 codes (0..s-1, s = missing),
 * rows of p bytes.  One host->device DMA (fast from pinned memory); the code
 * range is validated on the device.  A code > s returns
 * RRL_ERROR_OUT_OF_RANGE and leaves those tips all-missing. */
int rrl_set_tip_states_u8(int inst, int first_tip, int count,
                          const uint8_t *states /*[count][p]*/);
int rrl_set_tip_partials(int inst, int tip, const double *partials /*[p][s]*/);
/* Arbitrary partials for any buffer (tests / restarts), layout [c][p][s]. */
int rrl_set_partials(int inst, int buffer, const double *partials);
int rrl_get_partials(int inst, int buffer, double *out /*[c][p][s]*/);
/* Pattern weights wt_i: the multiplicity of unique site pattern i (PAPER.md:169
 * "--sites ... site patterns", :180 "unique site patterns"; reading A15),
 * applied only in the root/edge sum lnL = sum_i wt_i lnL_i.  Default 1. */
int rrl_set_pattern_weights(int inst, const double *w /*[p]*/);
/* Stationary frequencies pi of model slot idx: the root distribution of the
 * root/edge integration (reading A4; Felsenstein [7]).  Reroot
 * invariance holds only for the stationary pi of a reversible
 * model.  Default uniform. */
int rrl_set_state_frequencies(int inst, int idx, const double *pi /*[s]*/);
/* Rate multipliers r_c of the +Gamma categories (reading A3: P_c =
 * exp(Q r_c t), categories combined only at the root), every model slot. */
int rrl_set_category_rates(int inst, const double *r /*[c]*/);
/* Category weights w_c of model slot idx for the root/edge integration
 * (reading A3/A4).  Default 1/c. */
int rrl_set_category_weights(int inst, int idx, const double *w /*[c]*/);
/* Category rates of model slot idx (0 <= idx < eigen_count) for partitioned
 * analyses ("independent model parameters for each of these
 * different subsets"); rrl_set_category_rates sets every slot.  K1 uses the
 * rates of the slot passed as eigen_idx. */
int rrl_set_category_rates_idx(int inst, int idx, const double *r /*[c]*/);

/* --------------------------------------------------- transition matrices (K1)
 * P_{m,c} = V diag(exp(lambda * r_c * t_m)) Vinv for each listed matrix m and
 * every category c, computed in fp64 on the device.  Eq. (1)'s Pr(x|z,t). */
int rrl_set_eigen_decomposition(int inst, int idx, const double *V, const double *Vinv,
                                const double *lambda);
int rrl_update_transition_matrices(int inst, int eigen_idx, const int32_t *matrix_idx,
                                   const double *t, int count);
int rrl_set_transition_matrix(int inst, int idx, const double *P /*[c][s][s]*/);
int rrl_get_transition_matrix(int inst, int idx, double *out /*[c][s][s]*/);

/* ------------------------------------------------------ updatePartials (K2/K3)
 * Executes `op_count` operations grouped into `set_count` concurrent
 * operation sets: set k = ops[set_offsets[k] .. set_offsets[k+1]).  Each set
 * is ONE kernel launch over (pattern-block x operation) (PAPER.md:116, 128
 * §VI-A "multi-operation kernel"); sets run in order on the instance stream.
 * Operations inside a set must be mutually independent (no op reads another
 * op's dest in the same set): violating sets return RRL_ERROR_GENERAL.
 * set_offsets == NULL: the library batches the ops greedily in submission
 * order, starting a new set whenever an op depends on an op already in the
 * current set. */
int rrl_update_partials(int inst, const rrl_op *ops, int op_count,
                        const int32_t *set_offsets /*[set_count+1] or NULL*/,
                        int set_count);

/* Pattern-partition concurrency (§IV-A, "a multi-operation
 * kernel ... to compute multiple likelihood arrays in a single execution
 * launch, and use pointer arithmetic to allow different input and output
 * arrays for different execution blocks"): like rrl_update_partials, but
 * operation i only covers patterns [pattern_ranges[2i], pattern_ranges[2i+1]).
 * Operations of different partitions (disjoint ranges, each with its own
 * transition matrices) may share a set and a destination buffer, so a level
 * set of every partition runs as ONE launch.  Range starts must be multiples
 * of RRL_PATTERN_RANGE_ALIGN (RRL_ERROR_GENERAL otherwise). */
int rrl_update_partials_ranged(int inst, const rrl_op *ops, const int32_t *pattern_ranges /*[2*op_count]*/,
                               int op_count, const int32_t *set_offsets, int set_count);

/* ------------------------------------------------------------ scaling (K5)
 * cumulative[p] += sum_k scale[scale_idx[k]][p]  (int32, exact). */
int rrl_accumulate_scale_factors(int inst, const int32_t *scale_idx, int count,
                                 int cumulative_idx);
int rrl_reset_scale_factors(int inst, int cumulative_idx);
int rrl_get_scale_factors(int inst, int idx, int32_t *out /*[p]*/);

/* ------------------------------------------------------------- root (K4)
 * lnL_i = ln( sum_c w_c sum_z pi_z L_root[i][c][z] ) + E_i ln 2,
 * *out_sum = sum_i wt_i lnL_i (fp64, deterministic fixed-order reduction).
 * cumulative_idx = RRL_NONE means E = 0.  Blocks until the value is on the
 * host.  The _device variant writes the fp64 sum to `d_out` (device pointer)
 * asynchronously; the per-pattern values stay on the device for
 * rrl_get_site_log_likelihoods. */
int rrl_calculate_root_log_likelihoods(int inst, int root_buffer, int cat_weights_idx,
                                       int freqs_idx, int cumulative_idx, double *out_sum);
int rrl_calculate_root_log_likelihoods_device(int inst, int root_buffer, int cat_weights_idx,
                                              int freqs_idx, int cumulative_idx,
                                              double *d_out);

/* Root log-likelihood of the patterns [pattern_begin, pattern_end) only (one
 * partition of a partitioned analysis; per-pattern values for that range are
 * updated for rrl_get_site_log_likelihoods). */
int rrl_calculate_root_log_likelihoods_range(int inst, int root_buffer, int cat_weights_idx,
                                             int freqs_idx, int cumulative_idx, int pattern_begin,
                                             int pattern_end, double *out_sum);

/* ------------------------------------------------------------- edge (K6)
 * lnL_i = ln( sum_c w_c sum_z pi_z Lp[i][c][z] sum_x P_m[c][z][x] Lc[i][c][x] )
 *         + (Ep_i + Ec_i) ln 2
 * parent_scale_idx / child_scale_idx: cumulative exponents of each side
 * (RRL_NONE = 0).  child_buffer may be a tip. */
int rrl_calculate_edge_log_likelihoods(int inst, int parent_buffer, int child_buffer,
                                       int matrix_idx, int cat_weights_idx, int freqs_idx,
                                       int parent_scale_idx, int child_scale_idx,
                                       double *out_sum);
/* Per-pattern lnL_i of the last root/edge call (reading A4; each
 * pattern's likelihood is computed autonomously and combined afterwards). */
int rrl_get_site_log_likelihoods(int inst, double *out /*[p]*/);

/* ------------------------------------------------------------- profiling
 * The paper's metric is the throughput of the partial-likelihood kernel only
 * (§VI-C, --full-timing PAPER.md:180): these counters time
 * the updatePartials launches separately from K1/K4/K5 (reading A17). */
int rrl_set_profiling(int inst, int enable);
int rrl_get_profile(int inst, rrl_profile *out); /* synchronizes the stream */
int rrl_reset_profile(int inst);

/* ------------------------------------------------ host-only (no instance)
 * Reroot and schedule (readings A7-A11).
 * Input: tip_count n >= 2, parent[2n-1] (root = -1; tips 0..n-1, internal
 * n..2n-2, each internal node with exactly two children), blen[2n-1].
 * Modes: RRL_SCHED_SEQUENTIAL | LEVEL | REROOT, optionally
 * | RRL_SCHED_REUSE_BUFFERS.
 * REROOT picks, in O(n), the unrooted edge minimising the number of level
 * sets (= tree height), ties broken by (keep current root edge, min
 * |tips_left - tips_right|, min edge key; edge key = child id in the input
 * rooting, the root's merged edge = min of its two children), places the new
 * root (reusing the old root id) at the edge midpoint and merges the old
 * root's two branches (t1 + t2).
 * Outputs (caller-allocated):
 *   out_parent[2n-1], out_blen[2n-1]  -- the (re)rooted tree;
 *   out_root_edge                      -- key of the root edge chosen;
 *   out_ops[n-1]                       -- ops, set by set, sorted by dest id,
 *                                         child1 < child2, matrix = child id,
 *                                         dest_scale_write = dest - n;
 *   out_set_offsets[n]                 -- set k = [off[k], off[k+1]);
 *   out_set_count                      -- number of sets (= height);
 *   out_buffer_count                   -- partials buffers needed (2n-1, or
 *                                         fewer with REUSE_BUFFERS, in which
 *                                         case dest/child/scale ids refer to
 *                                         physical buffers and out_parent
 *                                         still uses logical node ids).
 * Any output pointer may be NULL.  Returns RRL_ERROR_INVALID_TREE for a
 * malformed tree. */
int rrl_reroot_and_schedule(int tip_count, const int32_t *parent, const double *blen,
                            uint32_t flags, int32_t *out_parent, double *out_blen,
                            int32_t *out_root_edge, rrl_op *out_ops,
                            int32_t *out_set_offsets, int32_t *out_set_count,
                            int32_t *out_buffer_count);

/* Per-edge objective table used by the reroot (for tests/reporting):
 * for each of the 2n-3 unrooted edges, out_key[e], out_sets[e], out_imbalance[e].
 * Returns the number of edges written. */
int rrl_reroot_edge_table(int tip_count, const int32_t *parent, int32_t *out_key,
                          int32_t *out_sets, int32_t *out_imbalance);

/* Partial-tree update schedule (host; only the part of
 * the tree above a change is recomputed).  nodes[node_count]: the lowest
 * internal nodes whose partials must be recomputed (e.g. parent(v) after the
 * branch above v changed); every ancestor up to the root is added.  Writes
 * the level-batched ops (same conventions as rrl_reroot_and_schedule, current
 * rooting, identity buffers) to out_ops[<= n-1] and out_set_offsets[<= n];
 * out_op_count / out_set_count receive the sizes.  Internal node ids only
 * (RRL_ERROR_OUT_OF_RANGE otherwise). */
int rrl_schedule_partial(int tip_count, const int32_t *parent, const int32_t *nodes, int node_count,
                         rrl_op *out_ops, int32_t *out_set_offsets, int32_t *out_op_count,
                         int32_t *out_set_count);

/* The paper's exhaustive O(n^2) rerooting search in C++, with
 * the same objective and tie-break as rrl_reroot_and_schedule's O(n) DP; for
 * cost comparisons.  blen may be NULL. */
int rrl_reroot_exhaustive(int tip_count, const int32_t *parent, const double *blen,
                          int32_t *out_root_edge, int32_t *out_set_count);

/* Topology moves (host; SURVEY.md NEXT-2, §VII-D "only a subtree
 * representing the modified portion of the overall tree is recomputed for
 * each topology change").  Node ids and the root id are kept; the input tree
 * is not modified; out_parent[2n-1] / out_blen[2n-1] receive the new tree.
 * SPR (reading A26): prune the subtree at prune_node (a non-root node whose
 *   parent p is not the root): p's other child s takes p's place, branch
 *   t_s + t_p; regraft p on the branch above regraft_node (not the root, not
 *   p, not inside the pruned subtree), splitting it in halves.
 *   RRL_ERROR_OUT_OF_RANGE for an illegal pair.
 * NNI (reading A27) on the unrooted internal edge keyed by edge_node (the
 *   branch above it; the root's merged branch is keyed by the root's smaller
 *   child, which must then be internal, as must the other root child):
 *   edge_node's child `which` (0 = smaller id) and the subtree across the
 *   edge (the sibling, or the other root child's smaller child) exchange
 *   places, keeping their branch lengths. */
int rrl_tree_spr(int tip_count, const int32_t *parent, const double *blen, int prune_node,
                 int regraft_node, int32_t *out_parent, double *out_blen);
int rrl_tree_nni(int tip_count, const int32_t *parent, const double *blen, int edge_node, int which,
                 int32_t *out_parent, double *out_blen);

/* Partial update after any change (SURVEY.md NEXT-2; PAPER.md:258, :268,
 * :282-288; reading A28).  The partials buffers (identity assignment: buffer
 * = node id) hold the partials of the stored tree (stored_parent /
 * stored_blen).  For the new tree (parent / blen, same tip set), a node's
 * stored partial is reused iff its children, their branch lengths and,
 * recursively, their subtrees are unchanged; every other internal node is
 * recomputed.  flags = RRL_SCHED_LEVEL: on the new tree's rooting.
 * flags = RRL_SCHED_REROOT: on the rooting (over all 2n-3 edges, O(n)) that
 * minimises the number of sets of this update, then the number of
 * operations (rerooting also recomputes every node whose orientation flips),
 * then keeps the current root edge, then the smallest key; the rerooted tree
 * is built as by rrl_reroot_and_schedule.
 * Outputs: out_parent / out_blen (the tree the ops refer to; use its branch
 * lengths for the transition matrices), out_root_edge, out_ops[<= n-1] (same
 * conventions as rrl_reroot_and_schedule, identity buffers), out_set_offsets
 * [<= n], out_op_count, out_set_count.  Any output may be NULL. */
int rrl_schedule_update(int tip_count, const int32_t *stored_parent, const double *stored_blen,
                        const int32_t *parent, const double *blen, uint32_t flags, int32_t *out_parent,
                        double *out_blen, int32_t *out_root_edge, rrl_op *out_ops,
                        int32_t *out_set_offsets, int32_t *out_op_count, int32_t *out_set_count);

/* Predicted time (microseconds) of one updatePartials pass over `ops` /
 * `set_offsets` (SURVEY.md NEXT-4; PAPER.md:270, :288 cost vs benefit of
 * rerooting): sum over level sets k of
 *   launch_us + (B_k - phi_k C_k) / hbm_gbs,
 * B_k = the set's algorithmic bytes (per pattern: every output c s B + 4,
 * every internal child c s B + 4, every tip child 1), C_k = its reads of
 * children written by set k-1, phi_k = clamp(1 - O_{k-1} / l2_bytes, 0, 1)
 * with O_{k-1} = set k-1's output bytes (the part still in L2).  B = precision
 * / 8.  Used to decide whether rerooting pays (DESIGN.md §9 "NEXT-4"). */
int rrl_schedule_cost(int tip_count, const rrl_op *ops, int op_count, const int32_t *set_offsets,
                      int set_count, int pattern_count, int state_count, int category_count, int precision,
                      double launch_us, double hbm_gbs, double l2_bytes, double *out_us);

/* Substitution model (host, fp64): builds the normalised rate matrix Q
 * (-sum_i pi_i Q_ii = 1) for model in {"jc69","hky","gtr","gy94"} and its
 * eigensystem through the symmetric form S = Pi^1/2 Q Pi^-1/2 (cyclic Jacobi).
 * params: hky {kappa}; gtr {rAC,rAG,rAT,rCG,rCT,rGT}; gy94 {kappa, omega};
 * jc69 none.  pi[s] must be positive.  Outputs (any may be NULL):
 * Q[s][s], V[s][s], Vinv[s][s], lambda[s].  s = 4, or 61 for gy94 (sense
 * codons of the standard code in ACGT order). */
int rrl_model_eigensystem(const char *model, int state_count, const double *pi,
                          const double *params, int param_count, double *Q, double *V,
                          double *Vinv, double *lambda);

#ifdef __cplusplus
}
#endif
#endif /* RRL_H */
