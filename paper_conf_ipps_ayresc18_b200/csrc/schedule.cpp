// Host-side reroot + level-set scheduling (C++, O(n)).
//
// Implements rrl_reroot_and_schedule / rrl_reroot_edge_table of include/rrl.h.
// The paper finds the optimal rooting by exhaustive search over every branch
// (§VI-E, O(n^2)) and notes "a more efficient algorithm could be
// employed" (§VIII).  This file is that algorithm: the number of
// concurrent operation sets of a rooting equals its height (BEAGLE's greedy
// batching of PAPER.md:128 breaks exactly once per dependency level; DESIGN.md
// reading A7), so one down pass (subtree heights) and one up pass (height of
// the complementary component) give the set count of every one of the 2n-3
// candidate root edges in O(n).  Tie-break and rebuild rules: DESIGN.md
// readings A9-A11.
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <queue>
#include <vector>

#include "rrl.h"
#include "rrl_internal.h"

namespace {

struct View {
  int n = 0, N = 0, root = -1;
  std::vector<int> parent, c1, c2;  // c1 < c2, -1 for tips
  std::vector<int> post;            // internal nodes, children before parents
};

int build_view(int n, const int32_t *parent, View &v) {
  if (n < 2 || parent == nullptr) return rrl::fail(RRL_ERROR_INVALID_TREE, "need tip_count >= 2");
  const int N = 2 * n - 1;
  v.n = n;
  v.N = N;
  v.parent.assign(parent, parent + N);
  v.c1.assign(N, -1);
  v.c2.assign(N, -1);
  int roots = 0;
  for (int x = 0; x < N; ++x) {
    const int p = parent[x];
    if (p == -1) {
      ++roots;
      v.root = x;
      continue;
    }
    if (p < 0 || p >= N || p == x || p < n)
      return rrl::fail(RRL_ERROR_INVALID_TREE, "bad parent id");
    if (v.c1[p] < 0) v.c1[p] = x;
    else if (v.c2[p] < 0) v.c2[p] = x;
    else return rrl::fail(RRL_ERROR_INVALID_TREE, "node with more than two children");
  }
  if (roots != 1 || v.root < n) return rrl::fail(RRL_ERROR_INVALID_TREE, "need exactly one internal root");
  for (int x = n; x < N; ++x) {
    if (v.c2[x] < 0) return rrl::fail(RRL_ERROR_INVALID_TREE, "internal node without two children");
    if (v.c1[x] > v.c2[x]) std::swap(v.c1[x], v.c2[x]);
  }
  // iterative post-order: child1 subtree, child2 subtree, node
  v.post.clear();
  v.post.reserve(n - 1);
  std::vector<std::pair<int, bool>> st;
  st.reserve(N);
  st.push_back({v.root, false});
  int visited = 0;
  while (!st.empty()) {
    auto [x, done] = st.back();
    st.pop_back();
    if (x < n) {
      ++visited;
      continue;
    }
    if (done) {
      v.post.push_back(x);
      ++visited;
    } else {
      st.push_back({x, true});
      st.push_back({v.c2[x], false});
      st.push_back({v.c1[x], false});
    }
    if ((int)st.size() > N + 1) return rrl::fail(RRL_ERROR_INVALID_TREE, "cycle");
  }
  if (visited != N) return rrl::fail(RRL_ERROR_INVALID_TREE, "tree is not connected");
  return RRL_SUCCESS;
}

struct EdgeRow {
  int sets, not_current, imbalance, key;
  bool operator<(const EdgeRow &o) const {
    if (sets != o.sets) return sets < o.sets;
    if (not_current != o.not_current) return not_current < o.not_current;
    if (imbalance != o.imbalance) return imbalance < o.imbalance;
    return key < o.key;
  }
};

// All 2n-3 unrooted edges with their set counts (O(n) down/up passes).
std::vector<EdgeRow> edge_table(const View &v) {
  const int n = v.n, N = v.N, R = v.root;
  std::vector<int> down(N, 0), tips(N, 0), up(N, 0);
  for (int x = 0; x < n; ++x) tips[x] = 1;
  for (int x : v.post) {
    down[x] = 1 + std::max(down[v.c1[x]], down[v.c2[x]]);
    tips[x] = tips[v.c1[x]] + tips[v.c2[x]];
  }
  const int a = v.c1[R], b = v.c2[R];
  // up[x] = height of the component on the far side of edge (parent(x), x),
  // rooted at the neighbour of x across that edge (root's edges merged).
  up[a] = down[b];
  up[b] = down[a];
  for (auto it = v.post.rbegin(); it != v.post.rend(); ++it) {  // parents first
    const int u = *it;
    if (u == R) continue;
    const int l = v.c1[u], r = v.c2[u];
    up[l] = 1 + std::max(down[r], up[u]);
    up[r] = 1 + std::max(down[l], up[u]);
  }
  std::vector<EdgeRow> rows;
  rows.reserve(2 * n - 3);
  const int cur = std::min(a, b);
  for (int x = 0; x < N; ++x) {
    if (x == R || x == a || x == b) continue;
    const int other = n - tips[x];
    rows.push_back({1 + std::max(down[x], up[x]), 1, std::abs(tips[x] - other), x});
  }
  rows.push_back({1 + std::max(down[a], down[b]), 0, std::abs(tips[a] - tips[b]), cur});
  std::sort(rows.begin(), rows.end(), [](const EdgeRow &p, const EdgeRow &q) { return p.key < q.key; });
  return rows;
}

// Re-root on the edge keyed `key` (reading A10/A11): path reversal from the
// chosen edge up to the old root; the old root id becomes the new root.
void reroot(const View &v, const double *blen, int key, std::vector<int> &par,
            std::vector<double> &bl) {
  const int R = v.root, a = v.c1[R], b = v.c2[R];
  par = v.parent;
  bl.assign(blen, blen + v.N);
  if (key == std::min(a, b)) return;  // already rooted on this edge: no-op (A9(2), A25)
  const int x0 = key;
  std::vector<int> path;  // x0, x1 = parent(x0), ..., xk = root child
  for (int x = x0; x != R; x = v.parent[x]) path.push_back(x);
  const int k = (int)path.size() - 1;
  const int c = path[k];
  const int d = (c == a) ? b : a;
  const double half = blen[x0] / 2.0;
  par[x0] = R;
  bl[x0] = half;
  par[path[1]] = R;
  bl[path[1]] = half;
  for (int i = 1; i <= k - 1; ++i) {
    par[path[i + 1]] = path[i];
    bl[path[i + 1]] = blen[path[i]];
  }
  par[d] = c;
  bl[d] = blen[a] + blen[b];
  par[R] = -1;
  bl[R] = 0.0;
}

}  // namespace

extern "C" int rrl_reroot_edge_table(int tip_count, const int32_t *parent, int32_t *out_key,
                                     int32_t *out_sets, int32_t *out_imbalance) {
  View v;
  int rc = build_view(tip_count, parent, v);
  if (rc < 0) return rc;
  auto rows = edge_table(v);
  for (size_t i = 0; i < rows.size(); ++i) {
    if (out_key) out_key[i] = rows[i].key;
    if (out_sets) out_sets[i] = rows[i].sets;
    if (out_imbalance) out_imbalance[i] = rows[i].imbalance;
  }
  return (int)rows.size();
}

extern "C" int rrl_reroot_and_schedule(int tip_count, const int32_t *parent, const double *blen,
                                       uint32_t flags, int32_t *out_parent, double *out_blen,
                                       int32_t *out_root_edge, rrl_op *out_ops,
                                       int32_t *out_set_offsets, int32_t *out_set_count,
                                       int32_t *out_buffer_count) {
  try {
    if (blen == nullptr) return rrl::fail(RRL_ERROR_GENERAL, "blen is NULL");
    View v;
    int rc = build_view(tip_count, parent, v);
    if (rc < 0) return rc;
    const int n = v.n, N = v.N;
    const uint32_t mode = flags & 0xffu;
    if (mode != RRL_SCHED_SEQUENTIAL && mode != RRL_SCHED_LEVEL && mode != RRL_SCHED_REROOT)
      return rrl::fail(RRL_ERROR_GENERAL, "unknown schedule mode");
    const bool reuse = (flags & RRL_SCHED_REUSE_BUFFERS) != 0;

    int key = std::min(v.c1[v.root], v.c2[v.root]);
    if (mode == RRL_SCHED_REROOT) {
      auto rows = edge_table(v);
      key = std::min_element(rows.begin(), rows.end())->key;
    }
    std::vector<int> par;
    std::vector<double> bl;
    reroot(v, blen, key, par, bl);
    View w;
    rc = build_view(n, par.data(), w);
    if (rc < 0) return rc;

    // Operation order and set boundaries.
    std::vector<int> order;  // internal node ids in execution order
    std::vector<int> offs;
    order.reserve(n - 1);
    if (mode == RRL_SCHED_SEQUENTIAL) {
      order = w.post;
      for (int i = 0; i <= (int)order.size(); ++i) offs.push_back(i);
    } else {
      std::vector<int> h(N, 0);
      for (int x : w.post) h[x] = 1 + std::max(h[w.c1[x]], h[w.c2[x]]);
      const int H = h[w.root];
      std::vector<int> count(H + 2, 0);
      for (int x = n; x < N; ++x) ++count[h[x]];
      offs.assign(H + 1, 0);
      for (int k = 1; k <= H; ++k) offs[k] = offs[k - 1] + count[k];
      std::vector<int> fill(offs.begin(), offs.end());
      order.assign(n - 1, -1);
      for (int x = n; x < N; ++x) order[fill[h[x] - 1]++] = x;  // ascending ids within a level
    }
    const int nsets = (int)offs.size() - 1;

    // Physical buffer assignment (identity unless reusing).
    std::vector<int> phys(N);
    for (int x = 0; x < N; ++x) phys[x] = x;
    int nbuf = N;
    if (reuse) {
      std::priority_queue<int, std::vector<int>, std::greater<int>> freeq;
      int next = n;
      for (int k = 0; k < nsets; ++k) {
        for (int i = offs[k]; i < offs[k + 1]; ++i) {
          const int x = order[i];
          if (!freeq.empty()) {
            phys[x] = freeq.top();
            freeq.pop();
          } else {
            phys[x] = next++;
          }
        }
        for (int i = offs[k]; i < offs[k + 1]; ++i) {
          const int x = order[i];
          if (w.c1[x] >= n) freeq.push(phys[w.c1[x]]);
          if (w.c2[x] >= n) freeq.push(phys[w.c2[x]]);
        }
      }
      nbuf = next;
    }

    if (out_parent) std::copy(par.begin(), par.end(), out_parent);
    if (out_blen) std::copy(bl.begin(), bl.end(), out_blen);
    if (out_root_edge) *out_root_edge = key;
    if (out_ops) {
      for (int i = 0; i < n - 1; ++i) {
        const int x = order[i];
        const int l = w.c1[x], r = w.c2[x];
        out_ops[i] = rrl_op{phys[x], phys[x] - n, RRL_NONE, phys[l], l, phys[r], r};
      }
    }
    if (out_set_offsets) std::copy(offs.begin(), offs.end(), out_set_offsets);
    if (out_set_count) *out_set_count = nsets;
    if (out_buffer_count) *out_buffer_count = nbuf;
    return RRL_SUCCESS;
  } catch (...) {
    return rrl::fail(RRL_ERROR_UNIDENTIFIED_EXCEPTION, "exception in rrl_reroot_and_schedule");
  }
}

// ---------------------------------------------------------------------------
// Partial-tree updates (§VII-D, §VIII:
// "phylogenetic analysis programs only calculate those subtree partial
// likelihoods as required for a topology change").  The caller names the
// lowest internal nodes whose partials must be recomputed (e.g. parent(v)
// after v's branch length changed); the library adds every ancestor up to the
// root and level-batches exactly those operations on the current rooting:
// level(v) = 1 + max level of v's children that are recomputed (1 if none).
extern "C" int rrl_schedule_partial(int tip_count, const int32_t *parent, const int32_t *nodes,
                                    int node_count, rrl_op *out_ops, int32_t *out_set_offsets,
                                    int32_t *out_op_count, int32_t *out_set_count) {
  try {
    View v;
    int rc = build_view(tip_count, parent, v);
    if (rc < 0) return rc;
    const int n = v.n, N = v.N;
    if (node_count < 0 || (node_count > 0 && !nodes)) return rrl::fail(RRL_ERROR_GENERAL, "nodes");
    std::vector<char> mark(N, 0);
    for (int i = 0; i < node_count; ++i) {
      int x = nodes[i];
      if (x < n || x >= N) return rrl::fail(RRL_ERROR_OUT_OF_RANGE, "partial-update node must be internal");
      while (x >= 0 && !mark[x]) {
        mark[x] = 1;
        x = v.parent[x];
      }
    }
    std::vector<int> lev(N, 0);
    int H = 0, cnt = 0;
    for (int x : v.post)
      if (mark[x]) {
        int l = 0;
        if (mark[v.c1[x]]) l = lev[v.c1[x]];
        if (mark[v.c2[x]]) l = std::max(l, lev[v.c2[x]]);
        lev[x] = l + 1;
        H = std::max(H, lev[x]);
        ++cnt;
      }
    std::vector<int> count(H + 2, 0), offs(H + 1, 0);
    for (int x = n; x < N; ++x)
      if (mark[x]) ++count[lev[x]];
    for (int k = 1; k <= H; ++k) offs[k] = offs[k - 1] + count[k];
    std::vector<int> fill(offs.begin(), offs.end()), order(cnt);
    for (int x = n; x < N; ++x)
      if (mark[x]) order[fill[lev[x] - 1]++] = x;
    if (out_ops)
      for (int i = 0; i < cnt; ++i) {
        const int x = order[i];
        out_ops[i] = rrl_op{x, x - n, RRL_NONE, v.c1[x], v.c1[x], v.c2[x], v.c2[x]};
      }
    if (out_set_offsets) std::copy(offs.begin(), offs.end(), out_set_offsets);
    if (out_op_count) *out_op_count = cnt;
    if (out_set_count) *out_set_count = H;
    return RRL_SUCCESS;
  } catch (...) {
    return rrl::fail(RRL_ERROR_UNIDENTIFIED_EXCEPTION, "exception in rrl_schedule_partial");
  }
}

// ---------------------------------------------------------------------------
// The paper's own search (§VI-E), in C++ for the cost comparison
// of SURVEY.md NEXT-4: for every one of the 2n-3 edges, rebuild the rooted
// tree there (path reversal) and measure its height; O(n^2).  Same tie-break
// as the O(n) DP (reading A9); returns the chosen edge key, writes its set
// count.
extern "C" int rrl_reroot_exhaustive(int tip_count, const int32_t *parent, const double *blen,
                                     int32_t *out_root_edge, int32_t *out_set_count) {
  try {
    View v;
    int rc = build_view(tip_count, parent, v);
    if (rc < 0) return rc;
    const int n = v.n, N = v.N, R = v.root, a = v.c1[R], b = v.c2[R];
    std::vector<double> zero;
    if (!blen) zero.assign(N, 0.0);
    const double *bl = blen ? blen : zero.data();
    const int cur = std::min(a, b);
    EdgeRow best{1 << 30, 1, 1 << 30, 1 << 30};
    std::vector<int> par;
    std::vector<double> nb;
    std::vector<int> h(N), tips(N);
    for (int key = 0; key < N; ++key) {
      if (key == R || key == std::max(a, b)) continue;  // the merged root edge is keyed by min(a, b)
      reroot(v, bl, key, par, nb);
      View w;
      rc = build_view(n, par.data(), w);
      if (rc < 0) return rc;
      std::fill(h.begin(), h.end(), 0);
      std::fill(tips.begin(), tips.begin() + n, 1);
      for (int x : w.post) {
        h[x] = 1 + std::max(h[w.c1[x]], h[w.c2[x]]);
        tips[x] = tips[w.c1[x]] + tips[w.c2[x]];
      }
      const EdgeRow row{h[w.root], key == cur ? 0 : 1, std::abs(tips[w.c1[w.root]] - tips[w.c2[w.root]]), key};
      if (row < best) best = row;
    }
    if (out_root_edge) *out_root_edge = best.key;
    if (out_set_count) *out_set_count = best.sets;
    return RRL_SUCCESS;
  } catch (...) {
    return rrl::fail(RRL_ERROR_UNIDENTIFIED_EXCEPTION, "exception in rrl_reroot_exhaustive");
  }
}

// ---------------------------------------------------------------------------
// Topology moves (§VII-D "only a subtree
// representing the modified portion of the overall tree is recomputed for each
// topology change").  The paper does not define the moves: DESIGN.md readings
// A26 (SPR) and A27 (NNI).  Node ids and the root are kept.
extern "C" int rrl_tree_spr(int tip_count, const int32_t *parent, const double *blen, int prune_node,
                            int regraft_node, int32_t *out_parent, double *out_blen) {
  try {
    if (!blen || !out_parent || !out_blen) return rrl::fail(RRL_ERROR_GENERAL, "NULL array");
    View v;
    int rc = build_view(tip_count, parent, v);
    if (rc < 0) return rc;
    const int N = v.N, R = v.root, x = prune_node, r = regraft_node;
    if (x < 0 || x >= N || x == R) return rrl::fail(RRL_ERROR_OUT_OF_RANGE, "prune node must be a non-root node");
    const int p = v.parent[x];
    if (p == R) return rrl::fail(RRL_ERROR_OUT_OF_RANGE, "prune node's parent must not be the root");
    if (r < 0 || r >= N || r == R || r == p) return rrl::fail(RRL_ERROR_OUT_OF_RANGE, "bad regraft node");
    for (int y = r; y != -1; y = v.parent[y])
      if (y == x) return rrl::fail(RRL_ERROR_OUT_OF_RANGE, "regraft node inside the pruned subtree");
    std::vector<int32_t> par(v.parent.begin(), v.parent.end());
    std::vector<double> bl(blen, blen + N);
    const int g = v.parent[p];
    const int s = (v.c1[p] == x) ? v.c2[p] : v.c1[p];
    par[s] = g;  // prune: the sibling takes p's place, branches merge
    bl[s] = bl[s] + bl[p];
    const int q = par[r];  // regraft: p on the branch above r, split in halves
    const double half = bl[r] / 2.0;
    par[p] = q;
    bl[p] = half;
    par[r] = p;
    bl[r] = half;
    std::copy(par.begin(), par.end(), out_parent);
    std::copy(bl.begin(), bl.end(), out_blen);
    return RRL_SUCCESS;
  } catch (...) {
    return rrl::fail(RRL_ERROR_UNIDENTIFIED_EXCEPTION, "exception in rrl_tree_spr");
  }
}

extern "C" int rrl_tree_nni(int tip_count, const int32_t *parent, const double *blen, int edge_node, int which,
                            int32_t *out_parent, double *out_blen) {
  try {
    if (!blen || !out_parent || !out_blen) return rrl::fail(RRL_ERROR_GENERAL, "NULL array");
    View v;
    int rc = build_view(tip_count, parent, v);
    if (rc < 0) return rc;
    const int n = v.n, N = v.N, R = v.root, x = edge_node;
    if (x < n || x >= N || x == R || (which != 0 && which != 1))
      return rrl::fail(RRL_ERROR_OUT_OF_RANGE, "NNI needs an internal non-root node and which in {0, 1}");
    std::vector<int32_t> par(v.parent.begin(), v.parent.end());
    const int u = v.parent[x];
    const int mine = which == 0 ? v.c1[x] : v.c2[x];
    if (u == R) {
      const int a = v.c1[R], b = v.c2[R];
      if (x != a) return rrl::fail(RRL_ERROR_OUT_OF_RANGE, "the root's merged edge is keyed by its smaller child");
      if (b < n) return rrl::fail(RRL_ERROR_OUT_OF_RANGE, "merged root edge is not internal");
      const int theirs = v.c1[b];
      par[mine] = b;
      par[theirs] = x;
    } else {
      const int w = (v.c1[u] == x) ? v.c2[u] : v.c1[u];
      par[mine] = u;
      par[w] = x;
    }
    std::copy(par.begin(), par.end(), out_parent);
    std::copy(blen, blen + N, out_blen);
    return RRL_SUCCESS;
  } catch (...) {
    return rrl::fail(RRL_ERROR_UNIDENTIFIED_EXCEPTION, "exception in rrl_tree_nni");
  }
}

// ---------------------------------------------------------------------------
// Partial update after any change (moves, branch lengths), optionally
// rerooted (reading A28).
// A node's stored partial (identity buffers) is reused iff its children, their
// branch lengths and, recursively, their subtrees equal the stored tree's: one
// O(n) pass.  Rerooting on the edge above x flips every node strictly between
// x and the root (x_1..x_k: their children change) and the root itself; all
// other nodes keep their rooted subtree.  So for every candidate edge the
// update's set count is 1 + max(dirty height below x, dirty height of the
// flipped side), computed for all 2n-3 edges by the same down/up passes as the
// full reroot (edge_table), with the flipped side always recomputed, and its
// operation count is |D| + (valid nodes among x_1..x_k) + (root valid).
extern "C" int rrl_schedule_update(int tip_count, const int32_t *stored_parent, const double *stored_blen,
                                   const int32_t *parent, const double *blen, uint32_t flags,
                                   int32_t *out_parent, double *out_blen, int32_t *out_root_edge,
                                   rrl_op *out_ops, int32_t *out_set_offsets, int32_t *out_op_count,
                                   int32_t *out_set_count) {
  try {
    if (!stored_blen || !blen) return rrl::fail(RRL_ERROR_GENERAL, "blen is NULL");
    const uint32_t mode = flags & 0xffu;
    if (mode != RRL_SCHED_LEVEL && mode != RRL_SCHED_REROOT)
      return rrl::fail(RRL_ERROR_GENERAL, "rrl_schedule_update: mode must be LEVEL or REROOT");
    View s, v;
    int rc = build_view(tip_count, stored_parent, s);
    if (rc < 0) return rc;
    rc = build_view(tip_count, parent, v);
    if (rc < 0) return rc;
    const int n = v.n, N = v.N, R = v.root, a = v.c1[R], b = v.c2[R];
    std::vector<char> valid(N, 1);
    std::vector<int> down(N, 0);
    int ndirty = 0;
    for (int x : v.post) {
      const int l = v.c1[x], r = v.c2[x];
      valid[x] = (s.c1[x] == l && s.c2[x] == r && stored_blen[l] == blen[l] && stored_blen[r] == blen[r] &&
                  valid[l] && valid[r]);
      if (!valid[x]) {
        down[x] = 1 + std::max(down[l], down[r]);
        ++ndirty;
      }
    }
    const int cur = std::min(a, b);
    int key = cur, best_sets = down[R];
    if (mode == RRL_SCHED_REROOT && ndirty > 0) {
      std::vector<int> up(N, 0), cnt(N, 0);
      up[a] = down[b];
      up[b] = down[a];
      for (auto it = v.post.rbegin(); it != v.post.rend(); ++it) {  // parents first
        const int u = *it;
        if (u == R) continue;
        const int l = v.c1[u], r = v.c2[u];
        up[l] = 1 + std::max(down[r], up[u]);
        up[r] = 1 + std::max(down[l], up[u]);
        cnt[l] = cnt[r] = cnt[u] + (valid[u] ? 1 : 0);
      }
      // (sets, ops, not current, key), reading A28
      long long best[4] = {down[R], ndirty, 0, cur};
      for (int x = 0; x < N; ++x) {
        if (x == R || x == a || x == b) continue;
        const long long row[4] = {1 + std::max(down[x], up[x]), ndirty + cnt[x] + (valid[R] ? 1 : 0), 1, x};
        if (std::lexicographical_compare(row, row + 4, best, best + 4)) std::copy(row, row + 4, best);
      }
      key = (int)best[3];
      best_sets = (int)best[0];
    }
    std::vector<int> par;
    std::vector<double> bl;
    reroot(v, blen, key, par, bl);
    View w;
    rc = build_view(n, par.data(), w);
    if (rc < 0) return rc;
    std::vector<char> dirty(N, 0);
    for (int x = n; x < N; ++x) dirty[x] = !valid[x];
    if (key != cur) {
      dirty[R] = 1;
      for (int y = v.parent[key]; y != R; y = v.parent[y]) dirty[y] = 1;
    }
    std::vector<int> lev(N, 0);
    int H = 0, cnt_ops = 0;
    for (int x : w.post)
      if (dirty[x]) {
        lev[x] = 1 + std::max(dirty[w.c1[x]] ? lev[w.c1[x]] : 0, dirty[w.c2[x]] ? lev[w.c2[x]] : 0);
        H = std::max(H, lev[x]);
        ++cnt_ops;
      }
    if (H != best_sets) return rrl::fail(RRL_ERROR_GENERAL, "internal: update set count mismatch");
    std::vector<int> count(H + 2, 0), offs(H + 1, 0);
    for (int x = n; x < N; ++x)
      if (dirty[x]) ++count[lev[x]];
    for (int k = 1; k <= H; ++k) offs[k] = offs[k - 1] + count[k];
    std::vector<int> fill(offs.begin(), offs.end()), order(cnt_ops);
    for (int x = n; x < N; ++x)
      if (dirty[x]) order[fill[lev[x] - 1]++] = x;
    if (out_parent) std::copy(par.begin(), par.end(), out_parent);
    if (out_blen) std::copy(bl.begin(), bl.end(), out_blen);
    if (out_root_edge) *out_root_edge = key;
    if (out_ops)
      for (int i = 0; i < cnt_ops; ++i) {
        const int x = order[i];
        out_ops[i] = rrl_op{x, x - n, RRL_NONE, w.c1[x], w.c1[x], w.c2[x], w.c2[x]};
      }
    if (out_set_offsets) std::copy(offs.begin(), offs.end(), out_set_offsets);
    if (out_op_count) *out_op_count = cnt_ops;
    if (out_set_count) *out_set_count = H;
    return RRL_SUCCESS;
  } catch (...) {
    return rrl::fail(RRL_ERROR_UNIDENTIFIED_EXCEPTION, "exception in rrl_schedule_update");
  }
}

// ---------------------------------------------------------------------------
// Schedule cost model ("the desired
// outcome is that the benefit gained by the increased concurrent computation
// on the rerooted tree is greater than the cost").  Per level set k:
//   T_k = t0 + (B_k - phi_k C_k) / BW,
// B_k = algorithmic bytes of the set (every op: output c s B + 4 B exponent;
// each internal child c s B + 4 B cumulative exponent, each tip child 1 B, per
// pattern), C_k = the part of it that reads children written by set k-1, and
// phi_k = clamp(1 - O_{k-1} / L2, 0, 1) the fraction of set k-1's output
// O_{k-1} still in L2.  t0 is the fixed cost of a level-set launch.  Fitted
// against the measured 1,024-pectinate sweep (DESIGN.md §9 "NEXT-4"): it
// predicts rerooting to win up to ~10^5 patterns and to lose at 10^6 (fp32),
// where a one-op chain re-reads its child from L2.
extern "C" int rrl_schedule_cost(int tip_count, const rrl_op *ops, int op_count, const int32_t *set_offsets,
                                 int set_count, int pattern_count, int state_count, int category_count,
                                 int precision, double launch_us, double hbm_gbs, double l2_bytes,
                                 double *out_us) {
  try {
    if (!ops || !set_offsets || !out_us || set_count < 0 || op_count < 0 || tip_count < 2 || pattern_count < 0 ||
        (precision != 32 && precision != 64) || hbm_gbs <= 0.0 || l2_bytes < 0.0)
      return rrl::fail(RRL_ERROR_GENERAL, "rrl_schedule_cost: bad arguments");
    if (set_offsets[0] != 0 || set_offsets[set_count] != op_count)
      return rrl::fail(RRL_ERROR_GENERAL, "rrl_schedule_cost: set offsets must span ops");
    const double p = pattern_count;
    const double vec = (double)category_count * state_count * (precision / 8);
    const double out_b = (vec + 4.0) * p, int_b = (vec + 4.0) * p, tip_b = 1.0 * p;
    int maxbuf = tip_count;
    for (int i = 0; i < op_count; ++i) maxbuf = std::max({maxbuf, ops[i].dest + 1, ops[i].child1 + 1, ops[i].child2 + 1});
    std::vector<int> written_in(maxbuf, -2);
    double total = 0.0, prev_out = 0.0;
    for (int k = 0; k < set_count; ++k) {
      double B = 0.0, Cprev = 0.0, O = 0.0;
      for (int i = set_offsets[k]; i < set_offsets[k + 1]; ++i) {
        const rrl_op &o = ops[i];
        for (int ch : {o.child1, o.child2}) {
          if (ch < tip_count) {
            B += tip_b;
          } else {
            B += int_b;
            if (written_in[ch] == k - 1) Cprev += int_b;
          }
        }
        B += out_b;
        O += out_b;
      }
      const double phi = l2_bytes > 0.0 ? std::min(1.0, std::max(0.0, 1.0 - prev_out / l2_bytes)) : 0.0;
      total += launch_us + (B - phi * Cprev) / (hbm_gbs * 1e3);  // bytes / (GB/s) -> us
      for (int i = set_offsets[k]; i < set_offsets[k + 1]; ++i) written_in[ops[i].dest] = k;
      prev_out = O;
    }
    *out_us = total;
    return RRL_SUCCESS;
  } catch (...) {
    return rrl::fail(RRL_ERROR_UNIDENTIFIED_EXCEPTION, "exception in rrl_schedule_cost");
  }
}
