// reorder.cpp -- Graph Clustering based Reordering (GCR, Fig. 8),
// host side (BASELINE.json: "optional host-side graph-clustering reorder").
//
// The paper runs a GPU Louvain (refs [29][30]) and converts the graph to a
// "reordered hybrid CSR/COO format according to the clustering result".  It gives no
// parameters; our reading (DESIGN.md §2 item 23):
//   * Louvain on the symmetric graph, self-loops ignored at the first level, resolution
//     1.0, nodes visited in id order, moves to the neighbouring community of largest
//     modularity gain (ties: smaller community id), a level stops when a pass improves
//     modularity by less than min_gain or after max_passes; up to max_levels levels of
//     aggregation;
//   * the new order groups nodes hierarchically: top-level communities ordered by their
//     smallest original member id, then the sub-communities of the level below the same
//     way, ..., then original id.  perm[old] = new.
// Then S' = P S P^T (gnn_permute_graph), X' = P X (gnn_permute_rows, device).
#include <math.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <new>
#include <vector>

#include "internal.cuh"

namespace gnn {
namespace {

struct LevelGraph {  // symmetric weighted graph in CSR (both directions stored)
  int64_t n = 0;
  std::vector<int64_t> ptr;
  std::vector<int32_t> adj;
  std::vector<double> w;  // empty = all weights 1
};

// One level of Louvain local moving.  Returns the community of every node (renumbered
// 0..nc-1 by first appearance) and the modularity of the final partition.
struct LevelResult {
  std::vector<int32_t> comm;
  int32_t nc = 0;
  double q = 0.0;
  bool moved = false;
};

LevelResult local_moving(const int32_t *ptr32, const int64_t *ptr64, const int32_t *adj,
                         const double *w, int64_t n, bool skip_self, double res, int max_passes,
                         double min_gain) {
  auto row_b = [&](int64_t i) -> int64_t { return ptr32 ? (int64_t)ptr32[i] - ptr32[0] : ptr64[i]; };
  auto row_e = [&](int64_t i) -> int64_t {
    return ptr32 ? (int64_t)ptr32[i + 1] - ptr32[0] : ptr64[i + 1];
  };
  std::vector<double> k(n, 0.0), self(n, 0.0);
  double m2 = 0.0;
  for (int64_t i = 0; i < n; ++i) {
    double s = 0.0;
    for (int64_t e = row_b(i); e < row_e(i); ++e) {
      const int32_t j = adj[e];
      const double we = w ? w[e] : 1.0;
      if (j == i) {
        if (skip_self) continue;
        self[i] += we;
      }
      s += we;
    }
    k[i] = s;
    m2 += s;
  }
  LevelResult r;
  r.comm.resize(n);
  for (int64_t i = 0; i < n; ++i) r.comm[i] = (int32_t)i;
  if (m2 <= 0.0) {
    r.nc = (int32_t)n;
    return r;
  }
  std::vector<double> tot(k), in(self);  // per community
  std::vector<double> nw(n, -1.0);       // weight from the current node to community c
  std::vector<int32_t> touched;
  touched.reserve(1024);
  auto modularity = [&]() {
    double q = 0.0;
    for (int64_t c = 0; c < n; ++c)
      if (tot[c] > 0) q += in[c] / m2 - res * (tot[c] / m2) * (tot[c] / m2);
    return q;
  };
  double q = modularity();
  for (int pass = 0; pass < max_passes; ++pass) {
    bool any = false;
    for (int64_t i = 0; i < n; ++i) {
      const int32_t ci = r.comm[i];
      touched.clear();
      nw[ci] = 0.0;
      touched.push_back(ci);
      for (int64_t e = row_b(i); e < row_e(i); ++e) {
        const int32_t j = adj[e];
        if (j == i) continue;
        const double we = w ? w[e] : 1.0;
        const int32_t cj = r.comm[j];
        if (nw[cj] < 0.0) {
          nw[cj] = 0.0;
          touched.push_back(cj);
        }
        nw[cj] += we;
      }
      // remove i from its community
      tot[ci] -= k[i];
      in[ci] -= 2.0 * nw[ci] + self[i];
      // best community: gain = k_i,in(c) - res * tot_c * k_i / m2
      int32_t best = ci;
      double best_gain = nw[ci] - res * tot[ci] * k[i] / m2;
      for (int32_t c : touched) {
        const double gain = nw[c] - res * tot[c] * k[i] / m2;
        if (gain > best_gain || (gain == best_gain && c < best)) {
          best = c;
          best_gain = gain;
        }
      }
      tot[best] += k[i];
      in[best] += 2.0 * nw[best] + self[i];
      if (best != ci) {
        r.comm[i] = best;
        any = true;
        r.moved = true;
      }
      for (int32_t c : touched) nw[c] = -1.0;
    }
    const double q2 = modularity();
    const double gain = q2 - q;
    q = q2;
    if (!any || gain < min_gain) break;
  }
  // renumber by first appearance
  std::vector<int32_t> ren(n, -1);
  int32_t nc = 0;
  for (int64_t i = 0; i < n; ++i) {
    int32_t &x = ren[r.comm[i]];
    if (x < 0) x = nc++;
    r.comm[i] = x;
  }
  r.nc = nc;
  r.q = q;
  return r;
}

// Aggregate: community graph with summed weights (self entries = internal weight).
LevelGraph aggregate(const int32_t *ptr32, const int64_t *ptr64, const int32_t *adj,
                     const double *w, int64_t n, bool skip_self, const std::vector<int32_t> &comm,
                     int32_t nc) {
  auto row_b = [&](int64_t i) -> int64_t { return ptr32 ? (int64_t)ptr32[i] - ptr32[0] : ptr64[i]; };
  auto row_e = [&](int64_t i) -> int64_t {
    return ptr32 ? (int64_t)ptr32[i + 1] - ptr32[0] : ptr64[i + 1];
  };
  std::vector<int64_t> moff(nc + 1, 0);
  for (int64_t i = 0; i < n; ++i) moff[comm[i] + 1]++;
  for (int32_t c = 0; c < nc; ++c) moff[c + 1] += moff[c];
  std::vector<int32_t> members(n);
  {
    std::vector<int64_t> fill(moff.begin(), moff.end() - 1);
    for (int64_t i = 0; i < n; ++i) members[fill[comm[i]]++] = (int32_t)i;
  }
  LevelGraph g;
  g.n = nc;
  g.ptr.assign(nc + 1, 0);
  std::vector<double> acc(nc, 0.0);
  std::vector<char> seen(nc, 0);
  std::vector<int32_t> touched;
  for (int32_t c = 0; c < nc; ++c) {
    touched.clear();
    for (int64_t m = moff[c]; m < moff[c + 1]; ++m) {
      const int32_t i = members[m];
      for (int64_t e = row_b(i); e < row_e(i); ++e) {
        const int32_t j = adj[e];
        if (skip_self && j == i) continue;
        const int32_t d = comm[j];
        if (!seen[d]) {
          seen[d] = 1;
          touched.push_back(d);
        }
        acc[d] += w ? w[e] : 1.0;
      }
    }
    std::sort(touched.begin(), touched.end());
    for (int32_t d : touched) {
      g.adj.push_back(d);
      g.w.push_back(acc[d]);
      acc[d] = 0.0;
      seen[d] = 0;
    }
    g.ptr[c + 1] = (int64_t)g.adj.size();
  }
  return g;
}

}  // namespace
}  // namespace gnn

using namespace gnn;

extern "C" {

GNN_API gnn_status_t gnn_reorder_gcr(const int32_t *row_ptr, const int32_t *col_ind, int64_t n,
                                     const gnn_reorder_opts_t *opts, int32_t *perm,
                                     int32_t *comm_out, double *modularity) {
  if (!row_ptr || n < 0 || !perm || (n > 0 && !col_ind))
    return fail(GNN_ERR_INVALID_ARG, "gnn_reorder_gcr: bad arguments");
  gnn_reorder_opts_t o{};
  if (opts) o = *opts;
  const int max_levels = o.max_levels > 0 ? o.max_levels : 3;
  const int max_passes = o.max_passes > 0 ? o.max_passes : 20;
  const double min_gain = o.min_gain > 0 ? o.min_gain : 1e-6;
  const double res = o.resolution > 0 ? o.resolution : 1.0;
  for (int64_t i = 0; i < n; ++i) {
    const int64_t b = (int64_t)row_ptr[i] - row_ptr[0], e = (int64_t)row_ptr[i + 1] - row_ptr[0];
    if (e < b) return fail(GNN_ERR_INVALID_ARG, "gnn_reorder_gcr: row_ptr decreasing at %lld", (long long)i);
    for (int64_t x = b; x < e; ++x)
      if (col_ind[x] < 0 || col_ind[x] >= n)
        return fail(GNN_ERR_INVALID_ARG, "gnn_reorder_gcr: col_ind out of range (square graph)");
  }
  try {
    // levels[l][v] = community (level l+1 node) of level-l node v
    std::vector<std::vector<int32_t>> levels;
    LevelGraph cur;
    double q = 0.0;
    int64_t nl = n;
    for (int lev = 0; lev < max_levels; ++lev) {
      LevelResult r = lev == 0 ? local_moving(row_ptr, nullptr, col_ind, nullptr, n, true, res,
                                              max_passes, min_gain)
                               : local_moving(nullptr, cur.ptr.data(), cur.adj.data(),
                                              cur.w.data(), nl, false, res, max_passes, min_gain);
      if (lev > 0 && !r.moved) break;
      q = r.q;
      LevelGraph next = lev == 0 ? aggregate(row_ptr, nullptr, col_ind, nullptr, n, true, r.comm,
                                             r.nc)
                                 : aggregate(nullptr, cur.ptr.data(), cur.adj.data(),
                                             cur.w.data(), nl, false, r.comm, r.nc);
      levels.push_back(std::move(r.comm));
      cur = std::move(next);
      nl = cur.n;
      if (nl == (int64_t)levels.back().size()) break;  // nothing merged
    }
    const int L = (int)levels.size();
    // community path of each original node and min original member id per community
    std::vector<std::vector<int32_t>> path(L, std::vector<int32_t>(n));
    std::vector<std::vector<int32_t>> minid(L);
    for (int l = 0; l < L; ++l) {
      minid[l].assign(levels[l].empty() ? 0 : (*std::max_element(levels[l].begin(), levels[l].end())) + 1,
                      INT32_MAX);
      for (int64_t i = 0; i < n; ++i) {
        const int32_t below = l == 0 ? (int32_t)i : path[l - 1][i];
        const int32_t c = levels[l][below];
        path[l][i] = c;
        if ((int32_t)i < minid[l][c]) minid[l][c] = (int32_t)i;
      }
    }
    std::vector<int32_t> order(n);
    for (int64_t i = 0; i < n; ++i) order[i] = (int32_t)i;
    std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
      for (int l = L - 1; l >= 0; --l) {
        const int32_t ka = minid[l][path[l][a]], kb = minid[l][path[l][b]];
        if (ka != kb) return ka < kb;
      }
      return a < b;
    });
    if (o.hub_rows > 0) {
      // hub block (B200 addition, DESIGN.md §5 "hub block"): the hub_rows nodes of largest
      // degree (ties: smaller id) move to the front, in the hierarchical order among
      // themselves; the rest keep theirs.  Their feature rows then form one contiguous
      // block of X that the kernels can keep L2-resident (plan option hub_rows).
      const int64_t H = o.hub_rows < n ? o.hub_rows : n;
      std::vector<int32_t> byd(n);
      for (int64_t i = 0; i < n; ++i) byd[i] = (int32_t)i;
      auto deg = [&](int32_t v) { return (int64_t)row_ptr[v + 1] - row_ptr[v]; };
      std::nth_element(byd.begin(), byd.begin() + (H - 1), byd.end(), [&](int32_t a, int32_t b) {
        const int64_t da = deg(a), db = deg(b);
        return da != db ? da > db : a < b;
      });
      std::vector<char> hub(n, 0);
      for (int64_t i = 0; i < H; ++i) hub[byd[i]] = 1;
      std::stable_partition(order.begin(), order.end(), [&](int32_t v) { return hub[v] != 0; });
    }
    for (int64_t p = 0; p < n; ++p) perm[order[p]] = (int32_t)p;
    if (comm_out) {
      for (int64_t i = 0; i < n; ++i) comm_out[i] = L ? path[L - 1][i] : (int32_t)i;
    }
    if (modularity) *modularity = q;
  } catch (const std::bad_alloc &) {
    return fail(GNN_ERR_INVALID_ARG, "gnn_reorder_gcr: out of host memory");
  }
  return GNN_OK;
}

GNN_API gnn_status_t gnn_permute_graph(const int32_t *row_ptr, const int32_t *col_ind,
                                       const float *val, int64_t n, const int32_t *perm,
                                       int32_t *row_ptr_out, int32_t *row_ind_out,
                                       int32_t *col_ind_out, float *val_out) {
  if (!row_ptr || !perm || !row_ptr_out || n < 0)
    return fail(GNN_ERR_INVALID_ARG, "gnn_permute_graph: bad arguments");
  const int64_t base = row_ptr[0];
  const int64_t nnz = (int64_t)row_ptr[n] - base;
  if (nnz > 0 && (!col_ind || !col_ind_out || (val && !val_out)))
    return fail(GNN_ERR_INVALID_ARG, "gnn_permute_graph: bad arguments");
  try {
    std::vector<int32_t> inv(n);
    std::vector<char> hit(n, 0);
    for (int64_t i = 0; i < n; ++i) {
      const int32_t p = perm[i];
      if (p < 0 || p >= n || hit[p]) return fail(GNN_ERR_INVALID_ARG, "gnn_permute_graph: perm is not a bijection");
      hit[p] = 1;
      inv[p] = (int32_t)i;
    }
    row_ptr_out[0] = 0;
    for (int64_t p = 0; p < n; ++p)
      row_ptr_out[p + 1] = row_ptr_out[p] + (row_ptr[inv[p] + 1] - row_ptr[inv[p]]);
    std::vector<uint64_t> tmp;
    for (int64_t p = 0; p < n; ++p) {
      const int64_t ob = (int64_t)row_ptr[inv[p]] - base, oe = (int64_t)row_ptr[inv[p] + 1] - base;
      const int64_t nb = row_ptr_out[p];
      tmp.resize(oe - ob);
      for (int64_t x = ob; x < oe; ++x) {
        const int32_t c = col_ind[x];
        if (c < 0 || c >= n) return fail(GNN_ERR_INVALID_ARG, "gnn_permute_graph: col out of range");
        // key = new column, then original position (stable for duplicates)
        tmp[x - ob] = ((uint64_t)(uint32_t)perm[c] << 32) | (uint64_t)(uint32_t)(x - ob);
      }
      std::sort(tmp.begin(), tmp.end());
      for (int64_t y = 0; y < oe - ob; ++y) {
        col_ind_out[nb + y] = (int32_t)(tmp[y] >> 32);
        if (row_ind_out) row_ind_out[nb + y] = (int32_t)p;
        if (val) val_out[nb + y] = val[ob + (int64_t)(tmp[y] & 0xffffffffu)];
      }
    }
  } catch (const std::bad_alloc &) {
    return fail(GNN_ERR_INVALID_ARG, "gnn_permute_graph: out of host memory");
  }
  return GNN_OK;
}

}  // extern "C"
