// ttemb_reorder.cu -- host-side (offline) part of the index bijection generator (Sec. IV-C,
// P:269-277): modularity-based community detection on the index graph of Alg. 2 by the Louvain
// method (the paper's refs [34], [35]).  Plain C++ on the host, no device code; exported through
// the C ABI (include/ttemb.h: ttemb_louvain) and called by paper_conf_sc_wangwfmmd22_b200/reorder.py.
//
// Local moving: vertices in index order move to the neighbouring community with the largest
// modularity gain  dQ ~ k_i,in(C) - tot(C) k_i / 2m  (ties to the smaller community id; a move
// needs a gain > 1e-12), repeated until no vertex moves; then communities are aggregated into
// vertices (internal weight -> self-loop) and the next level starts, until a level moves nothing.
// Deterministic; the same algorithm as reorder.louvain (the Python reference the tests compare).
#include <stdint.h>

#include <algorithm>
#include <unordered_map>
#include <vector>

#include "../../include/ttemb.h"

namespace {

struct Graph {
  int64_t n = 0;
  std::vector<int64_t> ptr, dst;
  std::vector<double> wt;
};

// symmetric CSR; a self-loop u == v is stored once with weight 2w
Graph build(int64_t n, const std::vector<int64_t>& u, const std::vector<int64_t>& v, const std::vector<double>& w) {
  Graph g;
  g.n = n;
  g.ptr.assign(n + 1, 0);
  for (size_t e = 0; e < u.size(); ++e) {
    g.ptr[u[e] + 1]++;
    if (u[e] != v[e]) g.ptr[v[e] + 1]++;
  }
  for (int64_t i = 0; i < n; ++i) g.ptr[i + 1] += g.ptr[i];
  g.dst.resize(g.ptr[n]);
  g.wt.resize(g.ptr[n]);
  std::vector<int64_t> fill(g.ptr.begin(), g.ptr.end() - 1);
  for (size_t e = 0; e < u.size(); ++e) {
    if (u[e] == v[e]) {
      g.dst[fill[u[e]]] = v[e]; g.wt[fill[u[e]]++] = 2.0 * w[e];
    } else {
      g.dst[fill[u[e]]] = v[e]; g.wt[fill[u[e]]++] = w[e];
      g.dst[fill[v[e]]] = u[e]; g.wt[fill[v[e]]++] = w[e];
    }
  }
  return g;
}

}  // namespace

extern "C" int ttemb_louvain(int64_t n, int64_t m, const int64_t* u, const int64_t* v, const double* w,
                             int64_t* labels) {
  if (n < 0 || m < 0 || (n > 0 && !labels) || (m > 0 && (!u || !v || !w))) return TTEMB_ERR_INVALID_ARG;
  for (int64_t e = 0; e < m; ++e)
    if (u[e] < 0 || u[e] >= n || v[e] < 0 || v[e] >= n) return TTEMB_ERR_INVALID_ARG;
  std::vector<int64_t> lab(n);
  for (int64_t i = 0; i < n; ++i) lab[i] = i;
  std::vector<int64_t> cu(u, u + m), cv(v, v + m);
  std::vector<double> cw(w, w + m);
  int64_t cn = n;
  for (int level = 0; level < 16 && !cw.empty(); ++level) {
    Graph g = build(cn, cu, cv, cw);
    std::vector<double> k(cn, 0.0);
    for (int64_t i = 0; i < cn; ++i)
      for (int64_t e = g.ptr[i]; e < g.ptr[i + 1]; ++e) k[i] += g.wt[e];
    double m2 = 0.0;
    for (double x : k) m2 += x;
    if (m2 <= 0.0) break;
    std::vector<int64_t> comm(cn);
    for (int64_t i = 0; i < cn; ++i) comm[i] = i;
    std::vector<double> tot(k);
    std::unordered_map<int64_t, double> kin;
    std::vector<int64_t> keys;
    bool improved = false;
    for (int pass = 0; pass < 32; ++pass) {
      int64_t moved = 0;
      for (int64_t i = 0; i < cn; ++i) {
        const int64_t ci = comm[i];
        tot[ci] -= k[i];
        kin.clear();
        keys.clear();
        for (int64_t e = g.ptr[i]; e < g.ptr[i + 1]; ++e) {
          if (g.dst[e] == i) continue;
          const int64_t c = comm[g.dst[e]];
          auto it = kin.find(c);
          if (it == kin.end()) { kin.emplace(c, g.wt[e]); keys.push_back(c); }
          else it->second += g.wt[e];
        }
        std::sort(keys.begin(), keys.end());
        int64_t best = ci;
        auto own = kin.find(ci);
        double best_gain = (own == kin.end() ? 0.0 : own->second) - tot[ci] * k[i] / m2;
        for (int64_t c : keys) {
          const double gain = kin[c] - tot[c] * k[i] / m2;
          if (gain > best_gain + 1e-12) { best = c; best_gain = gain; }
        }
        tot[best] += k[i];
        if (best != ci) { comm[i] = best; ++moved; }
      }
      if (moved == 0) break;
      improved = true;
    }
    if (!improved) break;
    // renumber communities 0..C-1 in increasing old id (== np.unique's inverse)
    std::vector<int64_t> ids(comm);
    std::sort(ids.begin(), ids.end());
    ids.erase(std::unique(ids.begin(), ids.end()), ids.end());
    std::vector<int64_t> re(cn);
    for (int64_t i = 0; i < cn; ++i) re[i] = std::lower_bound(ids.begin(), ids.end(), comm[i]) - ids.begin();
    for (int64_t i = 0; i < n; ++i) lab[i] = re[lab[i]];
    const int64_t nc = (int64_t)ids.size();
    // aggregate: merge parallel edges (keys lo * nc + hi, ascending like np.unique)
    std::vector<std::pair<int64_t, double>> ew(cu.size());
    for (size_t e = 0; e < cu.size(); ++e) {
      const int64_t a = re[cu[e]], b = re[cv[e]];
      ew[e] = {std::min(a, b) * nc + std::max(a, b), cw[e]};
    }
    std::sort(ew.begin(), ew.end(), [](const auto& x, const auto& y) { return x.first < y.first; });
    cu.clear(); cv.clear(); cw.clear();
    for (size_t e = 0; e < ew.size(); ++e) {
      if (e > 0 && ew[e].first == ew[e - 1].first) { cw.back() += ew[e].second; continue; }
      cu.push_back(ew[e].first / nc);
      cv.push_back(ew[e].first % nc);
      cw.push_back(ew[e].second);
    }
    cn = nc;
  }
  // labels numbered by first occurrence
  std::vector<int64_t> remap(n > 0 ? n : 1, -1);
  int64_t next = 0;
  for (int64_t i = 0; i < n; ++i) {
    if (remap[lab[i]] < 0) remap[lab[i]] = next++;
    labels[i] = remap[lab[i]];
  }
  return TTEMB_OK;
}
