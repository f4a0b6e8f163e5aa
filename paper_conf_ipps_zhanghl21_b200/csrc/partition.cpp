// Coarse-grained multi-phase partitioner (§IV-A; footnote 1 PAPER.md:111).
//
// A phased schedule S_1..S_t: phases are totally ordered, a phase is sequential (one subgraph)
// or multi-path (independent subgraphs), adjacent phases differ in kind, shared inputs get
// replicated placeholders.  Cut rule (DESIGN.md R-C2): separators = nodes on
// every source->sink path; regions between consecutive separators split into weakly connected
// components; >= 2 components -> multi-path phase, everything else merges into sequential phases.
#include <algorithm>
#include <queue>

#include "common.h"

namespace duet {

namespace {

std::vector<char> reach(int start, const std::vector<std::vector<int>>& adj, int blocked) {
  std::vector<char> seen(adj.size(), 0);
  std::vector<int> st{start};
  seen[start] = 1;
  while (!st.empty()) {
    int u = st.back();
    st.pop_back();
    for (int v : adj[u])
      if (!seen[v] && v != blocked) {
        seen[v] = 1;
        st.push_back(v);
      }
  }
  return seen;
}

}  // namespace

// Bytes of a b-byte row-major tensor in row shard j of k: the k shares
// floor(b (j+1) / k) - floor(b j / k) sum to b.
static int64_t share(int64_t b, int j, int k) { return b * (j + 1) / k - b * j / k; }

Partition* make_partition(const Graph* g, int granularity, int batch_shards) {
  if (granularity != 0 && granularity != 1) fail(DUET_EINVAL, "granularity must be 0 or 1");
  if (batch_shards < 1 || batch_shards > 64) fail(DUET_EINVAL, "batch_shards must be in [1, 64]");
  const int n0 = (int)g->nodes.size();
  std::vector<std::vector<int>> preds(n0), succs(n0);
  std::vector<char> is_input(n0);
  std::vector<int> alias(n0);
  for (int v = 0; v < n0; ++v) {
    preds[v] = g->nodes[v].inputs;
    is_input[v] = g->nodes[v].op == "input";
    alias[v] = v;
  }
  for (int v = 0; v < n0; ++v)
    for (int u : preds[v]) succs[u].push_back(v);
  for (auto& s : succs) std::sort(s.begin(), s.end());

  // step 1: replicated placeholders for shared inputs
  std::unique_ptr<Partition> P(new Partition());
  P->g = g;
  P->granularity = granularity;
  for (int i = 0; i < n0; ++i) {
    if (!is_input[i] || succs[i].size() <= 1) continue;
    std::vector<int> rest(succs[i].begin() + 1, succs[i].end());
    succs[i].resize(1);
    for (int c : rest) {
      int w = (int)preds.size();
      preds.push_back({});
      succs.push_back({c});
      alias.push_back(i);
      is_input.push_back(1);
      for (int& u : preds[c])
        if (u == i) u = w;
      P->n_placeholders++;
    }
  }
  const int N = (int)preds.size();
  // topological rank: Kahn, smallest ready id first
  std::vector<int> rank(N), indeg(N);
  {
    std::priority_queue<int, std::vector<int>, std::greater<int>> ready;
    for (int v = 0; v < N; ++v) {
      indeg[v] = (int)preds[v].size();
      if (!indeg[v]) ready.push(v);
    }
    int k = 0;
    while (!ready.empty()) {
      int u = ready.top();
      ready.pop();
      rank[u] = k++;
      for (int v : succs[u])
        if (--indeg[v] == 0) ready.push(v);
    }
    if (k != N) fail(DUET_ECYCLE, "graph has a cycle");
  }
  auto compute = [&](int v) { return !is_input[v]; };

  // step 2: virtual source S = N, sink T = N+1; separators
  const int S = N, T = N + 1;
  std::vector<std::vector<int>> fwd(N + 2), bwd(N + 2);
  for (int v = 0; v < N; ++v) {
    fwd[v] = succs[v];
    bwd[v] = preds[v];
  }
  for (int v = 0; v < N; ++v) {
    if (preds[v].empty()) {
      fwd[S].push_back(v);
      bwd[v].push_back(S);
    }
    // only nodes without successors reach the sink: an output that also feeds other nodes keeps
    // its boundary edge (step 6) but must not bypass the join, or the join would stop being a
    // separator and every branch concurrency behind it would be lost
    if (succs[v].empty()) {
      fwd[v].push_back(T);
      bwd[T].push_back(v);
    }
  }
  std::vector<int> seps;
  for (int v = 0; v < N; ++v)
    if (!reach(S, fwd, v)[T]) seps.push_back(v);
  std::sort(seps.begin(), seps.end(), [&](int a, int b) { return rank[a] < rank[b]; });
  std::vector<char> is_sep(N, 0);
  for (int v : seps) is_sep[v] = 1;

  // step 3: regions and components
  std::vector<int> bounds{S};
  bounds.insert(bounds.end(), seps.begin(), seps.end());
  bounds.push_back(T);
  struct Item {
    bool is_sep;
    int sep;
    std::vector<std::vector<int>> comps;
  };
  std::vector<Item> items;
  auto min_compute_rank = [&](const std::vector<int>& c) {
    int m = 1 << 30;
    for (int v : c)
      if (compute(v)) m = std::min(m, rank[v]);
    return m;
  };
  for (size_t bi = 0; bi + 1 < bounds.size(); ++bi) {
    auto down = reach(bounds[bi], fwd, -1);
    auto up = reach(bounds[bi + 1], bwd, -1);
    std::vector<char> in_region(N, 0);
    std::vector<int> region;
    for (int v = 0; v < N; ++v)
      if (!is_sep[v] && down[v] && up[v]) {
        in_region[v] = 1;
        region.push_back(v);
      }
    std::vector<int> comp_of(N, -1);
    std::vector<std::vector<int>> comps;
    std::sort(region.begin(), region.end(), [&](int a, int b) { return rank[a] < rank[b]; });
    for (int v : region) {
      if (comp_of[v] >= 0) continue;
      int cid = (int)comps.size();
      comps.push_back({});
      std::vector<int> st{v};
      comp_of[v] = cid;
      while (!st.empty()) {
        int u = st.back();
        st.pop_back();
        comps[cid].push_back(u);
        for (auto* lst : {&succs[u], &preds[u]})
          for (int w : *lst)
            if (in_region[w] && comp_of[w] < 0) {
              comp_of[w] = cid;
              st.push_back(w);
            }
      }
    }
    std::vector<std::vector<int>> kept;
    for (auto& c : comps) {
      bool any = false;
      for (int v : c) any |= compute(v);
      if (!any) continue;
      std::sort(c.begin(), c.end(), [&](int a, int b) { return rank[a] < rank[b]; });
      kept.push_back(c);
    }
    std::sort(kept.begin(), kept.end(), [&](const std::vector<int>& a, const std::vector<int>& b) {
      return min_compute_rank(a) < min_compute_rank(b);
    });
    items.push_back({false, -1, kept});
    if (bi + 2 < bounds.size()) items.push_back({true, bounds[bi + 1], {}});
  }

  // step 4: phases
  std::vector<std::pair<int, std::vector<std::vector<int>>>> phases;
  std::vector<int> cur;
  auto flush = [&]() {
    bool any = false;
    for (int v : cur) any |= compute(v);
    if (any) {
      std::sort(cur.begin(), cur.end(), [&](int a, int b) { return rank[a] < rank[b]; });
      phases.push_back({kSeq, {cur}});
    }
    cur.clear();
  };
  for (auto& it : items) {
    if (it.is_sep) {
      cur.push_back(it.sep);
    } else if (it.comps.size() >= 2) {
      flush();
      phases.push_back({kMulti, it.comps});
    } else {
      for (auto& c : it.comps) cur.insert(cur.end(), c.begin(), c.end());
    }
  }
  flush();

  // step 5: granularity
  std::vector<std::pair<int, std::vector<int>>> sgs;
  for (int p = 0; p < (int)phases.size(); ++p) {
    for (auto& grp : phases[p].second) {
      std::vector<int> nodes;
      for (int v : grp)
        if (compute(v)) nodes.push_back(v);
      if (granularity == 0) {
        sgs.push_back({p, nodes});
      } else {
        for (int v : nodes) sgs.push_back({p, {v}});
      }
    }
  }
  // step 6: ids by (phase, min rank); boundary tensors
  std::sort(sgs.begin(), sgs.end(), [&](const auto& a, const auto& b) {
    if (a.first != b.first) return a.first < b.first;
    return min_compute_rank(a.second) < min_compute_rank(b.second);
  });
  std::vector<int> sg_of(N, -1);
  for (int s = 0; s < (int)sgs.size(); ++s)
    for (int v : sgs[s].second) sg_of[v] = s;
  // step 7 (batch_shards = k > 1): every multi-path subgraph becomes k row-shard subgraphs with
  // consecutive ids; boundary bytes split by share(); shard-to-shard edges pair equal indices
  const int k = batch_shards;
  std::vector<std::vector<int>> ids(sgs.size());
  for (int s = 0; s < (int)sgs.size(); ++s) {
    const bool shard = k > 1 && phases[sgs[s].first].first == kMulti;
    for (int j = 0; j < (shard ? k : 1); ++j) {
      ids[s].push_back((int)P->sg_shard.size());
      P->sg_shard.push_back(shard ? j : -1);
      P->sg_origin.push_back(s);
    }
  }
  struct Pair { int a, b, j; };
  auto pairs = [&](int src, int dst) {
    std::vector<int> S = src >= 0 ? ids[src] : std::vector<int>{-1};
    std::vector<int> D = dst >= 0 ? ids[dst] : std::vector<int>{-1};
    std::vector<Pair> out;
    if (S.size() > 1 && D.size() > 1) {
      for (int j = 0; j < k; ++j) out.push_back({S[j], D[j], j});
    } else if (D.size() > 1) {
      for (int j = 0; j < k; ++j) out.push_back({S[0], D[j], j});
    } else if (S.size() > 1) {
      for (int i = 0; i < k; ++i) out.push_back({S[i], D[0], i});
    } else {
      out.push_back({S[0], D[0], -1});
    }
    return out;
  };
  std::map<std::pair<int, int>, std::pair<int, std::set<int>>> tensors;  // -> (shard index, tensors)
  for (int v = 0; v < N; ++v) {
    if (!compute(v)) continue;
    for (int u : preds[v]) {
      int src = compute(u) ? sg_of[u] : -1;
      if (src == sg_of[v]) continue;
      for (const Pair& e : pairs(src, sg_of[v])) {
        auto& t = tensors[{e.a, e.b}];
        t.first = e.j;
        t.second.insert(alias[u]);
      }
    }
  }
  for (int o : g->outputs)
    if (compute(o))
      for (const Pair& e : pairs(sg_of[o], -1)) {
        auto& t = tensors[{e.a, e.b}];
        t.first = e.j;
        t.second.insert(o);
      }
  for (auto& kv : tensors) {
    int64_t b = 0;
    for (int t : kv.second.second) {
      const int64_t nb = g->nodes[t].nbytes();
      b += kv.second.first < 0 ? nb : share(nb, kv.second.first, k);
    }
    P->edges[kv.first] = b;
  }
  P->batch_shards = k;
  P->node_to_sg.resize(n0);
  for (int v = 0; v < n0; ++v) P->node_to_sg[v] = sg_of[v] >= 0 ? ids[sg_of[v]][0] : -1;
  for (int s_new = 0; s_new < (int)P->sg_origin.size(); ++s_new) {
    const auto& s = sgs[P->sg_origin[s_new]];
    P->sg_nodes.push_back(s.second);
    P->sg_phase.push_back(s.first);
  }
  for (auto& ph : phases) P->phase_kind.push_back(ph.first);
  return P.release();
}

}  // namespace duet
