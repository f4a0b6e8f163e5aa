// Integer makespan model + greedy-correction scheduler + single-slot fallback.
//
// PAPER.md:81 (§IV-C): Step 1 places the critical path on the fastest device(s); Step 2 greedily
// places the remaining subgraphs on the device that minimises the increase of the critical path;
// Step 3 (Algorithm 1) refines each multi-path phase by swapping pairs / moving
// single subgraphs while the latency drops, stopping after x rounds without a decrease.
// fall back to the best single device.  The paper's `measure latency` is the
// integer model of SURVEY.md §8(c) C3 ("model mode", R-6); tie-breaks R-7..R-9.
#include <algorithm>
#include <tuple>

#include "common.h"

namespace duet {

Schedule::~Schedule() = default;

namespace {

struct Model {
  const Partition* p;
  const Profile* pr;
  int n, D;
  std::vector<std::vector<std::pair<int, int64_t>>> preds, succs;
  std::vector<int64_t> in_bytes, out_bytes;  // -1 = none
  std::vector<std::vector<int>> phases;

  Model(const Partition* p_, const Profile* pr_) : p(p_), pr(pr_) {
    n = p->n_sg();
    D = pr->n_slots;
    preds.resize(n);
    succs.resize(n);
    in_bytes.assign(n, -1);
    out_bytes.assign(n, -1);
    for (auto& kv : p->edges) {  // map order == lexicographic (src, dst)
      int u = kv.first.first, v = kv.first.second;
      if (u == -1)
        in_bytes[v] = kv.second;
      else if (v == -1)
        out_bytes[u] = kv.second;
      else {
        preds[v].push_back({u, kv.second});
        succs[u].push_back({v, kv.second});
      }
    }
    phases.resize(p->phase_kind.size());
    for (int s = 0; s < n; ++s) phases[p->sg_phase[s]].push_back(s);
  }

  int64_t T(int s, int d) const { return pr->T(s, d); }

  int64_t c(int from, int to, int64_t bytes) const {
    if (from == to) return 0;
    const duet_link& l =
        pr->slot_gpu[from] == pr->slot_gpu[to] ? pr->comm.same_gpu : pr->comm.cross_gpu;
    return l.alpha_ns + (bytes * l.ps_per_byte + 999) / 1000;
  }

  // simulate phase ph; finish/done carry earlier results; returns phase end, fills free
  int64_t sim_phase(const std::vector<int>& a, int ph, int64_t start_t, std::vector<int64_t>& finish,
                    std::vector<char>& done, std::vector<int64_t>* free_out) const {
    std::vector<int64_t> fr(D, start_t);
    int64_t pe = start_t;
    for (int s : phases[ph]) {
      if (a[s] < 0) continue;
      int d = a[s];
      int64_t ready = 0;
      if (in_bytes[s] >= 0) ready = c(0, d, in_bytes[s]);
      for (auto& e : preds[s])
        if (done[e.first]) ready = std::max(ready, finish[e.first] + c(a[e.first], d, e.second));
      int64_t st = std::max(fr[d], ready);
      finish[s] = st + T(s, d);
      done[s] = 1;
      fr[d] = finish[s];
      pe = std::max(pe, finish[s]);
    }
    if (free_out) *free_out = fr;
    return pe;
  }

  int64_t makespan(const std::vector<int>& a) const {
    std::vector<int64_t> finish(n, 0);
    std::vector<char> done(n, 0);
    int64_t t = 0;
    for (int ph = 0; ph < (int)phases.size(); ++ph) t = sim_phase(a, ph, t, finish, done, nullptr);
    int64_t m = t;
    for (int s = 0; s < n; ++s)
      if (out_bytes[s] >= 0) m = std::max(m, finish[s] + c(a[s], 0, out_bytes[s]));
    return m;
  }

  int64_t partial(const std::vector<int>& a, int ph, std::vector<int64_t>* free_out) const {
    std::vector<int64_t> finish(n, 0);
    std::vector<char> done(n, 0);
    int64_t t = 0;
    for (int q = 0; q < ph; ++q) t = sim_phase(a, q, t, finish, done, nullptr);
    return sim_phase(a, ph, t, finish, done, free_out);
  }

  int64_t comm_in(const std::vector<int>& a, int s, int d) const {
    int64_t r = 0;
    if (in_bytes[s] >= 0) r = c(0, d, in_bytes[s]);
    for (auto& e : preds[s])
      if (a[e.first] >= 0) r = std::max(r, c(a[e.first], d, e.second));
    return r;
  }

  int argmin_place(const std::vector<int>& a, int s) const {
    int best = 0;
    auto key = [&](int d) { return std::make_tuple(T(s, d), comm_in(a, s, d), d); };
    for (int d = 1; d < D; ++d)
      if (key(d) < key(best)) best = d;
    return best;
  }
};

std::vector<int> phase_chain(const Model& m, int ph, const std::vector<int64_t>& cost) {
  const auto& P = m.phases[ph];
  std::vector<char> inph(m.n, 0);
  for (int s : P) inph[s] = 1;
  int s_star = P[0];
  for (int s : P)
    if (cost[s] > cost[s_star]) s_star = s;  // ties: smallest id (P ascending)
  std::vector<int64_t> din(m.n, 0), dout(m.n, 0);
  for (int s : P) {
    int64_t b = 0;
    for (auto& e : m.preds[s])
      if (inph[e.first]) b = std::max(b, din[e.first]);
    din[s] = cost[s] + b;
  }
  for (auto it = P.rbegin(); it != P.rend(); ++it) {
    int s = *it;
    int64_t b = 0;
    for (auto& e : m.succs[s])
      if (inph[e.first]) b = std::max(b, dout[e.first]);
    dout[s] = cost[s] + b;
  }
  std::set<int> chain{s_star};
  int cur = s_star;
  while (true) {
    int best = -1;
    for (auto& e : m.preds[cur])
      if (inph[e.first] && (best < 0 || din[e.first] > din[best] ||
                            (din[e.first] == din[best] && e.first < best)))
        best = e.first;
    if (best < 0) break;
    chain.insert(best);
    cur = best;
  }
  cur = s_star;
  while (true) {
    int best = -1;
    for (auto& e : m.succs[cur])
      if (inph[e.first] && (best < 0 || dout[e.first] > dout[best] ||
                            (dout[e.first] == dout[best] && e.first < best)))
        best = e.first;
    if (best < 0) break;
    chain.insert(best);
    cur = best;
  }
  return std::vector<int>(chain.begin(), chain.end());
}

std::vector<int> greedy(const Model& m) {
  std::vector<int> a(m.n, -1);
  for (int ph = 0; ph < (int)m.phases.size(); ++ph) {
    const auto& P = m.phases[ph];
    if (m.p->phase_kind[ph] == kSeq) {
      for (int s : P) a[s] = m.argmin_place(a, s);
      continue;
    }
    std::vector<int64_t> cost(m.n, 0);
    for (int s : P) {
      int64_t c = m.T(s, 0);
      for (int d = 1; d < m.D; ++d) c = std::min(c, m.T(s, d));
      cost[s] = c;
    }
    for (int s : phase_chain(m, ph, cost)) a[s] = m.argmin_place(a, s);
    std::vector<int> rem;
    for (int s : P)
      if (a[s] < 0) rem.push_back(s);
    std::vector<char> inrem(m.n, 0);
    for (int s : rem) inrem[s] = 1;
    std::vector<int> indeg(m.n, 0);
    for (int s : rem)
      for (auto& e : m.preds[s])
        if (inrem[e.first]) indeg[s]++;
    std::vector<char> done(m.n, 0);
    for (size_t k = 0; k < rem.size(); ++k) {
      int s = -1;
      for (int x : rem) {
        if (done[x] || indeg[x]) continue;
        if (s < 0 || cost[x] > cost[s] || (cost[x] == cost[s] && x < s)) s = x;
      }
      int64_t before = m.partial(a, ph, nullptr);
      std::tuple<int64_t, int64_t, int64_t, int> best{0, 0, 0, -1};
      for (int d = 0; d < m.D; ++d) {
        a[s] = d;
        std::vector<int64_t> fr;
        int64_t after = m.partial(a, ph, &fr);
        auto key = std::make_tuple(after - before, fr[d], m.T(s, d), d);
        if (std::get<3>(best) < 0 || key < best) best = key;
      }
      a[s] = std::get<3>(best);
      done[s] = 1;
      for (auto& e : m.succs[s])
        if (inrem[e.first]) indeg[e.first]--;
    }
  }
  return a;
}

// `lat` is Algorithm 1's `measure latency`: the C3 model (model mode) or a device measurement of
// the whole assignment (measured mode); tie-breaks are the same in both.
void correct(const Model& m, std::vector<int>& a, int ph, int rounds, const Latency& lat) {
  int64_t t_old = lat(a);
  const auto& P = m.phases[ph];
  int idle = 0;
  while (true) {
    bool improved = false;
    std::vector<int> U(P.begin(), P.end());
    while (!U.empty()) {
      bool have = false;
      std::tuple<int64_t, int, int, int> best{};
      std::vector<int> b;
      for (int i : U)
        for (int d = 0; d < m.D; ++d) {
          if (d == a[i]) continue;
          b = a;
          b[i] = d;
          auto key = std::make_tuple(lat(b), 0, i, d);
          if (!have || key < best) best = key, have = true;
        }
      for (size_t x = 0; x < U.size(); ++x)
        for (size_t y = x + 1; y < U.size(); ++y) {
          int i = U[x], j = U[y];
          if (a[i] == a[j]) continue;
          b = a;
          std::swap(b[i], b[j]);
          auto key = std::make_tuple(lat(b), 1, i, j);
          if (!have || key < best) best = key, have = true;
        }
      if (!have) break;
      int64_t t_new = std::get<0>(best);
      int kind = std::get<1>(best), i = std::get<2>(best), y = std::get<3>(best);
      std::vector<int> U2;
      for (int s : U)
        if (s != i && !(kind == 1 && s == y)) U2.push_back(s);
      U.swap(U2);
      if (t_new < t_old) {
        if (kind == 0)
          a[i] = y;
        else
          std::swap(a[i], a[y]);
        t_old = t_new;
        improved = true;
      }
    }
    idle = improved ? 0 : idle + 1;
    if (idle >= rounds) break;
  }
}

uint32_t lowbias32(uint32_t x) {
  x ^= x >> 16;
  x *= 0x7feb352du;
  x ^= x >> 15;
  x *= 0x846ca68bu;
  x ^= x >> 16;
  return x;
}

}  // namespace

Schedule* make_schedule_with(const Partition* p, const Profile* pr, const duet_sched_opts* o, const Latency* measured) {
  if (pr->p != p) fail(DUET_EINVAL, "profile belongs to another partition");
  duet_sched_opts opts{0, 1, 1, nullptr, 0};
  if (o) opts = *o;
  if (opts.mode < 0 || opts.mode > 6) fail(DUET_EINVAL, "mode must be 0..6");
  if (opts.correction_rounds < 1) fail(DUET_EINVAL, "correction_rounds must be >= 1");
  Model m(p, pr);
  if (m.D < 1) fail(DUET_EINVAL, "no slots");
  const Latency model = [&](const std::vector<int>& b) { return m.makespan(b); };
  const Latency& lat = measured ? *measured : model;
  std::unique_ptr<Schedule> S(new Schedule());
  S->p = p;
  S->pr = pr;
  std::vector<int> a;
  if (opts.mode == 2) {
    a.assign(m.n, 0);
  } else if (opts.mode == 3) {
    if (!opts.fixed_slot_of) fail(DUET_EINVAL, "mode 3 needs fixed_slot_of");
    for (int s = 0; s < m.n; ++s) {
      int d = opts.fixed_slot_of[s];
      if (d < 0 || d >= m.D) fail(DUET_EINVAL, "fixed_slot_of out of range");
      a.push_back(d);
    }
  } else {
    if (opts.mode == 4 || opts.mode == 6) {
      for (int s = 0; s < m.n; ++s) a.push_back((int)(lowbias32(opts.seed * 0x9E3779B1u + (uint32_t)s) % (uint32_t)m.D));
    } else if (opts.mode == 5) {
      for (int s = 0; s < m.n; ++s) a.push_back(s % m.D);
    } else {
      a = greedy(m);
    }
    if (opts.mode == 0 || opts.mode == 6)
      for (int ph = 0; ph < (int)m.phases.size(); ++ph)
        if (p->phase_kind[ph] == kMulti) correct(m, a, ph, opts.correction_rounds, lat);
    if (opts.allow_fallback) {
      int64_t m_gc = lat(a);
      int64_t best = -1;
      int bd = 0;
      for (int d = 0; d < m.D; ++d) {
        int64_t v = lat(std::vector<int>(m.n, d));
        if (best < 0 || v < best) best = v, bd = d;
      }
      if (best <= m_gc) {
        a.assign(m.n, bd);
        S->fell_back = 1;
      }
    }
  }
  // measured mode: the slots are identical in the model but not on the device (the home slot's
  // stream has normal priority, the others high), so relabelling the slots
  // of the chosen assignment can change its measured latency -- c2 measured 5% faster with the
  // critical path off the home slot (profiles/r1c_fig13.md).  Step 3's `measure latency` therefore
  // also tries every relabelling (D <= 4) and keeps the fastest.
  if (measured && (opts.mode == 0 || opts.mode == 6) && m.D >= 2 && m.D <= 4) {
    std::vector<int> perm(m.D);
    for (int d = 0; d < m.D; ++d) perm[d] = d;
    int64_t best = lat(a);
    std::vector<int> best_a = a;
    while (std::next_permutation(perm.begin(), perm.end())) {
      std::vector<int> b(a.size());
      for (size_t s = 0; s < a.size(); ++s) b[s] = perm[a[s]];
      const int64_t v = lat(b);
      if (v < best) best = v, best_a = b;
    }
    a = best_a;
  }
  S->slot_of = a;
  for (int s = 0; s < m.n; ++s) S->order.push_back(s);
  S->makespan = m.makespan(a);
  if (measured) S->measured_ns = lat(a);
  return S.release();
}

Schedule* make_schedule(const Partition* p, const Profile* pr, const duet_sched_opts* o) {
  return make_schedule_with(p, pr, o, nullptr);
}

}  // namespace duet
