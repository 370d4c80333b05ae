// Host-side plan search (row a5): picks the plans to run.
//
// The paper searches the partition space with an HGGA (Alg. 1) and
// verifies small searches "using a deterministic method".  Here:
//   BRUTE  : every restricted-growth string, pruned on path closure (1.3) as kernels are
//            assigned, per-group verdicts memoised (the paper's pruning of inactive
//            constraints, in exact form);
//   GREEDY : agglomerative merging of groups that share an array, each merge closed under
//            (1.3), keeping the legal merge with the largest byte saving.
// Objective: total compulsory bytes (T = bytes / BW, Eq. 1 with the codeless bound);
// ties -> lexicographically smallest canonical labels (R17).
#include <algorithm>
#include <functional>
#include <random>
#include <unordered_map>

#include "kf_internal.hpp"

namespace kf {

struct GroupVerdict {
  bool ok;
  uint64_t bytes;
  double t_model;
};

class Evaluator {
 public:
  Evaluator(const Program& p, const kf_target& t) : p_(p), t_(t) {}
  // Legality of one group in isolation (V2, V3, V5..V8) and its bytes.
  const GroupVerdict& eval(const std::vector<int>& g) {
    std::string key(reinterpret_cast<const char*>(g.data()), g.size() * sizeof(int));
    auto it = cache_.find(key);
    if (it != cache_.end()) return it->second;
    GroupVerdict v{true, group_bytes(p_, g, nullptr, nullptr), 0.0};
    if (check_kinship(p_, g, 0, nullptr) || check_convex(p_, g, 0, nullptr)) {
      v.ok = false;
    } else {
      GroupLowering L = lower_group(p_, g, t_);
      if (check_hazard(p_, g, L, 0, nullptr) || check_halo(p_, L, t_, 0, nullptr) || L.smem > t_.smem_per_block ||
          !regs_ok(L, t_))
        v.ok = false;
      else {
        v.t_model = model_time(p_, L, t_, v.bytes);
        // experiment (KF_MODEL_PAIRS): project a group at the better of the point and pair canvas, as
        // autotuning picks -- its plans measured slower once tuned (round 2), so off by default
        if (t_.pblock[0] == 1 && t_.pblock[1] == 1 && t_.zunroll == 1 && getenv("KF_MODEL_PAIRS")) {
          kf_target tp = t_;
          tp.pblock[0] = 2;
          tp.pair_zq = 1;
          GroupLowering L2 = lower_group(p_, g, tp);
          if (L2.smem <= tp.smem_per_block && regs_ok(L2, tp))
            v.t_model = std::min(v.t_model, model_time(p_, L2, tp, v.bytes));
        }
      }
    }
    return cache_.emplace(key, v).first->second;
  }
  // Full legality of a canonical labelling.
  bool legal(const std::vector<int>& label, int m, uint64_t* bytes, double* tmodel = nullptr) {
    std::vector<std::vector<int>> gs(m);
    for (int k = 0; k < int(label.size()); k++) gs[label[k]].push_back(k);
    uint64_t tot = 0;
    double tt = 0.0;
    for (auto& g : gs) {
      const GroupVerdict& v = eval(g);
      if (!v.ok) return false;
      tot += v.bytes;
      tt += v.t_model;
    }
    if (!quotient_acyclic(p_, label, m, nullptr)) return false;
    if (bytes) *bytes = tot;
    if (tmodel) *tmodel = tt;
    return true;
  }

 private:
  const Program& p_;
  const kf_target& t_;
  std::unordered_map<std::string, GroupVerdict> cache_;
};

// Enumerate restricted-growth strings; `visit(label, m)` for every complete assignment that
// survives the incremental path-closure prune.  Pruning is exact: once a kernel c outside a
// group G lies on a path a ~> c ~> b with a, b in G, no completion can repair (1.3).
static void enumerate(const Program& p, const std::function<void(const std::vector<int>&, int)>& visit) {
  int n = p.nk;
  std::vector<int> label(n, -1);
  std::vector<std::vector<int>> members;
  std::function<void(int, int)> rec = [&](int i, int m) {
    if (i == n) { visit(label, m); return; }
    for (int gq = 0; gq <= m; gq++) {
      bool ok = true;
      if (gq < m) {
        // adding i to group gq: any already-assigned c outside gq with a ~> c ~> i, a in gq?
        for (int a : members[gq]) {
          for (int c = a + 1; c < i && ok; c++)
            if (label[c] != gq && p.reaches(a, c) && p.reaches(c, i)) ok = false;
          if (!ok) break;
        }
      }
      if (!ok) continue;
      label[i] = gq;
      if (gq == m) members.push_back({});
      members[gq].push_back(i);
      rec(i + 1, std::max(m, gq + 1));
      members[gq].pop_back();
      if (gq == m) members.pop_back();
      label[i] = -1;
    }
  };
  rec(0, 0);
}

static std::vector<int> canon(const std::vector<int>& lab, int* m) {
  std::map<int, int> mp;
  std::vector<int> out(lab.size());
  for (size_t k = 0; k < lab.size(); k++) {
    auto it = mp.find(lab[k]);
    if (it == mp.end()) it = mp.emplace(lab[k], int(mp.size())).first;
    out[k] = it->second;
  }
  if (m) *m = int(mp.size());
  return out;
}

static std::vector<int> greedy(const Program& p, Evaluator& ev, uint64_t* best_bytes, bool by_time) {
  std::vector<int> label(p.nk);
  for (int k = 0; k < p.nk; k++) label[k] = k;
  int m = p.nk;
  // objective: compulsory bytes, or projected time (scaled to an integer-like double)
  auto cost = [&](const std::vector<int>& lab, int mm, double* c) {
    uint64_t b = 0;
    double t = 0.0;
    if (!ev.legal(lab, mm, &b, &t)) return false;
    *c = by_time ? t : double(b);
    return true;
  };
  double cur = 0.0;
  cost(label, m, &cur);
  for (;;) {
    std::vector<std::vector<int>> gs(m);
    for (int k = 0; k < p.nk; k++) gs[label[k]].push_back(k);
    double best = cur;
    std::vector<int> best_lab;
    for (int gi = 0; gi < m; gi++)
      for (int gj = gi + 1; gj < m; gj++) {
        bool adj = false;
        for (int a : gs[gi]) {
          for (int b : gs[gj])
            if (p.share[a][b]) { adj = true; break; }
          if (adj) break;
        }
        if (!adj) continue;
        // close the union under paths (1.3): absorb every group holding a kernel on a path
        std::set<int> merged{gi, gj};
        for (bool grew = true; grew;) {
          grew = false;
          std::vector<int> mem;
          for (int g : merged) mem.insert(mem.end(), gs[g].begin(), gs[g].end());
          for (int c = 0; c < p.nk; c++) {
            if (merged.count(label[c])) continue;
            bool from = false, to = false;
            for (int a : mem) {
              if (p.reaches(a, c)) from = true;
              if (p.reaches(c, a)) to = true;
            }
            if (from && to) { merged.insert(label[c]); grew = true; }
          }
        }
        std::vector<int> lab(label);
        int tgt = *merged.begin();
        for (int k = 0; k < p.nk; k++)
          if (merged.count(lab[k])) lab[k] = tgt;
        int mm = 0;
        lab = canon(lab, &mm);
        double b = 0.0;
        if (!cost(lab, mm, &b)) continue;
        if (b < cur && (best_lab.empty() || b < best || (b == best && lab < best_lab))) {
          best = b;
          best_lab = lab;
        }
      }
    if (best_lab.empty() || best >= cur) break;
    label = best_lab;
    cur = best;
    m = 0;
    label = canon(label, &m);
  }
  if (best_bytes) {
    int mm = *std::max_element(label.begin(), label.end()) + 1;
    uint64_t b = 0;
    ev.legal(label, mm, &b);
    *best_bytes = b;
  }
  return label;
}

// ---------------------------------------------------------------- HGGA (NEXT-1)
// Hybrid Grouping Genetic Algorithm (Alg. 1; Falkenauer [19]): individuals
// are partitions whose genes are the groups (new kernels).  Group-aware crossover injects a
// random subset of the other parent's groups and repairs the rest; mutation dissolves or merges
// groups; every offspring is made legal (infeasible groups fall back to singletons, the first
// violated constraint rejects a merge -- the paper's active-constraint pruning) and then
// locally improved by legal merges.  Deterministic for a given seed.
struct Indiv {
  std::vector<int> lab;
  double cost = 0;
};

class Hgga {
 public:
  Hgga(const Program& p, Evaluator& ev, bool by_time, uint64_t seed) : p_(p), ev_(ev), by_time_(by_time), rng_(seed) {}

  std::vector<int> run(int pop_size, int max_gen, int stall_gen, uint64_t* bytes_out) {
    std::vector<Indiv> pop;
    for (int i = 0; i < pop_size; i++) pop.push_back(random_individual(i == 0 ? 0.0 : 0.6));
    auto better = [](const Indiv& a, const Indiv& b) { return a.cost < b.cost || (a.cost == b.cost && a.lab < b.lab); };
    Indiv best = *std::min_element(pop.begin(), pop.end(), better);
    int stall = 0;
    for (int gen = 0; gen < max_gen && stall < stall_gen; gen++) {
      std::vector<Indiv> next;
      // elitism: keep the two best
      std::sort(pop.begin(), pop.end(), better);
      next.push_back(pop[0]);
      if (pop.size() > 1) next.push_back(pop[1]);
      while (int(next.size()) < pop_size) {
        const Indiv& a = tournament(pop);
        const Indiv& b = tournament(pop);
        Indiv c = crossover(a, b);
        if (uni() < 0.3) c = mutate(c);
        next.push_back(c);
      }
      pop = std::move(next);
      Indiv gb = *std::min_element(pop.begin(), pop.end(), better);
      if (better(gb, best)) {
        best = gb;
        stall = 0;
      } else {
        stall++;
      }
    }
    if (bytes_out) {
      uint64_t b = 0;
      ev_.legal(best.lab, nm(best.lab), &b);
      *bytes_out = b;
    }
    return best.lab;
  }

 private:
  const Program& p_;
  Evaluator& ev_;
  bool by_time_;
  std::mt19937_64 rng_;

  double uni() { return std::uniform_real_distribution<double>(0.0, 1.0)(rng_); }
  int rint(int n) { return int(std::uniform_int_distribution<int>(0, n - 1)(rng_)); }
  static int nm(const std::vector<int>& lab) { return *std::max_element(lab.begin(), lab.end()) + 1; }

  bool cost(const std::vector<int>& lab, double* c) {
    uint64_t b = 0;
    double t = 0;
    if (!ev_.legal(lab, nm(lab), &b, &t)) return false;
    *c = by_time_ ? t : double(b);
    return true;
  }
  std::vector<std::vector<int>> groups(const std::vector<int>& lab) {
    std::vector<std::vector<int>> gs(nm(lab));
    for (int k = 0; k < p_.nk; k++) gs[lab[k]].push_back(k);
    return gs;
  }
  static std::vector<int> from_groups(const std::vector<std::vector<int>>& gs, int n) {
    std::vector<int> lab(n, -1);
    int g = 0;
    for (auto& grp : gs)
      if (!grp.empty()) {
        for (int k : grp) lab[k] = g;
        g++;
      }
    return canon(lab, nullptr);
  }
  // Make a plan legal: groups that are illegal alone dissolve into singletons; a cyclic quotient
  // dissolves groups until acyclic.
  std::vector<int> repair(std::vector<std::vector<int>> gs) {
    std::vector<std::vector<int>> out;
    for (auto& g : gs) {
      if (g.empty()) continue;
      std::sort(g.begin(), g.end());
      if (g.size() == 1 || ev_.eval(g).ok) out.push_back(g);
      else
        for (int k : g) out.push_back({k});
    }
    std::vector<int> lab = from_groups(out, p_.nk);
    while (!quotient_acyclic(p_, lab, nm(lab), nullptr)) {
      int bad = -1;
      quotient_acyclic(p_, lab, nm(lab), &bad);
      auto g2 = groups(lab);
      std::vector<std::vector<int>> o2;
      for (int i = 0; i < int(g2.size()); i++) {
        if (i == bad)
          for (int k : g2[i]) o2.push_back({k});
        else
          o2.push_back(g2[i]);
      }
      lab = from_groups(o2, p_.nk);
    }
    return lab;
  }
  // Local improvement: randomized legal merges of adjacent groups that lower the cost.
  Indiv improve(std::vector<int> lab, int tries) {
    double c = 0;
    cost(lab, &c);
    for (int t = 0; t < tries; t++) {
      auto gs = groups(lab);
      if (gs.size() < 2) break;
      int gi = rint(int(gs.size()));
      std::vector<int> cand;
      for (int gj = 0; gj < int(gs.size()); gj++) {
        if (gj == gi) continue;
        bool adj = false;
        for (int a : gs[gi]) {
          for (int b : gs[gj])
            if (p_.share[a][b]) { adj = true; break; }
          if (adj) break;
        }
        if (adj) cand.push_back(gj);
      }
      if (cand.empty()) continue;
      int gj = cand[rint(int(cand.size()))];
      std::vector<int> l2 = lab;
      for (int k = 0; k < p_.nk; k++)
        if (l2[k] == gj) l2[k] = gi;
      l2 = canon(l2, nullptr);
      double c2;
      if (cost(l2, &c2) && c2 < c) { lab = l2; c = c2; }
    }
    return Indiv{lab, c};
  }
  Indiv random_individual(double merge_p) {
    std::vector<int> lab(p_.nk);
    for (int k = 0; k < p_.nk; k++) lab[k] = k;
    if (merge_p > 0) {
      // random legal merges (not necessarily improving): diversity of the initial population
      for (int t = 0; t < 3 * p_.nk; t++) {
        if (uni() > merge_p) continue;
        int a = rint(p_.nk), b = rint(p_.nk);
        if (lab[a] == lab[b] || !p_.share[a][b]) continue;
        std::vector<int> l2 = lab;
        int ga = lab[a], gb = lab[b];
        for (int k = 0; k < p_.nk; k++)
          if (l2[k] == gb) l2[k] = ga;
        l2 = canon(l2, nullptr);
        double c2;
        if (cost(l2, &c2)) lab = l2;
      }
    }
    return improve(canon(lab, nullptr), p_.nk);
  }
  const Indiv& tournament(const std::vector<Indiv>& pop) {
    const Indiv& a = pop[rint(int(pop.size()))];
    const Indiv& b = pop[rint(int(pop.size()))];
    return (a.cost < b.cost || (a.cost == b.cost && a.lab < b.lab)) ? a : b;
  }
  Indiv crossover(const Indiv& A, const Indiv& B) {
    auto ga = groups(A.lab), gb = groups(B.lab);
    // inject a random subset of B's multi-kernel groups
    std::vector<std::vector<int>> inj;
    for (auto& g : gb)
      if (g.size() > 1 && uni() < 0.5) inj.push_back(g);
    std::vector<char> taken(p_.nk, 0);
    for (auto& g : inj)
      for (int k : g) taken[k] = 1;
    std::vector<std::vector<int>> out = inj;
    for (auto& g : ga) {
      std::vector<int> rest;
      for (int k : g)
        if (!taken[k]) rest.push_back(k);
      if (!rest.empty()) out.push_back(rest);
    }
    return improve(repair(out), p_.nk / 2 + 1);
  }
  Indiv mutate(const Indiv& A) {
    auto gs = groups(A.lab);
    std::vector<std::vector<int>> out;
    int victim = rint(int(gs.size()));
    for (int i = 0; i < int(gs.size()); i++) {
      if (i == victim && gs[i].size() > 1)
        for (int k : gs[i]) out.push_back({k});   // dissolve a group
      else
        out.push_back(gs[i]);
    }
    return improve(repair(out), p_.nk / 2 + 1);
  }
};

}  // namespace kf

using namespace kf;

extern "C" {

kf_status kf_plan_search(const kf_program* prog, const kf_target* target, int32_t method, uint64_t seed,
                         int32_t* plan_out, uint64_t* bytes_out) {
  (void)seed;
  KF_TRY({
    if (!prog || !plan_out) fail(KF_E_ARG, "null argument");
    check_target(target);
    const Program& p = prog->p;
    Evaluator ev(p, *target);
    if (method == KF_SEARCH_AUTO) method = p.nk <= 10 ? KF_SEARCH_BRUTE : KF_SEARCH_GREEDY;
    std::vector<int> best;
    uint64_t best_b = 0;
    if (method == KF_SEARCH_BRUTE || method == KF_SEARCH_BRUTE_TIME) {
      if (p.nk > 14) fail(KF_E_UNSUPPORTED, "brute-force search limited to 14 kernels");
      bool have = false;
      double best_t = 0.0;
      const bool by_time = method == KF_SEARCH_BRUTE_TIME;
      enumerate(p, [&](const std::vector<int>& lab, int m) {
        uint64_t b;
        double t;
        if (!ev.legal(lab, m, &b, &t)) return;
        bool better = by_time ? (!have || t < best_t) : (!have || b < best_b);   // RGS order = lexicographic
        if (better) { best = lab; best_b = b; best_t = t; have = true; }
      });
      if (!have) fail(KF_E_ILLEGAL_PLAN, "no legal plan");   // cannot happen: singletons are legal unless V6-V8 bind
    } else if (method == KF_SEARCH_GREEDY || method == KF_SEARCH_GREEDY_TIME) {
      best = greedy(p, ev, &best_b, method == KF_SEARCH_GREEDY_TIME);
      int m = 0;
      if (!ev.legal(best, *std::max_element(best.begin(), best.end()) + 1, nullptr))
        fail(KF_E_ILLEGAL_PLAN, "even the unfused plan is illegal under this target");
      (void)m;
    } else if (method == KF_SEARCH_HGGA || method == KF_SEARCH_HGGA_BYTES) {
      // population 100 as in Table VI; stop after 30 generations without improvement
      Hgga h(p, ev, method == KF_SEARCH_HGGA, seed);
      best = h.run(100, 2000, 30, &best_b);
    } else {
      fail(KF_E_ARG, "unknown search method");
    }
    std::copy(best.begin(), best.end(), plan_out);
    if (bytes_out) *bytes_out = best_b;
  });
}

kf_status kf_plan_count_legal(const kf_program* prog, const kf_target* target, uint64_t* count) {
  KF_TRY({
    if (!prog || !count) fail(KF_E_ARG, "null argument");
    check_target(target);
    const Program& p = prog->p;
    if (p.nk > 14) fail(KF_E_UNSUPPORTED, "counting limited to 14 kernels");
    Evaluator ev(p, *target);
    uint64_t c = 0;
    enumerate(p, [&](const std::vector<int>& lab, int m) {
      if (ev.legal(lab, m, nullptr)) c++;
    });
    *count = c;
  });
}

kf_status kf_plan_enumerate(const kf_program* prog, const kf_target* target, int32_t* plans, int64_t cap,
                            int64_t* count) {
  KF_TRY({
    if (!prog || !count || (cap > 0 && !plans)) fail(KF_E_ARG, "null argument");
    check_target(target);
    const Program& p = prog->p;
    if (p.nk > 14) fail(KF_E_UNSUPPORTED, "enumeration limited to 14 kernels");
    Evaluator ev(p, *target);
    int64_t c = 0;
    enumerate(p, [&](const std::vector<int>& lab, int m) {
      if (!ev.legal(lab, m, nullptr)) return;
      if (c < cap) std::copy(lab.begin(), lab.end(), plans + c * p.nk);
      c++;
    });
    *count = c;
  });
}

}  // extern "C"
