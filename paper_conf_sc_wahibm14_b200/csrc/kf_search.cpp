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
          L.regs > t_.regs_per_thread_max)
        v.ok = false;
      else
        v.t_model = model_time(p_, L, t_, v.bytes);
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

}  // extern "C"
