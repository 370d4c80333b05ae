// Fusion plans: lowering (a3), legality (a2), projection (a4).
//
// Legality follows the constraints of the paper's formulation (Fig. 4, Eq. 1.2-1.7,
// P:236-272) plus the two readings needed to execute a plan on a GPU: the quotient
// graph must be acyclic (R4) and no tile may read, outside its own tile, an array the
// group overwrites in HBM (the SMEM/GMEM incoherence of P:52 and P:107; R7).
// Extended regions implement the halo layers of complex fusion: producers are
// recomputed on the Minkowski sum of their consumers' regions and footprints (R8).
// The projection is the codeless upper bound of P:321 reduced to compulsory bytes over
// peak bandwidth (Eq. 11's LD/ST counts).
#include <algorithm>
#include <cstdio>
#include <climits>
#include <cstring>
#include <tuple>

#include "kf_internal.hpp"

namespace kf {

static int64_t rup(int64_t a, int64_t b) { return (a + b - 1) / b * b; }

Plan make_plan(const Program& p, const int32_t* labels) {
  Plan pl;
  std::map<int, int> m;
  pl.label.resize(p.nk);
  for (int k = 0; k < p.nk; k++) {
    if (labels[k] < 0) fail(KF_E_ILLEGAL_PLAN, "kernel " + std::to_string(k) + " has a negative group label");
    auto it = m.find(labels[k]);
    if (it == m.end()) it = m.emplace(labels[k], int(m.size())).first;
    pl.label[k] = it->second;
  }
  pl.m = int(m.size());
  pl.groups.assign(pl.m, {});
  for (int k = 0; k < p.nk; k++) pl.groups[pl.label[k]].push_back(k);
  return pl;
}

static bool in_group(const std::vector<int>& g, int k) { return std::binary_search(g.begin(), g.end(), k); }

std::vector<Ver> group_live_in(const Program& p, const std::vector<int>& g) {
  std::set<Ver> s;
  for (int k : g)
    for (auto& [x, _] : p.kernels[k].reads) {
      int v = p.vr(k, x);
      if (v == 0 || !in_group(g, p.writer_of(x, v))) s.insert(Ver{x, v});
    }
  return std::vector<Ver>(s.begin(), s.end());
}

std::vector<Ver> group_live_out(const Program& p, const std::vector<int>& g) {
  std::set<Ver> s;
  for (int k : g)
    for (int x : p.kernels[k].writes) {
      int v = p.vw(k, x);
      bool outside = false;
      for (int r : p.readers_of_version(x, v))
        if (!in_group(g, r)) { outside = true; break; }
      bool final_live = v == int(p.writers[x].size()) && p.step_live[x];
      if (outside || final_live) s.insert(Ver{x, v});
    }
  return std::vector<Ver>(s.begin(), s.end());
}

int GroupLowering::ring_of(const Ver& v) const {
  for (size_t i = 0; i < rings.size(); i++)
    if (rings[i].ver == v) return int(i);
  return -1;
}

GroupLowering lower_group(const Program& p, const std::vector<int>& g, const kf_target& t) {
  GroupLowering L;
  L.kernels = g;
  L.tile[0] = t.tile[0];
  L.tile[1] = t.tile[1];
  L.tile[2] = t.tile[2];
  L.stages = t.stages;
  L.threads = t.threads;
  L.zunroll = t.zunroll;
  L.ghost_write = t.ghostwrite && p.bc[2] != KF_BC_PERIODIC &&
                  (p.bc[0] == KF_BC_PERIODIC || p.bc[1] == KF_BC_PERIODIC) &&
                  (p.bc[0] != KF_BC_PERIODIC || p.n[0] >= 2 * p.ghost[0]) &&
                  (p.bc[1] != KF_BC_PERIODIC || p.n[1] >= 2 * p.ghost[1]);
  L.minblocks = t.minblocks;
  L.canvas_ld = t.canvas_ld;
  L.pair_zq = t.pair_zq;
  L.inline_xy = t.inline_xy;
  if (const char* v = getenv("KF_INLINE")) L.inline_xy = std::min(2, std::max(0, atoi(v)));   // A/B switch
  L.pblock[0] = t.pblock[0];
  L.pblock[1] = t.pblock[1];
  L.live_in = group_live_in(p, g);
  L.live_out = group_live_out(p, g);
  L.live_out_set = std::set<Ver>(L.live_out.begin(), L.live_out.end());
  // ---- extended regions, reverse program order (R8)
  for (auto it = g.rbegin(); it != g.rend(); ++it) {
    int k = *it;
    Ext e;
    auto merge = [&](const int lo[3], const int hi[3]) {
      if (!e.alive) {
        for (int a = 0; a < 3; a++) { e.elo[a] = lo[a]; e.ehi[a] = hi[a]; }
        e.alive = true;
      } else {
        for (int a = 0; a < 3; a++) { e.elo[a] = std::max(e.elo[a], lo[a]); e.ehi[a] = std::max(e.ehi[a], hi[a]); }
      }
    };
    for (int x : p.kernels[k].writes)
      if (L.live_out_set.count(Ver{x, p.vw(k, x)})) {
        int z[3] = {0, 0, 0};
        merge(z, z);
        break;
      }
    for (int c : g) {
      if (c <= k || !L.ext[c].alive) continue;
      for (auto& [x, offs] : p.kernels[c].reads) {
        int v = p.vr(c, x);
        if (v < 1 || p.writer_of(x, v) != k) continue;
        int lo[3], hi[3];
        for (int a = 0; a < 3; a++) {
          int dmin = INT_MAX, dmax = INT_MIN;
          for (auto& d : offs) { dmin = std::min(dmin, d[a]); dmax = std::max(dmax, d[a]); }
          lo[a] = L.ext[c].elo[a] - dmin;
          hi[a] = L.ext[c].ehi[a] + dmax;
        }
        merge(lo, hi);
      }
    }
    L.ext[k] = e;
  }
  std::vector<int> alive;
  for (int k : g)
    if (L.ext[k].alive) alive.push_back(k);
  // ---- z delays: a consumer runs behind its in-group producers by their dz reach; with the delay
  // skew (R20c) reads at a nonzero xy offset stay U planes further behind, so they only touch
  // planes written in earlier iterations (published by the end-of-iteration barrier)
  for (int k : alive) {
    int dk = 0;
    for (auto& [x, offs] : p.kernels[k].reads) {
      int v = p.vr(k, x);
      if (v < 1) continue;
      int pr = p.writer_of(x, v);
      if (!in_group(g, pr) || !L.ext[pr].alive) continue;
      for (auto& d : offs) {
        const bool xy = d[0] != 0 || d[1] != 0;
        dk = std::max(dk, L.delay[pr] + d[2] + (t.skew && xy ? t.zunroll : 0));
      }
    }
    L.delay[k] = dk;
  }
  const int es = p.es, TX = t.tile[0], TY = t.tile[1], S = t.stages, U = t.zunroll;
  auto finish_ring = [&](Ring& r) {
    const int a = 16 / es;
    // TMA box x start must be 16-byte aligned: round the lower x extent of a live-in box up to a
    // multiple of 16/es elements (ceil toward +inf also for negative extents).  (Round 2 tried the
    // same for in-group rings, so pair stores never split: no gain measured, KF_RING_ALIGN=1.)
    const bool align = r.live_in || getenv("KF_RING_ALIGN") != nullptr;
    r.ax_lo = !align ? r.blo[0] : r.blo[0] >= 0 ? (r.blo[0] + a - 1) / a * a : -((-r.blo[0]) / a * a);
    r.wx = TX + r.ax_lo + r.bhi[0];
    r.hy = TY + r.blo[1] + r.bhi[1];
    // row pitch: a multiple of 16 bytes.  (An odd number of 16-byte units would remove the 2-way
    // bank conflicts of the halo-column threads, but its ~5 % more shared memory cost the flux groups
    // a CTA per SM: measured 3.07 vs 2.58 ms per step, round 2 -- not used.)
    r.px = int(rup(r.wx, a));
    r.plane_bytes = int(rup(int64_t(r.px) * r.hy * es, 128));
  };
  // ---- live-in rings (TMA staged)
  for (const Ver& lv : L.live_in) {
    std::vector<int> rd;
    for (int c : alive)
      if (p.kernels[c].reads.count(lv.x) && p.vr(c, lv.x) == lv.v) rd.push_back(c);
    if (rd.empty()) continue;
    Ring r;
    r.ver = lv;
    r.live_in = true;
    int A = INT_MIN, B = INT_MAX;
    bool first = true;
    for (int c : rd) {
      for (auto& d : p.kernels[c].reads.at(lv.x)) {
        A = std::max(A, d[2] - L.delay[c]);
        B = std::min(B, d[2] - L.delay[c]);
        for (int a = 0; a < 3; a++) {
          int lo = L.ext[c].elo[a] - d[a], hi = L.ext[c].ehi[a] + d[a];
          if (first) { r.blo[a] = lo; r.bhi[a] = hi; }
          else { r.blo[a] = std::max(r.blo[a], lo); r.bhi[a] = std::max(r.bhi[a], hi); }
        }
        first = false;
      }
    }
    if (!p.relaxed[lv.x])
      for (int b : alive)
        if (p.kernels[b].writes_array(lv.x) && L.live_out_set.count(Ver{lv.x, p.vw(b, lv.x)}))
          A = std::max(A, -L.delay[b]);
    r.A = A;
    r.B = B;
    r.slots = (A - B + 1) + U * S - 1;   // planes in use [t+B, t+U-1+A] plus U*(S-1) prefetched
    finish_ring(r);
    L.rings.push_back(r);
  }
  // ---- in-group rings (intermediates kept on chip)
  for (int pk : alive)
    for (int x : p.kernels[pk].writes) {
      int v = p.vw(pk, x);
      int mx = INT_MIN;
      for (int c : alive)
        if (p.kernels[c].reads.count(x) && p.vr(c, x) == v)
          for (auto& d : p.kernels[c].reads.at(x)) mx = std::max(mx, L.delay[c] - d[2]);
      if (mx == INT_MIN) continue;
      Ring r;
      r.ver = Ver{x, v};
      r.live_in = false;
      r.producer = pk;
      for (int a = 0; a < 3; a++) { r.blo[a] = L.ext[pk].elo[a]; r.bhi[a] = L.ext[pk].ehi[a]; }
      r.slots = mx - L.delay[pk] + 1 + (U - 1);
      finish_ring(r);
      L.rings.push_back(r);
    }
  // ring unrolling (target.ringunroll): sizes rounded up to powers of two; N = the largest (<= 16)
  if (t.ringunroll) {
    int N = 1;
    for (auto& r : L.rings) {
      int q = 1;
      while (q < r.slots) q *= 2;
      r.slots = q;
      N = std::max(N, q);
    }
    L.ring_unroll = N <= 16 ? N : 0;
  }
  // ---- SMEM layout and the resource model (R20)
  int off = 0;
  for (auto& r : L.rings) {
    r.smem_off = off;
    off += r.slots * r.plane_bytes;
  }
  L.mbar_off = off;
  L.smem = off + 8 * S + 128;
  // threads per CTA: one per register block (bx x by points, pblock) of the largest extended
  // region, so the fast path covers every region in one pass without clamped duplicate lanes
  // (which would still issue shared loads); used when the tile itself fits the target's thread
  // count, capped at 512 (R20)
  {
    // the canvas = bounding box of all extended regions (per-axis max lo/hi halo): the fast path
    // gives each canvas point to one thread for every kernel of the group
    const int bx = std::max(1, t.pblock[0]), by = std::max(1, t.pblock[1]);
    int clo[2] = {0, 0}, chi[2] = {0, 0};
    for (int k : alive)
      for (int a = 0; a < 2; a++) {
        clo[a] = std::max(clo[a], L.ext[k].elo[a]);
        chi[a] = std::max(chi[a], L.ext[k].ehi[a]);
      }
    const int CW = TX + clo[0] + chi[0], CH = TY + clo[1] + chi[1];
    const int maxb = alive.empty() ? 0 : ((CW + std::min(bx, CW) - 1) / std::min(bx, CW)) * ((CH + std::min(by, CH) - 1) / std::min(by, CH));
    const int nt = (maxb + 31) / 32 * 32;
    const int tb = ((TX + bx - 1) / bx) * ((TY + by - 1) / by);
    L.threads = (tb <= t.threads && nt >= 32 && nt <= 512) ? nt : t.threads;
  }
  int depth = 1;
  for (int k : g) depth = std::max(depth, p.kernels[k].depth);
  L.depth = depth;
  // points computed concurrently per thread in the fast path: blocks x planes x rounds (R20)
  int rounds = 1;
  for (int k : alive) {
    const Ext& e = L.ext[k];
    const int WX = TX + e.elo[0] + e.ehi[0], WY = TY + e.elo[1] + e.ehi[1];
    const int bx = std::min(t.pblock[0], WX), by = std::min(t.pblock[1], WY);
    const int nb = ((WX + bx - 1) / bx) * ((WY + by - 1) / by);
    rounds = std::max(rounds, (nb + L.threads - 1) / L.threads);
  }
  const int P = std::min(8, t.pblock[0] * t.pblock[1] * U * rounds);
  // Register model (V8; R20, revised in round 2 after the hardware pin): the paper's Eq. 4/6
  // for one thread of a fused group,
  //     R_est = R_adr * U + RegFac * (es/4) * P * (ThrLD + depth),
  // R_adr = 32 address / index / predicate registers per plane of a stream iteration, R_fetch = 0
  // (TMA stages the live-ins without registers), RegFac = 1 (no register reuse: the upper end of
  // the paper's range 1/max(ThrLD) <= RegFac <= 1), P = points per thread (<= 8), depth = deepest
  // RPN stack, ThrLD = distinct values (array, version, offset) a thread loads and holds: the whole
  // group's on the canvas (its loads are reused across the phases of an iteration), the largest
  // single kernel's on the per-kernel path.  The kernel is compiled with this as its register cap
  // (__maxnreg__), so NUM_REGS <= R_est; a GPU test asserts it never spills at that cap.
  {
    int clo0 = 0, chi0 = 0, clo1 = 0, chi1 = 0;
    for (int k : alive) {
      clo0 = std::max(clo0, L.ext[k].elo[0]);
      chi0 = std::max(chi0, L.ext[k].ehi[0]);
      clo1 = std::max(clo1, L.ext[k].elo[1]);
      chi1 = std::max(chi1, L.ext[k].ehi[1]);
    }
    const int CW = TX + clo0 + chi0, CH = TY + clo1 + chi1;
    bool canvas = false;
    if (!alive.empty() && t.pblock[0] == 1 && t.pblock[1] == 1)
      canvas = (CW * CH + L.threads - 1) / L.threads == 1;
    if (!alive.empty() && t.pblock[0] == 2 && t.pblock[1] == 1 && U == 1 && TX % 2 == 0 && p.n[0] % 2 == 0) {
      const int cwp = TX / 2 + (clo0 + 1) / 2 + (chi0 + 1) / 2;
      canvas = (cwp * CH + L.threads - 1) / L.threads == 1;
    }
    std::set<std::tuple<int, int, int, int, int>> all;
    int kmax = 0;
    for (int k : alive) {
      int nk = 0;
      for (auto& [x, offs] : p.kernels[k].reads) {
        const int v = p.vr(k, x);
        for (auto& d : offs) {
          all.insert(std::make_tuple(x, v, d[0], d[1], d[2]));
          nk++;
        }
      }
      kmax = std::max(kmax, nk);
    }
    const int thrld = canvas ? int(all.size()) : kmax;
    L.regs = 32 * U + (es / 4) * P * (thrld + depth);
    L.thrld = thrld;
    L.pts = P;
  }
  return L;
}

std::vector<int> quotient_order(const Program& p, const Plan& pl) {
  int m = pl.m;
  std::vector<std::set<int>> succ(m);
  std::vector<int> indeg(m, 0);
  for (auto& e : p.edges) {
    int a = pl.label[e.src], b = pl.label[e.dst];
    if (a != b && succ[a].insert(b).second) indeg[b]++;
  }
  std::set<int> ready;
  for (int i = 0; i < m; i++)
    if (!indeg[i]) ready.insert(i);
  std::vector<int> order;
  while (!ready.empty()) {
    int gq = *ready.begin();
    ready.erase(ready.begin());
    order.push_back(gq);
    for (int h : succ[gq])
      if (--indeg[h] == 0) ready.insert(h);
  }
  if (int(order.size()) != m) order.clear();
  return order;
}

static bool nonlocal_read(const Program& p, const GroupLowering& L, int a, int x) {
  const Ext& e = L.ext.at(a);
  if (!e.alive) return false;
  for (auto& d : p.kernels[a].reads.at(x))
    for (int ax = 0; ax < 3; ax++)
      if (d[ax] - e.elo[ax] < 0 || e.ehi[ax] + d[ax] > 0) return true;
  return false;
}

// ---- per-group checks (each returns a kf_violation_code, filling why on failure)
int check_kinship(const Program& p, const std::vector<int>& g, int gi, kf_violation* why) {
  if (p.flags & KF_PROG_NO_KINSHIP) return KF_V_OK;
  std::set<int> seen{g[0]};
  std::vector<int> fr{g[0]};
  while (!fr.empty()) {
    std::vector<int> nx;
    for (int u : fr)
      for (int w : g)
        if (!seen.count(w) && p.share[u][w]) { seen.insert(w); nx.push_back(w); }
    fr = nx;
  }
  for (int b : g)
    if (!seen.count(b)) {
      if (why) *why = kf_violation{KF_V_KINSHIP, gi, g[0], b, -1};
      return KF_V_KINSHIP;
    }
  return KF_V_OK;
}

int check_convex(const Program& p, const std::vector<int>& g, int gi, kf_violation* why) {
  for (int c = 0; c < p.nk; c++) {
    if (in_group(g, c)) continue;
    int src = -1;
    for (int a : g)
      if (p.reaches(a, c)) { src = a; break; }
    if (src < 0) continue;
    for (int b : g)
      if (p.reaches(c, b)) {
        if (why) *why = kf_violation{KF_V_CONVEX, gi, src, c, -1};
        return KF_V_CONVEX;
      }
  }
  return KF_V_OK;
}

int check_hazard(const Program& p, const std::vector<int>& g, const GroupLowering& L, int gi, kf_violation* why) {
  std::set<Ver> lin(L.live_in.begin(), L.live_in.end());
  for (int b : g) {
    std::vector<int> ws = p.kernels[b].writes;
    std::sort(ws.begin(), ws.end());
    for (int x : ws) {
      if (p.relaxed[x] || !L.live_out_set.count(Ver{x, p.vw(b, x)})) continue;
      for (int a : g) {
        if (!p.kernels[a].reads.count(x)) continue;
        if (!lin.count(Ver{x, p.vr(a, x)})) continue;
        if (nonlocal_read(p, L, a, x)) {
          if (why) *why = kf_violation{KF_V_HAZARD, gi, a, b, x};
          return KF_V_HAZARD;
        }
      }
    }
  }
  return KF_V_OK;
}

int check_halo(const Program& p, const GroupLowering& L, const kf_target& t, int gi, kf_violation* why) {
  for (const auto& r : L.rings) {   // live-in rings come first, sorted by (array, version)
    if (!r.live_in) continue;
    for (int a = 0; a < 3; a++) {
      bool wrap = p.bc[a] == KF_BC_PERIODIC || ((t.internal_axes >> a) & 1);
      int ext = std::max(r.blo[a], r.bhi[a]);
      if ((wrap && ext > p.ghost[a]) || (a < 2 && ext > t.max_halo)) {
        if (why) *why = kf_violation{KF_V_HALO, gi, -1, -1, r.ver.x};
        return KF_V_HALO;
      }
    }
  }
  for (int k : L.kernels) {
    const Ext& e = L.ext.at(k);
    if (!e.alive) continue;
    if (std::max({e.elo[0], e.ehi[0], e.elo[1], e.ehi[1]}) > t.max_halo) {
      if (why) *why = kf_violation{KF_V_HALO, gi, k, -1, -1};
      return KF_V_HALO;
    }
  }
  return KF_V_OK;
}

bool quotient_acyclic(const Program& p, const std::vector<int>& label, int m, int* first_bad) {
  std::vector<std::vector<char>> q(m, std::vector<char>(m, 0));
  for (auto& e : p.edges) {
    int a = label[e.src], b = label[e.dst];
    if (a != b) q[a][b] = 1;
  }
  for (int k = 0; k < m; k++)
    for (int i = 0; i < m; i++)
      if (q[i][k])
        for (int j = 0; j < m; j++)
          if (q[k][j]) q[i][j] = 1;
  for (int gi = 0; gi < m; gi++)
    if (q[gi][gi]) {
      if (first_bad) *first_bad = gi;
      return false;
    }
  return true;
}

// Registers a thread of an NT-thread CTA can have: the register file is 4 sub-partitions of 16384
// (B200: 65536 per SM), a CTA's warps spread over them round-robin, allocation in units of 8
// registers per thread (256 per warp) -- measured: a 320-thread kernel at 192 registers reports
// CU_FUNC_ATTRIBUTE_MAX_THREADS_PER_BLOCK = 256.
int regs_limit(int threads) {
  const int warps = (threads + 31) / 32;
  const int per_quadrant = (warps + 3) / 4;
  return std::min(255, 16384 / (per_quadrant * 32) / 8 * 8);
}

// Register cap that keeps m CTAs of NT threads resident per SM: their m*warps warps spread evenly
// over the 4 sub-partitions (ncu: 3 CTAs of 5 warps at 126 registers fit, 4 warps per quadrant).
int regs_cap(int threads, int m) {
  const int warps = std::max(1, m) * ((threads + 31) / 32);
  return std::min(255, 16384 / (((warps + 3) / 4) * 32) / 8 * 8);
}

// V8 = Eq. 2 (R_T <= R_Max) and Eq. 3 with one CTA per SM (Thr * R_T <= R_SMX, per sub-partition)
bool regs_ok(const GroupLowering& L, const kf_target& t) {
  return L.regs <= t.regs_per_thread_max && L.regs <= regs_limit(L.threads);
}

int validate_plan_groups(const Program& p, const Plan& pl, const std::vector<kf_target>& T, kf_violation* why,
                         std::vector<GroupLowering>* lowered) {
  if (why) *why = kf_violation{KF_V_OK, -1, -1, -1, -1};
  int c;
  for (int gi = 0; gi < pl.m; gi++)
    if ((c = check_kinship(p, pl.groups[gi], gi, why))) return c;
  for (int gi = 0; gi < pl.m; gi++)
    if ((c = check_convex(p, pl.groups[gi], gi, why))) return c;
  int bad = -1;
  if (!quotient_acyclic(p, pl.label, pl.m, &bad)) {
    if (why) *why = kf_violation{KF_V_CYCLE, bad, -1, -1, -1};
    return KF_V_CYCLE;
  }
  std::vector<GroupLowering> Ls;
  for (int gi = 0; gi < pl.m; gi++) Ls.push_back(lower_group(p, pl.groups[gi], T[gi]));
  for (int gi = 0; gi < pl.m; gi++)
    if ((c = check_hazard(p, pl.groups[gi], Ls[gi], gi, why))) return c;
  for (int gi = 0; gi < pl.m; gi++)
    if ((c = check_halo(p, Ls[gi], T[gi], gi, why))) return c;
  for (int gi = 0; gi < pl.m; gi++)
    if (Ls[gi].smem > T[gi].smem_per_block) {
      if (why) *why = kf_violation{KF_V_SMEM, gi, -1, -1, -1};
      return KF_V_SMEM;
    }
  for (int gi = 0; gi < pl.m; gi++)
    if (!regs_ok(Ls[gi], T[gi])) {
      if (why) *why = kf_violation{KF_V_REGS, gi, -1, -1, -1};
      return KF_V_REGS;
    }
  if (lowered) *lowered = std::move(Ls);
  return KF_V_OK;
}

int validate_plan(const Program& p, const Plan& pl, const kf_target& t, kf_violation* why,
                  std::vector<GroupLowering>* lowered) {
  return validate_plan_groups(p, pl, std::vector<kf_target>(pl.m, t), why, lowered);
}

uint64_t group_bytes(const Program& p, const std::vector<int>& g, uint64_t* rd, uint64_t* wr) {
  uint64_t unit = uint64_t(p.npts) * uint64_t(p.es);
  uint64_t r = unit * group_live_in(p, g).size();
  uint64_t w = unit * group_live_out(p, g).size();
  if (rd) *rd = r;
  if (wr) *wr = w;
  return r + w;
}

double model_time(const Program& p, const GroupLowering& L, const kf_target& t, uint64_t bytes) {
  // NEXT-2 (R22, recalibrated in round 2 on 129 measured groups: 8 candidate plans' groups under the
  // default launch configuration + the autotuned configurations of the bench plan, clamped canvas
  // loads; median error 5 %, max 24 %, tools/round2/model_fit.py, profiles/round2_summary.md.  A
  // refit on the weather groups after inline recompute (RegFac 0.5, efficiency 0.8) brought the
  // committed groups within 15 % but made the config-2 search pick a 4.7 % slower plan: not kept).
  // The paper's Eq. 9 idea -- the memory bound scaled by the effectiveness of blocking B_eff
  // -- with B_eff from the warps a SM keeps resident:
  //   CTAs/SM   = the shared-memory / thread limit, lowered while a register NEED estimate
  //               (R_adr*U + 0.6*(es/4)*P*(ThrLD + depth): the register model with RegFac 0.6, the
  //               reuse ptxas achieves) does not fit the per-sub-partition register file (Eq. 3)
  //   warps     = CTAs * warps/CTA (a pair-canvas thread counts twice: two independent points)
  //   t_mem     = bytes / (copy rate 0.8185 * nominal) / 0.98 / min(1, warps / 8)
  //   t_smem    = canvas shared-memory traffic / (128 B/clk * n_sm * 1.9 GHz) / 0.7
  //   t         = max(t_mem, t_smem) + 0.1 * t_issue / min(1, warps / 24)   (x0.5 for pairs)
  // t_issue: ~17 issue slots of fixed cost per point of an extended region plus ~1.5 per RPN node.
  const double T = double(L.tile[0]) * L.tile[1];
  double work = 0.0;
  for (int k : L.kernels) {
    const Ext& e = L.ext.at(k);
    if (!e.alive) continue;
    const double R = double(L.tile[0] + e.elo[0] + e.ehi[0]) * (L.tile[1] + e.elo[1] + e.ehi[1]);
    int ops = 0;
    for (auto& st : p.kernels[k].stmts) ops += int(st.rpn.size()) + 1;
    work += (R / T) * (17.0 + 1.5 * ops);
  }
  const int old_ctas = std::max(1, std::min(2048 / std::max(32, L.threads), (t.smem_per_block + 1024) / std::max(1, L.smem + 1024)));
  const double old_eff = std::min(1.0, std::min(64.0, double(old_ctas) * (L.threads / 32)) / 32.0);
  const double t_comp = double(p.npts) * work / (2.5e13 * old_eff);
  const CanvasPlan cv = plan_canvas(p, L);
  const double per_plane = (cv.lds_bytes + cv.sts_bytes + cv.tma_bytes) / std::max(1, L.zunroll);
  const double t_smem = double(p.npts) / T * per_plane / (128.0 * t.n_sm * 1.9e9);
  // resident warps
  const int need = int(32 * L.zunroll + 0.6 * (p.es / 4) * L.pts * (L.thrld + L.depth));
  // shared memory per SM = the per-CTA limit + the 1 KB reserve (B200: 232448 + 1024); scales with a
  // hypothetical smem_per_block (the SMEM-capacity what-if of P:485)
  const int smem_sm = t.smem_per_block + 1024;
  int ctas = std::max(1, std::min({smem_sm / std::max(1, L.smem + 1024), 2048 / std::max(32, L.threads), 32}));
  while (ctas > 1 && regs_cap(L.threads, ctas) < need) ctas--;
  const bool pair = cv.ok && cv.pair;
  const double warps = double(ctas) * ((L.threads + 31) / 32) * (pair ? 2.0 : 1.0);
  const double t_mem = double(bytes) / (0.8185 * t.hbm_bytes_per_s) / 0.98 / std::min(1.0, warps / 8.0);
  const double t_issue = 0.1 * t_comp / std::min(1.0, warps / 24.0) * (pair ? 0.5 : 1.0);
  if (getenv("KF_DEBUG_MODEL"))
    fprintf(stderr, "model: group of %zu kernels: mem %.3f ms, smem %.3f ms (lds %.0f sts %.0f tma %.0f B/plane, canvas %d), comp %.3f ms, ctas %d warps %.0f"
            " | bytes %llu threads %d smemB %d need %d pts %d thrld %d depth %d u %d pair %d\n",
            L.kernels.size(), t_mem * 1e3, t_smem * 1e3, cv.lds_bytes, cv.sts_bytes, cv.tma_bytes, int(cv.ok), t_comp * 1e3, ctas, warps,
            (unsigned long long)bytes, L.threads, L.smem, need, L.pts, L.thrld, L.depth, L.zunroll, int(pair));
  return std::max(t_mem, t_smem / 0.7) + t_issue + 5e-6;
}

void check_target(const kf_target* t) {
  if (!t) fail(KF_E_ARG, "null target");
  if (t->tile[0] < 1 || t->tile[1] < 1 || t->tile[2] < 0 || t->tile[0] > 224 || t->tile[1] > 224)
    fail(KF_E_ARG, "tile must be TX,TY in [1,224], TZ >= 0");
  if (t->max_halo < 0 || t->max_halo > 16) fail(KF_E_ARG, "max_halo must be in [0,16] (TMA box <= 256)");
  if (t->tile[0] % 4) fail(KF_E_ARG, "tile TX must be a multiple of 4 (16-byte aligned TMA boxes)");
  if (t->stages < 2 || t->stages > 8) fail(KF_E_ARG, "stages must be in [2, 8]");
  if (t->zunroll < 1 || t->zunroll > 4) fail(KF_E_ARG, "zunroll must be in [1, 4]");
  if (t->ringunroll < 0 || t->ringunroll > 1) fail(KF_E_ARG, "ringunroll must be 0 or 1");
  if (t->ghostwrite < 0 || t->ghostwrite > 1) fail(KF_E_ARG, "ghostwrite must be 0 or 1");
  if (t->minblocks < -1 || t->minblocks > 32) fail(KF_E_ARG, "minblocks must be in [-1, 32]");
  if (t->skew < 0 || t->skew > 1) fail(KF_E_ARG, "skew must be 0 or 1");
  if (t->canvas_ld < 0 || t->canvas_ld > 1) fail(KF_E_ARG, "canvas_ld must be 0 or 1");
  if (t->pair_zq < 0 || t->pair_zq > 1) fail(KF_E_ARG, "pair_zq must be 0 or 1");
  if (t->inline_xy < 0 || t->inline_xy > 2) fail(KF_E_ARG, "inline_xy must be 0, 1 or 2");
  if (t->pblock[0] < 1 || t->pblock[0] > 4 || t->pblock[1] < 1 || t->pblock[1] > 4)
    fail(KF_E_ARG, "pblock must be in [1, 4] x [1, 4]");
  if (t->threads < 32 || t->threads > 1024 || t->threads % 32) fail(KF_E_ARG, "threads must be a multiple of 32 in [32,1024]");
  if (!(t->hbm_bytes_per_s > 0)) fail(KF_E_ARG, "hbm_bytes_per_s must be > 0");
}

}  // namespace kf

using namespace kf;

extern "C" {

kf_status kf_plan_canonical(const int32_t* plan, int32_t n, int32_t* out, int32_t* m) {
  KF_TRY({
    if (!plan || !out || n < 0) fail(KF_E_ARG, "null argument");
    std::map<int, int> mp;
    std::vector<int32_t> r(n);
    for (int i = 0; i < n; i++) {
      if (plan[i] < 0) fail(KF_E_ILLEGAL_PLAN, "negative label");
      auto it = mp.find(plan[i]);
      if (it == mp.end()) it = mp.emplace(plan[i], int(mp.size())).first;
      r[i] = it->second;
    }
    std::copy(r.begin(), r.end(), out);
    if (m) *m = int(mp.size());
  });
}

kf_status kf_plan_validate(const kf_program* prog, const int32_t* plan, const kf_target* target, kf_violation* why) {
  try {
    if (!prog || !plan) fail(KF_E_ARG, "null argument");
    check_target(target);
    const Program& p = prog->p;
    for (int k = 0; k < p.nk; k++)
      if (plan[k] < 0) {
        if (why) *why = kf_violation{KF_V_PARTITION, -1, k, -1, -1};
        set_error("V1 PARTITION: kernel " + std::to_string(k) + " has no group");
        return KF_E_ILLEGAL_PLAN;
      }
    Plan pl = make_plan(p, plan);
    kf_violation w{};
    int code = validate_plan(p, pl, *target, &w);
    if (why) *why = w;
    if (code != KF_V_OK) {
      static const char* names[] = {"OK", "V1 PARTITION", "V2 KINSHIP", "V3 CONVEX", "V4 CYCLE",
                                    "V5 HAZARD", "V6 HALO", "V7 SMEM", "V8 REGS"};
      set_error(std::string(names[code]) + " in group " + std::to_string(w.group));
      return KF_E_ILLEGAL_PLAN;
    }
    return KF_OK;
  } catch (const Error& e) {
    set_error(e.msg);
    return e.st;
  } catch (const std::exception& e) {
    set_error(e.what());
    return KF_E_ARG;
  }
}

kf_status kf_project(const kf_program* prog, const int32_t* plan, const kf_target* target, kf_group_proj* per_group,
                     int32_t cap, int32_t* m, uint64_t* bytes_total, double* t_total_s) {
  KF_TRY({
    if (!prog || !plan) fail(KF_E_ARG, "null argument");
    check_target(target);
    const Program& p = prog->p;
    Plan pl = make_plan(p, plan);
    if (cap > 0 && !per_group) fail(KF_E_ARG, "per_group is NULL");
    uint64_t tot = 0;
    double tt = 0.0;
    std::vector<kf_group_proj> res;
    for (int gi = 0; gi < pl.m; gi++) {
      const auto& g = pl.groups[gi];
      kf_group_proj r{};
      group_bytes(p, g, &r.bytes_read, &r.bytes_written);
      GroupLowering L = lower_group(p, g, *target);
      r.smem_bytes = uint32_t(L.smem);
      r.regs_est = uint32_t(L.regs);
      r.n_kernels = int(g.size());
      uint64_t unit = uint64_t(p.npts) * p.es;
      double halo = 0.0;
      for (auto& rg : L.rings)
        if (rg.live_in)
          halo += double(unit) * (double(rg.wx) * rg.hy / (double(L.tile[0]) * L.tile[1]) - 1.0);
      r.halo_bytes_est = uint64_t(std::max(0.0, halo));
      if (g.size() >= 2) {
        uint64_t alone = 0;
        for (int k : g) alone += group_bytes(p, std::vector<int>{k}, nullptr, nullptr);
        r.unprofitable = (r.bytes_read + r.bytes_written) >= alone;
      }
      r.t_s = double(r.bytes_read + r.bytes_written) / target->hbm_bytes_per_s;
      r.t_model_s = model_time(p, L, *target, r.bytes_read + r.bytes_written);
      tot += r.bytes_read + r.bytes_written;
      tt += r.t_s;
      res.push_back(r);
    }
    for (int i = 0; i < int(res.size()) && i < cap; i++) per_group[i] = res[i];
    if (m) *m = pl.m;
    if (bytes_total) *bytes_total = tot;
    if (t_total_s) *t_total_s = tt;
  });
}

kf_status kf_group_schedule(const kf_program* prog, const int32_t* plan, const kf_target* target, int32_t group,
                            kf_kernel_sched* out, int32_t cap, int32_t* n) {
  KF_TRY({
    if (!prog || !plan || !n) fail(KF_E_ARG, "null argument");
    check_target(target);
    const Program& p = prog->p;
    Plan pl = make_plan(p, plan);
    if (group < 0 || group >= pl.m) fail(KF_E_ARG, "group out of range");
    GroupLowering L = lower_group(p, pl.groups[group], *target);
    int i = 0;
    for (int k : L.kernels) {
      if (i < cap && out) {
        kf_kernel_sched s{};
        const Ext& e = L.ext.at(k);
        s.kernel = k;
        s.alive = e.alive;
        s.delay = e.alive ? L.delay.at(k) : -1;
        for (int a = 0; a < 3; a++) { s.elo[a] = e.elo[a]; s.ehi[a] = e.ehi[a]; }
        out[i] = s;
      }
      i++;
    }
    *n = i;
  });
}

}  // extern "C"

// ---------------------------------------------------------------- paper Eq. 2-10 (NEXT-2)
// The paper's codeless upper-bound projection for one new kernel, evaluated from
// the Table III / Table IV metadata exactly as printed.  Used to reproduce the worked example
// (B_Sh = 688, P_MemBound = 29.688 GFLOPS); not the B200 search objective (R22).
extern "C" kf_status kf_paper_projection(const kf_paper_meta* m, kf_paper_proj* out) {
  KF_TRY({
    if (!m || !out) fail(KF_E_ARG, "null argument");
    if (m->thr <= 0 || m->blocks <= 0 || m->shared_arrays <= 0 || m->gmem_bw_gbs <= 0 || m->elem_bytes <= 0)
      fail(KF_E_ARG, "thr, blocks, shared_arrays, gmem_bw_gbs, elem_bytes must be > 0");
    kf_paper_proj r{};
    const int c = m->halo ? 1 : 0;
    r.h_th = (m->hal + m->thr - 1) / m->thr;                                   // H_TH = ceil(Hal/Thr)
    const double denom = double(1 + c * r.h_th) * m->shared_arrays;
    r.b_sh = double(m->t_b) * m->blocks_smx / denom;                            // Eq. 8
    r.b_eff = r.b_sh * m->smx / (double(m->thr) * m->blocks);                   // B_eff
    r.p_membound_gflops = r.b_eff * m->gmem_bw_gbs / m->elem_bytes;             // Eq. 9 ("8" = fp64 bytes, R14)
    const double flops = m->fl_unfused_sum + m->flop_halo_sum * m->hal / (double(m->blocks) * m->thr);
    r.t_pro_s = flops * 1e-9 / r.p_membound_gflops;                             // Eq. 10 (R12)
    // constraints
    const double regs_blocking = m->regfac * m->max_thread_load + c * r.h_th + 1;   // Eq. 4 lower bound
    const double r_fetch = 1 + c * r.h_th;                                          // Eq. 5
    r.eq2_ok = m->r_t <= m->r_max;
    r.eq3_ok = double(m->blocks_smx) * m->thr * m->r_t <= m->r_smx;
    r.eq6_ok = r_fetch + regs_blocking + m->r_adr < m->r_t && m->r_t <= m->r_max;
    r.eq7_ok = double(1 + c * r.h_th) * m->t_b * m->blocks_smx * m->shared_arrays * m->elem_bytes + m->b_conf <= m->sh_smx;
    *out = r;
  });
}
