// Canvas plan of a fused group's fast iterations (row a8): which reads are forwarded in
// registers, which versions still need their shared-memory ring, where barriers go, and which
// shared loads remain (one per distinct address).  Used by the code generator (kf_codegen.cpp)
// and by the resource-aware projection (model_time), so the model counts the shared-memory
// traffic the generated kernel actually issues.
#include <algorithm>
#include <functional>
#include <set>

#include "kf_internal.hpp"

namespace kf {

static bool in_group(const GroupLowering& L, int k) { return std::binary_search(L.kernels.begin(), L.kernels.end(), k); }

// A read of an in-group version at xy offset 0 of a plane its producer computes in the same
// iteration (sub-plane uu' = uu + dz - D_k + D_p in [0, U)) takes the producer's register.
bool canvas_forward(const Program& p, const GroupLowering& L, int k, int x, const Off& d, int uu, int* prod, int* up) {
  const int v = p.vr(k, x);
  if (v < 1 || d[0] != 0 || d[1] != 0) return false;
  const int pr = p.writer_of(x, v);
  if (!in_group(L, pr) || !L.ext.at(pr).alive) return false;
  const int u2 = uu + d[2] - L.delay.at(k) + L.delay.at(pr);
  if (u2 < 0 || u2 >= L.zunroll) return false;
  *prod = pr;
  *up = u2;
  return true;
}

CanvasKey canvas_key(const Program& p, const GroupLowering& L, const CanvasPlan& c, int k, int x, const Off& d, int uu) {
  const int ring = L.ring_of(Ver{x, p.vr(k, x)});
  const Ring& R = L.rings[ring];
  const int off = (d[1] + R.blo[1] - c.clo[1]) * R.px + (d[0] + R.ax_lo - c.clo[0]);
  return CanvasKey{ring, -L.delay.at(k) + d[2] + uu, off};
}

Rect canvas_rect(const GroupLowering& L, const CanvasPlan& c, int k) {
  const Ext& e = L.ext.at(k);
  const int ox = c.clo[0] - e.elo[0], oy = c.clo[1] - e.elo[1];
  return Rect{ox, ox + L.tile[0] + e.elo[0] + e.ehi[0], oy, oy + L.tile[1] + e.elo[1] + e.ehi[1]};
}

CanvasPlan plan_canvas(const Program& p, const GroupLowering& L) {
  CanvasPlan c;
  std::vector<int> alive;
  for (int k : L.kernels)
    if (L.ext.at(k).alive) alive.push_back(k);
  const int TX = L.tile[0], TY = L.tile[1], U = L.zunroll;
  for (int k : alive)
    for (int a = 0; a < 2; a++) {
      c.clo[a] = std::max(c.clo[a], L.ext.at(k).elo[a]);
      c.chi[a] = std::max(c.chi[a], L.ext.at(k).ehi[a]);
    }
  c.cw = TX + c.clo[0] + c.chi[0];
  c.ch = TY + c.clo[1] + c.chi[1];
  c.pts = c.cw * c.ch;
  c.rounds = (c.pts + L.threads - 1) / L.threads;
  // one canvas point per thread only: with several rounds the forwarded values of all rounds stay
  // live together (register pressure), and the per-kernel fast path is used instead
  c.ok = !alive.empty() && L.pblock[0] == 1 && L.pblock[1] == 1 && c.rounds == 1 && !getenv("KF_NO_CANVAS");
  // pair mode: pairs aligned to even tile-relative x (TX and NX even), so a pair never straddles
  // the tile or domain edge; one pair per thread
  if (!alive.empty() && L.pblock[0] == 2 && L.pblock[1] == 1 && U == 1 && TX % 2 == 0 && p.n[0] % 2 == 0 &&
      !getenv("KF_NO_CANVAS")) {
    c.lop = (c.clo[0] + 1) / 2;
    c.hip = (c.chi[0] + 1) / 2;
    c.cwp = TX / 2 + c.lop + c.hip;
    c.rounds = (c.cwp * c.ch + L.threads - 1) / L.threads;
    c.pair = c.ok = c.rounds == 1;
  }
  // Inline recompute (pair mode, L.inline_xy): an in-group version whose statement reads only
  // staged live-in versions, and whose every in-group reader runs in the same stream iteration
  // (equal delay) and reads it in its own plane (dz = 0), is recomputed by each reader at each xy
  // offset it reads (the same IEEE operations in the same order: the same bits) instead of being
  // stored to and re-read from shared memory behind a barrier.  The loads this adds lie in the
  // live-in boxes (a box covers the producer's region grown by its footprint, and the producer's
  // region covers its readers' regions grown by theirs).  Fast iterations only: the slow path
  // keeps the ring (same-iteration readers: its contents never cross iterations).
  if (c.pair && L.inline_xy)
    for (int level = 0; level < (L.inline_xy >= 2 ? 2 : 1); level++) {   // level 1 (inline_xy 2): statements that also read level-0 values
      std::map<Ver, std::pair<int, int>> add;
      for (int k : alive) {
        const Kernel& K = p.kernels[k];
        for (size_t si = 0; si < K.stmts.size(); si++) {
          const Ver V{K.stmts[si].out, p.vw(k, K.stmts[si].out)};
          if (L.ring_of(V) < 0 || c.inl.count(V)) continue;
          bool ok = true, any_xy = false;
          int nloads = 0;
          std::set<std::pair<int, int>> xy_offs;   // distinct nonzero xy offsets it is read at
          for (const Insn& in : K.stmts[si].rpn)
            if (in.op == KF_OP_LOAD) {
              nloads++;
              const Ver W{in.arg, p.vr(k, in.arg)};
              const int r = L.ring_of(W);
              if (r < 0 || !(L.rings[r].live_in || c.inl.count(W))) ok = false;
            }
          for (int c2 : alive) {
            auto it = p.kernels[c2].reads.find(V.x);
            if (c2 == k || it == p.kernels[c2].reads.end() || p.vr(c2, V.x) != V.v) continue;
            if (L.delay.at(c2) != L.delay.at(k)) ok = false;
            for (auto& d : it->second) {
              if (d[2] != 0) ok = false;
              if (d[0] != 0 || d[1] != 0) {
                any_xy = true;
                xy_offs.insert({d[0], d[1]});
              }
            }
          }
          (void)any_xy;   // (values read only at offset 0 join too: the inputs of level-1 values)
          // cost bound: a cheap producer read at few offsets (a flux read at i-1: 1 offset x 5
          // loads); a wide stencil of a wide stencil (S13 of S27: 12 x 27) stays in shared memory
          if (int(xy_offs.size()) * nloads > 16) ok = false;
          if (ok) add[V] = {k, int(si)};
        }
      }
      if (add.empty()) break;
      c.inl.insert(add.begin(), add.end());
    }
  // versions whose every in-group read is forwarded (or recomputed) need no shared-memory copy in
  // fast iterations
  for (int k : alive)
    for (auto& [x, offs] : p.kernels[k].reads) {
      const int v = p.vr(k, x);
      if (v < 1 || L.ring_of(Ver{x, v}) < 0 || L.rings[L.ring_of(Ver{x, v})].live_in) continue;
      for (auto& d : offs)
        for (int uu = 0; uu < U; uu++) {
          int pr, u2;
          if (!canvas_forward(p, L, k, x, d, uu, &pr, &u2) && !c.inlined(p, k, x, d)) c.need_sts.insert(Ver{x, v});
        }
    }
  // phases: a barrier only before a kernel that reads through shared memory a plane written (to
  // shared memory) earlier in this iteration
  {
    std::set<int> dirty;
    for (int k : alive) {
      const Kernel& K = p.kernels[k];
      bool need = false;
      for (auto& [x, offs] : K.reads) {
        const int v = p.vr(k, x);
        if (v < 1) continue;
        const int pr = p.writer_of(x, v);
        if (!dirty.count(pr)) continue;
        for (auto& d : offs)
          for (int uu = 0; uu < U; uu++) {
            int q, u2;
            if (canvas_forward(p, L, k, x, d, uu, &q, &u2) || c.inlined(p, k, x, d)) continue;
            if (L.delay.at(k) - d[2] - L.delay.at(pr) < U) need = true;
          }
      }
      if (need || c.phases.empty()) {
        c.phases.emplace_back();
        dirty.clear();
      }
      c.phases.back().push_back(k);
      for (int x : K.writes)
        if (c.need_sts.count(Ver{x, p.vw(k, x)})) dirty.insert(k);
    }
  }
  // shared loads: one per (ring, plane, offset from the canvas point), predicated on the bounding
  // box of the regions of the kernels reading it (which lies in the ring's box)
  for (int k : alive) {
    const Rect rk = canvas_rect(L, c, k);
    for (auto& [x, offs] : p.kernels[k].reads)
      for (auto& d : offs)
        for (int uu = 0; uu < U; uu++) {
          int pr, u2;
          if (canvas_forward(p, L, k, x, d, uu, &pr, &u2)) continue;
          auto add = [&](int kr, int xr, const Off& dr) {
            const CanvasKey key = canvas_key(p, L, c, kr, xr, dr, uu);
            auto it = c.krect.find(key);
            if (it == c.krect.end()) c.krect[key] = rk;
            else {
              auto& a = it->second;
              a = {std::min(a[0], rk[0]), std::max(a[1], rk[1]), std::min(a[2], rk[2]), std::max(a[3], rk[3])};
            }
          };
          // an inlined read: the producer's loads shifted by the read's offset, recursively
          std::function<void(int, int, const Off&)> expand = [&](int kr, int xr, const Off& dr) {
            int q, u3;
            if (c.inlined(p, kr, xr, dr)) {
              const auto& [pk, si] = c.inl.at(Ver{xr, p.vr(kr, xr)});
              for (const Insn& in : p.kernels[pk].stmts[si].rpn)
                if (in.op == KF_OP_LOAD) expand(pk, in.arg, Off{dr[0] + in.d[0], dr[1] + in.d[1], dr[2] + in.d[2]});
            } else if (!canvas_forward(p, L, kr, xr, dr, uu, &q, &u3)) {
              add(kr, xr, dr);
            }
          };
          expand(k, x, d);
        }
  }
  // shared-memory traffic of one fast iteration (U planes of one tile)
  const int es = p.es;
  for (auto& [key, rc] : c.krect) c.lds_bytes += double(rc[1] - rc[0]) * (rc[3] - rc[2]) * es;
  for (int k : alive)
    for (int x : p.kernels[k].writes)
      if (c.need_sts.count(Ver{x, p.vw(k, x)})) {
        const Rect rk = canvas_rect(L, c, k);
        c.sts_bytes += double(rk[1] - rk[0]) * (rk[3] - rk[2]) * es * U;
      }
  for (auto& r : L.rings)
    if (r.live_in) c.tma_bytes += double(r.wx) * r.hy * es * U;
  return c;
}

}  // namespace kf
