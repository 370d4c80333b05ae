// Program ingest and dependency analysis (hot-path row a1).
//
// Builds, from the explicit program description, the paper's data-dependency graph
// (DDG: kernels and arrays with read/write edges), the array classes,
// the order-of-execution graph with relaxation of expandable arrays by redundant copies
// (P:53), its transitive closure, the sharing sets and kinship adjacency
// (Table II) and per-array step liveness (R15).
#include <algorithm>
#include <cmath>
#include <cstring>
#include <sstream>

#include "kf_internal.hpp"

namespace kf {

static thread_local std::string g_last_error;

void set_error(const std::string& msg) { g_last_error = msg; }
[[noreturn]] void fail(kf_status st, const std::string& msg) { throw Error{st, msg}; }

bool Kernel::writes_array(int x) const { return std::find(writes.begin(), writes.end(), x) != writes.end(); }

int Program::vr(int k, int x) const {
  const auto& w = writers[x];
  return int(std::lower_bound(w.begin(), w.end(), k) - w.begin());
}

std::vector<int> Program::readers_of_version(int x, int v) const {
  std::vector<int> out;
  for (int k : readers[x])
    if (vr(k, x) == v) out.push_back(k);
  return out;
}

static int rpn_depth(const std::vector<Insn>& rpn, std::string* err) {
  int d = 0, m = 0;
  for (const auto& in : rpn) {
    switch (in.op) {
      case KF_OP_CONST: case KF_OP_PARAM: case KF_OP_LOAD: d++; break;
      case KF_OP_NEG: case KF_OP_ABS: case KF_OP_SQRT:
        if (d < 1) { *err = "unary op on empty stack"; return -1; }
        break;
      case KF_OP_ADD: case KF_OP_SUB: case KF_OP_MUL: case KF_OP_DIV: case KF_OP_MIN: case KF_OP_MAX:
        if (d < 2) { *err = "binary op needs two operands"; return -1; }
        d--;
        break;
      default: *err = "unknown opcode " + std::to_string(in.op); return -1;
    }
    m = std::max(m, d);
  }
  if (d != 1) { *err = "RPN must leave exactly one value (left " + std::to_string(d) + ")"; return -1; }
  return m;
}

static int64_t roundup(int64_t a, int64_t b) { return (a + b - 1) / b * b; }

void build_program(const kf_program_desc* d, Program& p) {
  if (!d) fail(KF_E_ARG, "null program description");
  if (d->dtype != KF_F32 && d->dtype != KF_F64) fail(KF_E_PROGRAM, "dtype must be KF_F32 or KF_F64");
  p.dtype = d->dtype;
  p.es = d->dtype == KF_F32 ? 4 : 8;
  for (int a = 0; a < 3; a++) {
    if (d->n[a] < 1) fail(KF_E_PROGRAM, "grid extent n[" + std::to_string(a) + "] must be >= 1");
    if (d->ghost[a] < 0 || d->ghost[a] > 64) fail(KF_E_PROGRAM, "ghost width must be in [0, 64]");
    if (d->bc[a] != KF_BC_FROZEN && d->bc[a] != KF_BC_PERIODIC) fail(KF_E_PROGRAM, "bad boundary condition");
    p.n[a] = d->n[a];
    p.ghost[a] = d->ghost[a];
    p.bc[a] = d->bc[a];
  }
  if (d->n_arrays < 1 || !d->arrays) fail(KF_E_PROGRAM, "program needs >= 1 array");
  if (d->n_kernels < 1 || !d->kernels) fail(KF_E_PROGRAM, "program needs >= 1 kernel");
  if (d->n_params < 0) fail(KF_E_PROGRAM, "n_params < 0");
  if (d->flags & ~7u) fail(KF_E_PROGRAM, "unknown program flags");
  p.na = d->n_arrays;
  p.nk = d->n_kernels;
  p.n_params = d->n_params;
  p.flags = d->flags;
  for (int x = 0; x < p.na; x++) {
    p.array_names.push_back(d->arrays[x].name ? d->arrays[x].name : ("a" + std::to_string(x)));
    if (d->arrays[x].flags & ~3u) fail(KF_E_PROGRAM, "unknown array flags on " + p.array_names.back());
    p.array_flags.push_back(d->arrays[x].flags);
  }
  for (int k = 0; k < p.nk; k++) {
    const kf_kernel_desc& kd = d->kernels[k];
    Kernel K;
    K.name = kd.name ? kd.name : ("k" + std::to_string(k));
    auto where = [&](int s) { return "kernel " + std::to_string(k) + " (" + K.name + ") statement " + std::to_string(s) + ": "; };
    if (kd.n_stmt < 1 || !kd.stmt) fail(KF_E_PROGRAM, "kernel " + K.name + " has no statements");
    std::set<int> outs;
    std::map<int, std::set<Off>> rd;
    for (int s = 0; s < kd.n_stmt; s++) {
      const kf_stmt& sd = kd.stmt[s];
      if (sd.out_array < 0 || sd.out_array >= p.na) fail(KF_E_PROGRAM, where(s) + "output array out of range");
      if (!outs.insert(sd.out_array).second) fail(KF_E_PROGRAM, where(s) + "two statements write the same array (R1)");
      if (p.array_flags[sd.out_array] & KF_ARRAY_READONLY)
        fail(KF_E_PROGRAM, where(s) + "writes READONLY array " + p.array_names[sd.out_array]);
      if (sd.n_insn < 1 || !sd.insn) fail(KF_E_PROGRAM, where(s) + "empty RPN");
      Stmt S;
      S.out = sd.out_array;
      for (int i = 0; i < sd.n_insn; i++) {
        const kf_insn& in = sd.insn[i];
        Insn I{in.op, in.arg, {in.d[0], in.d[1], in.d[2]}, in.imm};
        if (in.op == KF_OP_LOAD) {
          if (in.arg < 0 || in.arg >= p.na) fail(KF_E_PROGRAM, where(s) + "LOAD array out of range");
          for (int a = 0; a < 3; a++)
            if (std::abs(int(in.d[a])) > p.ghost[a])
              fail(KF_E_PROGRAM, where(s) + "offset exceeds ghost width on axis " + std::to_string(a));
          rd[in.arg].insert(I.d);
        } else if (in.op == KF_OP_PARAM) {
          if (in.arg < 0 || in.arg >= p.n_params) fail(KF_E_PROGRAM, where(s) + "PARAM index out of range");
        } else {
          I.arg = 0;
          I.d = {0, 0, 0};
        }
        if (in.op != KF_OP_CONST) I.imm = 0.0;
        S.rpn.push_back(I);
      }
      std::string err;
      S.depth = rpn_depth(S.rpn, &err);
      if (S.depth < 0) fail(KF_E_PROGRAM, where(s) + err);
      K.depth = std::max(K.depth, S.depth);
      K.writes.push_back(S.out);
      K.stmts.push_back(std::move(S));
    }
    for (auto& [x, offs] : rd) K.reads[x] = std::vector<Off>(offs.begin(), offs.end());
    // R1: an array written by the kernel may be read only at offset (0,0,0)
    for (int x : K.writes) {
      auto it = K.reads.find(x);
      if (it != K.reads.end())
        for (const Off& o : it->second)
          if (o[0] || o[1] || o[2])
            fail(KF_E_PROGRAM, "kernel " + K.name + " reads array " + p.array_names[x] +
                                   " at a nonzero offset while writing it (R1; split the kernel)");
    }
    // optional declared footprint must equal the LOAD set
    if (kd.n_reads > 0) {
      if (!kd.reads) fail(KF_E_PROGRAM, "kernel " + K.name + ": n_reads > 0 but reads == NULL");
      std::map<int, std::set<Off>> decl;
      for (int r = 0; r < kd.n_reads; r++) {
        const kf_access& ac = kd.reads[r];
        if (ac.array < 0 || ac.array >= p.na) fail(KF_E_PROGRAM, "kernel " + K.name + ": declared read out of range");
        decl[ac.array].insert(Off{ac.d[0], ac.d[1], ac.d[2]});
      }
      if (decl != rd) fail(KF_E_PROGRAM, "kernel " + K.name + ": declared footprint differs from its LOADs");
    }
    for (auto& [x, _] : K.reads) K.touched.insert(x);
    for (int x : K.writes) K.touched.insert(x);
    p.kernels.push_back(std::move(K));
  }

  // ---- DDG: readers / writers of each array
  p.writers.assign(p.na, {});
  p.readers.assign(p.na, {});
  for (int k = 0; k < p.nk; k++) {
    for (auto& [x, _] : p.kernels[k].reads) p.readers[x].push_back(k);
    for (int x : p.kernels[k].writes) p.writers[x].push_back(k);
  }
  p.ver_read.assign(p.nk, {});
  for (int k = 0; k < p.nk; k++)
    for (int x : p.kernels[k].touched) p.ver_read[k][x] = p.vr(k, x);
  // ---- array classes
  p.cls.assign(p.na, KF_CLS_RO);
  for (int x = 0; x < p.na; x++) {
    size_t nw = p.writers[x].size(), nr = p.readers[x].size();
    p.cls[x] = nw == 0 ? KF_CLS_RO : (nr == 0 ? KF_CLS_WO : (nw >= 2 ? KF_CLS_EXPANDABLE : KF_CLS_RW));
  }
  // ---- relaxation by redundant arrays
  p.relaxed.assign(p.na, 0);
  for (int x = 0; x < p.na; x++) {
    if (p.flags & KF_PROG_RELAX_ALL) p.relaxed[x] = !p.writers[x].empty();
    else if (p.flags & KF_PROG_RELAX_EXPANDABLE) p.relaxed[x] = p.cls[x] == KF_CLS_EXPANDABLE;
  }
  // ---- step liveness (R15)
  p.step_live.assign(p.na, 0);
  for (int x = 0; x < p.na; x++) {
    int w = int(p.writers[x].size());
    if (w == 0) continue;
    bool up = !p.readers_of_version(x, 0).empty();
    bool out = p.array_flags[x] & KF_ARRAY_OUTPUT;
    bool unread_final = p.readers_of_version(x, w).empty();
    p.step_live[x] = up || out || unread_final;
  }
  // ---- order-of-execution graph, canonical nearest-access edges (R2)
  std::set<std::array<int, 4>> es;   // (dst, src, kind, array)
  for (int b = 0; b < p.nk; b++) {
    for (auto& [x, _] : p.kernels[b].reads) {
      int v = p.vr(b, x);
      if (v >= 1) es.insert({b, p.writer_of(x, v), KF_EDGE_RAW, x});
    }
    for (int x : p.kernels[b].writes) {
      if (p.relaxed[x]) continue;
      int v = p.vr(b, x);
      if (v >= 1) es.insert({b, p.writer_of(x, v), KF_EDGE_WAW, x});
      for (int a : p.readers_of_version(x, v))
        if (a < b) es.insert({b, a, KF_EDGE_WAR, x});
    }
  }
  for (auto& e : es) p.edges.push_back(kf_edge{e[1], e[0], e[2], e[3]});
  // ---- transitive closure (bitsets, kernels are topologically numbered: src < dst)
  int words = (p.nk + 63) / 64;
  p.reach.assign(p.nk, std::vector<uint64_t>(words, 0));
  std::vector<std::vector<int>> succ(p.nk);
  for (auto& e : p.edges) succ[e.src].push_back(e.dst);
  for (int a = p.nk - 1; a >= 0; a--)
    for (int b : succ[a]) {
      p.reach[a][b >> 6] |= 1ull << (b & 63);
      for (int w = 0; w < words; w++) p.reach[a][w] |= p.reach[b][w];
    }
  // ---- sharing adjacency (Table II)
  p.share.assign(p.nk, std::vector<char>(p.nk, 0));
  for (int a = 0; a < p.nk; a++)
    for (int b = 0; b < p.nk; b++) {
      if (a == b) continue;
      for (int x : p.kernels[a].touched)
        if (p.kernels[b].touched.count(x)) { p.share[a][b] = 1; break; }
    }
  // ---- device layout (P:82 horizontal padding; R13)
  int align = 128 / p.es;
  kf_layout L{};
  L.xoff = int(roundup(p.ghost[0], align));
  L.pitch = roundup(L.xoff + p.n[0] + p.ghost[0], align);
  L.rows = p.n[1] + 2 * p.ghost[1];
  L.plane = L.pitch * L.rows;
  L.origin = int64_t(p.ghost[2]) * L.plane + int64_t(p.ghost[1]) * L.pitch + L.xoff;
  L.elems = L.plane * (p.n[2] + 2 * p.ghost[2]);
  p.layout = L;
  p.npts = p.n[0] * p.n[1] * p.n[2];
}

}  // namespace kf

using namespace kf;

extern "C" {

const char* kf_last_error(void) { return g_last_error.c_str(); }
const char* kf_version(void) { return "kf 0.1 (sm_100a, NVRTC JIT, TMA+mbarrier group kernels)"; }

kf_status kf_program_create(const kf_program_desc* desc, kf_program** out) {
  KF_TRY({
    if (!out) fail(KF_E_ARG, "out is NULL");
    auto h = std::make_unique<kf_program>();
    build_program(desc, h->p);
    *out = h.release();
  });
}

void kf_program_destroy(kf_program* prog) { delete prog; }

kf_status kf_program_get_info(const kf_program* prog, kf_program_info* out) {
  KF_TRY({
    if (!prog || !out) fail(KF_E_ARG, "null argument");
    const Program& p = prog->p;
    kf_program_info r{};
    r.n_kernels = p.nk;
    r.n_arrays = p.na;
    r.n_edges = int(p.edges.size());
    r.es = p.es;
    r.npts = p.npts;
    for (char c : p.relaxed) r.n_relaxed += c ? 1 : 0;
    *out = r;
  });
}

kf_status kf_program_edges(const kf_program* prog, kf_edge* out, int32_t cap, int32_t* n) {
  KF_TRY({
    if (!prog || !n || (cap > 0 && !out)) fail(KF_E_ARG, "null argument");
    const auto& e = prog->p.edges;
    for (int i = 0; i < int(e.size()) && i < cap; i++) out[i] = e[i];
    *n = int(e.size());
  });
}

kf_status kf_program_reach(const kf_program* prog, uint8_t* reach) {
  KF_TRY({
    if (!prog || !reach) fail(KF_E_ARG, "null argument");
    const Program& p = prog->p;
    for (int a = 0; a < p.nk; a++)
      for (int b = 0; b < p.nk; b++) reach[a * p.nk + b] = p.reaches(a, b) ? 1 : 0;
  });
}

kf_status kf_program_array_class(const kf_program* prog, int32_t* cls) {
  KF_TRY({
    if (!prog || !cls) fail(KF_E_ARG, "null argument");
    const Program& p = prog->p;
    for (int x = 0; x < p.na; x++) cls[x] = p.cls[x];
  });
}

kf_status kf_program_array_info(const kf_program* prog, int32_t x, kf_array_info* out) {
  KF_TRY({
    if (!prog || !out) fail(KF_E_ARG, "null argument");
    const Program& p = prog->p;
    if (x < 0 || x >= p.na) fail(KF_E_ARG, "array index out of range");
    kf_array_info r{};
    r.cls = p.cls[x];
    r.n_writers = int(p.writers[x].size());
    r.n_readers = int(p.readers[x].size());
    r.relaxed = p.relaxed[x];
    r.step_live = p.step_live[x];
    r.upward_exposed = p.readers_of_version(x, 0).empty() ? 0 : 1;
    *out = r;
  });
}

kf_status kf_program_kinship(const kf_program* prog, int32_t a, int32_t b, const int32_t* group,
                             int32_t group_n, int32_t* degree) {
  KF_TRY({
    if (!prog || !degree || (group_n > 0 && !group)) fail(KF_E_ARG, "null argument");
    const Program& p = prog->p;
    std::vector<int> g(group, group + group_n);
    for (int k : g)
      if (k < 0 || k >= p.nk) fail(KF_E_ARG, "kernel index out of range");
    if (a == b) { *degree = 0; return KF_OK; }
    // BFS over the sharing graph induced on the group (Table II; R5)
    std::map<int, int> dist;
    dist[a] = 0;
    std::vector<int> fr{a};
    while (!fr.empty()) {
      std::vector<int> nx;
      for (int u : fr)
        for (int w : g)
          if (!dist.count(w) && p.share[u][w]) { dist[w] = dist[u] + 1; nx.push_back(w); }
      fr = nx;
    }
    *degree = dist.count(b) ? dist[b] : 0;
  });
}

kf_status kf_array_layout(const kf_program* prog, kf_layout* out) {
  KF_TRY({
    if (!prog || !out) fail(KF_E_ARG, "null argument");
    *out = prog->p.layout;
  });
}

kf_status kf_target_b200(kf_target* out) {
  KF_TRY({
    if (!out) fail(KF_E_ARG, "null argument");
    kf_target t{};
    t.hbm_bytes_per_s = 8.0e12;
    t.smem_per_block = 232448;
    t.regs_per_thread_max = 255;
    t.n_sm = 148;
    t.tile[0] = 64; t.tile[1] = 4; t.tile[2] = 0;
    t.stages = 2;
    t.threads = 256;
    t.max_halo = 16;
    t.internal_axes = 0;
    t.zunroll = 1;
    t.pblock[0] = 1;
    t.pblock[1] = 1;
    t.ringunroll = 0;
    t.ghostwrite = 0;   // measured slower than the fill kernels on B200 (tools/sweep.py, round 1)
    t.minblocks = 0;
    t.skew = 0;
    t.canvas_ld = 1;
    t.pair_zq = 1;
    t.inline_xy = 1;   // measured: -1.6 % step, flux groups -2 .. -6 % (profiles/round2_summary.md)
    *out = t;
  });
}

}  // extern "C"
