// Internal data structures of the kf host library (not part of the ABI).
// Host-side C++: program IR, DAG, lowering, legality, projection, search, codegen.
// Cites PAPER.md lines as P:n; readings Rn are in DESIGN.md.
#pragma once

#include <array>
#include <cstdlib>
#include <cstdint>
#include <map>
#include <memory>
#include <mutex>
#include <set>
#include <string>
#include <vector>

#include "kf.h"

namespace kf {

struct Error {
  kf_status st;
  std::string msg;
};
[[noreturn]] void fail(kf_status st, const std::string& msg);
void set_error(const std::string& msg);

using Off = std::array<int, 3>;

struct Insn {
  int op, arg;
  Off d;
  double imm;
};
struct Stmt {
  int out;
  std::vector<Insn> rpn;
  int depth;
};
struct Kernel {
  std::string name;
  std::vector<Stmt> stmts;
  std::map<int, std::vector<Off>> reads;  // array -> sorted distinct offsets (footprint)
  std::vector<int> writes;                // arrays written (statement order)
  std::set<int> touched;
  int depth = 0;                          // deepest RPN stack
  bool writes_array(int x) const;
};

// A version of an array inside one step: v = 0 is the value at step start, v >= 1 is
// produced by the v-th writer in program order.
struct Ver {
  int x, v;
  bool operator<(const Ver& o) const { return x != o.x ? x < o.x : v < o.v; }
  bool operator==(const Ver& o) const { return x == o.x && v == o.v; }
};

struct Program {
  int dtype = 0, es = 4;
  int64_t n[3] = {0, 0, 0};
  int ghost[3] = {0, 0, 0};
  int bc[3] = {0, 0, 0};
  std::vector<std::string> array_names;
  std::vector<uint32_t> array_flags;
  std::vector<Kernel> kernels;
  int n_params = 0;
  uint32_t flags = 0;

  // ---- derived (program.cpp)
  int nk = 0, na = 0;
  std::vector<std::vector<int>> writers;      // per array, writing kernels ascending
  std::vector<std::vector<int>> readers;      // per array, reading kernels ascending
  std::vector<std::map<int, int>> ver_read;   // per kernel: array -> version read
  std::vector<int> cls;                       // kf_array_class
  std::vector<char> relaxed, step_live;
  std::vector<kf_edge> edges;                 // canonical, sorted
  std::vector<std::vector<uint64_t>> reach;   // bitset rows
  std::vector<std::vector<char>> share;       // sharing adjacency
  kf_layout layout{};
  int64_t npts = 0;

  bool reaches(int a, int b) const { return (reach[a][b >> 6] >> (b & 63)) & 1ull; }
  int writer_of(int x, int v) const { return writers[x][v - 1]; }
  int vr(int k, int x) const;                 // version of x current before kernel k
  int vw(int k, int x) const { return vr(k, x) + 1; }   // version kernel k writes
  std::vector<int> readers_of_version(int x, int v) const;
};

void build_program(const kf_program_desc* d, Program& p);   // throws Error

// ---------------------------------------------------------------- plans / lowering
struct Plan {
  std::vector<int> label;                 // canonical labels
  std::vector<std::vector<int>> groups;   // kernels per group, ascending
  int m = 0;
};
Plan make_plan(const Program& p, const int32_t* labels);   // V1 checked by caller

struct Ext {
  bool alive = false;
  int elo[3] = {0, 0, 0}, ehi[3] = {0, 0, 0};
};

// SMEM-resident ring of a version inside a fused group (lowering a3).
struct Ring {
  Ver ver;
  bool live_in = false;   // staged by TMA from HBM; else produced in the group
  int producer = -1;      // kernel producing it (in-group rings)
  int blo[3], bhi[3];     // box extents beyond T (xy used for SMEM; z for plane range)
  int ax_lo = 0;          // x extent below T of the SMEM box: live-in boxes start on a 16-byte
                          // boundary (TMA faults on unaligned x starts, measured on B200)
  int wx, hy, px;         // box width, height, padded row pitch (elements)
  int plane_bytes;        // roundup(px*hy*es, 128)
  int slots;              // ring depth
  int A = 0, B = 0;       // live-in: newest/oldest plane offset needed at iteration t
  int smem_off = 0;       // byte offset in dynamic SMEM
};

struct GroupLowering;
// a11 overlap: the tile rectangle at least one ghost width inside the local domain (x, y)
struct Split { bool ok = false; int ix0 = 0, ix1 = 0, iy0 = 0, iy1 = 0; int interior_units = 0, boundary_units = 0; };

struct GroupLowering {
  std::vector<int> kernels;               // program order
  std::map<int, Ext> ext;                 // per kernel
  std::map<int, int> delay;               // per alive kernel
  std::vector<Ver> live_in, live_out;
  std::set<Ver> live_out_set;
  std::vector<Ring> rings;
  int smem = 0, regs = 0, depth = 0;
  int thrld = 0, pts = 1;                 // register model inputs (V8): values held, points per thread
  int mbar_off = 0;
  int tile[3];
  int stages = 2, threads = 256, zunroll = 1;
  int pblock[2] = {1, 1};   // points per thread in x, y (register blocking in the fast path)
  int ring_unroll = 0;      // 0, or N: every ring size a power of two dividing N, loop unrolled N times
  bool ghost_write = false; // live-out stores also write the periodic x/y ghost copies (no fills)
  int pair_zq = 1;          // pair canvas: z-column register queues (kf_target.pair_zq)
  int inline_xy = 0;        // pair canvas: readers recompute in-group versions at xy offsets
  int canvas_ld = 1;        // fast-iteration shared loads unpredicated where in bounds (kf_target.canvas_ld)
  int minblocks = 0;        // __launch_bounds__ min CTAs/SM: 0 auto (SMEM-limited), -1 none, n
  int ring_of(const Ver& v) const;        // index in rings or -1
};

std::vector<Ver> group_live_in(const Program& p, const std::vector<int>& g);
std::vector<Ver> group_live_out(const Program& p, const std::vector<int>& g);
GroupLowering lower_group(const Program& p, const std::vector<int>& g, const kf_target& t);
// Validation; returns code (0 ok) and fills why.
int validate_plan(const Program& p, const Plan& pl, const kf_target& t, kf_violation* why,
                  std::vector<GroupLowering>* lowered = nullptr);
// Same with one launch configuration per group (targets.size() == pl.m).
int validate_plan_groups(const Program& p, const Plan& pl, const std::vector<kf_target>& targets, kf_violation* why,
                         std::vector<GroupLowering>* lowered = nullptr);
std::vector<int> quotient_order(const Program& p, const Plan& pl);   // empty if cyclic
bool regs_ok(const GroupLowering& L, const kf_target& t);              // V8 (Eq. 2, Eq. 3)
int regs_limit(int threads);                                            // registers per thread of a CTA
int regs_cap(int threads, int m);                                       // ... with m CTAs per SM resident
int check_kinship(const Program& p, const std::vector<int>& g, int gi, kf_violation* why);
int check_convex(const Program& p, const std::vector<int>& g, int gi, kf_violation* why);
int check_hazard(const Program& p, const std::vector<int>& g, const GroupLowering& L, int gi, kf_violation* why);
int check_halo(const Program& p, const GroupLowering& L, const kf_target& t, int gi, kf_violation* why);
bool quotient_acyclic(const Program& p, const std::vector<int>& label, int m, int* first_bad);
void check_target(const kf_target* t);
uint64_t group_bytes(const Program& p, const std::vector<int>& g, uint64_t* rd, uint64_t* wr);
// Resource-aware projected time of one fused group (NEXT-2 direction, R22): HBM time of the
// compulsory bytes at the achievable copy rate, plus issue time of the recomputed regions.
double model_time(const Program& p, const GroupLowering& L, const kf_target& t, uint64_t bytes);

// ---------------------------------------------------------------- canvas (fast iterations)
// The fast iterations of a group kernel give each point of the canvas (bounding box of all
// extended regions) to one thread for every kernel; reads at xy offset 0 of a plane computed in
// the same iteration are forwarded in registers and identical shared loads are issued once.
struct CanvasKey {
  int ring, po, off;   // ring, plane offset from the stream position t, element offset from the canvas point
  bool operator<(const CanvasKey& o) const {
    return ring != o.ring ? ring < o.ring : po != o.po ? po < o.po : off < o.off;
  }
};
using Rect = std::array<int, 4>;   // canvas x0, x1, y0, y1 (half open)
struct CanvasPlan {
  bool ok = false;                 // one canvas point per thread (else the per-kernel fast path)
  int clo[2] = {0, 0}, chi[2] = {0, 0}, cw = 0, ch = 0, pts = 0, rounds = 1;
  std::set<Ver> need_sts;          // in-group versions still written to their SMEM ring
  std::vector<std::vector<int>> phases;   // kernels between barriers
  std::map<CanvasKey, Rect> krect; // shared loads and the rect of lanes that issue them
  double lds_bytes = 0, sts_bytes = 0, tma_bytes = 0;   // per fast iteration per U planes
  // pair mode (pblock 2x1, U = 1): a thread owns two x-adjacent canvas points whose pair starts on
  // an even (16-byte for fp64) element; shared loads/stores and live-out stores are 2-wide vectors
  bool pair = false;
  int lop = 0, hip = 0, cwp = 0;   // pair columns left of / right of the tile, per canvas row
  // pair mode with L.inline_xy: in-group versions whose readers recompute them at their xy
  // offsets instead of reading a shared-memory copy: version -> (producer, statement index)
  std::map<Ver, std::pair<int, int>> inl;
  bool inlined(const Program& p, int k, int x, const Off& d) const {
    return (d[0] != 0 || d[1] != 0) && inl.count(Ver{x, p.vr(k, x)}) > 0;
  }
};
bool canvas_forward(const Program& p, const GroupLowering& L, int k, int x, const Off& d, int uu, int* prod, int* up);
CanvasKey canvas_key(const Program& p, const GroupLowering& L, const CanvasPlan& c, int k, int x, const Off& d, int uu);
Rect canvas_rect(const GroupLowering& L, const CanvasPlan& c, int k);
CanvasPlan plan_canvas(const Program& p, const GroupLowering& L);

// ---------------------------------------------------------------- codegen
struct Codegen {
  std::string source;
  std::string name;
};
Codegen generate_group_kernel(const Program& p, const GroupLowering& L, int gid);
Split split_units(const Program& p, const GroupLowering& L);

}  // namespace kf

struct kf_program {
  kf::Program p;
  // kf_run state (kf_runtime.cpp): per-plan executors and the kf_dist_init context, freed with
  // the program
  void* run_cache = nullptr;
  void (*run_cache_free)(void*) = nullptr;
  ~kf_program() {
    if (run_cache && run_cache_free) run_cache_free(run_cache);
  }
};

#define KF_TRY(...)                                       \
  try {                                                   \
    __VA_ARGS__;                                               \
    return KF_OK;                                         \
  } catch (const Error& e) {                              \
    set_error(e.msg);                                     \
    return e.st;                                          \
  } catch (const std::bad_alloc&) {                       \
    set_error("host allocation failed");                  \
    return KF_E_OOM;                                      \
  } catch (const std::exception& e) {                     \
    set_error(std::string("internal error: ") + e.what()); \
    return KF_E_ARG;                                      \
  }

