// Code generation of one fused-group kernel for sm_100a (rows a6-a9).
//
// One CUDA kernel per fused group ("new kernel" F_j).  The template is
// written for Blackwell, not translated from the paper's Kepler listings (Fig. 3):
//   * a CTA owns an xy tile TX x TY and streams z (2.5-D blocking, the temporal
//     blocking of [15] cited at P:107) over a chunk of TZ planes;
//   * live-in arrays arrive by TMA (cp.async.bulk.tensor.3d) one plane per iteration
//     into per-array SMEM rings, completion tracked by an S-stage mbarrier ring (the
//     "specialized warps" of P:107 / [16] become the TMA engine);
//   * kernel k of the group runs D_k planes behind the stream front (z delay) on its
//     extended region E(k) (halo recompute); intermediates that later kernels
//     read stay in SMEM rings and never touch HBM unless live-out;
//   * live-out versions are stored from registers on T ∩ interior only;
//   * FROZEN boundaries: points of E(k) outside the interior take the stored ghost
//     values (R9), so fused results equal the unfused program bit for bit.
// Each RPN node becomes one IEEE operation, in order; NVRTC runs with --fmad=false.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <sstream>

#include "kf_internal.hpp"

namespace kf {

// Tile rectangle [ix0, ix1) x [iy0, iy1) whose tiles lie at least the ghost width inside the
// local domain on x and y (a11: they run while a halo exchange is in flight).
Split split_units(const Program& p, const GroupLowering& L) {
  Split s;
  const int TX = L.tile[0], TY = L.tile[1];
  const int NTX = int((p.n[0] + TX - 1) / TX), NTY = int((p.n[1] + TY - 1) / TY);
  const int gx = p.ghost[0], gy = p.ghost[1];
  s.ix0 = (gx + TX - 1) / TX;
  s.iy0 = (gy + TY - 1) / TY;
  s.ix1 = p.n[0] - gx - TX >= 0 ? int((p.n[0] - gx - TX) / TX) + 1 : 0;
  s.iy1 = p.n[1] - gy - TY >= 0 ? int((p.n[1] - gy - TY) / TY) + 1 : 0;
  s.ix1 = std::min(s.ix1, NTX);
  s.iy1 = std::min(s.iy1, NTY);
  s.ok = s.ix1 > s.ix0 && s.iy1 > s.iy0 && (s.ix1 - s.ix0) * (s.iy1 - s.iy0) < NTX * NTY;
  const int TZ = L.tile[2] > 0 ? std::min<int>(L.tile[2], int(p.n[2])) : int(p.n[2]);
  const int NTZ = int((p.n[2] + TZ - 1) / TZ);
  s.interior_units = s.ok ? (s.ix1 - s.ix0) * (s.iy1 - s.iy0) * NTZ : 0;
  s.boundary_units = s.ok ? NTX * NTY * NTZ - s.interior_units : 0;
  return s;
}

static std::string lit(double v, int dtype) {
  char buf[64];
  if (dtype == KF_F32) {
    float f = float(v);
    uint32_t u;
    std::memcpy(&u, &f, 4);
    snprintf(buf, sizeof buf, "__int_as_float(0x%08xu)", u);
  } else {
    uint64_t u;
    std::memcpy(&u, &v, 8);
    snprintf(buf, sizeof buf, "__longlong_as_double(0x%016llxull)", (unsigned long long)u);
  }
  return buf;
}

static std::string sanitize(const std::string& s) {
  std::string o;
  for (char c : s) o += (isalnum((unsigned char)c) ? c : '_');
  if (o.size() > 24) o = o.substr(0, 24);
  return o;
}

// Device-side helpers emitted at the top of every generated translation unit.
static const char* kPrelude = R"KF(
typedef unsigned int u32;
typedef unsigned long long u64;
struct __align__(64) KfTmap { u64 v[16]; };
static __device__ __forceinline__ u32 kf_smem_u32(const void* p) { return (u32)__cvta_generic_to_shared(p); }
static __device__ __forceinline__ void kf_mbar_init(u64* m, u32 cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(kf_smem_u32(m)), "r"(cnt) : "memory");
}
static __device__ __forceinline__ void kf_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
static __device__ __forceinline__ void kf_mbar_expect(u64* m, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(kf_smem_u32(m)), "r"(bytes) : "memory");
}
static __device__ __forceinline__ void kf_mbar_wait(u64* m, u32 parity) {
  u32 done = 0;
  do {
    asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                 : "=r"(done) : "r"(kf_smem_u32(m)), "r"(parity) : "memory");
  } while (!done);
}
static __device__ __forceinline__ void kf_tma_load3(void* dst, const KfTmap* map, int c0, int c1, int c2, u64* m) {
  asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
               :: "r"(kf_smem_u32(dst)), "l"((u64)map), "r"(c0), "r"(c1), "r"(c2), "r"(kf_smem_u32(m)) : "memory");
}
static __device__ __forceinline__ int kf_mod(int a, int m) { int r = a % m; return r < 0 ? r + m : r; }
static __device__ __forceinline__ int kf_slot(int c, int om, int n) { int s = c + om; return s >= n ? s - n : s; }
)KF";

Codegen generate_group_kernel(const Program& p, const GroupLowering& L, int gid) {
  std::ostringstream o;
  const int es = p.es;
  const std::string real = p.dtype == KF_F32 ? "float" : "double";
  const int TX = L.tile[0], TY = L.tile[1];
  const int64_t NX = p.n[0], NY = p.n[1], NZ = p.n[2];
  const int TZ = L.tile[2] > 0 ? std::min<int64_t>(L.tile[2], NZ) : int(NZ);
  const int64_t NTX = (NX + TX - 1) / TX, NTY = (NY + TY - 1) / TY, NTZ = (NZ + TZ - 1) / TZ;
  const int S = L.stages, NT = L.threads;
  const bool fx = p.bc[0] == KF_BC_FROZEN, fy = p.bc[1] == KF_BC_FROZEN, fz = p.bc[2] == KF_BC_FROZEN;
  const kf_layout& lay = p.layout;

  Codegen cg;
  {
    std::ostringstream nm;
    nm << "kf_g" << gid << "_" << sanitize(p.kernels[L.kernels.front()].name) << "_n" << L.kernels.size();
    cg.name = nm.str();
  }
  std::vector<int> alive;
  for (int k : L.kernels)
    if (L.ext.at(k).alive) alive.push_back(k);
  std::vector<int> in_rings, mid_rings;
  for (size_t i = 0; i < L.rings.size(); i++) (L.rings[i].live_in ? in_rings : mid_rings).push_back(int(i));
  auto in_group = [&](int k) { return std::binary_search(L.kernels.begin(), L.kernels.end(), k); };

  o << "// generated by kf " << kf_version() << " -- fused group " << gid << ": kernels";
  for (int k : L.kernels) o << " " << p.kernels[k].name;
  o << "\n" << kPrelude;
  o << "typedef " << real << " real;\n";
  o << "typedef " << (p.dtype == KF_F32 ? "float2" : "double2") << " real2;\n";
  o << "#define NX " << NX << "\n#define NY " << NY << "\n#define NZ " << NZ << "\n";
  o << "#define GX " << p.ghost[0] << "\n#define GY " << p.ghost[1] << "\n#define GZ " << p.ghost[2] << "\n";
  o << "#define PITCH " << lay.pitch << "ll\n#define PLANE " << lay.plane << "ll\n#define XOFF " << lay.xoff << "\n";
  o << "#define TX " << TX << "\n#define TY " << TY << "\n#define TZ " << TZ << "\n";
  o << "#define NTX " << NTX << "\n#define NTY " << NTY << "\n#define NTZ " << NTZ << "\n";
  o << "#define NT " << NT << "\n#define NSTAGE " << S << "\n";
  o << "struct KfArgs {\n";
  o << "  KfTmap tm[" << std::max<size_t>(1, in_rings.size()) << "];\n";
  o << "  real* out[" << std::max<size_t>(1, L.live_out.size()) << "];\n";
  o << "  const real* gsrc[" << std::max<size_t>(1, mid_rings.size()) << "];\n";
  o << "  double prm[" << std::max(1, p.n_params) << "];\n";
  o << "  int mode, pad_;   // units: 0 all, 1 interior tiles only, 2 the others (kf_split_units)\n";
  o << "};\n";
  // Registers.  minblocks -1: __launch_bounds__(NT), ptxas' own choice (measured: explicit budgets
  // make ptxas use up to the budget, e.g. 124 or 162 instead of 88 or 72 registers on the flux
  // groups, one CTA per SM less).  minblocks >= 0: __maxnreg__ at what keeps m CTAs per SM resident
  // (m = the shared-memory-limited count for 0, n for n >= 1), never above R_est.  Register cliffs
  // are steep (measured: 67 instead of 64 registers halved the CTAs per SM of a 448-thread group), so
  // a build that spills steps down the ladder m-1, m-2, ... CTAs and finally R_est (V8): the runtime
  // compiles "#define KF_CAP c" for the next cap of "// KF_CAPS" until ptxas neither spills nor
  // exceeds R_est.  So the loaded kernel never has more than R_est registers; a GPU test pins that it
  // does not spill either.
  {
    const int rest = std::max(24, std::min(L.regs, regs_limit(NT)));
    std::vector<int> caps;
    std::string primary;
    if (const char* fc = getenv("KF_MAXNREG")) {   // experiments only: force a register cap
      primary = "__maxnreg__(" + std::to_string(atoi(fc)) + ")";
    } else if (L.minblocks >= 0) {
      const int smem_ctas = 233472 / std::max(1, L.smem + 1024);
      const int minb = L.minblocks > 0 ? L.minblocks : std::max(1, std::min({smem_ctas, 2048 / std::max(1, NT), 8}));
      for (int m = minb; m >= 1; m--) {
        const int c = std::max(24, std::min(regs_cap(NT, m), rest));
        if (caps.empty() || c > caps.back()) caps.push_back(c);
      }
      primary = "__maxnreg__(KF_CAP)";
    } else {
      primary = "__launch_bounds__(NT)";
    }
    if (caps.empty() || caps.back() < rest) caps.push_back(rest);
    o << "#define KF_REST " << rest << "\n// KF_CAPS";
    for (int c : caps) o << " " << c;
    o << "\n";
    if (L.minblocks >= 0 && !getenv("KF_MAXNREG"))
      o << "#ifndef KF_CAP\n#define KF_CAP " << caps[0] << "\n#endif\n#define KF_BOUNDS __maxnreg__(KF_CAP)\n";
    else
      o << "#ifndef KF_CAP\n#define KF_BOUNDS " << primary << "\n#else\n#define KF_BOUNDS __maxnreg__(KF_CAP)\n#endif\n";
  }
  o << "/*@@KF_GCOPY@@*/";
  o << "extern \"C\" __global__ void KF_BOUNDS " << cg.name << "(const __grid_constant__ KfArgs a) {\n";
  // pointer arithmetic from the __shared__ array keeps the shared state space (LDS/STS, 32-bit
  // addressing); the pad realigns the dynamic window to 128 bytes (TMA destinations).
  o << "  extern __shared__ __align__(128) unsigned char kf_smem_raw[];\n";
  o << "  unsigned char* sm = kf_smem_raw + ((128u - (kf_smem_u32(kf_smem_raw) & 127u)) & 127u);\n";
  o << "  u64* mbar = (u64*)(sm + " << L.mbar_off << ");\n";
  o << "  const int tid = threadIdx.x;\n";
  // interior / boundary unit split (a11 overlap): interior tiles lie >= the ghost width inside the
  // local domain on x and y, so they neither read ghosts nor write the strips an exchange packs
  {
    const Split sp = split_units(p, L);
    o << "  int u = blockIdx.x;\n";
    if (sp.ok) {
      const int IW = sp.ix1 - sp.ix0, IH = sp.iy1 - sp.iy0;
      o << "  if (a.mode == 1) {\n"
        << "    const int tz = u / " << IW * IH << ", r = u - tz * " << IW * IH << ";\n"
        << "    u = (tz * NTY + " << sp.iy0 << " + r / " << IW << ") * NTX + " << sp.ix0 << " + r % " << IW << ";\n"
        << "  } else if (a.mode == 2) {\n"
        << "    const int nb = NTX * NTY - " << IW * IH << ", tz = u / nb;\n"
        << "    int b = u - tz * nb, tx, ty;\n"
        << "    if (b < " << sp.iy0 << " * NTX) { ty = b / NTX; tx = b % NTX; }\n"
        << "    else if ((b -= " << sp.iy0 << " * NTX) < " << IH * (NTX - IW) << ") {\n"
        << "      ty = " << sp.iy0 << " + b / " << NTX - IW << "; const int c = b % " << NTX - IW << "; tx = c < " << sp.ix0
        << " ? c : c + " << IW << ";\n"
        << "    } else { b -= " << IH * (NTX - IW) << "; ty = " << sp.iy1 << " + b / NTX; tx = b % NTX; }\n"
        << "    u = (tz * NTY + ty) * NTX + tx;\n"
        << "  }\n";
    }
  }
  o << "  const int x0 = (u % NTX) * TX; u /= NTX;\n";
  o << "  const int y0 = (u % NTY) * TY; u /= NTY;\n";
  o << "  const int z0 = u * TZ;\n";
  o << "  const int z1 = min(z0 + TZ, NZ);\n";
  o << "  const bool edge_tile = x0 < GX || x0 + TX > NX - GX || y0 < GY || y0 + TY > NY - GY;\n";
  o << "  if (tid == 0) {\n    for (int s = 0; s < NSTAGE; ++s) kf_mbar_init(&mbar[s], 1);\n    kf_fence_init();\n  }\n";
  // per-kernel starting point of the thread in its region (row-major, x fastest)
  for (int k : alive) {
    const Ext& e = L.ext.at(k);
    const int WX = TX + e.elo[0] + e.ehi[0];
    o << "  const int ly0_" << k << " = tid / " << WX << ", lx0_" << k << " = tid - ly0_" << k << " * " << WX << ";\n";
  }
  // ---- canvas (fast iterations): the bounding box of all extended regions, one point per thread
  // (rounds if larger than the CTA).  Canvas rows are covered by row-aligned warps over the tile's x
  // range [lo, lo+TX) (contiguous shared-memory rows: no extra wavefronts), the halo columns by
  // extra threads (column-major).  Every kernel of the group computes its region's points on the
  // same threads, so values a later kernel reads at xy offset 0 are forwarded in registers and
  // identical shared loads of different kernels are issued once.
  const CanvasPlan cv = plan_canvas(p, L);
  const int* clo = cv.clo;
  const int* chi = cv.chi;
  const int CH = cv.ch, CPTS = cv.pts, CROUNDS = cv.rounds;
  const bool canvas_mode = cv.ok;
  std::set<int> canvas_pitches;
  for (auto& r : L.rings) canvas_pitches.insert(r.px);
  const bool pair_mode = canvas_mode && cv.pair;
  const int PSH = 2 * cv.lop - clo[0];   // pair mode: canvas x of the thread's first point = 2 * pair column - PSH
  // Clamped canvas loads (canvas_ld): a lane outside the reading kernels' regions never stores (nor
  // forwards to a stored point) what it computes, so it may load any address -- it loads the one of
  // the nearest canvas point inside the regions' bounding rectangle (row and column clamped once,
  // before the stream loop).  No predicate, no zeroing move, and every address stays inside the
  // ring box of the plane being read, which no thread writes in the reading phase (an unclamped
  // load on such a lane could reach a neighbouring ring that another kernel stores to: a race,
  // compute-sanitizer racecheck, round 2).
  std::map<std::array<int, 5>, std::string> clamp_base;   // {x0, x1, y0, y1, pitch} -> variable
  std::string clamp_defs;
  auto cbase = [&](const Rect& rc, int pitch) {
    const std::array<int, 5> key{rc[0], rc[1], rc[2], rc[3], pitch};
    auto it = clamp_base.find(key);
    if (it != clamp_base.end()) return it->second;
    const std::string nm = "ckb" + std::to_string(clamp_base.size());
    const std::string cy = "min(max(cy_r0 + kz, " + std::to_string(rc[2]) + "), " + std::to_string(rc[3] - 1) + ")";
    std::string cx;
    if (pair_mode) {   // first-point x of an aligned pair inside [x0, x1): pair columns [lo, hi]
      const int lo = (rc[0] + PSH + 1) >> 1, hi = (rc[1] - 1 + PSH) >> 1;
      cx = "(2 * min(max(cxp_r0, " + std::to_string(lo) + "), " + std::to_string(std::max(lo, hi)) + ") - " + std::to_string(PSH) + ")";
    } else {
      cx = "min(max(cx_r0, " + std::to_string(rc[0]) + "), " + std::to_string(rc[1] - 1) + ")";
    }
    clamp_defs += "      const int " + nm + " = " + cy + " * " + std::to_string(pitch) + " + " + cx + ";\n";
    clamp_base.emplace(key, nm);
    return nm;
  };
  if (pair_mode) {
    // pair mode: row-aligned threads over the tile's TX/2 pair columns, then the halo pair columns
    // (column-major); cx = canvas x of the first point (even tile-relative x: pairs are 16-byte
    // aligned in every ring row and in HBM)
    const int TXp = TX / 2, LP = cv.lop, CWp = cv.cwp;
    o << "  int cxp_r0, cy_r0;\n";
    o << "  if (tid < " << TXp * CH << ") { cy_r0 = tid / " << TXp << "; cxp_r0 = " << LP << " + tid - cy_r0 * " << TXp << "; }\n";
    o << "  else { const int s = tid - " << TXp * CH << ", c = s / " << CH << "; cy_r0 = s - c * " << CH << "; cxp_r0 = c < " << LP
      << " ? c : c + " << TXp << "; }\n";
    o << "  const bool ca_r0 = tid < " << CWp * CH << ";\n";
    o << "  if (!ca_r0) { cxp_r0 = " << LP << "; cy_r0 = 0; }   // in bounds for unpredicated loads\n";
    o << "  const int cx_r0 = 2 * cxp_r0 - " << PSH << ";\n";
    for (int pch : canvas_pitches) o << "  const int cb" << pch << "_r0 = cy_r0 * " << pch << " + cx_r0;\n";
    o << "  const int cgx_r0 = x0 + cx_r0 - " << clo[0] << ", cgy_r0 = y0 + cy_r0 - " << clo[1] << ";\n";
    o << "  const bool cT_r0 = ca_r0 && cx_r0 >= " << clo[0] << " && cx_r0 < " << clo[0] + TX << " && cy_r0 >= " << clo[1]
      << " && cy_r0 < " << clo[1] + TY << " && cgx_r0 < NX && cgy_r0 < NY;\n";
    for (int k : alive) {
      const Ext& e = L.ext.at(k);
      const int ox = clo[0] - e.elo[0], oy = clo[1] - e.elo[1];
      const int WX = TX + e.elo[0] + e.ehi[0], WY = TY + e.elo[1] + e.ehi[1];
      for (int j = 0; j < 2; j++)
        o << "  const bool ce" << k << "_" << j << " = ca_r0 && cx_r0 + " << j << " >= " << ox << " && cx_r0 + " << j << " < "
          << ox + WX << " && cy_r0 >= " << oy << " && cy_r0 < " << oy + WY << ";\n";
    }
  }
  if (canvas_mode && !pair_mode)
    for (int r = 0; r < CROUNDS; r++) {
      const std::string rs = "_r" + std::to_string(r);
      o << "  const int ci" << rs << " = tid + " << r * NT << ";\n";
      o << "  int cx" << rs << ", cy" << rs << ";\n";
      o << "  if (ci" << rs << " < " << TX * CH << ") { cy" << rs << " = ci" << rs << " / " << TX << "; cx" << rs << " = "
        << clo[0] << " + ci" << rs << " - cy" << rs << " * " << TX << "; }\n";
      if (clo[0] + chi[0] > 0)
        o << "  else { const int s = ci" << rs << " - " << TX * CH << ", c = s / " << CH << "; cy" << rs << " = s - c * " << CH
          << "; cx" << rs << " = c < " << clo[0] << " ? c : c + " << TX << "; }\n";
      else
        o << "  else { cx" << rs << " = 0; cy" << rs << " = 0; }\n";
      o << "  const bool ca" << rs << " = ci" << rs << " < " << CPTS << ";\n";
      o << "  if (!ca" << rs << ") { cx" << rs << " = 0; cy" << rs << " = 0; }\n";
      for (int pch : canvas_pitches) o << "  const int cb" << pch << rs << " = cy" << rs << " * " << pch << " + cx" << rs << ";\n";
      // tile-interior predicate and global coordinates of the thread's canvas point
      o << "  const int cgx" << rs << " = x0 + cx" << rs << " - " << clo[0] << ", cgy" << rs << " = y0 + cy" << rs << " - " << clo[1]
        << ";\n";
      o << "  const bool cT" << rs << " = ca" << rs << " && cx" << rs << " >= " << clo[0] << " && cx" << rs << " < " << clo[0] + TX
        << " && cy" << rs << " >= " << clo[1] << " && cy" << rs << " < " << clo[1] + TY << " && cgx" << rs << " < NX && cgy" << rs
        << " < NY;\n";
      for (int k : alive) {
        const Ext& e = L.ext.at(k);
        const int ox = clo[0] - e.elo[0], oy = clo[1] - e.elo[1];
        const int WX = TX + e.elo[0] + e.ehi[0], WY = TY + e.elo[1] + e.ehi[1];
        o << "  const bool ce" << k << rs << " = ca" << rs << " && cx" << rs << " >= " << ox << " && cx" << rs << " < " << ox + WX
          << " && cy" << rs << " >= " << oy << " && cy" << rs << " < " << oy + WY << ";\n";
      }
    }
  o << "  __syncthreads();\n";
  // per-kernel compute / ghost plane ranges for this unit
  for (int k : alive) {
    const Ext& e = L.ext.at(k);
    o << "  // kernel " << k << " (" << p.kernels[k].name << "): E extents lo(" << e.elo[0] << "," << e.elo[1] << ","
      << e.elo[2] << ") hi(" << e.ehi[0] << "," << e.ehi[1] << "," << e.ehi[2] << "), delay " << L.delay.at(k) << "\n";
    if (fz) {
      o << "  const int plo" << k << " = max(z0 - " << e.elo[2] << ", 0), phi" << k << " = min(z1 + " << e.ehi[2] << ", NZ);\n";
      o << "  const int glo" << k << " = max(z0 - " << e.elo[2] << ", -GZ), ghi" << k << " = min(z1 + " << e.ehi[2] << ", NZ + GZ);\n";
    } else {
      o << "  const int plo" << k << " = z0 - " << e.elo[2] << ", phi" << k << " = z1 + " << e.ehi[2] << ";\n";
      o << "  const int glo" << k << " = plo" << k << ", ghi" << k << " = phi" << k << ";\n";
    }
  }
  // plane ranges needed per live-in ring
  for (int ri : in_rings) {
    const Ring& r = L.rings[ri];
    std::string lo, hi;
    bool first = true;
    for (int c : alive) {
      auto it = p.kernels[c].reads.find(r.ver.x);
      if (it == p.kernels[c].reads.end() || p.vr(c, r.ver.x) != r.ver.v) continue;
      int dmin = 1 << 30, dmax = -(1 << 30);
      for (auto& d : it->second) { dmin = std::min(dmin, d[2]); dmax = std::max(dmax, d[2]); }
      std::string l = "(plo" + std::to_string(c) + " + (" + std::to_string(dmin) + "))";
      std::string h = "(phi" + std::to_string(c) + " + (" + std::to_string(dmax) + "))";
      lo = first ? l : "min(" + lo + ", " + l + ")";
      hi = first ? h : "max(" + hi + ", " + h + ")";
      first = false;
    }
    o << "  const int rlo" << ri << " = " << lo << ", rhi" << ri << " = " << hi << ";  // ring " << ri << " ("
      << p.array_names[r.ver.x] << " v" << r.ver.v << ") planes [rlo, rhi)\n";
  }
  // iteration range
  {
    std::string ts, te;
    bool first = true;
    auto addmin = [&](const std::string& s) { ts = first ? s : "min(" + ts + ", " + s + ")"; };
    auto addmax = [&](const std::string& s) { te = first ? s : "max(" + te + ", " + s + ")"; };
    for (int k : alive) {
      std::string d = std::to_string(L.delay.at(k));
      addmin("(min(plo" + std::to_string(k) + ", glo" + std::to_string(k) + ") + " + d + ")");
      addmax("(max(phi" + std::to_string(k) + ", ghi" + std::to_string(k) + ") + " + d + ")");
      first = false;
    }
    for (int ri : in_rings) {
      addmin("(rlo" + std::to_string(ri) + " - (" + std::to_string(L.rings[ri].A) + "))");
      first = false;
    }
    if (alive.empty()) { ts = "0"; te = "0"; }
    o << "  const int t0 = " << ts << ", t1 = " << te << ";\n";
  }
  // The stream advances U planes per loop iteration ("z-unroll"): every kernel handles U
  // consecutive planes per point, giving each thread U independent computations (ILP) and
  // amortising barriers and ring bookkeeping over U planes.  Ring depths include U (R20).
  const int U = L.zunroll;
  // TMA issue for the super-iteration starting at t (thread 0): U planes per live-in ring
  o << "  auto issue = [&](int t) {\n";
  o << "    u64* mb = &mbar[((t - t0) / " << U << ") % NSTAGE];\n";
  o << "    u32 bytes = 0;\n";
  for (int ri : in_rings) {
    const Ring& r = L.rings[ri];
    for (int uu = 0; uu < U; uu++) {
      o << "    const int P" << ri << "_" << uu << " = t + " << uu << " + (" << r.A << ");\n";
      o << "    const bool ok" << ri << "_" << uu << " = P" << ri << "_" << uu << " >= rlo" << ri << " && P" << ri << "_" << uu
        << " < rhi" << ri << ";\n";
      o << "    if (ok" << ri << "_" << uu << ") bytes += " << (r.px * r.hy * es) << "u;\n";
    }
  }
  o << "    kf_mbar_expect(mb, bytes);\n";
  int ti = 0;
  for (int ri : in_rings) {
    const Ring& r = L.rings[ri];
    for (int uu = 0; uu < U; uu++)
      o << "    if (ok" << ri << "_" << uu << ") kf_tma_load3(sm + " << r.smem_off << " + kf_mod(P" << ri << "_" << uu << " - t0, "
        << r.slots << ") * " << r.plane_bytes << ", &a.tm[" << ti << "], XOFF + x0 - (" << r.ax_lo << "), GY + y0 - ("
        << r.blo[1] << "), GZ + P" << ri << "_" << uu << ", mb);\n";
    ti++;
  }
  o << "  };\n";
  o << "  if (tid == 0)\n    for (int t = t0; t < t1 && t < t0 + " << U << " * (NSTAGE - 1); t += " << U << ") issue(t);\n";
  // Ring slots are relative to the CTA's first iteration: plane P lives in slot (P - t0) mod n.
  // With ring unrolling (every ring size a power of two dividing N) the loop body is emitted N
  // times and every slot is a compile-time constant: no per-iteration pointer arithmetic.
  const int NU = L.ring_unroll;   // 0: per-ring counters cs_r; else unroll factor N
  // z register queues: a kernel whose fast-path thread keeps the same point(s) every iteration
  // (U == 1, at most 2 points per thread) and reads a ring at (0,0,dz) over a contiguous dz
  // range keeps that column of values in registers: one shared load per iteration (the newest
  // plane) instead of one per dz ("z-streaming register queues").
  struct ZQ { std::map<int, std::pair<int, int>> rings; std::vector<std::string> pss; };
  std::map<int, ZQ> zq;
  int zq_used = 0, zq_max = getenv("KF_ZQ_MAX") ? atoi(getenv("KF_ZQ_MAX")) : 0;   // off by default: measured neutral
  if (U == 1 && !getenv("KF_NO_ZQ"))   // KF_NO_ZQ: A/B switch for measurement
    for (int k : alive) {
      const Ext& e = L.ext.at(k);
      const int WX = TX + e.elo[0] + e.ehi[0], WY = TY + e.elo[1] + e.ehi[1];
      const int bx = std::min(L.pblock[0], WX), by = std::min(L.pblock[1], WY);
      const int NB = ((WX + bx - 1) / bx) * ((WY + by - 1) / by);
      const int rounds = (NB + NT - 1) / NT;
      if (rounds * bx * by > 2) continue;
      ZQ q;
      for (auto& [x, offs] : p.kernels[k].reads) {
        int ring = L.ring_of(Ver{x, p.vr(k, x)});
        std::set<int> dzs;
        for (auto& d : offs)
          if (d[0] == 0 && d[1] == 0) dzs.insert(d[2]);
        if (dzs.size() < 2) continue;
        const int lo = *dzs.begin(), hi = *dzs.rbegin();
        if (int(dzs.size()) != hi - lo + 1 || hi - lo > 4) continue;   // contiguous, short
        q.rings[ring] = {lo, hi};
      }
      if (q.rings.empty()) continue;
      for (int r = 0; r < rounds; r++)
        for (int jj = 0; jj < by; jj++)
          for (int ii = 0; ii < bx; ii++)
            q.pss.push_back("_r" + std::to_string(r) + "_" + std::to_string(ii) + "_" + std::to_string(jj));
      int cost = 0;
      for (auto& [ring, mm] : q.rings) cost += (mm.second - mm.first + 1) * int(q.pss.size());
      if (zq_used + cost > zq_max) continue;
      zq_used += cost;
      zq[k] = q;
    }
  // live-out output pointer index
  auto out_index = [&](const Ver& v) {
    for (size_t i = 0; i < L.live_out.size(); i++)
      if (L.live_out[i] == v) return int(i);
    return -1;
  };
  // ---- canvas plan (fast iterations; see the canvas comment above and kf_canvas.cpp)
  auto slot = [&](int ring, int po) { const int n = L.rings[ring].slots; return ((po % n) + n) % n; };
  auto fwd_src = [&](int k, int x, const Off& d, int uu, int* prod, int* up) {
    return canvas_forward(p, L, k, x, d, uu, prod, up);
  };
  using Key = CanvasKey;
  const std::set<Ver>& need_sts = cv.need_sts;
  const std::vector<std::vector<int>>& cph = cv.phases;
  std::map<Key, Rect> krect = cv.krect;
  auto rect_of = [&](int k) { return canvas_rect(L, cv, k); };
  auto contains = [](const Rect& a, const Rect& b) { return a[0] <= b[0] && a[1] >= b[1] && a[2] <= b[2] && a[3] >= b[3]; };
  auto load_key = [&](int k, int x, const Off& d, int uu) { return canvas_key(p, L, cv, k, x, d, uu); };
  // z register queues on the canvas ("z-streaming register queues"): the value a key (ring, po,
  // off) reads at iteration t is the value of (ring, po + U, off) at iteration t - U when that was
  // loaded (on a superset of lanes) or computed in registers by the producer.  Such keys are
  // carried in registers across fast iterations instead of re-read from shared memory; after a
  // slow iteration they are reloaded.  carry[key] = source: a load key or a forwarded value.
  struct Src { bool is_load; Key key; int x, v, uu; };
  std::map<Key, Src> carry;
  if (canvas_mode && !pair_mode && getenv("KF_CQ")) {   // off by default: the carried registers cost occupancy (measured slower)
    // widen the load predicate of (ring, po + U, off) to cover (ring, po, off): both lie in the
    // ring's box at every plane, and the wider load then feeds the next iteration's narrower read
    for (auto& [key, rc] : krect) {
      auto it = krect.find(Key{key.ring, key.po + U, key.off});
      if (it == krect.end()) continue;
      auto& a = it->second;
      a = {std::min(a[0], rc[0]), std::max(a[1], rc[1]), std::min(a[2], rc[2]), std::max(a[3], rc[3])};
    }
    for (auto& [key, rc] : krect) {
      Key nx{key.ring, key.po + U, key.off};
      auto it = krect.find(nx);
      if (it != krect.end() && contains(it->second, rc)) {
        carry[key] = Src{true, nx, 0, 0, 0};
        continue;
      }
      const Ring& R = L.rings[key.ring];
      if (R.live_in) continue;
      const int off0 = (R.blo[1] - clo[1]) * R.px + (R.ax_lo - clo[0]);
      const int pk = R.producer;
      const int u2 = key.po + U + L.delay.at(pk);
      if (key.off == off0 && u2 >= 0 && u2 < U && contains(rect_of(pk), rc))
        carry[key] = Src{false, nx, R.ver.x, R.ver.v, u2};
    }
  }
  auto key_name = [&](const char* pre, const Key& key, const std::string& rs) {
    return std::string(pre) + std::to_string(key.ring) + "_" + (key.po < 0 ? "m" + std::to_string(-key.po) : std::to_string(key.po)) +
           "_" + (key.off < 0 ? "m" + std::to_string(-key.off) : std::to_string(key.off)) + rs;
  };
  // shared loads reused across the phases of an iteration: a value cannot change within an
  // iteration, but the longer live ranges cost registers -- large groups (a 35-kernel group
  // spilled) keep per-phase loads.  KF_CANVAS_PHASE_LD=1: per-phase loads everywhere (A/B).
  const bool xphase_ld = alive.size() <= 16 && cv.phases.size() <= 4 && !getenv("KF_CANVAS_PHASE_LD");
  auto emit_canvas = [&]() {
    std::map<std::pair<Key, int>, std::string> ldname;
    std::map<std::tuple<int, int, int, int>, std::string> fwd;   // (x, v, round, sub-plane) -> value
    std::map<std::pair<Key, int>, std::string> ldfirst;   // first load of every key (carry sources)
    for (size_t ph = 0; ph < cph.size(); ph++) {
      if (ph > 0) o << "      __syncthreads();\n";
      // loads are shared across the phases of an iteration (a value cannot change within an
      // iteration; measured 1-5 % faster on the flux groups despite the longer live ranges);
      // KF_CANVAS_PHASE_LD=1: per-phase loads (A/B)
      if (!xphase_ld) ldname.clear();
      std::vector<std::tuple<int, int, int, std::vector<std::string>>> done;   // (k, r, uu, vals)
      for (int k : cph[ph]) {
        const Kernel& K = p.kernels[k];
        o << "      // kernel " << k << " " << K.name << " (canvas)\n";
        for (int r = 0; r < CROUNDS; r++) {
          const std::string rs = "_r" + std::to_string(r);
          for (int uu = 0; uu < U; uu++) {
            std::vector<std::string> vals;
            for (size_t si = 0; si < K.stmts.size(); si++) {
              std::vector<std::string> st;
              int tmp = 0;
              for (const Insn& in : K.stmts[si].rpn) {
                std::string t = "c" + std::to_string(k) + "s" + std::to_string(si) + "_" + std::to_string(tmp++) + "_" +
                                std::to_string(uu) + rs;
                std::string f;
                switch (in.op) {
                  case KF_OP_CONST: f = lit(in.imm, p.dtype); break;
                  case KF_OP_PARAM: f = "(real)a.prm[" + std::to_string(in.arg) + "]"; break;
                  case KF_OP_LOAD: {
                    int pr, u2;
                    if (fwd_src(k, in.arg, in.d, uu, &pr, &u2)) {
                      f = fwd.at(std::make_tuple(in.arg, p.vr(k, in.arg), r, u2));
                    } else {
                      Key key = load_key(k, in.arg, in.d, uu);
                      auto nk = std::make_pair(key, r);
                      auto it = ldname.find(nk);
                      if (it == ldname.end()) {
                        const auto& rc = krect.at(key);
                        std::string nm = key_name("cl", key, rs) + "_h" + std::to_string(ph);
                        const std::string acc = "P" + std::to_string(key.ring) + "_" + std::to_string(slot(key.ring, key.po)) +
                                                "[cb" + std::to_string(L.rings[key.ring].px) + rs + " + " + std::to_string(key.off) + "]";
                        // canvas_ld: clamped unpredicated load (see cbase); else predicated with a zero
                        const Ring& RR = L.rings[key.ring];
                        std::string ld;
                        if (L.canvas_ld)
                          ld = "P" + std::to_string(key.ring) + "_" + std::to_string(slot(key.ring, key.po)) + "[" +
                               cbase(rc, RR.px) + " + " + std::to_string(key.off) + "]";
                        else
                          ld = "(ca" + rs + " && cx" + rs + " >= " + std::to_string(rc[0]) + " && cx" + rs + " < " +
                               std::to_string(rc[1]) + " && cy" + rs + " >= " + std::to_string(rc[2]) + " && cy" + rs + " < " +
                               std::to_string(rc[3]) + ") ? " + acc + " : (real)0";
                        if (carry.count(key))
                          o << "      const real " << nm << " = cqv ? " << key_name("cq", key, rs) << " : (" << ld << ");\n";
                        else
                          o << "      const real " << nm << " = " << ld << ";\n";
                        it = ldname.emplace(nk, nm).first;
                        ldfirst.emplace(nk, nm);
                      }
                      f = it->second;
                    }
                    break;
                  }
                  case KF_OP_NEG: case KF_OP_ABS: case KF_OP_SQRT: {
                    std::string a1 = st.back(); st.pop_back();
                    f = in.op == KF_OP_NEG ? "-" + a1
                      : in.op == KF_OP_ABS ? (p.dtype == KF_F32 ? "fabsf(" : "fabs(") + a1 + ")"
                                           : (p.dtype == KF_F32 ? "sqrtf(" : "sqrt(") + a1 + ")";
                    break;
                  }
                  default: {
                    std::string b = st.back(); st.pop_back();
                    std::string a1 = st.back(); st.pop_back();
                    switch (in.op) {
                      case KF_OP_ADD: f = a1 + " + " + b; break;
                      case KF_OP_SUB: f = a1 + " - " + b; break;
                      case KF_OP_MUL: f = a1 + " * " + b; break;
                      case KF_OP_DIV: f = a1 + " / " + b; break;
                      case KF_OP_MIN: f = "(" + b + " < " + a1 + ") ? " + b + " : " + a1; break;
                      case KF_OP_MAX: f = "(" + a1 + " < " + b + ") ? " + b + " : " + a1; break;
                    }
                  }
                }
                o << "      const real " << t << " = " << f << ";\n";
                st.push_back(t);
              }
              vals.push_back(st.back());
            }
            for (size_t si = 0; si < K.stmts.size(); si++)
              fwd[std::make_tuple(K.stmts[si].out, p.vw(k, K.stmts[si].out), r, uu)] = vals[si];
            done.emplace_back(k, r, uu, vals);
          }
        }
      }
      // stores of the phase (after all its loads)
      for (auto& [k, r, uu, vals] : done) {
        const Kernel& K = p.kernels[k];
        const Ext& e = L.ext.at(k);
        const std::string rs = "_r" + std::to_string(r);
        const int ox = clo[0] - e.elo[0], oy = clo[1] - e.elo[1];
        bool any_out = false;
        for (size_t si = 0; si < K.stmts.size(); si++) {
          const Ver v{K.stmts[si].out, p.vw(k, K.stmts[si].out)};
          const int ring = L.ring_of(v);
          if (ring >= 0 && need_sts.count(v)) {
            const Ring& R = L.rings[ring];
            o << "      if (ce" << k << rs << ") P" << ring << "_" << slot(ring, -L.delay.at(k) + uu) << "[cb" << R.px << rs << " - "
              << (oy * R.px + (clo[0] - R.ax_lo)) << "] = " << vals[si] << ";\n";
          }
          if (out_index(v) >= 0) any_out = true;
        }
        if (!any_out) continue;
        const std::string pz = "(t - " + std::to_string(L.delay.at(k) - uu) + ")";
        o << "      if (cT" << rs << " && " << pz << " >= z0 && " << pz << " < z1) {\n";
        o << "        const long long gi = (long long)" << pz << " * PLANE + (long long)cgy" << rs << " * PITCH + cgx" << rs << ";\n";
        for (size_t si = 0; si < K.stmts.size(); si++) {
          const int oi = out_index(Ver{K.stmts[si].out, p.vw(k, K.stmts[si].out)});
          if (oi >= 0) o << "        a.out[" << oi << "][gi] = " << vals[si] << ";\n";
        }
        o << "      }\n";
      }
    }
    // carried z-queue registers for the next iteration (ascending plane: read before overwritten)
    for (int r = 0; r < CROUNDS; r++) {
      const std::string rs = "_r" + std::to_string(r);
      for (auto& [key, src] : carry) {
        const std::string val = src.is_load ? ldfirst.at(std::make_pair(src.key, r))
                                            : fwd.at(std::make_tuple(src.x, src.v, r, src.uu));
        o << "      " << key_name("cq", key, rs) << " = " << val << ";\n";
      }
    }
    if (!carry.empty()) o << "      cqv = true;\n";
  };
  // Pair mode (cv.pair): the same phases, forwarding and load CSE as emit_canvas, for two
  // x-adjacent points per thread.  A shared value is loaded as part of the 16-byte-aligned pair
  // (2 elements) containing it, one vector load per distinct (ring, plane, pair offset) in a phase:
  // a 4th-order x stencil on a point pair needs 3 vector loads instead of 8 scalar ones.  Ring and
  // live-out stores are vector stores where the pair is aligned.  U = 1, no z-queue carries.
  auto mod2 = [](int v) { return ((v % 2) + 2) % 2; };
  using PK = std::tuple<int, int, int>;   // ring, plane offset, element offset of the aligned pair
  auto pk_of = [&](int k, int x, const Off& d, int j, int* comp) {
    const Key key = load_key(k, x, d, 0);
    const int e = key.off + j;
    *comp = mod2(PSH + e);   // parity of the absolute element index (row pitches are even)
    return PK{key.ring, key.po, e - *comp};
  };
  // lanes (first point's canvas x, row) needing each pair load over the whole fast iteration, and
  // whether the load can be issued unpredicated (every address it can form lies in the rings)
  std::map<PK, Rect> pall;
  auto pair_nopred = [&](const PK&) { return L.canvas_ld != 0; };   // clamped loads (cbase)
  // z register queues of the pair canvas: a pair value (ring, po, rel) read at iteration t is the
  // value (ring, po + 1, rel) had at iteration t - 1 -- loaded then by the same thread, or computed
  // then by it (its own forwarded result one plane earlier).  Such values are carried in registers
  // across fast iterations instead of re-read from shared memory (fp64: centre-column z stencils
  // and the z-flux read at dz = -1); after a slow iteration they are reloaded once.
  struct PSrc { bool is_load; PK src; int x, v; };
  std::map<PK, PSrc> pcarry;
  // The reads a kernel issues for its point j of the pair: its own loads, a read of an inlined
  // version at an xy offset replaced by the producer's loads shifted by that offset -- none where
  // the offset lands on the thread's other point (the producer's value there is forwarded).
  // (recursively: an inlined producer may itself read inlined values, R20d)
  std::function<void(int, int, const Off&, int, const std::function<void(int, int, const Off&)>&)> eff_expand =
      [&](int kr, int x, const Off& d, int j, const std::function<void(int, int, const Off&)>& fn) {
        if (cv.inlined(p, kr, x, d)) {
          const int ax = j + d[0];
          if (d[1] == 0 && (ax == 0 || ax == 1)) return;
          const auto& [pk, si] = cv.inl.at(Ver{x, p.vr(kr, x)});
          for (const Insn& in : p.kernels[pk].stmts[si].rpn)
            if (in.op == KF_OP_LOAD) eff_expand(pk, in.arg, Off{d[0] + in.d[0], d[1] + in.d[1], d[2] + in.d[2]}, j, fn);
          return;
        }
        fn(kr, x, d);
      };
  auto eff_reads = [&](int k, int j, const std::function<void(int, int, const Off&)>& fn) {
    for (auto& [x, offs] : p.kernels[k].reads)
      for (auto& d : offs) eff_expand(k, x, d, j, fn);
  };
  if (pair_mode) {
    for (int k : alive)
      for (int j = 0; j < 2; j++)
        eff_reads(k, j, [&](int kr, int x, const Off& d) {
          int pr, u2, comp;
          if (fwd_src(kr, x, d, 0, &pr, &u2)) return;
          const Rect rc = krect.at(load_key(kr, x, d, 0));
          const PK pk = pk_of(kr, x, d, j, &comp);
          const Rect rj{rc[0] - j, rc[1] - j, rc[2], rc[3]};
          auto it = pall.find(pk);
          if (it == pall.end()) pall[pk] = rj;
          else {
            auto& a = it->second;
            a = {std::min(a[0], rj[0]), std::max(a[1], rj[1]), std::min(a[2], rj[2]), std::max(a[3], rj[3])};
          }
        });
    if (L.pair_zq)
      for (auto& [pk, rc] : pall) {   // ascending (ring, plane offset): widening propagates upward
        const auto& [ring, po, rel] = pk;
        const PK nx{ring, po + 1, rel};
        auto it = pall.find(nx);
        if (it != pall.end()) {
          // the source load must give every lane of this key's rectangle its true value: widen the
          // source's lanes to the union (both lie in the ring box at every plane)
          auto& a = it->second;
          a = {std::min(a[0], rc[0]), std::max(a[1], rc[1]), std::min(a[2], rc[2]), std::max(a[3], rc[3])};
          pcarry[pk] = PSrc{true, nx, 0, 0};
          continue;
        }
        // the thread's own result one plane earlier: an in-group ring, the pair of the thread's own
        // points (element offset of the canvas point, aligned), computed at plane t + po + 1
        const Ring& R = L.rings[ring];
        if (R.live_in) continue;
        const int off0 = (R.blo[1] - clo[1]) * R.px + (R.ax_lo - clo[0]);
        const int pk_ = R.producer;
        if (mod2(PSH + off0) != 0 || rel != off0 || po + 1 != -L.delay.at(pk_)) continue;
        // Valid wherever it is used: a reader uses element j of the pair only at a point of its
        // region, which lies in the producer's region (E(producer) covers its readers' regions
        // grown by their offsets, here (0, 0)), where the previous fast iteration computed it.
        // (Round 1 also required the key's lane rectangle -- widened by the pair's second element --
        // inside the producer's rectangle, which rejected the z-flux carries.)
        const Rect rp = canvas_rect(L, cv, pk_);   // the producer's region (first point's x, both points inside)
        if ((rp[0] <= rc[0] && rp[1] - 1 >= rc[1] && rp[2] <= rc[2] && rp[3] >= rc[3]) || !getenv("KF_OWN_CARRY_RECT"))
          pcarry[pk] = PSrc{false, nx, R.ver.x, R.ver.v};
      }
  }
  auto pq_name = [&](const PK& pk) {
    const auto& [ring, po, rel] = pk;
    return "pq" + std::to_string(ring) + "_" + (po < 0 ? "m" + std::to_string(-po) : std::to_string(po)) + "_" +
           (rel < 0 ? "m" + std::to_string(-rel) : std::to_string(rel));
  };
  auto pair_acc = [&](const PK& pk) {   // canvas_ld: the clamped base of the key's lanes (pall)
    const auto& [ring, po, rel] = pk;
    const std::string b = L.canvas_ld ? cbase(pall.at(pk), L.rings[ring].px) : "cb" + std::to_string(L.rings[ring].px) + "_r0";
    return "*(const real2*)&P" + std::to_string(ring) + "_" + std::to_string(slot(ring, po)) + "[" + b + " + " +
           std::to_string(rel) + "]";
  };
  auto pair_pred = [&](const Rect& rc) {
    return "ca_r0 && cx_r0 >= " + std::to_string(rc[0]) + " && cx_r0 < " + std::to_string(rc[1]) + " && cy_r0 >= " +
           std::to_string(rc[2]) + " && cy_r0 < " + std::to_string(rc[3]);
  };
  auto emit_canvas_pairs = [&]() {
    std::map<std::tuple<int, int, int>, std::string> fwd;   // (x, v, point) -> value
    std::map<PK, std::string> ldfirst_p;                     // first load of each pair key this iteration
    // carried pair values: loaded once after a slow iteration
    if (!pcarry.empty()) {
      o << "      if (!pqv) {\n";
      for (auto& [pk, src] : pcarry) {
        const Rect& rc = pall.at(pk);
        if (pair_nopred(pk)) o << "        " << pq_name(pk) << " = " << pair_acc(pk) << ";\n";
        else o << "        " << pq_name(pk) << " = (" << pair_pred(rc) << ") ? " << pair_acc(pk) << " : real2{(real)0, (real)0};\n";
      }
      o << "      }\n";
    }
    // Loads are shared across the phases of an iteration: a (ring, plane, offset) value cannot
    // change within an iteration (a reader of a version follows its producer's phase; ring depths
    // keep recycled slots dead), and pair mode has the registers to keep them (one point per
    // thread reloads after every barrier instead; xphase_ld above).
    const bool phase_ld = !xphase_ld;
    std::map<PK, Rect> prect;
    std::map<PK, int> pmask;   // elements of the pair needed (bit 0: first, bit 1: second)
    std::map<PK, std::string> ldname;
    size_t cur_ph = 0;
    // the value a reader's LOAD takes for point j: forwarded, carried, or a (CSE'd) shared load
    auto load_val = [&](int kr, int x, const Off& d, int j) -> std::string {
      int pr, u2, comp;
      if (fwd_src(kr, x, d, 0, &pr, &u2)) return fwd.at(std::make_tuple(x, p.vr(kr, x), j));
      const PK pk = pk_of(kr, x, d, j, &comp);
      if (pcarry.count(pk)) return pq_name(pk) + (comp ? ".y" : ".x");
      auto it = ldname.find(pk);
      if (it == ldname.end()) {
        const auto& [ring, po, rel] = pk;
        const Rect& rc = pall.at(pk);   // (widened for z-queue carries)
        const std::string nm = "pl" + std::to_string(ring) + "_" + (po < 0 ? "m" + std::to_string(-po) : std::to_string(po)) +
                               "_" + (rel < 0 ? "m" + std::to_string(-rel) : std::to_string(rel)) + "_h" + std::to_string(cur_ph);
        const int mask = pmask.at(pk);
        if (mask == 3) {
          if (pair_nopred(pk))
            o << "      const real2 " << nm << " = " << pair_acc(pk) << ";\n";
          else
            o << "      const real2 " << nm << " = (" << pair_pred(rc) << ") ? " << pair_acc(pk)
              << " : real2{(real)0, (real)0};\n";
        } else {
          const int c1 = mask == 2 ? 1 : 0;
          const std::string b1 = L.canvas_ld ? cbase(pall.at(pk), L.rings[ring].px)
                                             : "cb" + std::to_string(L.rings[ring].px) + "_r0";
          const std::string acc1 = "P" + std::to_string(ring) + "_" + std::to_string(slot(ring, po)) + "[" + b1 + " + " +
                                   std::to_string(rel + c1) + "]";
          if (pair_nopred(pk)) o << "      const real " << nm << " = " << acc1 << ";\n";
          else o << "      const real " << nm << " = (" << pair_pred(rc) << ") ? " << acc1 << " : (real)0;\n";
        }
        it = ldname.emplace(pk, nm).first;
        ldfirst_p.emplace(pk, nm);
      }
      return it->second + (pmask.at(pk) == 3 ? (comp ? ".y" : ".x") : "");
    };
    // an inlined version at xy offset d of point j: the producer's statement re-evaluated there
    // (same operations, same order), once per (statement, point) per iteration
    std::map<std::tuple<int, int, int, int>, std::string> inl_memo;
    std::function<std::string(int, int, const Off&, int)> inline_val = [&](int k, int x, const Off& d, int j) -> std::string {
      const auto [pk, si] = cv.inl.at(Ver{x, p.vr(k, x)});
      const int ax = j + d[0];
      if (d[1] == 0 && (ax == 0 || ax == 1)) return fwd.at(std::make_tuple(x, p.vr(k, x), ax));
      const auto mk = std::make_tuple(pk, si, ax, d[1]);
      auto mit = inl_memo.find(mk);
      if (mit != inl_memo.end()) return mit->second;
      auto sg = [](int v) { return v < 0 ? "m" + std::to_string(-v) : std::to_string(v); };
      const std::string pre = "n" + std::to_string(pk) + "s" + std::to_string(si) + "_" + sg(ax) + "_" + sg(d[1]) + "_";
      std::vector<std::string> st;
      int tmp = 0;
      for (const Insn& in : p.kernels[pk].stmts[si].rpn) {
        std::string f;
        switch (in.op) {
          case KF_OP_CONST: f = lit(in.imm, p.dtype); break;
          case KF_OP_PARAM: f = "(real)a.prm[" + std::to_string(in.arg) + "]"; break;
          case KF_OP_LOAD: {
            const Off dd{d[0] + in.d[0], d[1] + in.d[1], d[2] + in.d[2]};
            f = cv.inlined(p, pk, in.arg, dd) ? inline_val(pk, in.arg, dd, j) : load_val(pk, in.arg, dd, j);
            break;
          }
          case KF_OP_NEG: case KF_OP_ABS: case KF_OP_SQRT: {
            std::string a1 = st.back(); st.pop_back();
            f = in.op == KF_OP_NEG ? "-" + a1
              : in.op == KF_OP_ABS ? (p.dtype == KF_F32 ? "fabsf(" : "fabs(") + a1 + ")"
                                   : (p.dtype == KF_F32 ? "sqrtf(" : "sqrt(") + a1 + ")";
            break;
          }
          default: {
            std::string b = st.back(); st.pop_back();
            std::string a1 = st.back(); st.pop_back();
            switch (in.op) {
              case KF_OP_ADD: f = a1 + " + " + b; break;
              case KF_OP_SUB: f = a1 + " - " + b; break;
              case KF_OP_MUL: f = a1 + " * " + b; break;
              case KF_OP_DIV: f = a1 + " / " + b; break;
              case KF_OP_MIN: f = "(" + b + " < " + a1 + ") ? " + b + " : " + a1; break;
              case KF_OP_MAX: f = "(" + a1 + " < " + b + ") ? " + b + " : " + a1; break;
            }
          }
        }
        const std::string t = pre + std::to_string(tmp++);
        o << "      const real " << t << " = " << f << ";\n";
        st.push_back(t);
      }
      inl_memo.emplace(mk, st.back());
      return st.back();
    };
    for (size_t ph = 0; ph < cph.size(); ph++) {
      cur_ph = ph;
      if (ph > 0) o << "      __syncthreads();\n";
      // lanes (first point's canvas x, row) needing each pair load in this phase (all phases
      // unless per-phase loads)
      if (phase_ld || ph == 0) {
        prect.clear();
        pmask.clear();
        ldname.clear();
      }
      for (int k : (phase_ld ? cph[ph] : ph == 0 ? alive : std::vector<int>{}))
        for (int j = 0; j < 2; j++)
          eff_reads(k, j, [&](int kr, int x, const Off& d) {
            int pr, u2, comp;
            if (fwd_src(kr, x, d, 0, &pr, &u2)) return;
            const Rect rc = krect.at(load_key(kr, x, d, 0));
            const PK pk = pk_of(kr, x, d, j, &comp);
            const Rect rj{rc[0] - j, rc[1] - j, rc[2], rc[3]};
            pmask[pk] |= 1 << comp;
            auto it = prect.find(pk);
            if (it == prect.end()) prect[pk] = rj;
            else {
              auto& a = it->second;
              a = {std::min(a[0], rj[0]), std::max(a[1], rj[1]), std::min(a[2], rj[2]), std::max(a[3], rj[3])};
            }
          });
      // a pair of which only one element is needed (e.g. y/z neighbours in a ring whose pairs are
      // offset by one from the canvas pairs) is a scalar load: same instruction count as the
      // vector load, half the wavefronts; carry sources and carried values stay vectors
      for (auto& [pk, src] : pcarry) {
        pmask[pk] = 3;
        if (src.is_load) pmask[src.src] = 3;
      }
      std::vector<std::tuple<int, std::vector<std::string>, std::vector<std::string>>> done;   // (k, vals pt0, vals pt1)
      for (int k : cph[ph]) {
        const Kernel& K = p.kernels[k];
        o << "      // kernel " << k << " " << K.name << " (canvas pairs)\n";
        std::vector<std::string> vals[2];
        for (int j = 0; j < 2; j++)
          for (size_t si = 0; si < K.stmts.size(); si++) {
            std::vector<std::string> st;
            int tmp = 0;
            for (const Insn& in : K.stmts[si].rpn) {
              std::string t = "c" + std::to_string(k) + "s" + std::to_string(si) + "_" + std::to_string(tmp++) + "_p" + std::to_string(j);
              std::string f;
              switch (in.op) {
                case KF_OP_CONST: f = lit(in.imm, p.dtype); break;
                case KF_OP_PARAM: f = "(real)a.prm[" + std::to_string(in.arg) + "]"; break;
                case KF_OP_LOAD:
                  f = cv.inlined(p, k, in.arg, in.d) ? inline_val(k, in.arg, in.d, j) : load_val(k, in.arg, in.d, j);
                  break;
                case KF_OP_NEG: case KF_OP_ABS: case KF_OP_SQRT: {
                  std::string a1 = st.back(); st.pop_back();
                  f = in.op == KF_OP_NEG ? "-" + a1
                    : in.op == KF_OP_ABS ? (p.dtype == KF_F32 ? "fabsf(" : "fabs(") + a1 + ")"
                                         : (p.dtype == KF_F32 ? "sqrtf(" : "sqrt(") + a1 + ")";
                  break;
                }
                default: {
                  std::string b = st.back(); st.pop_back();
                  std::string a1 = st.back(); st.pop_back();
                  switch (in.op) {
                    case KF_OP_ADD: f = a1 + " + " + b; break;
                    case KF_OP_SUB: f = a1 + " - " + b; break;
                    case KF_OP_MUL: f = a1 + " * " + b; break;
                    case KF_OP_DIV: f = a1 + " / " + b; break;
                    case KF_OP_MIN: f = "(" + b + " < " + a1 + ") ? " + b + " : " + a1; break;
                    case KF_OP_MAX: f = "(" + a1 + " < " + b + ") ? " + b + " : " + a1; break;
                  }
                }
              }
              o << "      const real " << t << " = " << f << ";\n";
              st.push_back(t);
            }
            vals[j].push_back(st.back());
          }
        for (int j = 0; j < 2; j++)
          for (size_t si = 0; si < K.stmts.size(); si++)
            fwd[std::make_tuple(K.stmts[si].out, p.vw(k, K.stmts[si].out), j)] = vals[j][si];
        done.emplace_back(k, vals[0], vals[1]);
      }
      // stores of the phase (after all its loads)
      for (auto& [k, v0, v1] : done) {
        const Kernel& K = p.kernels[k];
        const Ext& e = L.ext.at(k);
        const int ox = clo[0] - e.elo[0], oy = clo[1] - e.elo[1];
        const std::string c0 = "ce" + std::to_string(k) + "_0", c1 = "ce" + std::to_string(k) + "_1";
        bool any_out = false;
        for (size_t si = 0; si < K.stmts.size(); si++) {
          const Ver v{K.stmts[si].out, p.vw(k, K.stmts[si].out)};
          const int ring = L.ring_of(v);
          if (ring >= 0 && need_sts.count(v)) {
            const Ring& R = L.rings[ring];
            const int oxr = clo[0] - R.ax_lo;   // ring column of canvas x 0 is -oxr
            const std::string base = "P" + std::to_string(ring) + "_" + std::to_string(slot(ring, -L.delay.at(k))) + "[cb" +
                                     std::to_string(R.px) + "_r0 - " + std::to_string(oy * R.px + oxr);
            if (mod2(PSH + oxr) == 0)   // the pair is aligned in this ring
              o << "      if (" << c0 << " && " << c1 << ") *(real2*)&" << base << "] = real2{" << v0[si] << ", " << v1[si]
                << "};\n      else { if (" << c0 << ") " << base << "] = " << v0[si] << "; if (" << c1 << ") " << base
                << " + 1] = " << v1[si] << "; }\n";
            else
              o << "      if (" << c0 << ") " << base << "] = " << v0[si] << ";\n      if (" << c1 << ") " << base << " + 1] = " << v1[si]
                << ";\n";
          }
          if (out_index(v) >= 0) any_out = true;
        }
        if (!any_out) continue;
        const std::string pz = "(t - " + std::to_string(L.delay.at(k)) + ")";
        o << "      if (cT_r0 && " << pz << " >= z0 && " << pz << " < z1) {\n";
        o << "        const long long gi = (long long)" << pz << " * PLANE + (long long)cgy_r0 * PITCH + cgx_r0;\n";
        for (size_t si = 0; si < K.stmts.size(); si++) {
          const int oi = out_index(Ver{K.stmts[si].out, p.vw(k, K.stmts[si].out)});
          if (oi >= 0) o << "        *(real2*)&a.out[" << oi << "][gi] = real2{" << v0[si] << ", " << v1[si] << "};\n";
        }
        o << "      }\n";
      }
    }
    // carried values for the next iteration (ascending plane offset: read before overwritten)
    for (auto& [pk, src] : pcarry) {
      std::string val;
      if (!src.is_load) val = "real2{" + fwd.at(std::make_tuple(src.x, src.v, 0)) + ", " + fwd.at(std::make_tuple(src.x, src.v, 1)) + "}";
      else if (pcarry.count(src.src)) val = pq_name(src.src);
      else val = ldfirst_p.at(src.src);
      o << "      " << pq_name(pk) << " = " << val << ";\n";
    }
    if (!pcarry.empty()) o << "      pqv = true;\n";
  };
  auto qname = [](int k, const std::string& ps, int ring, int dz) {
    return "q" + std::to_string(k) + ps + "_" + std::to_string(ring) + "_" + (dz < 0 ? "m" + std::to_string(-dz) : std::to_string(dz));
  };
  // fast-iteration plane conditions fold into one range [cf0, cf1) computed once per unit
  std::string canvas_bounds;
  if (canvas_mode) {
    std::string lo, hi;
    for (int k : alive)
      for (int uu = 0; uu < U; uu++) {
        const std::string ks = std::to_string(k), d = std::to_string(L.delay.at(k) - uu);
        lo = lo.empty() ? "plo" + ks + " + " + d : "max(" + lo + ", plo" + ks + " + " + d + ")";
        hi = hi.empty() ? "phi" + ks + " + " + d : "min(" + hi + ", phi" + ks + " + " + d + ")";
      }
    std::string cxy = "true";
    for (int k : alive) {
      const Ext& e = L.ext.at(k);
      const int WX = TX + e.elo[0] + e.ehi[0], WY = TY + e.elo[1] + e.ehi[1];
      if (fx) cxy += " && x0 - " + std::to_string(e.elo[0]) + " >= 0 && x0 - " + std::to_string(e.elo[0]) + " + " +
                     std::to_string(WX) + " <= NX";
      if (fy) cxy += " && y0 - " + std::to_string(e.elo[1]) + " >= 0 && y0 - " + std::to_string(e.elo[1]) + " + " +
                     std::to_string(WY) + " <= NY";
    }
    canvas_bounds = "  const bool cfxy = " + cxy + ";\n  const int cf0 = cfxy ? " + lo + " : 0, cf1 = cfxy ? " + hi + " : 0;\n";
  }
  // rotated slot offsets are loop-carried uniform registers: with many ring slots they spill into
  // vector registers (a 35-kernel group: 66 -> 88 registers), so large groups keep the counters
  int rot_slots = 0;
  for (const Ring& R : L.rings) rot_slots += R.slots > 1 ? R.slots : 0;
  const bool rotate = rot_slots <= 32 && !getenv("KF_SLOT_COUNTERS");   // A/B switch: per-ring counters + kf_slot
  if (getenv("KF_DEBUG")) fprintf(stderr, "codegen %s: %d rotated ring slots%s\n", cg.name.c_str(), rot_slots, rotate ? "" : " (counters)");
  // Periodic ghost copies written by the producer (ghostwrite; no ghost-fill launches): after its z
  // loop an edge tile copies, for every live-out and plane it stored, the points within the ghost
  // width of a periodic x / y boundary to the opposite ghost layer (corners too), re-reading them
  // from global memory (written by this CTA before the barrier).  x images are whole 32-byte
  // sectors when the row origin and NX allow it (a ghost span widened into the padding: no
  // partial-sector stores, which cost the L2 an ECC read-modify-write -- ncu, round 2).
  const bool ghost_copy_on = L.ghost_write && !L.live_out.empty();
  const int ESEC = 32 / es;
  const bool xsector = lay.xoff >= ESEC && p.ghost[0] <= ESEC && NX % ESEC == 0 && (lay.xoff * es) % 32 == 0 &&
                       (lay.pitch * es) % 32 == 0;
  auto emit_ghost_copy_body = [&](std::ostream& o, const std::string& tt, const std::string& ind, bool delays) {
    const bool px_ = p.bc[0] == KF_BC_PERIODIC, py_ = p.bc[1] == KF_BC_PERIODIC;
    const std::string EX = xsector ? std::to_string(ESEC) : "GX";
    o << ind << "{ const int tw = min(TX, NX - x0), th = min(TY, NY - y0);\n";
    o << ind << "  const int xa0 = x0, xa1 = " << (px_ ? "min(" + EX + ", x0 + tw)" : "x0") << ";\n";
    o << ind << "  const int xb0 = " << (px_ ? "max(NX - " + EX + ", x0 + max(xa1 - x0, 0))" : "x0 + tw") << ", xb1 = x0 + tw;\n";
    o << ind << "  const int ya0 = y0, ya1 = " << (py_ ? "min(GY, y0 + th)" : "y0") << ";\n";
    o << ind << "  const int yb0 = " << (py_ ? "max(NY - GY, y0 + max(ya1 - y0, 0))" : "y0 + th") << ", yb1 = y0 + th;\n";
    o << ind << "  const int na = max(xa1 - xa0, 0), nb = max(xb1 - xb0, 0), ncx = na + nb;\n";
    o << ind << "  const int nya = max(ya1 - ya0, 0), ncy = nya + max(yb1 - yb0, 0);\n";
    o << ind << "  const int per = ncx * th + (tw - ncx) * ncy;   // x strips (all rows), then y strips (other columns)\n";
    o << ind << "  #pragma unroll 1\n";
    o << ind << "  for (int i = tid; i < per * " << U << "; i += NT) {\n";
    o << ind << "    const int uu = i / per, r = i - uu * per;\n";
    o << ind << "    int gx, gy;\n";
    o << ind << "    if (r < ncx * th) { const int c = r / th; gy = y0 + (r - c * th); gx = c < na ? xa0 + c : xb0 + (c - na); }\n";
    o << ind << "    else { const int q = r - ncx * th, w = tw - ncx, c = q / w;   // columns [x0 + na, x0 + tw - nb)\n";
    o << ind << "           gy = c < nya ? ya0 + c : yb0 + (c - nya); gx = x0 + na + (q - c * w); }\n";
    o << ind << "    const bool wx = " << (px_ ? "(gx < " + EX + " || gx >= NX - " + EX + ")" : "false") << ", wy = "
      << (py_ ? "(gy < GY || gy >= NY - GY)" : "false") << ";\n";
    o << ind << "    const int gx2 = gx < " << EX << " ? gx + NX : gx - NX, gy2 = gy < GY ? gy + NY : gy - NY;\n";
    for (size_t oi = 0; oi < L.live_out.size(); oi++) {
      const Ver v = L.live_out[oi];
      const int k = p.writer_of(v.x, v.v);
      o << ind << "    { const int pz = " << tt << " - " << (delays ? L.delay.at(k) : 0) << " + uu;\n";
      o << ind << "      if (pz >= z0 && pz < z1) {\n";
      o << ind << "        const long long pb = (long long)pz * PLANE;\n";
      o << ind << "        const real v = a.out[" << oi << "][pb + (long long)gy * PITCH + gx];\n";
      o << ind << "        if (wx) a.out[" << oi << "][pb + (long long)gy * PITCH + gx2] = v;\n";
      o << ind << "        if (wy) a.out[" << oi << "][pb + (long long)gy2 * PITCH + gx] = v;\n";
      o << ind << "        if (wx && wy) a.out[" << oi << "][pb + (long long)gy2 * PITCH + gx2] = v;\n";
      o << ind << "      }\n    }\n";
    }
    o << ind << "  }\n" << ind << "}\n";
  };
  // the copy is a __noinline__ function (emitted before the kernel), called per plane by edge tiles
  // after their z loop
  auto emit_body = [&](int j) {
  o << "    if (tid == 0 && t + " << U << " * (NSTAGE - 1) < t1) issue(t + " << U << " * (NSTAGE - 1));\n";

  o << "    kf_mbar_wait(&mbar[((t - t0) / " << U << ") % NSTAGE], (((t - t0) / " << U << ") / NSTAGE) & 1);\n";

  auto mid_index = [&](int ring) {
    for (size_t i = 0; i < mid_rings.size(); i++)
      if (mid_rings[i] == ring) return int(i);
    return -1;
  };
  auto us = [](int uu) { return std::to_string(uu); };

  // every (ring, slot offset) pointer used in this iteration
  std::vector<std::pair<int, int>> undefs;
  {
    std::set<std::pair<int, int>> need;
    for (int k : alive) {
      const Kernel& K = p.kernels[k];
      for (auto& [x, offs] : K.reads) {
        int ring = L.ring_of(Ver{x, p.vr(k, x)});
        if (ring < 0) continue;
        const int n = L.rings[ring].slots;
        for (auto& d : offs)
          for (int uu = 0; uu < U; uu++) need.insert({ring, ((-L.delay.at(k) + d[2] + uu) % n + n) % n});
      }
      for (int x : K.writes) {
        int ring = L.ring_of(Ver{x, p.vw(k, x)});
        if (ring < 0) continue;
        const int n = L.rings[ring].slots;
        for (int uu = 0; uu < U; uu++) need.insert({ring, ((-L.delay.at(k) + uu) % n + n) % n});
      }
    }
    // with per-ring counters: one pointer per (ring, slot offset) per iteration; with ring
    // unrolling: compile-time constants
    for (auto& [ring, om] : need) {
      const Ring& R = L.rings[ring];
      if (j < 0 && rotate)   // slot offsets rotated at the end of every iteration
        o << "    real* P" << ring << "_" << om << " = (real*)(sm + so" << ring << "_" << om << ");\n";
      else if (j < 0)   // computed once per iteration (measured slightly faster than per-use macros)
        o << "    real* P" << ring << "_" << om << " = (real*)(sm + " << R.smem_off << " + kf_slot(cs" << ring << ", " << om
          << ", " << R.slots << ") * " << R.plane_bytes << ");\n";
      else
        o << "#define P" << ring << "_" << om << " ((real*)(sm + " << (R.smem_off + ((j * U + om) % R.slots) * R.plane_bytes)
          << "))\n";
    }
    undefs.assign(need.begin(), need.end());
  }
  // barrier phases: a barrier is needed before k only if k reads, in this iteration, a plane
  // another kernel wrote in this iteration (0 <= D_k - dz - D_p < U); older planes were
  // published by the end-of-iteration barrier.  Within a phase no thread loads an address any
  // thread stores in the same phase (ring depths keep overwritten slots dead, R20).
  std::vector<std::vector<int>> phases;
  {
    std::set<int> dirty;   // kernels that wrote ring planes since the last barrier of this iteration
    for (int k : alive) {
      const Kernel& K = p.kernels[k];
      bool need = false;
      for (auto& [x, offs] : K.reads) {
        int v = p.vr(k, x);
        if (v < 1) continue;
        int pr = p.writer_of(x, v);
        if (!dirty.count(pr)) continue;
        for (auto& d : offs)
          if (L.delay.at(k) - d[2] - L.delay.at(pr) < U) need = true;
      }
      if (need || phases.empty()) {
        phases.emplace_back();
        dirty.clear();
      }
      phases.back().push_back(k);
      for (int x : K.writes)
        if (L.ring_of(Ver{x, p.vw(k, x)}) >= 0) dirty.insert(k);
    }
  }
  // emit_kernel(ph, pi, pm): kernel ph[pi].  pm (phase mode): fast-path code only, loads and
  // arithmetic of ph[pi+1..] nested inside before this kernel's stores, so every load of the
  // phase precedes every store in program order and the compiler can overlap the kernels'
  // SMEM latencies (it cannot reorder loads above stores through unprovable aliasing).
  std::function<void(const std::vector<int>&, size_t, bool)> emit_kernel = [&](const std::vector<int>& ph, size_t pi,
                                                                              bool pm) {
    const int k = ph[pi];
    const Kernel& K = p.kernels[k];
    const Ext& e = L.ext.at(k);
    const int WX = TX + e.elo[0] + e.ehi[0], WY = TY + e.elo[1] + e.ehi[1];
    const std::string ks = std::to_string(k);
    // outputs of this kernel
    struct OutInfo { int stmt; Ver ver; int ring; int outi; };
    std::vector<OutInfo> outs;
    bool has_mid = false, any_store = false;
    for (size_t s = 0; s < K.stmts.size(); s++) {
      Ver v{K.stmts[s].out, p.vw(k, K.stmts[s].out)};
      OutInfo oi{int(s), v, L.ring_of(v), out_index(v)};
      if (oi.ring >= 0) has_mid = true;
      if (oi.outi >= 0) any_store = true;
      outs.push_back(oi);
    }
    o << "    { // ---- kernel " << k << " " << K.name << "\n";
    o << "      const int pzb = t - " << L.delay.at(k) << ";\n";
    std::string guard, allc;
    for (int uu = 0; uu < U; uu++) {
      o << "      const int pz" << uu << " = pzb + " << uu << ";\n";
      o << "      const bool cm" << uu << " = pz" << uu << " >= plo" << ks << " && pz" << uu << " < phi" << ks << ";\n";
      o << "      const bool gf" << uu << " = !cm" << uu << " && pz" << uu << " >= glo" << ks << " && pz" << uu << " < ghi" << ks
        << ";\n";
      guard += (uu ? " || " : "") + std::string("cm") + us(uu) + (has_mid ? " || gf" + us(uu) : "");
      allc += (uu ? " && " : "") + std::string("cm") + us(uu);
    }
    const bool has_q = !pm && zq.count(k) > 0;
    if (has_q) o << "      const bool qw" << k << " = qv" << k << ";\n      qv" << k << " = false;\n";
    o << "      if (" << (pm ? std::string("true") : guard) << ") {\n";
    // slot pointers of inputs, per (ring, dz, u)
    std::map<std::tuple<int, int, int>, std::string> rp;
    for (auto& [x, offs] : K.reads) {
      int v = p.vr(k, x);
      int ring = L.ring_of(Ver{x, v});
      if (ring < 0) fail(KF_E_UNSUPPORTED, "internal: no ring for an input of " + K.name);
      (void)in_group;
      const Ring& R = L.rings[ring];
      for (auto& d : offs)
        for (int uu = 0; uu < U; uu++) {
          const int po = d[2] + uu;   // plane offset relative to pzb: one pointer per plane (CSE across U)
          auto key = std::make_tuple(ring, po, 0);
          if (rp.count(key)) continue;
          std::string nm = "r" + std::to_string(ring) + "_p" + (po < 0 ? "m" + std::to_string(-po) : std::to_string(po));
          rp[key] = nm;
          const int om = ((-L.delay.at(k) + d[2] + uu) % R.slots + R.slots) % R.slots;
          o << "        const real* " << nm << " = P" << ring << "_" << om << ";\n";
        }
    }
    for (auto& oi : outs)
      if (oi.ring >= 0) {
        const Ring& R = L.rings[oi.ring];
        for (int uu = 0; uu < U; uu++) {
          const int om = ((-L.delay.at(k) + uu) % R.slots + R.slots) % R.slots;
          // writes use the producer's region coordinates; the ring box starts ax_lo - blo0 columns
          // further left (16-byte aligned box origin)
          o << "        real* w" << oi.ring << "_" << uu << " = P" << oi.ring << "_" << om << " + " << (R.ax_lo - R.blo[0]) << ";\n";
        }
      }
    o << "        const int gx0 = x0 - " << e.elo[0] << ", gy0 = y0 - " << e.elo[1] << ";\n";
    const int R = WX * WY;
    // statements of sub-iteration uu at point suffix ps (one IEEE op per RPN node, in order)
    bool blocked = false;   // fast path with register blocking: loads index a per-pitch block base
    // fast path: every distinct shared-memory address (ring, plane, offset from the round's block
    // origin) is loaded once per round and reused by every point and plane of the block that
    // reads it (explicit CSE: the compiler does not merge these loads itself)
    std::map<std::tuple<int, int, int>, std::string> ldcache;
    int cur_i = 0, cur_j = 0;
    std::string cur_rs;
    auto emit = [&](int uu, const std::string& ind, const std::string& ps) {
      std::vector<std::string> vals;
      for (size_t s = 0; s < K.stmts.size(); s++) {
        const Stmt& S_ = K.stmts[s];
        std::vector<std::string> st;
        int tmp = 0;
        for (const Insn& in : S_.rpn) {
          std::string t = "s" + std::to_string(s) + "_" + std::to_string(tmp++) + "_" + us(uu) + ps;
          switch (in.op) {
            case KF_OP_CONST: o << ind << "const real " << t << " = " << lit(in.imm, p.dtype) << ";\n"; break;
            case KF_OP_PARAM: o << ind << "const real " << t << " = (real)a.prm[" << in.arg << "];\n"; break;
            case KF_OP_LOAD: {
              int v = p.vr(k, in.arg);
              int ring = L.ring_of(Ver{in.arg, v});
              const Ring& Rg = L.rings[ring];
              int cx = Rg.ax_lo - e.elo[0] + in.d[0];
              int cy = Rg.blo[1] - e.elo[1] + in.d[1];
              if (blocked && has_q && in.d[0] == 0 && in.d[1] == 0 && zq[k].rings.count(ring))
                o << ind << "const real " << t << " = " << qname(k, ps, ring, in.d[2]) << ";\n";
              else if (blocked) {   // round base per row pitch + constant offset, loaded once per address
                const int po = int(in.d[2]) + uu;
                const int off = (cy + cur_j) * Rg.px + cx + cur_i;
                auto key = std::make_tuple(ring, po, off);
                auto it = ldcache.find(key);
                if (it == ldcache.end()) {
                  std::string nm = "ld" + std::to_string(k) + "_" + std::to_string(ring) + "_" +
                                   (po < 0 ? "m" + std::to_string(-po) : std::to_string(po)) + "_" +
                                   (off < 0 ? "m" + std::to_string(-off) : std::to_string(off)) + cur_rs;
                  o << ind << "const real " << nm << " = " << rp[std::make_tuple(ring, po, 0)] << "[bb" << Rg.px << cur_rs
                    << " + " << off << "];\n";
                  it = ldcache.emplace(key, nm).first;
                }
                o << ind << "const real " << t << " = " << it->second << ";\n";
              }
              else
                o << ind << "const real " << t << " = " << rp[std::make_tuple(ring, int(in.d[2]) + uu, 0)] << "[(ly" << ps
                  << " + " << cy << ") * " << Rg.px << " + lx" << ps << " + " << cx << "];\n";
              break;
            }
            case KF_OP_NEG: case KF_OP_ABS: case KF_OP_SQRT: {
              std::string a1 = st.back(); st.pop_back();
              std::string f = in.op == KF_OP_NEG ? "-" + a1
                            : in.op == KF_OP_ABS ? (p.dtype == KF_F32 ? "fabsf(" : "fabs(") + a1 + ")"
                                                 : (p.dtype == KF_F32 ? "sqrtf(" : "sqrt(") + a1 + ")";
              o << ind << "const real " << t << " = " << f << ";\n";
              break;
            }
            default: {
              std::string b = st.back(); st.pop_back();
              std::string a1 = st.back(); st.pop_back();
              std::string f;
              switch (in.op) {
                case KF_OP_ADD: f = a1 + " + " + b; break;
                case KF_OP_SUB: f = a1 + " - " + b; break;
                case KF_OP_MUL: f = a1 + " * " + b; break;
                case KF_OP_DIV: f = a1 + " / " + b; break;
                case KF_OP_MIN: f = "(" + b + " < " + a1 + ") ? " + b + " : " + a1; break;
                case KF_OP_MAX: f = "(" + a1 + " < " + b + ") ? " + b + " : " + a1; break;
              }
              o << ind << "const real " << t << " = " << f << ";\n";
            }
          }
          st.push_back(t);
        }
        vals.push_back(st.back());
      }
      return vals;
    };
    // outputs: SMEM ring and/or HBM (interior of the tile only); `act` predicates padded lanes
    auto emit_out = [&](int uu, const std::vector<std::string>& vals, const std::string& ind, const std::string& ps,
                        const std::string& act) {
      for (auto& oi : outs)
        if (oi.ring >= 0)
          o << ind << (act.empty() ? "" : "if (" + act + ") ") << "w" << oi.ring << "_" << uu << "[ly" << ps << " * "
            << L.rings[oi.ring].px << " + lx" << ps << "] = " << vals[oi.stmt] << ";\n";
      if (any_store) {
        o << ind << "if (" << (act.empty() ? "" : act + " && ") << "inT" << ps << " && pz" << uu << " >= z0 && pz" << uu
          << " < z1) {\n";
        o << ind << "  const long long gi = (long long)pz" << uu << " * PLANE + (long long)gy" << ps << " * PITCH + gx" << ps
          << ";\n";
        for (auto& oi : outs)
          if (oi.outi >= 0) o << ind << "  a.out[" << oi.outi << "][gi] = " << vals[oi.stmt] << ";\n";
        o << ind << "}\n";
      }
    };
    // FROZEN axes: outside the interior the ring holds the version's stored ghost (R9).  Ghost
    // cells of PERIODIC axes in frozen-ghost rows/planes are constant and filled once per run
    // (wrap, or the neighbour's values in a decomposition), so the stored cell is read as is;
    // reads are range-checked (ragged tiles reach past the ghost layer).
    auto emit_ghost = [&](int uu, const std::string& ind) {
      o << ind << "const int qx = gx, qy = gy, qz = pz" << us(uu) << ";\n";
      std::string valid = "qx >= -GX && qx < NX + GX && qy >= -GY && qy < NY + GY";
      if (!fz) valid += " && qz >= -GZ && qz < NZ + GZ";
      o << ind << "if (" << valid << ") {\n";
      o << ind << "  const long long gi = (long long)qz * PLANE + (long long)qy * PITCH + qx;\n";
      for (auto& oi : outs)
        if (oi.ring >= 0)
          o << ind << "  w" << oi.ring << "_" << uu << "[ly * " << L.rings[oi.ring].px << " + lx] = a.gsrc["
            << mid_index(oi.ring) << "][gi];\n";
      o << ind << "}\n";
    };
    // ---- fast path (CTA-uniform): every sub-iteration computes and, on FROZEN xy axes, the
    // whole region lies in the interior.  Rounds are unrolled straight-line code: lanes past
    // the region recompute its last point (clamped index) and skip the stores, so all loads and
    // arithmetic of all rounds and planes are independent and can be interleaved (ILP).
    {
      std::string fast = allc;
      if (fx) fast += " && gx0 >= 0 && gx0 + " + std::to_string(WX) + " <= NX";
      if (fy) fast += " && gy0 >= 0 && gy0 + " + std::to_string(WY) + " <= NY";
      o << "        if (" << (pm ? std::string("true") : fast) << ") {\n";
      // register blocking: each thread computes a bx x by block of adjacent points; block origins
      // are clamped inside the region (edge blocks overlap and recompute identical values), and
      // lanes past the last block redo it -- duplicate stores write the same bits.
      const int bx = std::min(L.pblock[0], WX), by = std::min(L.pblock[1], WY);
      const int nbx = (WX + bx - 1) / bx, nby = (WY + by - 1) / by, NB = nbx * nby;
      const int rounds = (NB + NT - 1) / NT;
      std::set<int> pitches;
      for (auto& [x, offs] : K.reads) pitches.insert(L.rings[L.ring_of(Ver{x, p.vr(k, x)})].px);
      std::vector<std::vector<std::vector<std::string>>> V;
      std::vector<std::string> pss;
      blocked = true;
      for (int r = 0; r < rounds; r++) {
        const std::string rs = "_r" + std::to_string(r);
        o << "          const int ib" << rs << " = min(tid + " << r * NT << ", " << (NB - 1) << ");\n";
        o << "          const int iby" << rs << " = ib" << rs << " / " << nbx << ", ibx" << rs << " = ib" << rs << " - iby" << rs
          << " * " << nbx << ";\n";
        o << "          const int bx0" << rs << " = min(ibx" << rs << " * " << bx << ", " << (WX - bx) << "), by0" << rs
          << " = min(iby" << rs << " * " << by << ", " << (WY - by) << ");\n";
        for (int pch : pitches)
          o << "          const int bb" << pch << rs << " = by0" << rs << " * " << pch << " + bx0" << rs << ";\n";
        cur_rs = rs;
        ldcache.clear();   // loads are per round (each round is a different block of points)
        for (int j = 0; j < by; j++)
          for (int i = 0; i < bx; i++) {
            const std::string ps = rs + "_" + std::to_string(i) + "_" + std::to_string(j);
            pss.push_back(ps);
            o << "          const int lx" << ps << " = bx0" << rs << " + " << i << ", ly" << ps << " = by0" << rs << " + " << j
              << ";\n";
            o << "          const int gx" << ps << " = gx0 + lx" << ps << ", gy" << ps << " = gy0 + ly" << ps << ";\n";
            for (int pch : pitches)
              o << "          const int b" << pch << ps << " = ly" << ps << " * " << pch << " + lx" << ps << ";\n";
            if (any_store)
              o << "          const bool inT" << ps << " = lx" << ps << " >= " << e.elo[0] << " && lx" << ps << " < "
                << (e.elo[0] + TX) << " && gx" << ps << " < NX && ly" << ps << " >= " << e.elo[1] << " && ly" << ps << " < "
                << (e.elo[1] + TY) << " && gy" << ps << " < NY;\n";
            if (has_q)
              for (auto& [ring, mm] : zq[k].rings) {
                const Ring& Rg = L.rings[ring];
                const int cx = Rg.ax_lo - e.elo[0], cy = Rg.blo[1] - e.elo[1];
                auto ld = [&](int dz) {
                  return rp[std::make_tuple(ring, dz, 0)] + "[b" + std::to_string(Rg.px) + ps + " + " +
                         std::to_string(cy * Rg.px + cx) + "]";
                };
                o << "          if (qw" << k << ") {";
                for (int dz = mm.first; dz < mm.second; dz++) o << " " << qname(k, ps, ring, dz) << " = " << qname(k, ps, ring, dz + 1) << ";";
                o << " } else {";
                for (int dz = mm.first; dz < mm.second; dz++) o << " " << qname(k, ps, ring, dz) << " = " << ld(dz) << ";";
                o << " }\n";
                o << "          " << qname(k, ps, ring, mm.second) << " = " << ld(mm.second) << ";\n";
              }
            std::vector<std::vector<std::string>> vu;
            cur_i = i;
            cur_j = j;
            for (int uu = 0; uu < U; uu++) vu.push_back(emit(uu, "          ", ps));
            V.push_back(vu);
          }
      }
      blocked = false;
      if (pm && pi + 1 < ph.size()) emit_kernel(ph, pi + 1, true);
      for (size_t q = 0; q < pss.size(); q++)
        for (int uu = 0; uu < U; uu++) emit_out(uu, V[q][uu], "          ", pss[q], "");
      if (has_q) o << "          qv" << k << " = true;\n";
      if (pm) {
        o << "        }\n      }\n    }\n";
        return;
      }
      o << "        } else {\n";
    }
    // ---- general path: per point boundary handling (frozen ghosts, ghost planes, ragged tiles)
    if (R <= NT) {
      o << "        if (tid < " << R << ") {\n";
      o << "          const int lx = lx0_" << ks << ", ly = ly0_" << ks << ";\n";
    } else {
      o << "        int lx = lx0_" << ks << ", ly = ly0_" << ks << ";\n";
      o << "        for (int i = tid; i < " << R << "; i += NT, lx += " << (NT % WX) << ", ly += " << (NT / WX) << ") {\n";
      o << "          if (lx >= " << WX << ") { lx -= " << WX << "; ++ly; }\n";
    }
    o << "          const int gx = gx0 + lx, gy = gy0 + ly;\n";
    std::string inxy = "true";
    if (fx) inxy += " && (unsigned)gx < (unsigned)NX";
    if (fy) inxy += " && (unsigned)gy < (unsigned)NY";
    o << "          const bool inxy = " << inxy << ";\n";
    if (any_store)
      o << "          const bool inT = lx >= " << e.elo[0] << " && lx < " << (e.elo[0] + TX) << " && gx < NX && ly >= " << e.elo[1]
        << " && ly < " << (e.elo[1] + TY) << " && gy < NY;\n";
    for (int uu = 0; uu < U; uu++) {
      o << "          if (cm" << uu << " && inxy) {\n";
      auto vals = emit(uu, "            ", "");
      emit_out(uu, vals, "            ", "", "");
      o << "          }";
      if (has_mid) {
        o << " else if (cm" << uu << " || gf" << uu << ") {\n";
        emit_ghost(uu, "            ");
        o << "          }\n";
      } else {
        o << "\n";
      }
    }
    o << "        }\n";   // point loop
    o << "        }\n";   // fast / general
    o << "      }\n";     // guard
    o << "    }\n";
    (void)has_mid;
  };
  const bool phase_batch = zq.empty() && !getenv("KF_NO_PHASE");   // KF_NO_PHASE: A/B switch
  const bool use_canvas = canvas_mode && zq.empty();
  if (use_canvas) {
    // CTA-uniform: every kernel computes all its planes this iteration (and, on FROZEN xy axes,
    // its region lies in the interior)
    std::string c;
    for (int k : alive) {
      const Ext& e = L.ext.at(k);
      const int WX = TX + e.elo[0] + e.ehi[0], WY = TY + e.elo[1] + e.ehi[1];
      const std::string ks = std::to_string(k);
      for (int uu = 0; uu < U; uu++) {
        const std::string pz = "(t - " + std::to_string(L.delay.at(k) - uu) + ")";
        c += std::string(c.empty() ? "" : " && ") + pz + " >= plo" + ks + " && " + pz + " < phi" + ks;
      }
      if (fx) c += " && x0 - " + std::to_string(e.elo[0]) + " >= 0 && x0 - " + std::to_string(e.elo[0]) + " + " +
                   std::to_string(WX) + " <= NX";
      if (fy) c += " && y0 - " + std::to_string(e.elo[1]) + " >= 0 && y0 - " + std::to_string(e.elo[1]) + " + " +
                   std::to_string(WY) + " <= NY";
    }
    if (!getenv("KF_CANVAS_COND")) c = "t >= cf0 && t < cf1";   // A/B switch: the per-kernel conjunction
    o << "    if (" << c << ") {   // ---- fast iteration on the canvas\n";
    // clamped load bases (canvas_ld), recomputed every iteration from an opaque zero so the compiler
    // does not keep them live across the stream loop (cheap integer ops instead of registers)
    o << "      int kz;\n      asm volatile(\"mov.u32 %0, 0;\" : \"=r\"(kz));\n/*@@KF_CLAMP_BASES@@*/";
    if (pair_mode) emit_canvas_pairs();
    else emit_canvas();
    o << "    } else {\n";
    if (!carry.empty()) o << "    cqv = false;\n";
    if (!pcarry.empty()) o << "    pqv = false;\n";
  }
  for (size_t pi = 0; pi < phases.size(); pi++) {
    const auto& ph = phases[pi];
    if (pi > 0) o << "    __syncthreads();\n";
    const bool batch = phase_batch && ph.size() > 1;
    if (batch) {
      // CTA-uniform: every kernel of the phase takes its fast path this iteration
      std::string c;
      for (int k : ph) {
        const Ext& e = L.ext.at(k);
        const int WX = TX + e.elo[0] + e.ehi[0], WY = TY + e.elo[1] + e.ehi[1];
        const std::string ks = std::to_string(k);
        for (int uu = 0; uu < U; uu++) {
          const std::string pz = "(t - " + std::to_string(L.delay.at(k) - uu) + ")";
          c += std::string(c.empty() ? "" : " && ") + pz + " >= plo" + ks + " && " + pz + " < phi" + ks;
        }
        if (fx) c += " && x0 - " + std::to_string(e.elo[0]) + " >= 0 && x0 - " + std::to_string(e.elo[0]) + " + " +
                     std::to_string(WX) + " <= NX";
        if (fy) c += " && y0 - " + std::to_string(e.elo[1]) + " >= 0 && y0 - " + std::to_string(e.elo[1]) + " + " +
                     std::to_string(WY) + " <= NY";
      }
      o << "    if (" << c << ") {   // ---- phase: loads of all kernels before their stores\n";
      emit_kernel(ph, 0, true);
      o << "    } else {\n";
    }
    for (int k : ph) emit_kernel(std::vector<int>{k}, 0, false);
    if (batch) o << "    }\n";
  }
  if (use_canvas) o << "    }\n";
  o << "    __syncthreads();\n";
  if (NU != 0)
    for (auto& [ring, om] : undefs) o << "#undef P" << ring << "_" << om << "\n";
  };   // emit_body
  // z register queues (declared before the stream loop: they carry values across iterations)
  for (auto& [k, qs] : zq) {
    o << "  bool qv" << k << " = false;\n";
    for (auto& ps : qs.pss)
      for (auto& [ring, mm] : qs.rings)
        for (int dz = mm.first; dz <= mm.second; dz++)
          o << "  real q" << k << ps << "_" << ring << "_" << (dz < 0 ? "m" + std::to_string(-dz) : std::to_string(dz))
            << " = 0;\n";
  }
  if (!pcarry.empty()) {
    o << "  bool pqv = false;\n";
    for (auto& [pk, src] : pcarry) o << "  real2 " << pq_name(pk) << " = real2{(real)0, (real)0};\n";
  }
  if (canvas_mode && zq.empty() && !carry.empty()) {
    o << "  bool cqv = false;\n";
    for (int r = 0; r < CROUNDS; r++)
      for (auto& [key, src] : carry) o << "  real " << key_name("cq", key, "_r" + std::to_string(r)) << " = 0;\n";
  }
  o << canvas_bounds;

  if (NU == 0 && rotate) {
    // slot byte offsets of every ring, rotated by U slots per iteration: slot (c + om) mod n of a
    // per-ring counter c costs ~5 uniform instructions per pointer and iteration (ncu: ~35 % of all
    // instructions were uniform-datapath bookkeeping), a rotation one move per slot
    for (size_t ri = 0; ri < L.rings.size(); ri++)
      for (int sl = 0; sl < L.rings[ri].slots; sl++)
        o << "  u32 so" << ri << "_" << sl << " = " << L.rings[ri].smem_off + sl * L.rings[ri].plane_bytes << "u;\n";
    o << "  for (int t = t0; t < t1; t += " << U << ") {\n";
    emit_body(-1);
    for (size_t ri = 0; ri < L.rings.size(); ri++) {
      const int n = L.rings[ri].slots;
      if (n == 1 || U % n == 0) continue;
      o << "    { const u32";
      for (int sl = 0; sl < n; sl++) o << (sl ? ", " : " ") << "r" << sl << " = so" << ri << "_" << sl;
      o << ";";
      for (int sl = 0; sl < n; sl++) o << " so" << ri << "_" << sl << " = r" << (sl + U) % n << ";";
      o << " }\n";
    }
    o << "  }\n";
  } else if (NU == 0) {
    for (size_t ri = 0; ri < L.rings.size(); ri++) o << "  int cs" << ri << " = 0;\n";
    o << "  for (int t = t0; t < t1; t += " << U << ") {\n";
    emit_body(-1);
    for (size_t ri = 0; ri < L.rings.size(); ri++)
      o << "    cs" << ri << " += " << U << "; if (cs" << ri << " >= " << L.rings[ri].slots << ") cs" << ri << " -= "
        << L.rings[ri].slots << ";\n";
    o << "  }\n";
  } else {
    o << "  for (int tb = t0; tb < t1; tb += " << NU * U << ") {\n";
    for (int j = 0; j < NU; j++) {
      o << "   { const int t = tb + " << j * U << ";\n";
      o << "   if (t < t1) {\n";
      emit_body(j);
      o << "   } }\n";
    }
    o << "  }\n";
  }
  if (ghost_copy_on) {
    // after the whole z range (round 2: per-iteration copies, even in a __noinline__ function, made
    // every group 10-30 % slower; the epilogue 5-15 %; the fills are the default)
    o << "  __syncthreads();\n";
    o << "  if (edge_tile) {\n";
    o << "    for (int tz = z0; tz < z1; tz += " << U << ") kf_gcopy(a, tz, x0, y0, z0, z1);\n";
    o << "  }\n";
  }
  o << "}\n";
  cg.source = o.str();
  {
    std::ostringstream fo;
    if (ghost_copy_on) {
      fo << "static __device__ __noinline__ void kf_gcopy(const KfArgs& a, const int tt, const int x0, const int y0,"
            " const int z0, const int z1) {\n  const int tid = threadIdx.x;\n";
      emit_ghost_copy_body(fo, "tt", "  ", false);
      fo << "}\n";
    }
    const std::string mark = "/*@@KF_GCOPY@@*/";
    const size_t at = cg.source.find(mark);
    if (at != std::string::npos) cg.source.replace(at, mark.size(), fo.str());
  }
  {
    const std::string mark = "/*@@KF_CLAMP_BASES@@*/";
    for (size_t at = cg.source.find(mark); at != std::string::npos; at = cg.source.find(mark, at))
      cg.source.replace(at, mark.size(), clamp_defs);
  }
  return cg;
}

}  // namespace kf
