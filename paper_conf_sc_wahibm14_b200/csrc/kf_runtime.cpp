// Runtime executor (rows a6, a10): NVRTC JIT of the generated group kernels for sm_100a,
// module/tensor-map management, renamed-buffer ping-pong, periodic ghost fills, and the
// step loop (a CUDA graph of one replay period).
//
// Host -> device boundary: one graph launch per period; everything inside the step runs
// in this library's kernels (JIT'd group kernels + AOT helpers in kf_kernels.cu).
// The paper fused kernels by hand and replaced the calls "from the host by a
// single call to the newly constructed kernel" (P:39(c)); here the host issues groups in
// quotient-topological order (R18).
#include <cuda.h>
#include <cuda_runtime.h>
#include <nvrtc.h>

#include <algorithm>
#include <atomic>
#include <cstring>
#include <functional>
#include <sstream>
#include <thread>

#include "kf_internal.hpp"
#include "kf_kernels.hpp"

namespace kf {

// ---------------------------------------------------------------- driver entry points
struct Drv {
  CUresult (*moduleLoadData)(CUmodule*, const void*) = nullptr;
  CUresult (*moduleUnload)(CUmodule) = nullptr;
  CUresult (*moduleGetFunction)(CUfunction*, CUmodule, const char*) = nullptr;
  CUresult (*funcSetAttribute)(CUfunction, CUfunction_attribute, int) = nullptr;
  CUresult (*funcGetAttribute)(int*, CUfunction_attribute, CUfunction) = nullptr;
  CUresult (*launchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, CUstream,
                           void**, void**) = nullptr;
  CUresult (*tensorMapEncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill) = nullptr;
  CUresult (*getErrorString)(CUresult, const char**) = nullptr;
};

// (a failing runtime call also leaves its error as the thread's "last error": clear it, or the next
// launch helper's cudaGetLastError() would report it again)
#define CK(x)                                                                                       \
  do {                                                                                              \
    cudaError_t e_ = (x);                                                                           \
    if (e_ != cudaSuccess) {                                                                        \
      cudaGetLastError();                                                                           \
      fail(KF_E_CUDA, std::string(#x) + ": " + cudaGetErrorString(e_));                             \
    }                                                                                               \
  } while (0)

static Drv& drv() {
  static Drv d;
  static std::once_flag once;
  static std::string err;
  std::call_once(once, [] {
    auto get = [](const char* sym, void** fp) {
      cudaDriverEntryPointQueryResult q;
      cudaError_t e = cudaGetDriverEntryPoint(sym, fp, cudaEnableDefault, &q);
      if (e != cudaSuccess || q != cudaDriverEntryPointSuccess) *fp = nullptr;
    };
    get("cuModuleLoadData", (void**)&d.moduleLoadData);
    get("cuModuleUnload", (void**)&d.moduleUnload);
    get("cuModuleGetFunction", (void**)&d.moduleGetFunction);
    get("cuFuncSetAttribute", (void**)&d.funcSetAttribute);
    get("cuFuncGetAttribute", (void**)&d.funcGetAttribute);
    get("cuLaunchKernel", (void**)&d.launchKernel);
    get("cuTensorMapEncodeTiled", (void**)&d.tensorMapEncodeTiled);
    get("cuGetErrorString", (void**)&d.getErrorString);
  });
  if (!d.moduleLoadData || !d.launchKernel || !d.tensorMapEncodeTiled)
    fail(KF_E_UNSUPPORTED, "CUDA driver entry points unavailable (no GPU / driver?)");
  return d;
}

static void ckd(CUresult r, const char* what) {
  if (r == CUDA_SUCCESS) return;
  const char* s = nullptr;
  if (drv().getErrorString) drv().getErrorString(r, &s);
  fail(KF_E_CUDA, std::string(what) + ": " + (s ? s : "CUDA driver error " + std::to_string(int(r))));
}

// ---------------------------------------------------------------- NVRTC
struct Compiled {
  std::vector<char> cubin;
  std::string log;
  int regs_ptxas = -1, spill = -1;
  bool nocap = false;   // a fallback build ("#define KF_CAP c" prepended)
  int cap_idx = -1;     // position on the source's KF_CAPS ladder (-1: the primary build)
};

static Compiled nvrtc_compile(const std::string& src, const std::string& name) {
  nvrtcProgram prog;
  if (nvrtcCreateProgram(&prog, src.c_str(), (name + ".cu").c_str(), 0, nullptr, nullptr) != NVRTC_SUCCESS)
    fail(KF_E_NVRTC, "nvrtcCreateProgram failed");
  // IEEE semantics, no FMA contraction (R16): fused results must equal the unfused program bit for bit.
  const char* opts[] = {"--gpu-architecture=sm_100a", "--fmad=false", "--prec-div=true", "--prec-sqrt=true",
                        "--ftz=false", "-std=c++17", "-lineinfo", "--ptxas-options=-v"};
  if (getenv("KF_DEBUG")) fprintf(stderr, "nvrtc: compiling %s\n", name.c_str());
  nvrtcResult r = nvrtcCompileProgram(prog, int(sizeof(opts) / sizeof(opts[0])), opts);
  if (getenv("KF_DEBUG")) fprintf(stderr, "nvrtc: done %d\n", int(r));
  Compiled c;
  size_t ls = 0;
  nvrtcGetProgramLogSize(prog, &ls);
  c.log.resize(ls);
  if (ls) nvrtcGetProgramLog(prog, &c.log[0]);
  if (r != NVRTC_SUCCESS) {
    nvrtcDestroyProgram(&prog);
    // the errors, not the warnings, first
    std::string errs;
    for (size_t a = 0, b; a < c.log.size(); a = b + 1) {
      b = c.log.find('\n', a);
      if (b == std::string::npos) b = c.log.size();
      const std::string line = c.log.substr(a, b - a);
      if (line.find("error") != std::string::npos) errs += line + "\n";
    }
    if (const char* dir = getenv("KF_DUMP_DIR")) {
      if (FILE* f = fopen((std::string(dir) + "/" + name + "_failed.cu").c_str(), "w")) { fwrite(src.data(), 1, src.size(), f); fclose(f); }
    }
    fail(KF_E_NVRTC, "NVRTC failed for " + name + ": " + errs.substr(0, 3000) + c.log.substr(0, 1000));
  }
  size_t cs = 0;
  nvrtcGetCUBINSize(prog, &cs);
  c.cubin.resize(cs);
  nvrtcGetCUBIN(prog, c.cubin.data());
  nvrtcDestroyProgram(&prog);
  if (const char* dir = getenv("KF_DUMP_DIR")) {   // debugging aid: keep the generated source and cubin
    std::string base = std::string(dir) + "/" + name + (src.rfind("#define KF_CAP", 0) == 0 ? "_cap" + std::to_string(atoi(src.c_str() + 15)) : "");
    if (FILE* f = fopen((base + ".log").c_str(), "w")) { fwrite(c.log.data(), 1, c.log.size(), f); fclose(f); }
    if (FILE* f = fopen((base + ".cu").c_str(), "w")) { fwrite(src.data(), 1, src.size(), f); fclose(f); }
    if (FILE* f = fopen((base + ".cubin").c_str(), "wb")) { fwrite(c.cubin.data(), 1, c.cubin.size(), f); fclose(f); }
  }
  auto p = c.log.find("Used ");
  if (p != std::string::npos) c.regs_ptxas = atoi(c.log.c_str() + p + 5);
  auto q = c.log.find("bytes spill stores");
  if (q != std::string::npos) {
    size_t b = c.log.rfind(',', q);
    b = b == std::string::npos ? 0 : b + 1;
    c.spill = atoi(c.log.c_str() + b);
  }
  return c;
}

static std::mutex g_cache_mu;
static std::map<std::string, std::shared_ptr<Compiled>> g_cubin_cache;   // source -> cubin

// register model bound the kernel was generated for (#define KF_REST n)
static int source_rest(const std::string& src) {
  const auto p = src.find("#define KF_REST ");
  return p == std::string::npos ? 255 : atoi(src.c_str() + p + 16);
}

// fallback register caps of a generated kernel ("// KF_CAPS c0 c1 ... R_est")
static std::vector<int> source_caps(const std::string& src) {
  std::vector<int> caps;
  const auto p = src.find("// KF_CAPS");
  if (p == std::string::npos) return caps;
  std::istringstream is(src.substr(p + 10, src.find('\n', p) - p - 10));
  for (int c; is >> c;) caps.push_back(c);
  return caps;
}

static bool needs_next(const Compiled& c, const std::string& src) {
  return c.spill > 0 || c.regs_ptxas > source_rest(src);
}

// The build after `c` on the cap ladder (c->cap_idx + 1), or nullptr at the end of it.
static std::shared_ptr<Compiled> compile_next(const std::string& src, const std::string& name, int cap_idx) {
  const std::vector<int> caps = source_caps(src);
  // minblocks >= 0 sources start at caps[0] (KF_CAP default): the first fallback is caps[1]
  const bool capped_primary = src.find("#define KF_BOUNDS __maxnreg__(KF_CAP)\n") != std::string::npos &&
                              src.find("#ifndef KF_CAP\n#define KF_CAP") != std::string::npos;
  const int next = cap_idx + 1 + (cap_idx < 0 && capped_primary ? 1 : 0);
  if (next >= int(caps.size())) return nullptr;
  auto c = std::make_shared<Compiled>(nvrtc_compile("#define KF_CAP " + std::to_string(caps[next]) + "\n" + src, name));
  c->cap_idx = next;
  c->nocap = true;
  return c;
}

static std::shared_ptr<Compiled> compile_cached(const std::string& src, const std::string& name) {
  {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    auto it = g_cubin_cache.find(src);
    if (it != g_cubin_cache.end()) return it->second;
  }
  auto c = std::make_shared<Compiled>(nvrtc_compile(src, name));
  // the build must neither spill nor exceed the register model (V8): walk down the cap ladder
  while (needs_next(*c, src)) {
    auto n = compile_next(src, name, c->cap_idx);
    if (!n) break;
    c = n;
  }
  std::lock_guard<std::mutex> lk(g_cache_mu);
  g_cubin_cache[src] = c;
  return c;
}

// The ptxas statistics come from the NVRTC log, which is empty when NVRTC serves a program from
// its own on-disk cache (seen on reused GPU boxes): the checks above then never fire.  The loader
// checks the loaded function's registers and local memory instead and comes here for the next cap.
static std::shared_ptr<Compiled> compile_after(const std::string& src, const std::string& name, int cap_idx) {
  auto c = compile_next(src, name, cap_idx);
  if (!c) return nullptr;
  std::lock_guard<std::mutex> lk(g_cache_mu);
  g_cubin_cache[src] = c;
  return c;
}

// ---------------------------------------------------------------- executor
struct Op {
  int kind;   // 0 = periodic fill of a buffer, 1 = group launch
  int group;
  int buf;
};

struct GroupExec {
  int gid = 0;
  GroupLowering L;
  Codegen cg;
  std::shared_ptr<Compiled> comp;
  CUmodule mod = nullptr;
  CUfunction fn = nullptr;
  int grid = 0, smem = 0, regs = -1, local = -1, maxthr = -1;
  Split split;   // interior / boundary units (a11 overlap)
  uint64_t bytes = 0;
  std::vector<Ver> ins, outs, mids;
  size_t blob_size = 0;
};

}  // namespace kf

using namespace kf;

struct kf_exec {
  kf_program* prog = nullptr;
  Plan plan;
  kf_target t{};
  std::vector<int> order;
  std::vector<GroupExec> G;
  int period = 1;
  std::vector<std::vector<Op>> sched;      // per parity (fills dropped when groups write ghost copies)
  std::vector<std::vector<Op>> sched_full; // per parity, every fill (domain decomposition exchanges)
  std::vector<Ver> scratch_vers;           // scratch buffer i holds (x, v)
  uint64_t scratch_bytes = 0, array_bytes = 0;
  std::vector<int> fill_all;               // buffers filled once at the start of a run
  int device = -1;
  // current pointers / argument blobs
  std::vector<void*> cur_arrays;
  void* cur_scratch = nullptr;
  std::vector<double> cur_params;
  std::vector<std::vector<std::vector<unsigned char>>> blobs;   // [parity][group]
  bool blobs_valid = false;
  uint64_t blob_gen = 0;                   // bumped whenever the argument blobs are rebuilt
  void* shell_init_scratch = nullptr;
  std::vector<void*> shell_init_arrays;
  // graph
  bool use_graph = true;
  cudaStream_t cap_stream = nullptr;
  cudaGraphExec_t gexec = nullptr;
  // profiling
  bool profiling = false;
  std::vector<double> gms;
  int64_t launches = 0;
  std::vector<std::tuple<int, cudaEvent_t, cudaEvent_t>> pending;
  std::vector<cudaEvent_t> evpool;
  // host-buffer runs
  std::vector<void*> dev_arrays;
  void* dev_scratch = nullptr;
  bool host_first = true;
  uint64_t step_bytes = 0;
};

namespace kf {

// Renamed array versions that need their own buffer ("redundant arrays"): every version of a
// relaxed array except the final version of a TEMP array (which lives in the array itself).
// *period = 2 when a renamed array is step-live (its buffers ping-pong between steps).
static std::vector<Ver> renamed_versions(const Program& p, int* period) {
  std::vector<Ver> out;
  *period = 1;
  for (int x = 0; x < p.na; x++) {
    if (!p.relaxed[x]) continue;
    int w = int(p.writers[x].size());
    for (int v = 1; v <= w; v++) {
      if (v == w && !p.step_live[x]) continue;
      out.push_back(Ver{x, v});
    }
    if (p.step_live[x]) *period = 2;
  }
  return out;
}

static uint64_t padded_array_bytes(const Program& p) {
  return (uint64_t(p.layout.elems) * p.es + 255) / 256 * 256;
}

static int buffer_id(const kf_exec* E, const Ver& v, int parity) {
  const Program& p = E->prog->p;
  int x = v.x;
  if (!p.relaxed[x]) return x;
  int w = int(p.writers[x].size());
  auto scr = [&](int ver) {
    for (size_t i = 0; i < E->scratch_vers.size(); i++)
      if (E->scratch_vers[i] == Ver{x, ver}) return p.na + int(i);
    fail(KF_E_ARG, "internal: missing scratch buffer");
  };
  if (!p.step_live[x]) {
    if (v.v == 0 || v.v == w) return x;
    return scr(v.v);
  }
  if (v.v == 0) return parity == 0 ? x : scr(w);
  if (v.v == w) return parity == 0 ? scr(w) : x;
  return scr(v.v);
}

static Geom geom(const Program& p) {
  Geom g;
  g.pitch = p.layout.pitch;
  g.plane = p.layout.plane;
  g.xoff = p.layout.xoff;
  g.nx = int(p.n[0]); g.ny = int(p.n[1]); g.nz = int(p.n[2]);
  g.gx = p.ghost[0]; g.gy = p.ghost[1]; g.gz = p.ghost[2];
  return g;
}

static void* buf_ptr(const kf_exec* E, int id) {
  const Program& p = E->prog->p;
  if (id < p.na) return E->cur_arrays[id];
  return (char*)E->cur_scratch + uint64_t(id - p.na) * E->array_bytes;
}

static void build_blobs(kf_exec* E) {
  const Program& p = E->prog->p;
  const int es = p.es;
  E->blobs.assign(E->period, std::vector<std::vector<unsigned char>>(E->G.size()));
  for (int par = 0; par < E->period; par++)
    for (auto& g : E->G) {
      size_t ni = std::max<size_t>(1, g.ins.size()), no = std::max<size_t>(1, g.outs.size()),
             nm = std::max<size_t>(1, g.mids.size()), np = std::max(1, p.n_params);
      size_t sz = 128 * ni + 8 * (no + nm + np) + 8;   // + int mode, pad (zero: every unit)
      sz = (sz + 63) / 64 * 64;
      g.blob_size = sz;
      std::vector<unsigned char> b(sz + 64, 0);
      // keep 64-byte alignment of the tensor maps inside the blob
      unsigned char* base = b.data() + ((64 - (reinterpret_cast<uintptr_t>(b.data()) & 63)) & 63);
      for (size_t i = 0; i < g.ins.size(); i++) {
        const Ring& R = g.L.rings[g.L.ring_of(g.ins[i])];
        void* ptr = buf_ptr(E, buffer_id(E, g.ins[i], par));
        cuuint64_t dims[3] = {cuuint64_t(p.layout.pitch), cuuint64_t(p.layout.rows), cuuint64_t(p.n[2] + 2 * p.ghost[2])};
        cuuint64_t strides[2] = {cuuint64_t(p.layout.pitch * es), cuuint64_t(p.layout.plane * es)};
        cuuint32_t box[3] = {cuuint32_t(R.px), cuuint32_t(R.hy), 1};
        cuuint32_t estr[3] = {1, 1, 1};
        CUtensorMap* tm = reinterpret_cast<CUtensorMap*>(base + 128 * i);
        if (getenv("KF_DEBUG"))
          fprintf(stderr, "tmap g%d in%zu ptr=%p dims=%llu,%llu,%llu strides=%llu,%llu box=%u,%u,%u\n", g.gid, i, ptr,
                  (unsigned long long)dims[0], (unsigned long long)dims[1], (unsigned long long)dims[2],
                  (unsigned long long)strides[0], (unsigned long long)strides[1], box[0], box[1], box[2]);
        ckd(drv().tensorMapEncodeTiled(tm, es == 4 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3,
                                       ptr, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                       CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE),
            "cuTensorMapEncodeTiled");
      }
      unsigned char* q = base + 128 * ni;
      for (size_t j = 0; j < no; j++) {
        void* ptr = j < g.outs.size() ? (char*)buf_ptr(E, buffer_id(E, g.outs[j], par)) + p.layout.origin * es : nullptr;
        std::memcpy(q + 8 * j, &ptr, 8);
      }
      q += 8 * no;
      for (size_t j = 0; j < nm; j++) {
        void* ptr = j < g.mids.size() ? (char*)buf_ptr(E, buffer_id(E, g.mids[j], par)) + p.layout.origin * es : nullptr;
        std::memcpy(q + 8 * j, &ptr, 8);
      }
      q += 8 * nm;
      for (int j = 0; j < p.n_params; j++) std::memcpy(q + 8 * j, &E->cur_params[j], 8);
      std::vector<unsigned char> out(base, base + sz);
      E->blobs[par][&g - &E->G[0]] = std::move(out);
    }
  E->blobs_valid = true;
  E->blob_gen++;
}

// mode 0: every unit; 1: interior tiles only; 2: the other tiles (the group's Split)
static void launch_group(kf_exec* E, int gi, int par, cudaStream_t s, int mode = 0) {
  GroupExec& g = E->G[gi];
  std::vector<unsigned char>& blob = E->blobs[par][gi];
  // The argument block is one __grid_constant__ struct; the driver copies it at launch.
  alignas(64) unsigned char tmp[32768];
  if (blob.size() > sizeof(tmp)) fail(KF_E_RESOURCE, "kernel argument block too large");
  std::memcpy(tmp, blob.data(), blob.size());
  int grid = g.grid;
  if (mode != 0) {
    if (!g.split.ok) fail(KF_E_ARG, "group has no interior/boundary split");
    grid = mode == 1 ? g.split.interior_units : g.split.boundary_units;
    const size_t off = 128 * std::max<size_t>(1, g.ins.size()) +
                       8 * (std::max<size_t>(1, g.outs.size()) + std::max<size_t>(1, g.mids.size()) +
                            std::max(1, E->prog->p.n_params));
    const int32_t m = mode;
    std::memcpy(tmp + off, &m, 4);
    if (grid == 0) return;
  }
  void* params[] = {tmp};
  if (getenv("KF_DEBUG")) {
    fprintf(stderr, "launch %s grid=%d threads=%d smem=%d blob=%zu:", g.cg.name.c_str(), g.grid, g.L.threads, g.smem, blob.size());
    for (size_t i = 0; i < blob.size(); i += 8) fprintf(stderr, " %016llx", *(unsigned long long*)(tmp + i));
    fprintf(stderr, "\n");
  }
  if (g.maxthr > 0 && g.L.threads > g.maxthr)
    fail(KF_E_RESOURCE, g.cg.name + ": " + std::to_string(g.L.threads) + " threads per CTA but the compiled kernel allows " +
                            std::to_string(g.maxthr) + " (" + std::to_string(g.regs) + " registers)");
  ckd(drv().launchKernel(g.fn, grid, 1, 1, g.L.threads, 1, 1, g.smem, (CUstream)s, params, nullptr),
      ("cuLaunchKernel " + g.cg.name).c_str());
}

static void run_fill(kf_exec* E, int buf, cudaStream_t s) {
  const Program& p = E->prog->p;
  Geom gm = geom(p);
  for (int a = 0; a < 3; a++)
    if (p.bc[a] == KF_BC_PERIODIC) CK(launch_fill(a, buf_ptr(E, buf), p.es, gm, s));
}

// Consecutive fills of a schedule in one launch (x and y together; z, if periodic, after them).
static void run_fills(kf_exec* E, const std::vector<int>& bufs, cudaStream_t s, int frozen_only = 0) {
  if (bufs.empty()) return;
  const Program& p = E->prog->p;
  Geom gm = geom(p);
  if (getenv("KF_FILL_SINGLE")) {   // A/B switch: one launch per buffer and axis
    for (int b : bufs) run_fill(E, b, s);
    return;
  }
  std::vector<void*> ptr;
  for (int b : bufs) ptr.push_back(buf_ptr(E, b));
  CK(launch_fill_xy_multi(ptr.data(), int(ptr.size()), p.bc[0] == KF_BC_PERIODIC, p.bc[1] == KF_BC_PERIODIC, p.es, gm, s,
                          frozen_only));
  if (p.bc[2] == KF_BC_PERIODIC)
    for (void* b : ptr) CK(launch_fill(2, b, p.es, gm, s));
}

static void run_step(kf_exec* E, int par, cudaStream_t s) {
  std::vector<int> pend;
  for (const Op& op : E->sched[par]) {
    if (op.kind == 0) {
      pend.push_back(op.buf);
      continue;
    }
    run_fills(E, pend, s);
    pend.clear();
    if (E->profiling) {
      cudaEvent_t a, b;
      if (E->evpool.size() >= 2) {
        a = E->evpool.back(); E->evpool.pop_back();
        b = E->evpool.back(); E->evpool.pop_back();
      } else {
        CK(cudaEventCreate(&a));
        CK(cudaEventCreate(&b));
      }
      CK(cudaEventRecord(a, s));
      launch_group(E, op.group, par, s);
      CK(cudaEventRecord(b, s));
      E->pending.emplace_back(op.group, a, b);
      E->launches++;
    } else {
      launch_group(E, op.group, par, s);
    }
  }
  run_fills(E, pend, s);
}

static void ensure_device(kf_exec* E) {
  int dev = 0;
  CK(cudaGetDevice(&dev));
  if (E->device >= 0 && dev != E->device) fail(KF_E_ARG, "kf_exec used on a different device than it was created on");
  if (E->device >= 0) return;
  CK(cudaFree(nullptr));   // make the primary context current
  E->device = dev;
  const Program& p = E->prog->p;
  for (auto& g : E->G) {
    for (int attempt = 0; attempt < 12; attempt++) {
      ckd(drv().moduleLoadData(&g.mod, g.comp->cubin.data()), ("cuModuleLoadData " + g.cg.name).c_str());
      ckd(drv().moduleGetFunction(&g.fn, g.mod, g.cg.name.c_str()), "cuModuleGetFunction");
      ckd(drv().funcSetAttribute(g.fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, g.smem),
          "cuFuncSetAttribute(MAX_DYNAMIC_SHARED_SIZE_BYTES)");
      drv().funcGetAttribute(&g.regs, CU_FUNC_ATTRIBUTE_NUM_REGS, g.fn);
      drv().funcGetAttribute(&g.local, CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES, g.fn);
      drv().funcGetAttribute(&g.maxthr, CU_FUNC_ATTRIBUTE_MAX_THREADS_PER_BLOCK, g.fn);
      // no spills, no more registers than R_est: else the next build of the cap ladder
      std::shared_ptr<Compiled> nx;
      if ((g.local > 0 || g.regs > source_rest(g.cg.source)) && (nx = compile_after(g.cg.source, g.cg.name, g.comp->cap_idx))) {
        g.comp = nx;
        if (drv().moduleUnload) drv().moduleUnload(g.mod);
        g.mod = nullptr;
        g.fn = nullptr;
      } else {
        break;
      }
    }
  }
  (void)p;
}

static void build_schedule(kf_exec* E) {
  const Program& p = E->prog->p;
  // periodic-fill needs: live-in rings whose box reaches beyond T on a periodic axis
  auto needs_fill = [&](const GroupExec& g, const Ver& v) {
    const Ring& R = g.L.rings[g.L.ring_of(v)];
    for (int a = 0; a < 3; a++)
      if (p.bc[a] == KF_BC_PERIODIC && std::max(R.blo[a], R.bhi[a]) > 0) return true;
    return false;
  };
  std::set<int> all_fill;
  std::vector<std::vector<Op>> sched(E->period);
  std::set<int> dirty;
  for (int pass = 0; pass < 2; pass++)
    for (int par = 0; par < E->period; par++) {
      std::vector<Op> ops;
      for (int gi : E->order) {
        const GroupExec& g = E->G[gi];
        std::set<int> filled;
        for (const Ver& v : g.ins) {
          if (!needs_fill(g, v)) continue;
          int b = buffer_id(E, v, par);
          all_fill.insert(b);
          if (dirty.count(b) && !filled.count(b)) {
            ops.push_back(Op{0, gi, b});
            filled.insert(b);
            dirty.erase(b);
          }
        }
        ops.push_back(Op{1, gi, -1});
        for (const Ver& v : g.outs) dirty.insert(buffer_id(E, v, par));
      }
      if (pass == 1) sched[par] = ops;
    }
  // Buffers whose stored ghosts are read for in-group versions (frozen-boundary rule R9): their
  // ghost cells on PERIODIC axes at frozen-ghost rows/planes are the wrap (or the neighbour's
  // values in a decomposition) of never-written ghost rows, i.e. constant -- fill them once at
  // the start of a run so kernels read them directly.
  bool any_frozen = false, any_periodic = false;
  for (int a = 0; a < 3; a++) (p.bc[a] == KF_BC_PERIODIC ? any_periodic : any_frozen) = true;
  if (any_frozen && any_periodic)
    for (int par = 0; par < E->period; par++)
      for (const GroupExec& g : E->G)
        for (const Ver& v : g.mids) all_fill.insert(buffer_id(E, v, par));
  E->sched_full = sched;
  // when every group writes periodic ghost copies with its live-out stores, buffers are never
  // dirty: drop the in-loop fills (the one-time fills at run start stay)
  bool all_gw = true;
  for (const GroupExec& g : E->G) all_gw = all_gw && g.L.ghost_write;
  if (all_gw)
    for (auto& ops : sched) {
      std::vector<Op> k;
      for (const Op& op : ops)
        if (op.kind != 0) k.push_back(op);
      ops = k;
    }
  E->sched = sched;
  E->fill_all.assign(all_fill.begin(), all_fill.end());
}

static void invalidate_graph(kf_exec* E) {
  if (E->gexec) {
    cudaGraphExecDestroy(E->gexec);
    E->gexec = nullptr;
  }
}

static void prepare_pointers(kf_exec* E, void* const* arrays, void* scratch, const double* params) {
  const Program& p = E->prog->p;
  std::vector<void*> arr(arrays, arrays + p.na);
  std::vector<double> prm(params ? params : nullptr, params ? params + p.n_params : nullptr);
  if (!params) prm.assign(p.n_params, 0.0);
  if (!E->blobs_valid || arr != E->cur_arrays || scratch != E->cur_scratch || prm != E->cur_params) {
    E->cur_arrays = arr;
    E->cur_scratch = scratch;
    E->cur_params = prm;
    build_blobs(E);
    invalidate_graph(E);
  }
}

static void exec_run(kf_exec* E, void* const* arrays, void* scratch, uint64_t scratch_bytes, int64_t nsteps,
                     const double* params, cudaStream_t s) {
  const Program& p = E->prog->p;
  if (!arrays) fail(KF_E_ARG, "arrays is NULL");
  for (int x = 0; x < p.na; x++) {
    if (!arrays[x]) fail(KF_E_ARG, "array pointer " + std::to_string(x) + " is NULL");
    if (reinterpret_cast<uintptr_t>(arrays[x]) & 127) fail(KF_E_ARG, "array base pointers must be 128-byte aligned");
  }
  if (scratch_bytes < E->scratch_bytes || (E->scratch_bytes && !scratch))
    fail(KF_E_RESOURCE, "scratch too small: need " + std::to_string(E->scratch_bytes) + " bytes");
  if (nsteps < 0) fail(KF_E_ARG, "nsteps < 0");
  if (p.n_params > 0 && !params) fail(KF_E_ARG, "params is NULL but the program has PARAM slots");
  ensure_device(E);
  prepare_pointers(E, arrays, scratch, params);
  if (nsteps == 0) return;
  // renamed copies share the array's ghost values (frozen boundaries, R9)
  std::vector<void*> arr(arrays, arrays + p.na);
  if (!E->scratch_vers.empty() && (E->shell_init_scratch != scratch || E->shell_init_arrays != arr)) {
    Geom gm = geom(p);
    for (size_t i = 0; i < E->scratch_vers.size(); i++)
      CK(launch_copy_shell(buf_ptr(E, p.na + int(i)), arrays[E->scratch_vers[i].x], p.es, gm, s));
    E->shell_init_scratch = scratch;
    E->shell_init_arrays = arr;
  }
  // run-start fills: the caller's arrays whole; renamed scratch versions (not written yet: their
  // periodic ghosts are filled / ghost-written after their producer) only where the cell lies in a
  // FROZEN axis' ghost layer (constant cells, R9)
  {
    std::vector<int> arr_b, scr_b;
    for (int b : E->fill_all) (b < p.na ? arr_b : scr_b).push_back(b);
    run_fills(E, arr_b, s);
    const int frozen = (p.bc[0] == KF_BC_FROZEN ? 1 : 0) | (p.bc[1] == KF_BC_FROZEN ? 2 : 0) | (p.bc[2] == KF_BC_FROZEN ? 4 : 0);
    if (frozen && p.bc[2] != KF_BC_PERIODIC) run_fills(E, scr_b, s, frozen);
    else run_fills(E, scr_b, s);
  }
  int64_t reps = nsteps / E->period, rem = nsteps % E->period;
  if (E->use_graph && !E->profiling && reps > 0) {
    if (!E->gexec) {
      if (!E->cap_stream) CK(cudaStreamCreateWithFlags(&E->cap_stream, cudaStreamNonBlocking));
      cudaGraph_t graph;
      CK(cudaStreamBeginCapture(E->cap_stream, cudaStreamCaptureModeThreadLocal));
      try {
        for (int par = 0; par < E->period; par++) run_step(E, par, E->cap_stream);
      } catch (...) {
        cudaStreamEndCapture(E->cap_stream, &graph);
        throw;
      }
      CK(cudaStreamEndCapture(E->cap_stream, &graph));
      CK(cudaGraphInstantiate(&E->gexec, graph, 0));
      cudaGraphDestroy(graph);
    }
    for (int64_t r = 0; r < reps; r++) CK(cudaGraphLaunch(E->gexec, s));
  } else {
    for (int64_t r = 0; r < reps; r++)
      for (int par = 0; par < E->period; par++) run_step(E, par, s);
  }
  for (int64_t r = 0; r < rem; r++) run_step(E, int(r), s);
  // after an odd number of steps the renamed final versions sit in scratch: copy back
  if (E->period == 2 && (nsteps % 2) == 1) {
    for (int x = 0; x < p.na; x++)
      if (p.relaxed[x] && p.step_live[x]) {
        int b = buffer_id(E, Ver{x, int(p.writers[x].size())}, 0);
        CK(cudaMemcpyAsync(arrays[x], buf_ptr(E, b), E->array_bytes, cudaMemcpyDeviceToDevice, s));
      }
  }
  CK(cudaGetLastError());
}

}  // namespace kf

extern "C" {

kf_status kf_exec_create_ex(kf_program* prog, const int32_t* plan, const kf_target* targets, int32_t n_targets,
                            kf_exec** out) {
  KF_TRY({
    if (!prog || !plan || !out || !targets || n_targets < 1) fail(KF_E_ARG, "null argument");
    const Program& p = prog->p;
    for (int k = 0; k < p.nk; k++)
      if (plan[k] < 0) fail(KF_E_ILLEGAL_PLAN, "V1 PARTITION: kernel " + std::to_string(k) + " has no group");
    auto E = std::make_unique<kf_exec>();
    E->prog = prog;
    E->plan = make_plan(p, plan);
    if (n_targets != 1 && n_targets != E->plan.m)
      fail(KF_E_ARG, "n_targets must be 1 or the number of groups (" + std::to_string(E->plan.m) + ")");
    std::vector<kf_target> T;
    for (int gi = 0; gi < E->plan.m; gi++) {
      const kf_target& t = targets[n_targets == 1 ? 0 : gi];
      check_target(&t);
      T.push_back(t);
    }
    E->t = T[0];
    kf_violation why{};
    std::vector<GroupLowering> Ls;
    int code = validate_plan_groups(p, E->plan, T, &why, &Ls);
    if (code != KF_V_OK)
      fail(KF_E_ILLEGAL_PLAN, "plan violates constraint V" + std::to_string(code) + " in group " + std::to_string(why.group));
    E->order = quotient_order(p, E->plan);
    // renamed versions -> scratch buffers ("redundant arrays")
    E->scratch_vers = renamed_versions(p, &E->period);
    E->array_bytes = padded_array_bytes(p);
    E->scratch_bytes = E->array_bytes * E->scratch_vers.size();
    E->G.resize(E->plan.m);
    for (int gi = 0; gi < E->plan.m; gi++) {
      GroupExec& g = E->G[gi];
      const kf_target& t = T[gi];
      const int TZ = t.tile[2] > 0 ? std::min<int64_t>(t.tile[2], p.n[2]) : int(p.n[2]);
      int64_t units = ((p.n[0] + t.tile[0] - 1) / t.tile[0]) * ((p.n[1] + t.tile[1] - 1) / t.tile[1]) *
                      ((p.n[2] + TZ - 1) / TZ);
      if (units > 2147483647) fail(KF_E_UNSUPPORTED, "grid too large");
      g.gid = gi;
      g.L = std::move(Ls[gi]);
      g.cg = generate_group_kernel(p, g.L, gi);
      g.grid = int(units);
      g.split = split_units(p, g.L);
      g.smem = g.L.smem;
      uint64_t rd, wr;
      g.bytes = group_bytes(p, E->plan.groups[gi], &rd, &wr);
      for (auto& r : g.L.rings) (r.live_in ? g.ins : g.mids).push_back(r.ver);
      g.outs = g.L.live_out;
      E->step_bytes += g.bytes;
    }
    // JIT all groups (NVRTC, sm_100a) on parallel host threads; identical sources are compiled once
    // per process (the cache), each nvrtcProgram is private to its thread
    {
      const int nthr = std::max(1, std::min<int>(int(E->G.size()), int(std::thread::hardware_concurrency())));
      std::atomic<int> next{0};
      std::vector<std::string> errs(E->G.size());
      std::vector<kf_status> sts(E->G.size(), KF_OK);
      auto work = [&]() {
        for (int i = next++; i < int(E->G.size()); i = next++) {
          try {
            E->G[i].comp = compile_cached(E->G[i].cg.source, E->G[i].cg.name);
          } catch (const Error& e) {
            sts[i] = e.st;
            errs[i] = e.msg;
          } catch (const std::exception& e) {
            sts[i] = KF_E_NVRTC;
            errs[i] = e.what();
          }
        }
      };
      std::vector<std::thread> th;
      for (int t = 1; t < nthr; t++) th.emplace_back(work);
      work();
      for (auto& t : th) t.join();
      for (size_t i = 0; i < sts.size(); i++)
        if (sts[i] != KF_OK) fail(sts[i], errs[i]);
    }
    build_schedule(E.get());
    *out = E.release();
  });
}

kf_status kf_exec_create(kf_program* prog, const int32_t* plan, const kf_target* target, kf_exec** out) {
  return kf_exec_create_ex(prog, plan, target, 1, out);
}

void kf_exec_destroy(kf_exec* ex) {
  if (!ex) return;
  try {
    invalidate_graph(ex);
    if (ex->cap_stream) cudaStreamDestroy(ex->cap_stream);
    for (auto& t : ex->pending) {
      cudaEventDestroy(std::get<1>(t));
      cudaEventDestroy(std::get<2>(t));
    }
    for (auto e : ex->evpool) cudaEventDestroy(e);
    for (void* d : ex->dev_arrays) cudaFree(d);
    if (ex->dev_scratch) cudaFree(ex->dev_scratch);
    for (auto& g : ex->G)
      if (g.mod && drv().moduleUnload) drv().moduleUnload(g.mod);
  } catch (...) {
  }
  delete ex;
}

kf_status kf_exec_scratch_bytes(const kf_exec* ex, uint64_t* bytes) {
  KF_TRY({
    if (!ex || !bytes) fail(KF_E_ARG, "null argument");
    *bytes = ex->scratch_bytes;
  });
}

kf_status kf_exec_run(kf_exec* ex, void* const* arrays, void* scratch, uint64_t scratch_bytes, int64_t nsteps,
                      const double* params, void* cuda_stream) {
  KF_TRY({
    if (!ex) fail(KF_E_ARG, "null exec");
    exec_run(ex, arrays, scratch, scratch_bytes, nsteps, params, (cudaStream_t)cuda_stream);
  });
}

kf_status kf_run_host(kf_exec* ex, void* const* host_arrays, int64_t nsteps, const double* params, void* cuda_stream,
                      uint64_t* h2d_bytes, uint64_t* d2h_bytes) {
  KF_TRY({
    if (!ex || !host_arrays) fail(KF_E_ARG, "null argument");
    const Program& p = ex->prog->p;
    cudaStream_t s = (cudaStream_t)cuda_stream;
    CK(cudaFree(nullptr));
    if (ex->dev_arrays.empty()) {
      for (int x = 0; x < p.na; x++) {
        void* d = nullptr;
        if (cudaMalloc(&d, ex->array_bytes) != cudaSuccess) fail(KF_E_OOM, "cudaMalloc failed in kf_run_host");
        ex->dev_arrays.push_back(d);
      }
      if (ex->scratch_bytes && cudaMalloc(&ex->dev_scratch, ex->scratch_bytes) != cudaSuccess)
        fail(KF_E_OOM, "cudaMalloc (scratch) failed in kf_run_host");
      ex->host_first = true;
    }
    uint64_t h2d = 0, d2h = 0;
    for (int x = 0; x < p.na; x++) {
      // inputs of a step: arrays read before being written (upward-exposed) and read-only arrays;
      // the first call also uploads every array (ghost values of temporaries)
      bool input = !p.readers_of_version(x, 0).empty();
      if (input || ex->host_first) {
        CK(cudaMemcpyAsync(ex->dev_arrays[x], host_arrays[x], uint64_t(p.layout.elems) * p.es, cudaMemcpyHostToDevice, s));
        h2d += uint64_t(p.layout.elems) * p.es;
      }
    }
    ex->host_first = false;
    // the uploaded arrays carry their (FROZEN) ghost values: renamed copies must take them again
    ex->shell_init_scratch = nullptr;
    ex->shell_init_arrays.clear();
    exec_run(ex, ex->dev_arrays.data(), ex->dev_scratch, ex->scratch_bytes, nsteps, params, s);
    for (int x = 0; x < p.na; x++)
      if (p.step_live[x]) {
        CK(cudaMemcpyAsync(host_arrays[x], ex->dev_arrays[x], uint64_t(p.layout.elems) * p.es, cudaMemcpyDeviceToHost, s));
        d2h += uint64_t(p.layout.elems) * p.es;
      }
    CK(cudaStreamSynchronize(s));
    if (h2d_bytes) *h2d_bytes = h2d;
    if (d2h_bytes) *d2h_bytes = d2h;
  });
}

kf_status kf_exec_get_info(const kf_exec* ex, kf_exec_info* out) {
  KF_TRY({
    if (!ex || !out) fail(KF_E_ARG, "null argument");
    kf_exec_info r{};
    r.n_groups = int(ex->G.size());
    int fills = 0, launches = 0;
    const Program& p = ex->prog->p;
    int naxes = 0;
    for (int a = 0; a < 3; a++) naxes += p.bc[a] == KF_BC_PERIODIC;
    // fill launches: one per run of consecutive fills (x and y batched, kMaxFillBufs buffers per
    // launch) plus one per buffer for a periodic z axis; KF_FILL_SINGLE: one per buffer and axis
    const bool single = getenv("KF_FILL_SINGLE") != nullptr;
    const int nxy = (p.bc[0] == KF_BC_PERIODIC) + (p.bc[1] == KF_BC_PERIODIC);
    for (auto& sc : ex->sched) {
      int run = 0;
      auto flush = [&]() {
        if (run == 0) return;
        fills += single ? run * naxes : (nxy ? (run + kMaxFillBufs - 1) / kMaxFillBufs : 0) +
                                            (p.bc[2] == KF_BC_PERIODIC ? run : 0);
        run = 0;
      };
      for (auto& op : sc) {
        if (op.kind == 0) { run++; continue; }
        flush();
        launches += 1;
      }
      flush();
    }
    r.fills_per_step = fills / ex->period;
    r.launches_per_step = launches / ex->period + r.fills_per_step;
    r.period = ex->period;
    r.compulsory_bytes_per_step = ex->step_bytes;
    *out = r;
  });
}

kf_status kf_exec_group_info(const kf_exec* ex, int32_t group, kf_group_info* out) {
  KF_TRY({
    if (!ex || !out) fail(KF_E_ARG, "null argument");
    if (group < 0 || group >= int(ex->G.size())) fail(KF_E_ARG, "group out of range");
    const GroupExec& g = ex->G[group];
    kf_group_info r{};
    r.group = group;
    r.grid = g.grid;
    r.threads = g.L.threads;
    r.smem_bytes = g.smem;
    r.regs = g.regs >= 0 ? g.regs : g.comp->regs_ptxas;
    r.local_bytes = g.local >= 0 ? g.local : g.comp->spill;
    r.n_kernels = int(g.L.kernels.size());
    r.max_threads = g.maxthr;
    r.bytes_per_launch = g.bytes;
    {
      const Program& p = ex->prog->p;
      const CanvasPlan cv = plan_canvas(p, g.L);
      const double per_plane = (cv.lds_bytes + cv.sts_bytes + cv.tma_bytes) / std::max(1, g.L.zunroll);
      r.onchip_bytes_per_launch = uint64_t(double(p.npts) / (double(g.L.tile[0]) * g.L.tile[1]) * per_plane);
    }
    std::strncpy(r.name, g.cg.name.c_str(), sizeof(r.name) - 1);
    *out = r;
  });
}

kf_status kf_exec_group_source(const kf_exec* ex, int32_t group, char* buf, int64_t cap, int64_t* len) {
  KF_TRY({
    if (!ex || !len) fail(KF_E_ARG, "null argument");
    if (group < 0 || group >= int(ex->G.size())) fail(KF_E_ARG, "group out of range");
    const std::string& s = ex->G[group].cg.source;
    *len = int64_t(s.size());
    if (buf && cap > 0) {
      int64_t n = std::min<int64_t>(cap - 1, int64_t(s.size()));
      std::memcpy(buf, s.data(), size_t(n));
      buf[n] = 0;
    }
  });
}

kf_status kf_exec_set_profiling(kf_exec* ex, int32_t on) {
  KF_TRY({
    if (!ex) fail(KF_E_ARG, "null exec");
    for (auto& t : ex->pending) {   // drop unread measurements (e.g. of a warm-up)
      cudaEventSynchronize(std::get<2>(t));
      ex->evpool.push_back(std::get<1>(t));
      ex->evpool.push_back(std::get<2>(t));
    }
    ex->pending.clear();
    ex->profiling = on != 0;
    ex->gms.assign(ex->G.size(), 0.0);
    ex->launches = 0;
  });
}

kf_status kf_exec_group_times(kf_exec* ex, double* ms, int32_t cap, int32_t* n, int64_t* launches) {
  KF_TRY({
    if (!ex || !n) fail(KF_E_ARG, "null argument");
    if (ex->gms.size() != ex->G.size()) ex->gms.assign(ex->G.size(), 0.0);
    for (auto& t : ex->pending) {
      float f = 0.f;
      CK(cudaEventSynchronize(std::get<2>(t)));
      CK(cudaEventElapsedTime(&f, std::get<1>(t), std::get<2>(t)));
      ex->gms[std::get<0>(t)] += f;
      ex->evpool.push_back(std::get<1>(t));
      ex->evpool.push_back(std::get<2>(t));
    }
    ex->pending.clear();
    for (int i = 0; i < int(ex->gms.size()) && i < cap && ms; i++) ms[i] = ex->gms[i];
    *n = int(ex->gms.size());
    if (launches) *launches = ex->launches;
  });
}

kf_status kf_exec_load(kf_exec* ex) {
  KF_TRY({
    if (!ex) fail(KF_E_ARG, "null exec");
    ensure_device(ex);
  });
}

kf_status kf_exec_invalidate(kf_exec* ex) {
  KF_TRY({
    if (!ex) fail(KF_E_ARG, "null exec");
    ex->shell_init_scratch = nullptr;
    ex->shell_init_arrays.clear();
  });
}

kf_status kf_exec_set_graph(kf_exec* ex, int32_t on) {
  KF_TRY({
    if (!ex) fail(KF_E_ARG, "null exec");
    ex->use_graph = on != 0;
  });
}

kf_status kf_flush_l2(void* buf, uint64_t bytes, void* cuda_stream) {
  KF_TRY({
    static unsigned v = 1;
    CK(launch_flush(buf, (long long)bytes, v++, (cudaStream_t)cuda_stream));
  });
}

kf_status kf_jit_check(const kf_program* prog, const int32_t* plan, const kf_target* target, int32_t group,
                       int32_t* regs, int32_t* spill_bytes, char* log, int64_t cap) {
  KF_TRY({
    if (!prog || !plan || !target) fail(KF_E_ARG, "null argument");
    check_target(target);
    const Program& p = prog->p;
    Plan pl = make_plan(p, plan);
    if (group < 0 || group >= pl.m) fail(KF_E_ARG, "group out of range");
    GroupLowering L = lower_group(p, pl.groups[group], *target);
    if (getenv("KF_DEBUG")) fprintf(stderr, "jit_check: lowered\n");
    Codegen cg = generate_group_kernel(p, L, group);
    if (getenv("KF_DEBUG")) fprintf(stderr, "jit_check: generated %zu bytes\n", cg.source.size());
    auto c = compile_cached(cg.source, cg.name);
    if (regs) *regs = c->regs_ptxas;
    if (spill_bytes) *spill_bytes = c->spill;
    if (log && cap > 0) {
      int64_t n = std::min<int64_t>(cap - 1, int64_t(c->log.size()));
      std::memcpy(log, c->log.data(), size_t(n));
      log[n] = 0;
    }
  });
}

}  // extern "C"

// ============================================================================ a11: multi-GPU
// Domain decomposition over a px x py process grid (x, y split; z whole; rank = iy*px + ix).
// Each part runs the same plan on its local sub-domain; the periodic ghost fills of the
// single-domain schedule become halo exchanges with the neighbouring parts (x strips first,
// then y strips including the x ghosts, which covers corners).  Every exchange point handles all
// its pending buffers at once: one pack launch, one ncclGroupStart/End of all sends and receives,
// one unpack launch per phase.  Transports: loopback (all parts in one process/GPU,
// strips copied device-to-device in one launch per phase; tests the decomposition bit-exactly on
// one GPU) and NCCL send/recv (one process per GPU, NVLink/NVSwitch).  A replay period of steps
// is captured in a CUDA graph (exchanges, overlap fork/join and NCCL calls included).
#include <dlfcn.h>

namespace kf {

struct Nccl {
  void* h = nullptr;
  int (*getUniqueId)(void*) = nullptr;                          // ncclUniqueId* (128 bytes)
  int (*commInitRank)(void**, int, const void*, int) = nullptr; // comm*, nranks, ncclUniqueId (by value: 128 B)
  int (*send)(const void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  int (*recv)(void*, size_t, int, int, void*, cudaStream_t) = nullptr;
  int (*groupStart)() = nullptr;
  int (*groupEnd)() = nullptr;
  int (*commDestroy)(void*) = nullptr;
  const char* (*errStr)(int) = nullptr;
};

// ncclCommInitRank takes ncclUniqueId by value (struct of 128 chars): declare it that way.
struct NcclId { char internal[128]; };

static Nccl& nccl() {
  static Nccl n;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);   // prefer the copy already in the process
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    n.h = h;
    n.getUniqueId = (int (*)(void*))dlsym(h, "ncclGetUniqueId");
    n.commInitRank = (int (*)(void**, int, const void*, int))dlsym(h, "ncclCommInitRank");
    n.send = (int (*)(const void*, size_t, int, int, void*, cudaStream_t))dlsym(h, "ncclSend");
    n.recv = (int (*)(void*, size_t, int, int, void*, cudaStream_t))dlsym(h, "ncclRecv");
    n.groupStart = (int (*)())dlsym(h, "ncclGroupStart");
    n.groupEnd = (int (*)())dlsym(h, "ncclGroupEnd");
    n.commDestroy = (int (*)(void*))dlsym(h, "ncclCommDestroy");
    n.errStr = (const char* (*)(int))dlsym(h, "ncclGetErrorString");
  });
  if (!n.h || !n.getUniqueId || !n.commInitRank || !n.send || !n.recv || !n.groupStart || !n.groupEnd)
    fail(KF_E_UNSUPPORTED, "NCCL (libnccl.so.2) not available");
  return n;
}

static void ckn(int r, const char* what) {
  if (r == 0) return;
  fail(KF_E_NCCL, std::string(what) + ": " + (nccl().errStr ? nccl().errStr(r) : std::to_string(r)));
}

// One NCCL communicator, shared by the kf_dist objects of one kf_dist_init context.
struct Comm {
  void* comm = nullptr;
  ~Comm() {
    if (comm && nccl().commDestroy) nccl().commDestroy(comm);
  }
};

static std::shared_ptr<Comm> make_comm(int rank, int world, const uint8_t* id) {
  NcclId u;
  std::memcpy(&u, id, 128);
  CK(cudaFree(nullptr));
  auto c = std::make_shared<Comm>();
  // ncclCommInitRank(ncclComm_t*, int nranks, ncclUniqueId commId, int rank): id passed by value
  auto init = (int (*)(void**, int, NcclId, int))nccl().commInitRank;
  ckn(init(&c->comm, world, u, rank), "ncclCommInitRank");
  return c;
}

}  // namespace kf

struct kf_dist {
  std::vector<kf_exec*> parts;   // loopback: px*py parts; NCCL: 1 part
  int px = 1, py = 1, rank = 0, world = 1;
  bool use_nccl = false;
  std::shared_ptr<kf::Comm> comm;
  void* stage = nullptr;         // NCCL staging (device): 4 strip slots per buffer of a batch
  uint64_t slot_bytes = 0;       // bytes of one strip slot (the larger face)
  int max_batch = 1;             // buffers per exchange batch the staging holds
  // overlap (a11): exchanges on a second stream while the group's interior tiles run
  int overlap = 1;
  cudaStream_t xs = nullptr;
  cudaEvent_t ev_ready = nullptr, ev_done = nullptr;
  // CUDA graph of one replay period
  bool use_graph = true, graph_failed = false;
  cudaStream_t cap = nullptr;
  cudaGraphExec_t gexec = nullptr;
  std::vector<uint64_t> gens;    // parts' blob generations the graph was captured with
  int gexec_overlap = -1;
};

namespace kf {

static void dist_neighbors(int px, int py, int rank, int out[4]) {
  const int ix = rank % px, iy = rank / px;
  out[0] = iy * px + (ix + px - 1) % px;   // left  (x-)
  out[1] = iy * px + (ix + 1) % px;        // right (x+)
  out[2] = ((iy + py - 1) % py) * px + ix; // down  (y-)
  out[3] = ((iy + 1) % py) * px + ix;      // up    (y+)
}

// Strip boxes of one buffer, in elements relative to the allocation base.
struct Box { long long off; int w, h, d; };

static void strip_boxes(const Program& p, int axis, Box* send_lo, Box* send_hi, Box* recv_lo, Box* recv_hi) {
  const kf_layout& L = p.layout;
  const int nx = int(p.n[0]), ny = int(p.n[1]), g0 = p.ghost[0], g1 = p.ghost[1];
  const int d = int(p.n[2]) + 2 * p.ghost[2];
  if (axis == 0) {
    const int h = ny + 2 * g1;                    // every row, y ghosts included
    *send_lo = Box{L.xoff, g0, h, d};
    *send_hi = Box{L.xoff + nx - g0, g0, h, d};
    *recv_lo = Box{L.xoff - g0, g0, h, d};
    *recv_hi = Box{L.xoff + nx, g0, h, d};
  } else {
    const int w = int(L.pitch);                   // whole padded rows: x ghosts (and corners) included
    *send_lo = Box{(long long)g1 * L.pitch, w, g1, d};
    *send_hi = Box{(long long)ny * L.pitch, w, g1, d};
    *recv_lo = Box{0, w, g1, d};
    *recv_hi = Box{(long long)(g1 + ny) * L.pitch, w, g1, d};
  }
}

static uint64_t box_bytes(const Box& b, int es) { return uint64_t(b.w) * b.h * b.d * es; }

// Halo exchange of the buffers `bufs` on every part: decomposed axes exchange with the
// neighbours, other periodic axes wrap locally.  Batches larger than the staging are split.
static void dist_exchange(kf_dist* D, const std::vector<int>& all, cudaStream_t s) {
  if (all.empty()) return;
  for (size_t c0 = 0; c0 < all.size(); c0 += size_t(D->max_batch)) {
    const std::vector<int> bufs(all.begin() + c0, all.begin() + std::min(all.size(), c0 + size_t(D->max_batch)));
    const Program& p = D->parts[0]->prog->p;
    const Geom gm = geom(p);
    const int es = p.es;
    const kf_layout& L = p.layout;
    for (int axis = 0; axis < 3; axis++) {
      if (p.bc[axis] != KF_BC_PERIODIC) continue;
      const int np = axis == 0 ? D->px : (axis == 1 ? D->py : 1);
      if (np == 1) {
        if (axis < 2) {
          std::vector<void*> ptr;
          for (kf_exec* E : D->parts)
            for (int b : bufs) ptr.push_back(buf_ptr(E, b));
          CK(launch_fill_xy_multi(ptr.data(), int(ptr.size()), axis == 0, axis == 1, es, gm, s));
        } else {
          for (kf_exec* E : D->parts)
            for (int b : bufs) CK(launch_fill(2, buf_ptr(E, b), es, gm, s));
        }
        continue;
      }
      Box slo, shi, rlo, rhi;
      strip_boxes(p, axis, &slo, &shi, &rlo, &rhi);
      auto at = [&](void* base, const Box& b) { return (void*)((char*)base + b.off * es); };
      std::vector<BoxCopy> boxes;
      if (!D->use_nccl) {
        // my low ghost <- low neighbour's high interior strip; my high ghost <- high neighbour's low strip
        for (int r = 0; r < int(D->parts.size()); r++) {
          int nb[4];
          dist_neighbors(D->px, D->py, r, nb);
          const int lo = axis == 0 ? nb[0] : nb[2], hi = axis == 0 ? nb[1] : nb[3];
          for (int b : bufs) {
            boxes.push_back(BoxCopy{at(buf_ptr(D->parts[r], b), rlo), at(buf_ptr(D->parts[lo], b), shi), L.pitch, L.plane,
                                    L.pitch, L.plane, shi.w, shi.h, shi.d, 0});
            boxes.push_back(BoxCopy{at(buf_ptr(D->parts[r], b), rhi), at(buf_ptr(D->parts[hi], b), slo), L.pitch, L.plane,
                                    L.pitch, L.plane, slo.w, slo.h, slo.d, 0});
          }
        }
        CK(launch_copy_boxes(boxes.data(), int(boxes.size()), es, s));
        continue;
      }
      kf_exec* E = D->parts[0];
      int nb[4];
      dist_neighbors(D->px, D->py, D->rank, nb);
      const int lo = axis == 0 ? nb[0] : nb[2], hi = axis == 0 ? nb[1] : nb[3];
      const uint64_t strip = box_bytes(slo, es);
      if (strip > D->slot_bytes) fail(KF_E_RESOURCE, "internal: halo strip larger than the staging slot");
      auto slot = [&](size_t i, int j) { return (char*)D->stage + (4 * i + j) * D->slot_bytes; };   // 0 s_lo 1 s_hi 2 r_lo 3 r_hi
      // pack the send strips of every buffer (one launch)
      for (size_t i = 0; i < bufs.size(); i++) {
        void* base = buf_ptr(E, bufs[i]);
        boxes.push_back(BoxCopy{slot(i, 0), at(base, slo), slo.w, (long long)slo.w * slo.h, L.pitch, L.plane, slo.w, slo.h, slo.d, 0});
        boxes.push_back(BoxCopy{slot(i, 1), at(base, shi), shi.w, (long long)shi.w * shi.h, L.pitch, L.plane, shi.w, shi.h, shi.d, 0});
      }
      CK(launch_copy_boxes(boxes.data(), int(boxes.size()), es, s));
      // one group of every send and receive of the phase.  Per peer, the order of matching
      // operations is the buffer order on both sides: my low strip goes to the low neighbour's
      // high ghost, which it receives (r_hi) in the same buffer order (also when lo == hi).
      Nccl& n = nccl();
      ckn(n.groupStart(), "ncclGroupStart");
      for (size_t i = 0; i < bufs.size(); i++) {
        ckn(n.send(slot(i, 0), strip, 1 /*ncclUint8*/, lo, D->comm->comm, s), "ncclSend");
        ckn(n.send(slot(i, 1), strip, 1, hi, D->comm->comm, s), "ncclSend");
        ckn(n.recv(slot(i, 3), strip, 1, hi, D->comm->comm, s), "ncclRecv");
        ckn(n.recv(slot(i, 2), strip, 1, lo, D->comm->comm, s), "ncclRecv");
      }
      ckn(n.groupEnd(), "ncclGroupEnd");
      boxes.clear();
      for (size_t i = 0; i < bufs.size(); i++) {
        void* base = buf_ptr(E, bufs[i]);
        boxes.push_back(BoxCopy{at(base, rlo), slot(i, 2), L.pitch, L.plane, rlo.w, (long long)rlo.w * rlo.h, rlo.w, rlo.h, rlo.d, 0});
        boxes.push_back(BoxCopy{at(base, rhi), slot(i, 3), L.pitch, L.plane, rhi.w, (long long)rhi.w * rhi.h, rhi.w, rhi.h, rhi.d, 0});
      }
      CK(launch_copy_boxes(boxes.data(), int(boxes.size()), es, s));
    }
  }
}

static void profiled_launch(kf_exec* E, int gi, int par, cudaStream_t s) {
  if (!E->profiling) {
    launch_group(E, gi, par, s);
    return;
  }
  cudaEvent_t a, b;
  if (E->evpool.size() >= 2) {
    a = E->evpool.back(); E->evpool.pop_back();
    b = E->evpool.back(); E->evpool.pop_back();
  } else {
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
  }
  CK(cudaEventRecord(a, s));
  launch_group(E, gi, par, s);
  CK(cudaEventRecord(b, s));
  E->pending.emplace_back(gi, a, b);
  E->launches++;
}

// One step (schedule parity `par`) of every part: exchanges before the groups that need them.
static void dist_step(kf_dist* D, int par, cudaStream_t s) {
  kf_exec* E0 = D->parts[0];
  const Program& p = E0->prog->p;
  std::vector<int> pend;   // exchanges due before the next group
  for (const Op& op : E0->sched_full[par]) {
    if (op.kind == 0) {
      pend.push_back(op.buf);
      continue;
    }
    // Overlap: the exchanges run on a second stream, ordered after everything issued
    // so far, while the group's interior tiles -- at least one ghost width inside the local domain
    // in x and y, so they read no x/y ghost and write no strip an exchange packs -- run on the
    // compute stream; the remaining tiles wait for the exchanges.  Not with a periodic z axis: its
    // wrap rewrites the z ghost planes, which interior tiles read.
    const bool split = D->overlap && !pend.empty() && E0->G[op.group].split.ok && !E0->profiling &&
                       p.bc[2] != KF_BC_PERIODIC;
    if (split) {
      CK(cudaEventRecord(D->ev_ready, s));
      CK(cudaStreamWaitEvent(D->xs, D->ev_ready, 0));
      dist_exchange(D, pend, D->xs);
      CK(cudaEventRecord(D->ev_done, D->xs));
      for (kf_exec* E : D->parts) launch_group(E, op.group, par, s, 1);
      CK(cudaStreamWaitEvent(s, D->ev_done, 0));
      for (kf_exec* E : D->parts) launch_group(E, op.group, par, s, 2);
      pend.clear();
      continue;
    }
    dist_exchange(D, pend, s);
    pend.clear();
    for (kf_exec* E : D->parts) profiled_launch(E, op.group, par, s);
  }
  dist_exchange(D, pend, s);
}

static void dist_invalidate_graph(kf_dist* D) {
  if (D->gexec) {
    cudaGraphExecDestroy(D->gexec);
    D->gexec = nullptr;
  }
}

static void dist_run(kf_dist* D, void* const* arrays, void* const* scratch, uint64_t scratch_bytes, int64_t nsteps,
                     const double* params, cudaStream_t s) {
  const Program& p = D->parts[0]->prog->p;
  const int np = int(D->parts.size());
  if (!arrays) fail(KF_E_ARG, "arrays is NULL");
  if (p.n_params > 0 && !params) fail(KF_E_ARG, "params is NULL but the program has PARAM slots");
  for (int r = 0; r < np; r++) {
    kf_exec* E = D->parts[r];
    void* const* arr = arrays + size_t(r) * p.na;
    for (int x = 0; x < p.na; x++)
      if (!arr[x] || (reinterpret_cast<uintptr_t>(arr[x]) & 127)) fail(KF_E_ARG, "array pointers must be 128-byte aligned");
    void* scr = scratch ? scratch[r] : nullptr;
    if (scratch_bytes < E->scratch_bytes || (E->scratch_bytes && !scr))
      fail(KF_E_RESOURCE, "scratch too small: need " + std::to_string(E->scratch_bytes) + " bytes per part");
    ensure_device(E);
    prepare_pointers(E, arr, scr, params);
    std::vector<void*> av(arr, arr + p.na);
    if (!E->scratch_vers.empty() && (E->shell_init_scratch != scr || E->shell_init_arrays != av)) {
      Geom gm = geom(p);
      for (size_t i = 0; i < E->scratch_vers.size(); i++)
        CK(launch_copy_shell(buf_ptr(E, p.na + int(i)), arr[E->scratch_vers[i].x], p.es, gm, s));
      E->shell_init_scratch = scr;
      E->shell_init_arrays = av;
    }
  }
  kf_exec* E0 = D->parts[0];
  dist_exchange(D, E0->fill_all, s);
  if (!D->xs) {
    CK(cudaStreamCreateWithFlags(&D->xs, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&D->ev_ready, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&D->ev_done, cudaEventDisableTiming));
  }
  bool profiling = false;
  std::vector<uint64_t> gens;
  for (kf_exec* E : D->parts) {
    profiling = profiling || E->profiling;
    gens.push_back(E->blob_gen);
  }
  const int64_t reps = nsteps / E0->period, rem = nsteps % E0->period;
  bool done = false;
  if (D->use_graph && !D->graph_failed && !profiling && reps > 0) {
    if (D->gexec && (gens != D->gens || D->gexec_overlap != D->overlap)) dist_invalidate_graph(D);
    if (!D->gexec) {
      if (!D->cap) CK(cudaStreamCreateWithFlags(&D->cap, cudaStreamNonBlocking));
      cudaGraph_t graph = nullptr;
      CK(cudaStreamBeginCapture(D->cap, cudaStreamCaptureModeThreadLocal));
      try {
        for (int par = 0; par < E0->period; par++) dist_step(D, par, D->cap);
      } catch (...) {
        cudaStreamEndCapture(D->cap, &graph);
        if (graph) cudaGraphDestroy(graph);
        cudaGetLastError();
        throw;
      }
      cudaError_t e = cudaStreamEndCapture(D->cap, &graph);
      if (e == cudaSuccess && graph) e = cudaGraphInstantiate(&D->gexec, graph, 0);
      if (graph) cudaGraphDestroy(graph);
      if (e != cudaSuccess) {   // e.g. a transport that cannot be captured: run eagerly from now on
        cudaGetLastError();
        D->gexec = nullptr;
        D->graph_failed = true;
      } else {
        D->gens = gens;
        D->gexec_overlap = D->overlap;
      }
    }
    if (D->gexec) {
      // the graph's first node must follow the stream's earlier work (ghost exchanges above)
      for (int64_t r = 0; r < reps; r++) CK(cudaGraphLaunch(D->gexec, s));
      done = true;
    }
  }
  if (!done)
    for (int64_t r = 0; r < reps; r++)
      for (int par = 0; par < E0->period; par++) dist_step(D, par, s);
  for (int64_t r = 0; r < rem; r++) dist_step(D, int(r), s);
  if (E0->period == 2 && (nsteps % 2) == 1)
    for (kf_exec* E : D->parts)
      for (int x = 0; x < p.na; x++)
        if (p.relaxed[x] && p.step_live[x]) {
          int b = buffer_id(E, Ver{x, int(p.writers[x].size())}, 0);
          CK(cudaMemcpyAsync(E->cur_arrays[x], buf_ptr(E, b), E->array_bytes, cudaMemcpyDeviceToDevice, s));
        }
  CK(cudaGetLastError());
}

// Builds a kf_dist over parts (loopback when comm is null and n_parts == px*py; NCCL otherwise).
static kf_dist* dist_make(kf_exec* const* parts, int n_parts, int px, int py, int rank, int world,
                          std::shared_ptr<Comm> comm) {
  if (!parts || n_parts < 1 || px < 1 || py < 1) fail(KF_E_ARG, "bad arguments");
  auto D = std::make_unique<kf_dist>();
  D->px = px;
  D->py = py;
  D->rank = rank;
  D->world = world;
  for (int i = 0; i < n_parts; i++) {
    if (!parts[i]) fail(KF_E_ARG, "null part");
    D->parts.push_back(parts[i]);
  }
  const Program& p = parts[0]->prog->p;
  for (int i = 1; i < n_parts; i++)
    if (parts[i]->prog != parts[0]->prog || parts[i]->plan.label != parts[0]->plan.label)
      fail(KF_E_ARG, "all parts must run the same program and plan");
  if ((px > 1 && p.bc[0] != KF_BC_PERIODIC) || (py > 1 && p.bc[1] != KF_BC_PERIODIC))
    fail(KF_E_UNSUPPORTED, "decomposed axes must be PERIODIC in the local program (halo exchange replaces the wrap)");
  if ((px > 1 && p.n[0] < p.ghost[0]) || (py > 1 && p.n[1] < p.ghost[1]))
    fail(KF_E_ARG, "local extent smaller than the ghost width");
  // the largest batch of buffers one exchange point handles (the schedule's, and the run-start fills)
  int batch = 1, run = 0;
  for (auto& ops : parts[0]->sched_full) {
    for (const Op& op : ops) {
      if (op.kind == 0) batch = std::max(batch, ++run);
      else run = 0;
    }
    run = 0;
  }
  D->max_batch = std::max(batch, 1);
  if (n_parts == px * py && world == 1 && !comm) {
    D->use_nccl = false;   // loopback: every part in this process
  } else if (n_parts == 1 && world == px * py && rank >= 0 && rank < world && comm) {
    D->use_nccl = true;
    D->comm = comm;
    Box a, b, c, d;
    strip_boxes(p, 0, &a, &b, &c, &d);
    uint64_t fx = box_bytes(a, p.es);
    strip_boxes(p, 1, &a, &b, &c, &d);
    uint64_t fy = box_bytes(a, p.es);
    D->slot_bytes = (std::max(fx, fy) + 255) / 256 * 256;
    const uint64_t bytes = 4 * D->slot_bytes * uint64_t(D->max_batch);
    if (cudaMalloc(&D->stage, bytes) != cudaSuccess) fail(KF_E_OOM, "cudaMalloc (halo staging) failed");
  } else {
    fail(KF_E_ARG, "either n_parts == px*py with world == 1 (loopback) or n_parts == 1 with world == px*py (NCCL)");
  }
  return D.release();
}

static void dist_free(kf_dist* d) {
  if (!d) return;
  try {
    dist_invalidate_graph(d);
    if (d->cap) cudaStreamDestroy(d->cap);
    if (d->stage) cudaFree(d->stage);
    if (d->xs) cudaStreamDestroy(d->xs);
    if (d->ev_ready) cudaEventDestroy(d->ev_ready);
    if (d->ev_done) cudaEventDestroy(d->ev_done);
  } catch (...) {
  }
  delete d;
}

// ---------------------------------------------------------------- kf_run (§8(b) entry point)
// Per-program cache of executors by canonical plan (JIT once per plan and device), plus the
// distributed context of kf_dist_init.
struct RunCache {
  std::map<std::pair<int, std::vector<int>>, kf_exec*> execs;   // (device, canonical plan)
  std::map<kf_exec*, kf_dist*> dists;
  bool dist = false;
  int rank = 0, world = 1, px = 1, py = 1;
  std::shared_ptr<Comm> comm;
};

static void run_cache_free(void* v) {
  RunCache* c = static_cast<RunCache*>(v);
  for (auto& [e, d] : c->dists) dist_free(d);
  for (auto& [k, e] : c->execs) kf_exec_destroy(e);
  delete c;
}

static RunCache& run_cache(kf_program* prog) {
  if (!prog->run_cache) {
    prog->run_cache = new RunCache();
    prog->run_cache_free = run_cache_free;
  }
  return *static_cast<RunCache*>(prog->run_cache);
}

}  // namespace kf

extern "C" {

kf_status kf_dist_unique_id(uint8_t id[128]) {
  KF_TRY({
    if (!id) fail(KF_E_ARG, "null argument");
    NcclId u;
    ckn(nccl().getUniqueId(&u), "ncclGetUniqueId");
    std::memcpy(id, &u, 128);
  });
}

kf_status kf_dist_neighbors(int32_t px, int32_t py, int32_t rank, int32_t out[4]) {
  KF_TRY({
    if (!out || px < 1 || py < 1 || rank < 0 || rank >= px * py) fail(KF_E_ARG, "bad process grid or rank");
    int nb[4];
    dist_neighbors(px, py, rank, nb);
    for (int i = 0; i < 4; i++) out[i] = nb[i];
  });
}

kf_status kf_dist_strips(const kf_program* prog, int32_t axis, kf_box out[4]) {
  KF_TRY({
    if (!prog || !out) fail(KF_E_ARG, "null argument");
    if (axis < 0 || axis > 1) fail(KF_E_ARG, "axis must be 0 (x) or 1 (y)");
    Box b[4];
    strip_boxes(prog->p, axis, &b[0], &b[1], &b[2], &b[3]);
    for (int i = 0; i < 4; i++) out[i] = kf_box{b[i].off, b[i].w, b[i].h, b[i].d, 0};
  });
}

kf_status kf_dist_create(kf_exec* const* parts, int32_t n_parts, int32_t px, int32_t py, int32_t rank, int32_t world,
                         const uint8_t* nccl_id, kf_dist** out) {
  KF_TRY({
    if (!out) fail(KF_E_ARG, "null argument");
    std::shared_ptr<Comm> comm;
    if (!(n_parts == px * py && world == 1)) {
      if (!nccl_id) fail(KF_E_ARG, "nccl_id required for the NCCL transport");
      if (n_parts != 1 || world != px * py || rank < 0 || rank >= world)
        fail(KF_E_ARG, "either n_parts == px*py with world == 1 (loopback) or n_parts == 1 with world == px*py (NCCL)");
      comm = make_comm(rank, world, nccl_id);
    }
    *out = dist_make(parts, n_parts, px, py, rank, world, comm);
  });
}

kf_status kf_dist_run(kf_dist* d, void* const* arrays, void* const* scratch, uint64_t scratch_bytes, int64_t nsteps,
                      const double* params, void* cuda_stream) {
  KF_TRY({
    if (!d) fail(KF_E_ARG, "null dist");
    if (nsteps < 0) fail(KF_E_ARG, "nsteps < 0");
    dist_run(d, arrays, scratch, scratch_bytes, nsteps, params, (cudaStream_t)cuda_stream);
  });
}

kf_status kf_dist_set_overlap(kf_dist* d, int32_t on) {
  KF_TRY({
    if (!d) fail(KF_E_ARG, "null dist");
    d->overlap = on ? 1 : 0;
  });
}

kf_status kf_dist_set_graph(kf_dist* d, int32_t on) {
  KF_TRY({
    if (!d) fail(KF_E_ARG, "null dist");
    d->use_graph = on != 0;
    if (!d->use_graph) dist_invalidate_graph(d);
  });
}

void kf_dist_destroy(kf_dist* d) { dist_free(d); }

kf_status kf_dist_init(kf_program* prog, int32_t rank, int32_t world, int32_t px, int32_t py, const uint8_t id[128]) {
  KF_TRY({
    if (!prog) fail(KF_E_ARG, "null program");
    if (px < 1 || py < 1 || world != px * py || rank < 0 || rank >= world) fail(KF_E_ARG, "bad process grid or rank");
    const Program& p = prog->p;
    if ((px > 1 && p.bc[0] != KF_BC_PERIODIC) || (py > 1 && p.bc[1] != KF_BC_PERIODIC))
      fail(KF_E_UNSUPPORTED, "decomposed axes must be PERIODIC in the local program");
    RunCache& c = run_cache(prog);
    if (c.dist) fail(KF_E_ARG, "kf_dist_init already called for this program");
    std::shared_ptr<Comm> comm;
    if (world > 1) {
      if (!id) fail(KF_E_ARG, "id required when world > 1");
      comm = make_comm(rank, world, id);
    }
    c.dist = world > 1;
    c.rank = rank;
    c.world = world;
    c.px = px;
    c.py = py;
    c.comm = comm;
  });
}

kf_status kf_scratch_bytes(const kf_program* prog, const int32_t* plan, uint64_t* bytes) {
  KF_TRY({
    if (!prog || !bytes) fail(KF_E_ARG, "null argument");
    (void)plan;   // renamed versions depend on the program only, not on the plan
    int period = 1;
    *bytes = padded_array_bytes(prog->p) * renamed_versions(prog->p, &period).size();
  });
}

kf_status kf_run(kf_program* prog, const int32_t* plan, void* const* arrays, void* scratch, uint64_t scratch_bytes,
                 int64_t nsteps, const double* params, void* cuda_stream) {
  KF_TRY({
    if (!prog || !plan) fail(KF_E_ARG, "null argument");
    const Program& p = prog->p;
    for (int k = 0; k < p.nk; k++)
      if (plan[k] < 0) fail(KF_E_ILLEGAL_PLAN, "V1 PARTITION: kernel " + std::to_string(k) + " has no group");
    const Plan pl = make_plan(p, plan);
    int dev = 0;
    CK(cudaGetDevice(&dev));
    RunCache& c = run_cache(prog);
    auto key = std::make_pair(dev, pl.label);
    auto it = c.execs.find(key);
    if (it == c.execs.end()) {
      kf_target t;
      kf_target_b200(&t);
      if (c.dist) t.internal_axes = (c.px > 1 ? 1 : 0) | (c.py > 1 ? 2 : 0);
      kf_exec* e = nullptr;
      kf_status st = kf_exec_create(prog, pl.label.data(), &t, &e);
      if (st != KF_OK) fail(st, kf_last_error());
      it = c.execs.emplace(key, e).first;
    }
    kf_exec* E = it->second;
    if (!c.dist) {
      exec_run(E, arrays, scratch, scratch_bytes, nsteps, params, (cudaStream_t)cuda_stream);
      return KF_OK;
    }
    auto dit = c.dists.find(E);
    if (dit == c.dists.end()) dit = c.dists.emplace(E, dist_make(&E, 1, c.px, c.py, c.rank, c.world, c.comm)).first;
    void* sc[1] = {scratch};
    dist_run(dit->second, arrays, sc, scratch_bytes, nsteps, params, (cudaStream_t)cuda_stream);
  });
}

}  // extern "C"
