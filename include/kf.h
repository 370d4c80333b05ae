/*
 * kf.h -- C ABI of the B200-native fused stencil-program executor.
 *
 * Implements the problem statement of Wahib & Maruyama, "Scalable Kernel Fusion
 * for Memory-Bound GPU Applications" (SC'14), PAPER.md:238 (Fig. 4):
 *     Input : original kernels K, |K| = n;  data arrays D, |D| = l
 *     Output: new kernels F, |F| = m
 * and executes the chosen fusion plan on sm_100a.  Line references "P:n" are
 * lines of /root/reference/PAPER.md.  Readings "Rn" are listed in DESIGN.md.
 *
 * Conventions (all entry points):
 *  - Every call returns kf_status; KF_OK == 0.  On error a thread-local message is
 *    available from kf_last_error() and output parameters are left untouched.
 *    No C++ exception crosses this boundary.
 *  - Handles (kf_program, kf_exec) are opaque, owned by the caller until *_destroy.
 *    Const queries on a handle are thread-safe; kf_exec_run on one kf_exec is not.
 *  - Device memory (arrays, scratch) is caller-owned (e.g. torch tensors) and laid
 *    out as kf_array_layout() says.  The library never allocates device memory
 *    except inside kf_run_host() (documented there).
 *  - A plan is a caller-owned int32_t[n] giving the group label of every kernel;
 *    any non-negative labels are accepted and canonicalised internally
 *    (groups renumbered by first appearance = restricted-growth string).
 */
#ifndef KF_H
#define KF_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------ status */
typedef enum {
  KF_OK = 0,
  KF_E_ARG = 1,           /* null pointer, bad size, out-of-range index            */
  KF_E_PROGRAM = 2,       /* ill-formed program description                        */
  KF_E_ILLEGAL_PLAN = 3,  /* plan violates a constraint (see kf_plan_validate)     */
  KF_E_RESOURCE = 4,      /* scratch too small, capacity exceeded                  */
  KF_E_CUDA = 5,          /* CUDA driver/runtime error (launch or async fault)     */
  KF_E_NVRTC = 6,         /* JIT compilation failed                                */
  KF_E_NCCL = 7,          /* NCCL error                                            */
  KF_E_OOM = 8,           /* host or device allocation failed                      */
  KF_E_UNSUPPORTED = 9    /* feature not available (e.g. no GPU, no NCCL)          */
} kf_status;

/* Thread-local message of the last failing kf_* call on this thread; valid until the
 * next kf_* call on the same thread.  Never NULL. */
const char* kf_last_error(void);
/* Library version string, e.g. "kf 0.1 (sm_100a)". */
const char* kf_version(void);

/* ------------------------------------------------------------------ program description
 * One program = an ordered list of original kernels over a set of 3D arrays sharing one
 * interior grid n[0] x n[1] x n[2] (x fastest) and one dtype.  A kernel is a list of
 * statements `out_array = expr`, expr in RPN.  Readings:
 *   R1  all reads of a kernel see pre-kernel values; a kernel may read an array it
 *       writes only at offset (0,0,0) (P:138-155 races otherwise); statements of one
 *       kernel write distinct arrays.
 *   R9  per-axis boundary: FROZEN = ghost cells are user-initialised and never written;
 *       PERIODIC = reads wrap modulo n.
 *   R16 each RPN node is one IEEE operation in the program dtype, left to right;
 *       CONST/PARAM values are rounded to the dtype; MIN(a,b)=(b<a)?b:a,
 *       MAX(a,b)=(a<b)?b:a; no FMA contraction anywhere.                            */
typedef enum { KF_F32 = 0, KF_F64 = 1 } kf_dtype;
typedef enum { KF_BC_FROZEN = 0, KF_BC_PERIODIC = 1 } kf_bc;

enum { KF_ARRAY_OUTPUT = 1u << 0,      /* final value must be kept (step-live, R15)       */
       KF_ARRAY_READONLY = 1u << 1 };  /* asserted never written (checked)                */

enum { KF_PROG_RELAX_EXPANDABLE = 1u << 0,  /* rename expandable arrays        */
       KF_PROG_RELAX_ALL = 1u << 1,         /* extension: rename every written array      */
       KF_PROG_NO_KINSHIP = 1u << 2 };      /* experiments only: skip constraint (1.5)    */

typedef enum {
  KF_OP_CONST = 0, KF_OP_PARAM = 1, KF_OP_LOAD = 2, KF_OP_ADD = 3, KF_OP_SUB = 4,
  KF_OP_MUL = 5, KF_OP_DIV = 6, KF_OP_MIN = 7, KF_OP_MAX = 8, KF_OP_NEG = 9,
  KF_OP_ABS = 10, KF_OP_SQRT = 11
} kf_opcode;

/* RPN instruction (24 bytes).  LOAD: arg = array index, d = (di,dj,dk) offset.
 * PARAM: arg = parameter index.  CONST: imm.  Others: arg, d, imm ignored. */
typedef struct { int32_t op; int32_t arg; int8_t d[3]; int8_t pad0; int32_t pad1; double imm; } kf_insn;
typedef struct { int32_t out_array; int32_t n_insn; const kf_insn* insn; } kf_stmt;
/* Optional declared footprint (Table III "ThrLD"): if n_reads > 0 the set of
 * (array, offset) pairs must equal the set of LOADs of the kernel exactly. */
typedef struct { int32_t array; int8_t d[3]; int8_t pad; } kf_access;
typedef struct {
  const char* name;
  int32_t n_stmt; const kf_stmt* stmt;
  int32_t n_reads; const kf_access* reads;
} kf_kernel_desc;
typedef struct { const char* name; uint32_t flags; } kf_array_desc;
typedef struct {
  int32_t dtype;                 /* kf_dtype                                        */
  int32_t pad;
  int64_t n[3];                  /* interior extents, each >= 1                     */
  int32_t ghost[3];              /* ghost width per axis (>= every |offset|)        */
  int32_t bc[3];                 /* kf_bc per axis                                  */
  int32_t n_arrays; const kf_array_desc* arrays;
  int32_t n_kernels; const kf_kernel_desc* kernels;
  int32_t n_params;              /* PARAM slots, values given to kf_exec_run        */
  uint32_t flags;                /* KF_PROG_*                                       */
} kf_program_desc;

typedef struct kf_program kf_program;

/* Deep-copies and checks the description (RPN well-formed, indices in range, offsets
 * within ghost, R1 in-place rule, READONLY arrays not written), then builds the
 * data-dependency graph, precedence DAG and derived sets.
 * Errors: KF_E_ARG (null), KF_E_PROGRAM (message names kernel/statement). */
kf_status kf_program_create(const kf_program_desc* desc, kf_program** out);
void kf_program_destroy(kf_program* prog);

typedef struct {
  int32_t n_kernels, n_arrays, n_edges, es;   /* es = element size in bytes */
  int64_t npts;                               /* interior points             */
  int32_t n_relaxed;                          /* arrays renamed       */
  int32_t pad;
} kf_program_info;
kf_status kf_program_get_info(const kf_program* prog, kf_program_info* out);

/* Precedence edges of the order-of-execution graph, canonical form (R2):
 * RAW from the writer of the version read; for arrays not renamed also WAW from the
 * previous writer and WAR from every reader of the overwritten version.  Sorted by
 * (dst, src, kind, array).  *n receives the total; at most cap are written. */
typedef enum { KF_EDGE_RAW = 0, KF_EDGE_WAR = 1, KF_EDGE_WAW = 2 } kf_edge_kind;
typedef struct { int32_t src, dst, kind, array; } kf_edge;
kf_status kf_program_edges(const kf_program* prog, kf_edge* out, int32_t cap, int32_t* n);

/* reach[a*n+b] = 1 iff a path a ~> b of length >= 1 exists (n = n_kernels). */
kf_status kf_program_reach(const kf_program* prog, uint8_t* reach);

/* Array classes: RO never written; WO written never read; EXPANDABLE >= 2
 * writing kernels; RW otherwise.  Also: renamed (relaxed) flag, step-live flag (R15) and
 * upward_exposed (read before any write in a step = an input of every step). */
typedef enum { KF_CLS_RO = 0, KF_CLS_RW = 1, KF_CLS_EXPANDABLE = 2, KF_CLS_WO = 3 } kf_array_class;
typedef struct { int32_t cls, n_writers, n_readers, relaxed, step_live, upward_exposed; } kf_array_info;
kf_status kf_program_array_info(const kf_program* prog, int32_t array, kf_array_info* out);
/* The class of every array at once: cls[n_arrays] (caller-owned) receives kf_array_class values
 * (SURVEY 8(b)). */
kf_status kf_program_array_class(const kf_program* prog, int32_t* cls);

/* Degree of kinship (Table II) of kernels a and b inside `group` (R5: the chain
 * must stay inside the group; 0 if none). */
kf_status kf_program_kinship(const kf_program* prog, int32_t a, int32_t b,
                             const int32_t* group, int32_t group_n, int32_t* degree);

/* Device layout of every array (all arrays share it): element (i,j,k) of the ghosted
 * grid, i in [-ghost[0], n[0]+ghost[0]) etc., lives at
 *     base + origin + k*plane + j*pitch + i          (elements)
 * pitch >= n[0]+2*ghost[0], origin 128-byte aligned (P:82 horizontal padding, R13).
 * elems = total elements to allocate per array. */
typedef struct { int64_t pitch, rows, plane, origin, elems; int32_t xoff, pad; } kf_layout;
kf_status kf_array_layout(const kf_program* prog, kf_layout* out);

/* ------------------------------------------------------------------ target (Table IV analogue) */
typedef struct {
  double hbm_bytes_per_s;        /* peak used by the projection (B200 nominal 8.0e12)     */
  int32_t smem_per_block;        /* usable dynamic SMEM per CTA (232448 on B200)          */
  int32_t regs_per_thread_max;   /* R_Max (255)                                           */
  int32_t n_sm;                  /* 148                                                   */
  int32_t tile[3];               /* TX, TY, TZ of a fused-group tile; TZ = 0: whole column */
  int32_t stages;                /* TMA ring stages S >= 2                                */
  int32_t threads;               /* threads per CTA (multiple of 32)                      */
  int32_t max_halo;              /* cap on xy extended-region extent                      */
  int32_t internal_axes;         /* bitmask of axes split across ranks (V6 treats as wrap) */
  int32_t zunroll;               /* planes per stream iteration U in [1,4] (ILP; ring depth) */
  int32_t pblock[2];             /* points per thread in x, y (register blocking), [1,4] each */
  int32_t ringunroll;            /* 1: ring sizes rounded to powers of two and the stream loop
                                    unrolled so every SMEM slot is a compile-time constant    */
  int32_t ghostwrite;            /* 1: stores also write periodic x/y ghost copies, so the step
                                    needs no ghost-fill kernels (single-domain runs)          */
  int32_t minblocks;             /* register cap of the group kernels (__maxnreg__): keep this
                                    many CTAs per SM resident -- 0 = as many as shared memory
                                    allows, n >= 1 = n; never above R_est (V8); dropped if ptxas
                                    would spill.  -1 = no cap                                   */
  int32_t skew;                  /* 1: a kernel reading an in-group version at a nonzero xy offset
                                    runs U more planes behind its producer (delay skew, R20c), so
                                    it reads planes the previous iteration's barrier published and
                                    fast iterations need no barrier between kernels             */
  int32_t canvas_ld;             /* fast-iteration shared loads: 1 = unpredicated wherever every
                                    address they can form lies in the rings' SMEM (fewer
                                    instructions; lanes outside the readers' regions load values
                                    nobody stores), 0 = predicated on the readers' regions      */
  int32_t pair_zq;               /* pair canvas (pblock 2x1): 1 = z-column values carried in
                                    registers across stream iterations instead of re-read
                                    from shared memory (more registers), 0 = off             */
  int32_t inline_xy;             /* pair canvas: 1 = a reader recomputes an in-group value it reads
                                    at an xy offset (the producer's statement re-evaluated there
                                    from the staged inputs: same operations, same bits) instead
                                    of a shared-memory copy behind a barrier, where the producer
                                    reads only staged inputs and every reader runs in the same
                                    stream iteration at dz = 0; 2 = also producers reading such
                                    recomputed values (two levels: more recompute, registers);
                                    0 = shared-memory copies                                  */
} kf_target;
/* Fills the B200 defaults: 8.0e12, 232448, 255, 148, {64,4,0}, 2, 256, 16, 0, 1, {1,1}, 0, 0, 0, 0, 1, 1, 1. */
kf_status kf_target_b200(kf_target* out);

/* ------------------------------------------------------------------ legality (Eq. 1.1-1.7) */
typedef enum {
  KF_V_OK = 0,
  KF_V_PARTITION = 1,  /* (1.2),(1.4) a kernel without a group (negative label)          */
  KF_V_KINSHIP = 2,    /* (1.5) group not connected by shared arrays (R5)                */
  KF_V_CONVEX = 3,     /* (1.3) a kernel on a path between two fused kernels is outside  */
  KF_V_CYCLE = 4,      /* groups cannot be ordered: quotient graph has a cycle (R4)      */
  KF_V_HAZARD = 5,     /* cross-tile read of an array the group overwrites (P:52,107;R7) */
  KF_V_HALO = 6,       /* accumulated halo > ghost (wrap/internal axes) or > max_halo    */
  KF_V_SMEM = 7,       /* (1.6) on-chip bytes > smem_per_block (resource model, R20)     */
  KF_V_REGS = 8        /* (1.7) register estimate > regs_per_thread_max (R20)            */
} kf_violation_code;
/* First violation in the canonical order: all groups for V1, then all groups for V2, ...
 * Fields not meaningful for a code are -1:
 *   V1 {kernel_a = kernel}; V2 {group, kernel_a = first kernel, kernel_b = unreachable};
 *   V3 {group, kernel_a = min in-group source, kernel_b = outside kernel on the path};
 *   V4 {group}; V5 {group, kernel_a = reader, kernel_b = writer, array};
 *   V6 {group, array} for a load box, or {group, kernel_a} for an extended region;
 *   V7, V8 {group}. */
typedef struct { int32_t code, group, kernel_a, kernel_b, array; } kf_violation;
/* Returns KF_OK if legal, KF_E_ILLEGAL_PLAN with *why filled otherwise. */
kf_status kf_plan_validate(const kf_program* prog, const int32_t* plan, const kf_target* target,
                           kf_violation* why);
/* Canonical labels (restricted-growth string) of a plan; returns m (number of groups). */
kf_status kf_plan_canonical(const int32_t* plan, int32_t n, int32_t* out, int32_t* m);

/* ------------------------------------------------------------------ projection (Eq. 11) */
/* Codeless upper bound: per group, compulsory bytes = es*N*(|LiveIn|+|LiveOut|) over the
 * interior (R15); t = bytes / hbm_bytes_per_s; totals are a left fold in canonical group
 * order.  Also the resource model used by V7/V8 and advisory (1.1): unprofitable = the
 * group (>= 2 kernels) saves no bytes over its kernels run alone (R6).
 * Works for any plan passing V1 (m <= cap groups written). */
typedef struct {
  uint64_t bytes_read, bytes_written;
  uint64_t halo_bytes_est;       /* tile-halo re-reads over the interior (not compulsory)  */
  uint32_t smem_bytes, regs_est;
  int32_t n_kernels, unprofitable;
  double t_s;                    /* codeless bound: compulsory bytes / hbm_bytes_per_s            */
  double t_model_s;              /* resource-aware projection (R22): HBM + issue time of regions  */
} kf_group_proj;
kf_status kf_project(const kf_program* prog, const int32_t* plan, const kf_target* target,
                     kf_group_proj* per_group, int32_t cap, int32_t* m,
                     uint64_t* bytes_total, double* t_total_s);

/* Lowering of one group (a3): per kernel its extended region E(k) as extents beyond the
 * tile T per axis (R8, may be negative), whether it is alive (non-empty E) and its z
 * delay (planes it runs behind the stream front).  Useful for tests and tools. */
typedef struct { int32_t kernel, alive, delay, pad; int32_t elo[3], ehi[3]; } kf_kernel_sched;
kf_status kf_group_schedule(const kf_program* prog, const int32_t* plan, const kf_target* target,
                            int32_t group, kf_kernel_sched* out, int32_t cap, int32_t* n);

/* The paper's own projection for one new kernel (Eq. 2-10) from Table III/IV
 * metadata, as printed (readings R11-R14: Hal in points, "8" = element bytes).  Reproduces the
 * worked example of P:372 (B_Sh = 688, P_MemBound = 29.688 GFLOPS); the B200 search uses
 * kf_group_proj.t_model_s instead (R22). */
typedef struct {
  int32_t t_b, blocks_smx, thr, blocks, hal, halo, shared_arrays, smx;   /* T_B, Blocks_SMX, Thr, B, Hal, c, |ShrLst|, #SMX */
  int32_t r_t, r_max, r_smx, r_adr, sh_smx, b_conf, elem_bytes, pad;      /* R_T, R_Max, R_SMX (regs), R_Adr, Sh_SMX (B), B_conf (B) */
  double gmem_bw_gbs, regfac, max_thread_load, fl_unfused_sum, flop_halo_sum;
} kf_paper_meta;
typedef struct {
  int32_t h_th, eq2_ok, eq3_ok, eq6_ok, eq7_ok, pad;
  double b_sh, b_eff, p_membound_gflops, t_pro_s;
} kf_paper_proj;
kf_status kf_paper_projection(const kf_paper_meta* meta, kf_paper_proj* out);

/* ------------------------------------------------------------------ plan search */
typedef enum {
  KF_SEARCH_BRUTE = 0,   /* all restricted-growth strings with pruning (n <= 14)           */
  KF_SEARCH_GREEDY = 1,  /* agglomerative merging of groups by largest byte saving          */
  KF_SEARCH_AUTO = 2,    /* brute if n <= 10 else greedy                                    */
  KF_SEARCH_GREEDY_TIME = 3,  /* greedy merging on the resource-aware projected time (R22)    */
  KF_SEARCH_BRUTE_TIME = 4,   /* brute force on the resource-aware projected time (n <= 14)    */
  KF_SEARCH_HGGA = 5,         /* hybrid grouping GA (Alg. 1) on projected time; seed  */
  KF_SEARCH_HGGA_BYTES = 6    /* the same GA on compulsory bytes (comparable to BRUTE)           */
} kf_search_method;
/* Minimises total compulsory bytes (or, for the *_TIME methods, total projected time) over
 * legal plans; ties -> lexicographically smallest canonical labels (R17).  plan_out:
 * int32_t[n] canonical.  bytes_out (compulsory bytes of the result) may be NULL. */
kf_status kf_plan_search(const kf_program* prog, const kf_target* target, int32_t method,
                         uint64_t seed, int32_t* plan_out, uint64_t* bytes_out);
/* Number of legal partitions (brute force; n <= 14). */
kf_status kf_plan_count_legal(const kf_program* prog, const kf_target* target, uint64_t* count);
/* Every legal partition (brute force over restricted-growth strings, n <= 14) in enumeration order:
 * plans[i*n .. i*n+n) = canonical labels of the i-th legal plan for i < cap; *count = the total
 * (call with cap = 0 to size the buffer).  Config 2 "every legal plan run". */
kf_status kf_plan_enumerate(const kf_program* prog, const kf_target* target, int32_t* plans, int64_t cap,
                            int64_t* count);

/* ------------------------------------------------------------------ execution (sm_100a) */
typedef struct kf_exec kf_exec;
/* Validates the plan (KF_E_ILLEGAL_PLAN), lowers every group, generates one CUDA kernel
 * per group and JIT-compiles it with NVRTC for sm_100a (--fmad=false, IEEE div/sqrt).
 * Needs a CUDA device (current device of the calling thread). */
kf_status kf_exec_create(kf_program* prog, const int32_t* plan, const kf_target* target, kf_exec** out);
/* Same with one launch configuration per fused group: targets[n_targets], n_targets = 1 (all
 * groups) or m (canonical group order).  Legality V6-V8 is checked per group with its own
 * target (tile, stages, zunroll, limits) -- e.g. the result of per-group autotuning. */
kf_status kf_exec_create_ex(kf_program* prog, const int32_t* plan, const kf_target* targets, int32_t n_targets,
                            kf_exec** out);
void kf_exec_destroy(kf_exec* ex);
/* Bytes of caller-provided device scratch: one buffer per renamed array version. */
kf_status kf_exec_scratch_bytes(const kf_exec* ex, uint64_t* bytes);
/* Runs nsteps steps asynchronously on `cuda_stream` (a cudaStream_t; NULL = legacy
 * default stream).  arrays: n_arrays device pointers to the *allocation base* of each
 * array (kf_array_layout).  params: n_params values (NULL if none).  After the call
 * completes, every array that is not TEMP (written but not step-live, R15) holds its
 * post-nsteps value in the interior; TEMP contents are unspecified.  Ghost cells of FROZEN
 * axes are never written; ghost layers of PERIODIC axes are overwritten with wrapped copies
 * of the interior (their contents after a run are the wrap of some step's values).
 * Read-only arrays' interiors are never written.
 * Errors: KF_E_ARG, KF_E_RESOURCE (scratch too small), KF_E_CUDA (launch failure; async
 * faults surface at the next synchronising call). */
kf_status kf_exec_run(kf_exec* ex, void* const* arrays, void* scratch, uint64_t scratch_bytes,
                      int64_t nsteps, const double* params, void* cuda_stream);
/* Same, with HOST arrays (same layout): allocates device buffers once per kf_exec (freed by
 * kf_exec_destroy), copies the arrays read before they are written in a step (upward-exposed
 * and read-only arrays) host->device, runs, copies every step-live array device->host, and
 * synchronises `cuda_stream`.  h2d/d2h receive the bytes copied (may be NULL). */
kf_status kf_run_host(kf_exec* ex, void* const* host_arrays, int64_t nsteps, const double* params,
                      void* cuda_stream, uint64_t* h2d_bytes, uint64_t* d2h_bytes);

typedef struct {
  int32_t n_groups;             /* fused kernels launched per step                        */
  int32_t launches_per_step;    /* group kernels + ghost fills                            */
  int32_t fills_per_step;       /* ghost-fill kernel launches per step (consecutive fills batched) */
  int32_t period;               /* steps per replay period (2 with renamed step-live)     */
  uint64_t compulsory_bytes_per_step;
} kf_exec_info;
kf_status kf_exec_get_info(const kf_exec* ex, kf_exec_info* out);
/* Per-group launch details: grid, threads, dynamic SMEM, registers (cuFuncGetAttribute),
 * local (spill) bytes, the loaded function's maximum threads per CTA (-1 before loading),
 * compulsory HBM bytes per launch, shared-memory bytes per launch of the canvas fast iterations
 * (loads + stores + TMA writes; the on-chip roofline's algorithmic bytes), kernel name.
 * name: >= 64 chars. */
typedef struct {
  int32_t group, grid, threads, smem_bytes, regs, local_bytes, n_kernels, max_threads;
  uint64_t bytes_per_launch;
  uint64_t onchip_bytes_per_launch;
  char name[64];
} kf_group_info;
kf_status kf_exec_group_info(const kf_exec* ex, int32_t group, kf_group_info* out);
/* Loads every group kernel of the executor onto the calling thread's current device (the first
 * kf_exec_run does it implicitly); afterwards kf_exec_group_info reports the loaded functions'
 * CU_FUNC_ATTRIBUTE_NUM_REGS / LOCAL_SIZE_BYTES (the V7/V8 hardware pin).  Needs a GPU. */
kf_status kf_exec_load(kf_exec* ex);
/* Generated CUDA source of a group (for inspection); *len receives the full length. */
kf_status kf_exec_group_source(const kf_exec* ex, int32_t group, char* buf, int64_t cap, int64_t* len);
/* Profiling mode: when on, kf_exec_run records a CUDA event around every group launch on
 * the launching stream and accumulates per-group device milliseconds, readable (after the
 * stream is synchronised) with kf_exec_group_times; reset clears the accumulators. */
kf_status kf_exec_set_profiling(kf_exec* ex, int32_t on);
kf_status kf_exec_group_times(kf_exec* ex, double* ms, int32_t cap, int32_t* n, int64_t* launches);
/* Use a captured CUDA graph for the step loop (default on). */
kf_status kf_exec_set_graph(kf_exec* ex, int32_t on);
/* The caller changed array contents outside the interior (e.g. FROZEN ghost values) while keeping
 * the same device pointers: the next run re-copies them into the renamed scratch versions (R9).
 * Without this call, FROZEN ghost values must stay constant for a given pointer set.
 * (kf_run_host does it itself after every upload.) */
kf_status kf_exec_invalidate(kf_exec* ex);

/* ------------------------------------------------------------------ multi-GPU (row a11) */
/* Domain decomposition over a px x py process grid (x, y split; z whole; part/rank index
 * iy*px + ix).  Every part runs the same kf_exec plan on its LOCAL sub-domain (the local
 * program has n = global n / (px, py) and PERIODIC bc on decomposed axes); the periodic
 * ghost fills of the schedule become halo exchanges with neighbouring parts (x strips, then
 * y strips incl. x ghosts = corners), so results equal the single-domain run bit for bit.
 * Transports: loopback -- n_parts == px*py, world == 1: all parts in this process on one
 * device (strips copied device-to-device; for testing); NCCL -- n_parts == 1,
 * world == px*py, rank in [0, world): ncclSend/ncclRecv per neighbour over NVLink/NVSwitch,
 * nccl_id from kf_dist_unique_id() on rank 0, broadcast by the caller (e.g. torch.distributed). */
typedef struct kf_dist kf_dist;
kf_status kf_dist_unique_id(uint8_t id[128]);
kf_status kf_dist_neighbors(int32_t px, int32_t py, int32_t rank, int32_t out[4]);   /* x-, x+, y-, y+ */
kf_status kf_dist_create(kf_exec* const* parts, int32_t n_parts, int32_t px, int32_t py, int32_t rank, int32_t world,
                         const uint8_t* nccl_id, kf_dist** out);
/* arrays: n_parts * n_arrays device pointers (part-major); scratch: n_parts pointers (or NULL
 * if the plan needs none), each >= kf_exec_scratch_bytes.  Asynchronous on cuda_stream. */
kf_status kf_dist_run(kf_dist* d, void* const* arrays, void* const* scratch, uint64_t scratch_bytes, int64_t nsteps,
                      const double* params, void* cuda_stream);
/* Overlap of halo exchange with interior compute (default on): before a group that needs fresh
 * ghosts, the exchanges run on an internal second stream (ordered after all work issued on
 * cuda_stream) while the group's interior tiles -- those at least one ghost width inside the
 * local domain in x and y, which read no ghost and write no exchanged strip -- run on
 * cuda_stream; the other tiles are launched after the exchanges complete.  Results are
 * identical either way; off = exchanges and whole-group launches in stream order. */
kf_status kf_dist_set_overlap(kf_dist* d, int32_t on);
/* Capture one replay period of kf_dist_run (exchanges, overlap and NCCL calls included) in a CUDA
 * graph (default on; if the capture fails the dist runs eagerly from then on). */
kf_status kf_dist_set_graph(kf_dist* d, int32_t on);
/* Halo strip geometry of the LOCAL program on a decomposed axis (0 = x, 1 = y), in elements of
 * kf_array_layout: out[0] send_lo (first ghost-deep interior strip, goes to the low neighbour's
 * high ghost), out[1] send_hi, out[2] recv_lo (low ghost), out[3] recv_hi.  x strips cover every
 * padded row; y strips are whole padded rows (x ghosts = corners included). */
typedef struct { int64_t offset; int32_t w, h, d, pad; } kf_box;
kf_status kf_dist_strips(const kf_program* prog, int32_t axis, kf_box out[4]);
void kf_dist_destroy(kf_dist* d);

/* ------------------------------------------------------------------ §8(b) one-call interface
 * The problem statement's boundary (Fig. 4): a program, a plan F (group label per kernel),
 * the data arrays D -- run N timesteps.  kf_run keeps one kf_exec per (device, canonical plan)
 * inside the program handle (validated, lowered and JIT-compiled on the first call for that plan
 * with the kf_target_b200 defaults; freed by kf_program_destroy), so repeated calls only launch.
 *
 * kf_scratch_bytes: device scratch kf_run needs for `plan` (one buffer per renamed version,
 * P:53; it depends on the program only, plan may be NULL).
 * kf_run: arrays = n_arrays caller-owned device pointers (allocation bases, kf_array_layout,
 * 128-byte aligned); scratch >= kf_scratch_bytes; params = n_params values (NULL if none);
 * asynchronous on cuda_stream.  Results/errors as kf_exec_run (KF_E_ILLEGAL_PLAN for an illegal
 * plan, KF_E_NVRTC if the JIT fails).  Not thread-safe per program.
 * kf_dist_init: makes later kf_run calls on this program distributed over a px x py process grid
 * (rank = iy*px + ix, world = px*py, the program describing the LOCAL sub-domain with PERIODIC
 * decomposed axes): halo exchange by NCCL over NVLink replaces the periodic wrap (row a11).  id =
 * kf_dist_unique_id() of rank 0, broadcast by the caller; ignored when world == 1.  Once per
 * program; KF_E_NCCL if the communicator cannot be created. */
kf_status kf_scratch_bytes(const kf_program* prog, const int32_t* plan, uint64_t* bytes);
kf_status kf_run(kf_program* prog, const int32_t* plan, void* const* arrays, void* scratch, uint64_t scratch_bytes,
                 int64_t nsteps, const double* params, void* cuda_stream);
kf_status kf_dist_init(kf_program* prog, int32_t rank, int32_t world, int32_t px, int32_t py, const uint8_t id[128]);

/* ------------------------------------------------------------------ utilities */
/* Overwrite `bytes` of caller-provided device memory on `cuda_stream` (benchmarks: evict
 * the 126 MB L2 between timed iterations). */
kf_status kf_flush_l2(void* buf, uint64_t bytes, void* cuda_stream);
/* Generate and JIT-compile (NVRTC, sm_100a) the kernel of one group without running it;
 * works without a GPU.  regs/spill_bytes from ptxas (-v); log receives the NVRTC log. */
kf_status kf_jit_check(const kf_program* prog, const int32_t* plan, const kf_target* target, int32_t group,
                       int32_t* regs, int32_t* spill_bytes, char* log, int64_t cap);

#ifdef __cplusplus
}
#endif
#endif /* KF_H */
