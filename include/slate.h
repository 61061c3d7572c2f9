/*
 * slate.h -- C ABI of libslate, the B200 (sm_100a) runtime of the Slate
 * slate-kernel path (Allen, Feng, Ge, "Slate: Enabling Workload-Aware
 * Efficient Multiprocessing for Modern GPGPUs", IPDPS 2019).
 *
 * Citations "P:L<n> §<sec>" are lines of the paper text.
 *
 * What the library does (north star):
 *   Client processes submit kernels to a single-context server (P:L133-139
 *   §IV-A).  Every kernel K(B,T) is run as the transformed kernel
 *   K*(B*,T) (§III-A-1): persistent worker CTAs bound to a per-queue SM
 *   range (Lst1) pull original block indices from a device-side
 *   atomic task counter (slateIdx, Lst2 P:L199-231), decode them to (x,y,z),
 *   run the tenant body, and check a device-visible resize word at every task
 *   boundary, so a kernel shrinks or grows its SM share on the fly with no
 *   relaunch (§III-C).  A workload-aware selector (Tab I,
 *   P:L99-121 §III-B) decides which kernels co-run.
 *
 * Conventions
 *   - Every call returns slate_status: 0 = SLATE_OK, > 0 informational,
 *     < 0 an error.  No exception or abort crosses the ABI.  After an error,
 *     slate_last_error(session) holds a one-line message (CUDA's text kept).
 *   - Device pointers are passed as uint64_t device addresses.  In-process
 *     (endpoint == NULL) they are used as is.  Through a server endpoint every
 *     pointer must lie inside a buffer registered with slate_share_buffer; the
 *     server rewrites it to its own mapping of that buffer (the paper's
 *     shared-buffer -> GPU-pointer table).
 *   - Sessions are thread-safe (one mutex per session).  Handles
 *     (slate_kernel, slate_launch_id) are never reused within a server's life.
 *   - SM ranges are inclusive [sm_lo, sm_hi] in *rank* space (P:L185-186,
 *     reading Q5): rank r is the r-th smallest %smid the server observed at
 *     start-up (calibration), 0 <= r < slate_info.num_sms.
 */
#ifndef SLATE_H
#define SLATE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SLATE_ABI_VERSION 1u

/* ------------------------------------------------------------------ status */
typedef int32_t slate_status;
#define SLATE_OK            0
#define SLATE_DONE          1   /* informational: the launch had already completed */
#define SLATE_EINVAL       (-1) /* bad argument */
#define SLATE_ENOMEM       (-2) /* out of device memory or control blocks */
#define SLATE_ECUDA        (-3) /* a CUDA call failed (sticky kernel errors included) */
#define SLATE_EIPC         (-4) /* no server at the endpoint / transport failure */
#define SLATE_ETIMEDOUT    (-5) /* slate_sync timed out */
#define SLATE_ENOTFOUND    (-6) /* unknown kernel or launch handle */
#define SLATE_ESTATE       (-7) /* call not valid in the current state */
#define SLATE_EUNSUPPORTED (-8) /* kind not built into this library */

typedef struct slate_session slate_session;
typedef uint64_t slate_kernel;   /* 0 is never a valid handle */
typedef uint64_t slate_launch_id; /* monotonically increasing per server, 0 never valid */

/* ------------------------------------------------------------------ kinds
 * The tenant kernels built into this library.  The paper
 * injects the Slate code into arbitrary user kernels at run time with a FLEX
 * scanner + NVRTC; its static alternative ("OMP-like pragma",
 * P:L157) is what this build does: each kind is compiled into the worker
 * template at build time.  Block geometry T is fixed per kind. */
typedef enum {
  SLATE_KIND_TRIAD = 1,        /* a = b + s*c, fp32; 1024 elems/block, T = 256          */
  SLATE_KIND_COPY = 2,         /* a = b, fp32; 4096 elems (16 KiB)/block, T = 128       */
  SLATE_KIND_SGEMM_NAIVE = 3,  /* C = A B, fp32 row-major; 16x16 C tile/block, T = 256  */
  SLATE_KIND_SPMV_CSR = 4,     /* y = A x, CSR int32/fp32; 32 rows/block, T = 256       */
  SLATE_KIND_BLACKSCHOLES = 5, /* mean call/put over P sigmas; 1024 options/block, T=256 */
  SLATE_KIND_STENCIL2D = 6,    /* 5-point Jacobi sweep; 128x8 points/block, T = 256     */
  SLATE_KIND_GEMM_BF16 = 7,    /* C(fp32) = A B^T, bf16 K-major; 128x128 tile/block     */
  /* The paper's own applications (Tab II; NEXT-2).  Black-Scholes
   * (BS) is SLATE_KIND_BLACKSCHOLES with one scenario. */
  SLATE_KIND_TRANSPOSE = 8,    /* TR: out = in^T, fp32 h x w -> w x h; 32x32 tile/block, T = 256 */
  SLATE_KIND_SGEMM_TILED = 9,  /* MM: C = A B, fp32 row-major, the SDK matrixMul; 32x32 C tile/block
                                  through shared memory, T = 256 (args: slate_args_sgemm)          */
  SLATE_KIND_QRNG = 10,        /* RG: quasirandom points; 1024 points of one dimension/block     */
  SLATE_KIND_GAUSS_FAN1 = 11,  /* GS step t, Fan1: m[i][t] = a[i][t] / a[t][t]; 256 rows/block   */
  SLATE_KIND_GAUSS_FAN2 = 12,  /* GS step t, Fan2: a[i][j] -= m[i][t] a[t][j] (j >= t),
                                  b[i] -= m[i][t] b[t]; 16 rows x 128 columns/block              */
  SLATE_KIND_USER = 13,        /* a user kernel compiled at run time (slate_register_source, NEXT-3) */
  SLATE_KIND_MAX_ = 14
} slate_kind;

/* Per-kind argument blocks (passed by value in slate_launch_desc.args).
 * All arrays are densely packed, 16-byte aligned, row-major. */
typedef struct { uint64_t a, b, c; uint64_t n; float s; uint32_t pad_; } slate_args_triad;
typedef struct { uint64_t a, b; uint64_t n; } slate_args_copy;
typedef struct { uint64_t A, B, C; uint32_t m, n, k, pad_; } slate_args_sgemm;      /* A m x k, B k x n */
typedef struct { uint64_t rowptr, col, val, x, y; uint32_t n_rows, n_cols; } slate_args_spmv;
typedef struct {
  uint64_t S, X, T;        /* inputs [n] fp32: spot, strike, years to expiry */
  uint64_t call, put;      /* outputs [n] fp32: mean over the P scenarios    */
  uint64_t sigmas;         /* [n_scen] fp32 volatilities (reading Q16)       */
  uint64_t n; float r; uint32_t n_scen;
} slate_args_bs;
typedef struct { uint64_t in, out; uint32_t h, w; } slate_args_stencil;
/* gemm: A m x k, B n x k bf16 K-major, C m x n fp32; any m, k % 8 == 0, n % 4 == 0 (16-byte row
 * strides); grid (ceil(n/tile_n), ceil(m/tile_m)), a ragged last tile row/column/K slice allowed */
typedef struct { uint64_t A, B, C; uint32_t m, n, k, pad_; } slate_args_gemm;
/* TR: in h x w fp32, out w x h fp32 (out[j][i] = in[i][j]); grid (ceil(w/32), ceil(h/32)) */
typedef struct { uint64_t in, out; uint32_t h, w; } slate_args_transpose;
/* RG (the CUDA SDK quasirandomGenerator kernel): out[d][i] = float(q_d(seed + i) + 1) * 2^-31,
 * q_d(k) = XOR of table[d][b] over the set bits b < 31 of k; table dims x 31 uint32 (< 2^31),
 * out dims x n fp32; grid (ceil(n/1024), dims) */
typedef struct { uint64_t table, out; uint32_t n, dims, seed, pad_; } slate_args_qrng;
/* GS (Rodinia gaussian, forward elimination without pivoting), step t < n-1 of an n x n
 * system: a n x n, m n x n (multipliers, column t written by Fan1), b n; all fp32 row-major.
 * Fan1 grid (ceil((n-1-t)/256)); Fan2 grid (ceil((n-t)/128), ceil((n-1-t)/16)). */
typedef struct { uint64_t a, b, m; uint32_t n, t; } slate_args_gauss;

/* ------------------------------------------------------------------ attach */
/* Open a session ("the daemon creates a session for each application
 * process upon its first Slate API call").
 *   endpoint  NULL -> an in-process server on CUDA device `device` (created on
 *             first use, shared by every in-process session on that device);
 *             otherwise the POSIX shared-memory name of a running `slated`
 *             (e.g. "/slate-gpu0"); `device` is then ignored.
 *   out       receives the session; the caller owns it until slate_detach.
 * Errors: EINVAL (out == NULL, bad device), EIPC (no server answering at the
 * endpoint), ECUDA (context creation / calibration failed). */
slate_status slate_attach(const char* endpoint, int device, slate_session** out);

/* Close a session: waits for all of its outstanding launches (watchdog 60 s),
 * releases its queue's SMs, closes IPC imports, frees the session.
 * Errors: ETIMEDOUT (a launch did not finish; the session is freed anyway). */
slate_status slate_detach(slate_session* s);

typedef struct {
  uint32_t abi_version;
  uint32_t num_sms;          /* N: ranks 0..N-1 (calibrated, see header) */
  uint32_t max_smid;         /* largest %smid observed */
  uint32_t device;
  uint64_t server_pid;       /* 0 in-process */
  double peak_hbm_gbps;      /* peaks the classifier uses (MEASURED_PEAKS.json or defaults) */
  double peak_fp32_gflops;
  double peak_tc_tflops;
} slate_info;
/* Static facts about the server behind a session.  Errors: EINVAL. */
slate_status slate_get_info(slate_session* s, slate_info* out);

/* ------------------------------------------------------------------ buffers */
/* Make client-owned device memory [dev_ptr, dev_ptr+bytes) usable by the
 * server (kernel IO data travels in buffers shared between
 * client and daemon).  Through an endpoint: exports a cudaIpcMemHandle of the
 * allocation, the server opens it once and caches base -> server pointer
 * (the paper's hash table).  In-process: records the range (identity map).
 *   handle  receives an opaque id (for slate_unshare_buffer).
 * Ownership: the CLIENT owns the memory and must keep it alive until every
 * launch that uses it has completed and the buffer is unshared/detached.
 * Through an endpoint the server drops its mapping asynchronously once no
 * session references the allocation: when the device is idle, else within
 * 30 s or once unreferenced mappings exceed 8 GiB (a mapping is never closed
 * on a session's issue path, because closing waits for the device).  CUDA
 * leaves freeing exported memory before every importer closed it undefined:
 * a client that frees a buffer while other tenants keep the server busy
 * relies on the driver's reference to the allocation until then.
 * Errors: EINVAL (null/zero range, not device memory), EIPC. */
slate_status slate_share_buffer(slate_session* s, void* dev_ptr, size_t bytes, uint64_t* handle);
slate_status slate_unshare_buffer(slate_session* s, uint64_t handle);

/* ------------------------------------------------------------------ kernels */
#define SLATE_KFLAG_COVERAGE 1u   /* launches may pass a coverage log (debug) */
/* Rank log (debug; needs SLATE_KFLAG_COVERAGE): the coverage log is then
 * u32[2B], and for every original block b the word cov[B + b] records who
 * took the task holding b, written by the fetching thread when it hands the
 * task out: bits 0-7 the worker's SM rank (for a GEMM CTA pair, the leader's),
 * bits 8-15 / 16-23 the range [lo, hi] of the resize word the worker acted on
 * (as published; a top-up worker is also bound to the ranks it was launched
 * for), bit 24 set if the worker was outside its range and kept the task only
 * because it was the last live worker
 * (reading Q22), bit 31 set (valid).  It makes "the kernel only runs on these
 * SMs" (§IV-C, Lst1) checkable per task. */
#define SLATE_KFLAG_RANKLOG 2u

typedef struct {
  uint32_t abi_version;    /* SLATE_ABI_VERSION */
  uint32_t kind;           /* slate_kind */
  uint32_t iters;          /* SLATE_ITERS, blocks per task; 0 -> auto per launch (reading
                              Q11): min(cap, max(1, B / (t * occ * N))), cap = 10, t = 8;
                              SPMV_CSR cap 32, t = 6; GEMM_BF16 -> 1.  SPMV_CSR accepts
                              iters <= 32 (its task buffer holds 32 blocks' row pointers) */
  uint32_t flags;          /* SLATE_KFLAG_* */
} slate_kernel_desc;

/* Register a kernel kind (the injector's output).  Computes the
 * worker's occupancy (the "maximum number of thread blocks that the
 * designated SMs can support").  Idempotent per
 * (kind, iters, flags): registering twice returns the same handle.
 * Errors: EINVAL (bad abi_version / kind / flags, iters above the kind's
 * maximum), EUNSUPPORTED. */
slate_status slate_register_kernel(slate_session* s, const slate_kernel_desc* d, slate_kernel* out);

/* ------------------------------------------------------------------ launch */
#define SLATE_PLACE_AUTO  0u  /* the selector decides co-run or solo (Tab I) */
#define SLATE_PLACE_SOLO  1u  /* wait for a free GPU, run on all SMs */
#define SLATE_PLACE_CORUN 2u  /* run now on [sm_lo, sm_hi] (resizes this queue's range) */

#define SLATE_MODE_SLATE      0u  /* transformed kernel K*(B*,T): persistent workers */
#define SLATE_MODE_STANDALONE 1u  /* the original K(B,T) on the hardware block
                                     scheduler, same body code (bit-exact reference,
                                     and the "vanilla CUDA" schedule) */

typedef struct {
  uint32_t grid[3];        /* original grid (Gx, Gy, Gz); must equal the grid the
                              kind's args imply (e.g. triad: ceil(n/1024), 1, 1) */
  uint32_t placement;      /* SLATE_PLACE_* */
  uint32_t sm_lo, sm_hi;   /* CORUN: inclusive rank range */
  uint32_t mode;           /* SLATE_MODE_* */
  uint32_t args_size;      /* sizeof the kind's slate_args_* */
  const void* args;        /* copied before the call returns */
  uint64_t coverage;       /* 0, or device u32[Gx*Gy*Gz] zero-filled by the caller:
                              every executed original block b does cov[b] += 1;
                              u32[2*Gx*Gy*Gz] for a kernel with SLATE_KFLAG_RANKLOG */
} slate_launch_desc;

/* Submit one kernel launch, asynchronously (the API "wraps ... launch",
 * P:L139).  Launches of one session run in submission order, one after
 * another (one queue per process); launches of different sessions may
 * run concurrently on disjoint SM ranges.  Returns once the launch is queued
 * (it may already be running).
 *   out  receives the launch id.
 * Ordering: the server runs launches on its own non-blocking streams, which do
 * not wait for the caller's streams: the caller must have finished writing the
 * inputs (and zeroing a coverage log) before the call, and must slate_sync
 * before reading the outputs.
 * Errors: EINVAL (grid inconsistent with args, zero grid, B >= 2^31, a pointer
 * outside every shared buffer through an endpoint, lo > hi, hi >= N),
 * ENOTFOUND (kernel), ENOMEM (control-block pool exhausted), ECUDA. */
slate_status slate_launch(slate_session* s, slate_kernel k, const slate_launch_desc* d, slate_launch_id* out);

/* n (>= 1) launches of the same kernel and descriptor in one call: a job of
 * n back-to-back kernels (the paper's applications loop over their kernels,
 * P:L291).  All n are queued before the selector considers the queue, so a
 * co-run decision and its split see the whole job (reading Q31), and the
 * client pays one round trip to the server instead of n.  The ids
 * are *first .. *first + n - 1.  Errors: as slate_launch; on an error after
 * some launches were queued, those stay queued and *first names the first. */
slate_status slate_launch_n(slate_session* s, slate_kernel k, const slate_launch_desc* d, uint32_t n,
                            slate_launch_id* first);

/* n (>= 1) launches of possibly different kernels and descriptors in one call,
 * in order: ks[i] with ds[i].  A job whose launches differ (e.g. Gaussian
 * elimination, a Fan1 and a Fan2 launch per step with the step in the args,
 * Tab II GS) goes out as one batch: no event between its kernels and
 * programmatic dependent launch, as slate_launch_n.  Stream order between the
 * launches is kept (launch i+1 starts after launch i completed).  ks and ds are
 * caller-owned arrays of n entries, read during the call.  The ids are
 * *first .. *first + n - 1.  Through an endpoint the launches are sent one by
 * one (same ids and order, no batch).  Errors: as slate_launch_n. */
slate_status slate_launch_many(slate_session* s, uint32_t n, const slate_kernel* ks, const slate_launch_desc* ds,
                               slate_launch_id* first);

/* ------------------------------------------------------------------ runtime kernel transformation
 * NEXT-3 (Slate scans a user kernel's source, injects its task
 * loop and compiles it with NVRTC; "a compiled kernel image can be further
 * cached").  `source` holds a CUDA C++ kernel
 *     __global__ void <kernel_name>(<parameters>) { ... blockIdx ... threadIdx ... }
 * with blocks of block_threads x block_y x block_z threads (block_y, block_z:
 * 0 means 1) and `smem_bytes` of dynamic shared memory.  The server renames
 * it into a device function that takes the block index, the original grid,
 * the thread index and the block shape (every blockIdx / gridDim / threadIdx /
 * blockDim token of the source is renamed), generates the slate worker
 * (Lst1/Lst2: SM binding, task counter, decode, resize word) -- a 1-D worker
 * CTA of the same thread count, threads linearised x-fastest as the hardware
 * forms warps -- and an original-kernel wrapper around the same body launched
 * with the real block shape, compiles both for sm_100a with NVRTC and
 * registers the result as a kernel of kind SLATE_KIND_USER.  If the source
 * uses shared memory (a __shared__ declaration or smem_bytes > 0) the worker
 * puts a CTA barrier between the blocks it runs back to back.
 * Compiled images are cached, keyed by a hash of the generated source, the
 * options and the NVRTC version: in process (a second registration, e.g. with
 * another task size, reuses the loaded image) and on disk in
 * $SLATE_RTC_CACHE (default $HOME/.cache/slate-rtc; "off" disables it).
 * Launch it with slate_launch / slate_launch_n: desc.grid is the original grid
 * (any x, y, z), desc.args the parameters packed as a C struct in declaration
 * order (args_size bytes; checked against the compiled struct's size).
 * bytes_per_block / flops_per_block declare its work for slate_profile's
 * classification (0 if unknown).  Through an endpoint the source travels over
 * the command channel and the server rewrites every pointer parameter (a
 * parameter whose type contains '*') to its mapping of the shared buffers.
 * flags: SLATE_KFLAG_COVERAGE / SLATE_KFLAG_RANKLOG as for slate_register_kernel.
 * Errors: EINVAL (no such kernel in the source, bad sizes, args_size not the
 * parameter struct's), EUNSUPPORTED (no NVRTC), ECUDA (compile or load
 * failed; the compiler log is in slate_last_error). */
typedef struct {
  uint32_t abi_version;
  uint32_t block_threads;      /* blockDim.x */
  uint32_t smem_bytes;
  uint32_t args_size;
  uint32_t iters;              /* task size; 0 = automatic */
  uint32_t flags;              /* SLATE_KFLAG_COVERAGE / SLATE_KFLAG_RANKLOG */
  const char* source;
  const char* kernel_name;
  double bytes_per_block, flops_per_block;
  uint32_t block_y, block_z;   /* blockDim.y, blockDim.z (0 = 1) */
} slate_source_desc;
slate_status slate_register_source(slate_session* s, const slate_source_desc* d, slate_kernel* out);
/* The transformed source slate_register_source would compile (no GPU, no
 * NVRTC needed): writes up to cap bytes (NUL-terminated) to out and the full
 * length to *len.  Errors: EINVAL (no such kernel, bad block shape). */
slate_status slate_transform_source(const char* source, const char* kernel_name, uint32_t block_x, uint32_t block_y,
                                    uint32_t block_z, uint32_t smem_bytes, char* out, size_t cap, size_t* len);
/* Counters of this process's compiled-image cache: NVRTC compiles, in-process
 * hits, on-disk hits (any pointer may be NULL). */
void slate_rtc_stats(uint64_t* compiles, uint64_t* mem_hits, uint64_t* disk_hits);

/* NEXT-1, the fused co-run worker (a kernel shrinks when another
 * arrives and "seamlessly claims" the SMs of one that completes
 * the workers' exit conditions).  Launches da (session sa) and db (session
 * sb) as ONE persistent kernel: every CTA holds the uniform shape of the pair
 * and, at each task boundary, works for the tenant whose range (its session's
 * resize word) holds its SM rank -- or for the other one once its own tenant
 * has no task left -- so a resize in either direction and the grow on
 * completion need no launch, no top-up grid and no standby CTA.  B starts on
 * the top sm_b ranks, A on the rest.  Each launch keeps its own id, control
 * block, coverage / rank log, counters and resize-latency stamps: slate_sync,
 * slate_query and slate_resize work on either as on separate launches.
 * Both sessions must be in-process sessions of the same server with no launch
 * queued or running.  Pairs: any two of TRIAD, SGEMM_NAIVE, SGEMM_TILED,
 * BLACKSCHOLES, STENCIL2D, TRANSPOSE (the kinds sharing a 256-thread CTA with
 * no per-CTA state).  *la / *lb receive the two ids.
 * Errors: EINVAL (sm_b outside [1, N-1], bad descriptors, sa == sb's queue),
 * ESTATE (a session busy), EUNSUPPORTED (kind pair, or not in-process),
 * ENOMEM (control blocks), ECUDA. */
slate_status slate_launch_fused(slate_session* sa, slate_kernel ka, const slate_launch_desc* da, slate_session* sb,
                                slate_kernel kb, const slate_launch_desc* db, uint32_t sm_b, slate_launch_id* la,
                                slate_launch_id* lb);

/* Resize the SM range of the queue that owns launch l to [sm_lo, sm_hi]
 * (§III-C; the dispatcher's start_sm/end_sm, Lst3 P:L250-251).
 * Publishes {epoch+1, lo, hi} to the device with a stream memory write that
 * needs no SM; workers outside the range retire at their next task boundary
 * (shrink), and ranks newly in range get workers (grow: waiting CTAs join, plus
 * a top-up launch bound to the new ranks sharing the same task counter).  The
 * running workers are never relaunched; progress is only in the counter.
 * Returns once the write is enqueued; completion is visible in slate_query.
 * Errors: EINVAL (lo > hi, hi >= N), ENOTFOUND.  SLATE_DONE (+1) if l had
 * already completed (the queue's range is still updated). */
slate_status slate_resize(slate_session* s, slate_launch_id l, uint32_t sm_lo, uint32_t sm_hi);

/* Wait until launch l (0 = every launch of this session) has run every block
 * and all its worker CTAs have exited.  timeout_us < 0 waits forever.  A
 * launch id older than the server's retention window (SLATE_KEEP_FINISHED,
 * default 65536 completed launches) has completed: SLATE_OK.
 * The server watchdog: a launch still running SLATE_WATCHDOG_S seconds after
 * its issue (default 120, 0 = off) is reported -- this call returns ECUDA
 * ("watchdog") instead of waiting; the kernel itself cannot be preempted.
 * Errors: ETIMEDOUT, ECUDA (sticky kernel error, watchdog), ENOTFOUND. */
slate_status slate_sync(slate_session* s, slate_launch_id l, int64_t timeout_us);

/* ------------------------------------------------------------------ profile */
#define SLATE_PROF_CURVE 1u  /* also time the kernel on N, 3N/4, N/2, N/3, N/4, N/8 SMs */
#define SLATE_PROF_FORCE 2u  /* ignore the cached entry */

typedef struct {
  double solo_ms;          /* time on all SMs */
  double hbm_gbps;         /* algorithmic bytes / solo time */
  double fp32_gflops;      /* algorithmic fp32 flops / solo time */
  double tc_tflops;        /* algorithmic tensor-core flops / solo time */
  double hbm_frac, fp32_frac, tc_frac;   /* of the server's peaks (slate_info) */
  uint32_t c_level, m_level;             /* 0 = L, 1 = M, 2 = H (reading Q9) */
  uint32_t category;       /* 0 L_C, 1 M_C, 2 H_C, 3 M_M, 4 H_M (Tab I order) */
  uint32_t n_curve;        /* points in curve_* */
  uint32_t curve_sms[8];
  double curve_ms[8];
  double bytes, flops;     /* algorithmic bytes and flops of the sample launch */
} slate_profile_t;

/* Profile a kernel solo on a sample launch ("The daemon profiles
 * kernels at their first time run, and saves the profile data in the kernel
 * profile table").  Runs the sample through the worker on all SMs (and on
 * fewer SMs with SLATE_PROF_CURVE), times it with CUDA events, and classifies
 * it; the entry is cached per (kind, shape) and used by SLATE_PLACE_AUTO.
 * The sample launch's outputs are written (the kernel really runs).
 * Requires an idle GPU for this session's server (waits for it).
 * Errors: EINVAL, ECUDA, ENOTFOUND. */
slate_status slate_profile(slate_session* s, slate_kernel k, const slate_launch_desc* sample,
                           uint32_t flags, slate_profile_t* out);

/* ------------------------------------------------------------------ query */
typedef struct {
  uint32_t state;          /* 0 queued, 1 issued, 2 complete */
  uint32_t blocks_done;    /* original blocks executed (== B when complete) */
  uint32_t tasks_done;     /* tasks executed (== ceil(B/iters)) */
  uint32_t total_blocks;   /* B */
  uint32_t next_clamped;   /* min(slateIdx, ceil(B/iters)*iters) */
  uint32_t next_raw;       /* raw slateIdx (overshoots; nondeterministic) */
  uint32_t live_workers;   /* worker CTAs (or warps) still live */
  uint32_t iters;
  uint32_t sm_lo, sm_hi;   /* the queue's current range */
  uint32_t n_resizes;      /* resizes applied while the launch ran */
  uint32_t n_topups;       /* top-up worker launches (grow) */
  uint32_t workers_started;/* worker CTAs/warps that ran at least one prologue */
  uint32_t coverage_ok;    /* 1 if a coverage log was given and every entry is 1 */
  uint32_t epoch;          /* the queue's resize-word epoch now */
  uint32_t shrink_epoch;   /* last epoch whose shrink the device saw complete */
  uint32_t join_epoch;     /* last epoch in which a worker joined (grow) */
  uint32_t pad_;
  uint64_t t_first_ns;     /* %globaltimer at the first task start (device clock) */
  uint64_t t_last_ns;      /* %globaltimer when the last block finished */
  double start_ms, end_ms; /* CUDA-event times of the launch relative to the server's epoch */
  double resize_us[16];    /* latency of the first 16 resizes applied while the launch ran
                              (reading Q30: from the slate_resize call to, for a shrink, the
                              last worker retiring outside the range, for a grow, the first
                              worker joining on a new rank; device clock mapped to the host
                              clock); -1 if not observed (e.g. the launch ended first) */
  uint8_t resize_kind[16]; /* 1 shrink, 2 grow, 0 none, for each resize_us entry */
  uint64_t t_enter_ns;     /* %globaltimer when the first worker CTA started (device clock; 0 if standalone) */
  uint64_t t_exit_ns;      /* %globaltimer when the last worker CTA that ran a task exited (0 unless the
                              library is built with SLATE_DIAG_EXIT) */
  uint32_t n_superseded;   /* resizes with no completion to time: shrinks overtaken by a grow before
                              they completed, grows of a queue with no block left to run */
  uint32_t pad2_;
} slate_launch_info;

/* Counters and timing of a launch (copied out).  Errors: ENOTFOUND. */
slate_status slate_query(slate_session* s, slate_launch_id l, slate_launch_info* out);

/* ------------------------------------------------------------------ server */
/* Run a Slate server for CUDA device `device` on the calling thread (the body
 * of the `slated` daemon): creates the single CUDA context every client's
 * kernels run in, publishes the POSIX shared-memory endpoint (e.g.
 * "/slate-gpu0"; replaced if stale), gives every attaching client session its
 * own server thread and queue, and returns after SIGINT/SIGTERM, when
 * it unlinks the endpoint.  flags: reserved, 0.
 * Errors: EINVAL (endpoint must start with '/'), ECUDA (no usable device),
 * EIPC (shared memory could not be created). */
slate_status slate_serve(const char* endpoint, int device, uint32_t flags);

/* ------------------------------------------------------------------ strings */
const char* slate_status_string(slate_status st);     /* static string */
const char* slate_last_error(slate_session* s);       /* session-owned, valid until the next call */

/* The block geometry of a kind (what one original block of K(B,T) owns):
 * elements per block for 1-D kinds (tile_m = 1), else the output tile rows x
 * columns (sgemm 16 x 16, stencil 8 x 32, gemm 128 x tile_n of this build).
 * Returns SLATE_EINVAL for an unknown kind.  No GPU needed. */
slate_status slate_kind_geometry(uint32_t kind, uint32_t* tile_m, uint32_t* tile_n);

/* ------------------------------------------------------------------ host logic
 * The selector's pure functions, exported so they can be checked without a GPU.
 * Categories: 0 L_C, 1 M_C, 2 H_C, 3 M_M, 4 H_M. */
/* Classify fractions of peak (reading Q9). Returns the category;
 * *c_level and *m_level receive 0 = L, 1 = M, 2 = H (may be NULL). */
uint32_t slate_classify(double hbm_frac, double fp32_frac, double tc_frac, uint32_t* c_level, uint32_t* m_level);
/* Tab I: 1 = corun, 0 = solo.  literal != 0 uses the table as
 * printed, otherwise the symmetric reading (Q8). */
int slate_policy(uint32_t cat_active, uint32_t cat_candidate, int literal);
/* Selection algorithm (reading Q13): index of the first queued
 * candidate to co-run with the active kernel, or -1 for solo.  bypassed may
 * be NULL. */
int slate_select(uint32_t cat_active, const uint32_t* queue_cats, const uint32_t* bypassed, uint32_t n,
                 uint32_t max_bypass, int literal);
/* SM split for a co-run (reading Q10): SMs for candidate B (A keeps n - s),
 * minimising the fluid-model makespan with grow-on-completion, given solo
 * time curves (sms ascending, ms).  s ranges over the multiples of step in
 * [step, n_sms - step], further limited to [lo_b, hi_b] where those are
 * non-zero (reading Q29; if that leaves nothing, the bound nearest the range
 * is used).  Returns s and the predicted makespan in *makespan_ms (may be
 * NULL). */
uint32_t slate_choose_split(const uint32_t* sms_a, const double* ms_a, uint32_t n_a,
                            const uint32_t* sms_b, const double* ms_b, uint32_t n_b,
                            uint32_t n_sms, uint32_t step, uint32_t lo_b, uint32_t hi_b,
                            double* makespan_ms);
/* The split objective (reading Q41).  MAKESPAN: slate_choose_split's.  ANTT:
 * among the splits whose fluid-model makespan is within `slack` (e.g. 0.05) of
 * the best, the one with the least ANTT = mean over the two jobs of co-run
 * completion / solo time on all SMs (Eyerman; a makespan-only split can double
 * the shorter job's turnaround).  *makespan_ms and *antt (may be NULL) receive
 * the chosen split's predictions. */
#define SLATE_SPLIT_MAKESPAN 0u
#define SLATE_SPLIT_ANTT     1u
uint32_t slate_choose_split_obj(const uint32_t* sms_a, const double* ms_a, uint32_t n_a,
                                const uint32_t* sms_b, const double* ms_b, uint32_t n_b,
                                uint32_t n_sms, uint32_t step, uint32_t lo_b, uint32_t hi_b,
                                uint32_t objective, double slack, double* makespan_ms, double* antt);
/* Reading Q29 (bandwidth saturation cap): the fewest SMs (1..n_sms) on which
 * a solo curve (sms ascending, ms) comes within frac (0 < frac <= 1) of its
 * full-chip rate: interp(s) <= interp(n_sms) / frac.  The scheduler caps a
 * memory-bound co-runner at saturation_sms(curve, f), f = SLATE_SATURATION_FRAC
 * in the server's environment (default 0.95, 1.0 = no cap): past that point it
 * gains little bandwidth but raises the HBM latency its compute-bound partner
 * sees. */
uint32_t slate_saturation_sms(const uint32_t* sms, const double* ms, uint32_t n, uint32_t n_sms, double frac);
/* NEXT-4, the task size from a solo profile: a
 * worker's time per block is t = solo_ms * occ * n_sms / B; the task takes
 * floor(budget_us / t) blocks, at most floor(B / (2 occ n_sms)) (every worker
 * gets two tasks), clamped to [1, cap].  The server uses it for launches of
 * kernels registered with iters 0 once their shape has been profiled. */
uint32_t slate_choose_iters(double solo_ms, uint32_t occ, uint32_t n_sms, uint32_t B, uint32_t cap, double budget_us);
/* NEXT-4, k co-runners: the fluid-model makespan of k jobs (curve i: npts[i]
 * points sms[i][*] -> ms[i][*], job times) on disjoint shares, a finishing
 * job's SMs going to the unfinished one with the most time left; and the
 * shares (multiples of step, each >= step, summing to n_sms) minimising it,
 * by exhaustive search (returns the makespan, -1 if n_sms / step < k).  Pure
 * functions for the selector and its tests; the server co-runs at most two
 * queues (Q13, Q37). */
double slate_corun_makespan_k(const uint32_t* const* sms, const double* const* ms, const uint32_t* npts, uint32_t k,
                              const uint32_t* shares);
double slate_choose_split_k(const uint32_t* const* sms, const double* const* ms, const uint32_t* npts, uint32_t k,
                            uint32_t n_sms, uint32_t step, uint32_t* shares_out);
/* NEXT-4 / reading Q49 ("examines other kernels in the queue"): should
 * a candidate job (curve k, category cats[k]) join a co-running group of k
 * jobs (curves 0..k-1 on shares_cur)?  Only if the group keeps at most one
 * memory-intensive job (categories 3, 4; reading Q37) and the fluid model
 * predicts gain = (slate_corun_makespan_k(group, shares_cur) + T_k(n_sms)) /
 * the best (k+1)-way makespan >= min_gain.  shares_out (k+1 entries) receives
 * the best shares, *gain the prediction.  Returns 1 to admit.  The server
 * admits a third co-runner this way (SLATE_MAX_CORUN, default 3). */
int slate_kway_admit(const uint32_t* const* sms, const double* const* ms, const uint32_t* npts, const uint32_t* cats,
                     uint32_t k, const uint32_t* shares_cur, uint32_t n_sms, uint32_t step, double min_gain,
                     uint32_t* shares_out, double* gain);
/* Reading Q31 (the B200 selector): should kernel B co-run with the active A
 * although Tab I says solo?  Job curves are `work` launches of each kernel
 * (the launches queued or running) back to back, time = work * curve(s); the
 * split is slate_choose_split over the job curves and the predicted gain is
 * (T_A(n) + T_B(n)) / makespan(split).  Returns 1 iff gain >= min_gain;
 * *split and *gain (may be NULL) receive the split and the gain. */
int slate_fluid_corun(const uint32_t* sms_a, const double* ms_a, uint32_t n_a, double work_a,
                      const uint32_t* sms_b, const double* ms_b, uint32_t n_b, double work_b,
                      uint32_t n_sms, uint32_t step, uint32_t lo_b, uint32_t hi_b, double min_gain,
                      uint32_t* split, double* gain);

/* slate_fluid_corun with the split taken under `objective` / `slack`
 * (slate_choose_split_obj); the gain is T_seq over that split's makespan. */
int slate_fluid_corun_obj(const uint32_t* sms_a, const double* ms_a, uint32_t n_a, double work_a,
                          const uint32_t* sms_b, const double* ms_b, uint32_t n_b, double work_b,
                          uint32_t n_sms, uint32_t step, uint32_t lo_b, uint32_t hi_b, double min_gain,
                          uint32_t objective, double slack, uint32_t* split, double* gain);

/* The split objective of the server's co-runs (process-wide; initial value
 * from SLATE_SPLIT_OBJECTIVE = makespan | antt and SLATE_SPLIT_SLACK in the
 * server's environment, default makespan; slack 0.05).  Errors: EINVAL. */
slate_status slate_set_split_objective(slate_session* s, uint32_t objective, double slack);

/* Selector policy of the server (process-wide; the initial value comes from
 * SLATE_POLICY = table | literal | hybrid in the server's environment, default
 * hybrid).  TABLE: Tab I, symmetric reading (Q8); LITERAL: Tab I as printed;
 * HYBRID: Tab I, and where it says solo the fluid model over the measured
 * solo curves and the queued work (slate_fluid_corun, gain >= 1.05) may still
 * co-run the pair (Q31).  In every policy a co-running pair's split is re-taken
 * from the job curves as launches arrive (resizing both queues).
 * Errors: EINVAL (unknown policy). */
#define SLATE_POLICY_TABLE   0u
#define SLATE_POLICY_LITERAL 1u
#define SLATE_POLICY_HYBRID  2u
slate_status slate_set_policy(slate_session* s, uint32_t policy);

#ifdef __cplusplus
}
#endif
#endif /* SLATE_H */
