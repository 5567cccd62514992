/* hpl.h — C ABI of the B200-native NPB-EP hot path (libhpl.so).
 *
 * What this library is.  The paper (Bozkus & Fraguela, "A Portable
 * High-Productivity Approach to Program Heterogeneous Systems", IPDPSW'12)
 * evaluates HPL — a C++ library whose `Array<T,N>` objects track host and
 * device copies and whose `eval(f)` runs a
 * kernel over an index domain — on the NAS EP
 * benchmark.  This header is the boundary of the
 * B200 re-design of that hot path: an `Array` coherence layer and a fixed
 * `eval` of EP, implemented by hand-written sm_100a CUDA kernels.
 *
 * Conventions (all functions):
 *   - extern "C", plain pointers and integers, no C++ or torch types;
 *   - return an int status (HPL_OK = 0 or a negative HPL_E* code); they never
 *     throw, abort or exit across the ABI; hpl_last_error() gives detail;
 *   - outputs are written only when HPL_OK is returned;
 *   - "device" means the CUDA device current on the calling thread unless a
 *     device argument says otherwise ("by default the kernel
 *     is evaluated in the first device found in the system that is not a
 *     standard general-purpose CPU" — here: the current CUDA device);
 *   - `stream` arguments are cudaStream_t values passed as void* (NULL = the
 *     legacy default stream), e.g. torch.cuda.current_stream().cuda_stream.
 *
 * EP stream convention (NPB ep.f/randdp.f, the paper's reference [16],
 * PAPER.md:1322-1323; readings R1-R10):
 *   x_0 = seed, x_{k+1} = a * x_k mod 2^46, uniform u_j = x_{j+1} * 2^-46,
 *   pair i = (u_{2i}, u_{2i+1}), x1 = 2u_{2i} - 1, x2 = 2u_{2i+1} - 1,
 *   t = RN(RN(x1*x1) + RN(x2*x2)); accepted iff t <= 1;
 *   X = x1*sqrt(-2 ln t / t), Y = x2*sqrt(-2 ln t / t);
 *   l = trunc(max(|X|,|Y|)), q[l] += 1, sx += X, sy += Y.
 * Valid parameters: 0 <= M <= 43 (the stream period is 2^44 uniforms),
 * seed < 2^46 and seed != 2^45, a odd and 1 <= a < 2^46 (reading R9).
 */
#ifndef HPL_H_
#define HPL_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes ------------------------------------------------------ */
#define HPL_OK 0
#define HPL_EINVAL (-1)  /* bad argument                                    */
#define HPL_ENOMEM (-2)  /* host or device allocation failed                */
#define HPL_ECUDA (-3)   /* CUDA runtime error; detail in hpl_last_error()  */
#define HPL_ENODEV (-4)  /* no CUDA device / device is not sm_100           */
#define HPL_ERANGE (-5)  /* an annulus index l >= 10 occurred; result withheld */
#define HPL_ESTATE (-6)  /* coherence misuse (e.g. data() of an invalid copy) */

/* Static string for a status code (never NULL). */
const char* hpl_strerror(int code);
/* Thread-local detail of the last failing call on this thread ("" if none);
 * valid until the next hpl_* call on the same thread. */
const char* hpl_last_error(void);
/* Library ABI version: (major << 16) | minor. */
int hpl_version(void);

/* ---- device memory and library state ----------------------------------
 * Device memory the library allocates for the caller (hpl_array device
 * copies, the temporary buffers of the test hooks) comes from cudaMalloc
 * unless an allocator is installed: alloc(bytes, device, ctx) returns device
 * memory on `device` (NULL = out of memory, reported as HPL_ENOMEM) and
 * free(ptr, bytes, device, ctx) releases it.  The Python binding installs
 * torch's caching allocator, so arrays share the pool of the caller's tensors
 * (reading B1).  An array is always freed with the
 * allocator that allocated it.  alloc and free must both be NULL (restore
 * cudaMalloc) or both non-NULL.  Internal per-device state (the EP log table,
 * reduction workspaces) stays on cudaMalloc and is released by hpl_shutdown. */
typedef void* (*hpl_alloc_fn)(size_t bytes, int device, void* ctx);
typedef void (*hpl_free_fn)(void* ptr, size_t bytes, int device, void* ctx);
int hpl_set_device_allocator(hpl_alloc_fn alloc, hpl_free_fn free_fn, void* ctx);
/* Release every library-owned buffer: the calling thread's hpl_ep_run result
 * arrays (other threads' are freed at their exit), the EP log tables and
 * workspaces and the reduction workspaces of every device (each synchronised
 * first), and restore the cudaMalloc allocator.  Call with no library work
 * pending; the next call re-creates what it needs. */
int hpl_shutdown(void);

/* ---- devices ----------------------------------------------------------- */
int hpl_device_count(int* n);
/* Make `device` current for this thread's subsequent hpl_* calls.  Multi-GPU
 * callers (one process per GPU) call this with their local rank. */
int hpl_set_device(int device);
int hpl_get_device(int* device);

/* ---- Array<T, ndim>: host/device coherence ----------
 * An hpl_array owns (or borrows) a host copy and owns a device copy of an
 * ndim-dimensional dense row-major array (ndim 0 = scalar, PAPER.md:361-364;
 * ndim <= 3 like the paper's index domains).  Two valid bits record which
 * copies are current; hpl_array_sync() copies only when the requested copy
 * is stale (the paper's transfer minimisation, PAPER.md:1064-1069,
 * 1174-1178).  Kernels launched through this library mark their output
 * arrays device-valid / host-stale. */
typedef struct hpl_array_s* hpl_array;
typedef enum { HPL_F64 = 0, HPL_F32 = 1, HPL_U64 = 2, HPL_I64 = 3, HPL_I32 = 4, HPL_U32 = 5 } hpl_dtype;
typedef enum { HPL_HOST = 1, HPL_DEVICE = 2 } hpl_where;
typedef enum { HPL_READ = 1, HPL_WRITE = 2, HPL_READWRITE = 3 } hpl_access;

/* Allocate an array of dims[0..ndim-1] elements of type t on `device`
 * (-1 = current).  host_ptr == NULL: the library allocates a pinned host
 * buffer and frees it in hpl_array_free; both copies start valid (contents
 * undefined).  host_ptr != NULL: the caller owns that storage, which must
 * hold the array and outlive it; the host copy starts
 * valid and the device copy stale.  Errors: EINVAL (ndim not in 0..3, a dim
 * <= 0, bad dtype, out == NULL), ENOMEM, ECUDA. */
int hpl_array_alloc(hpl_array* out, hpl_dtype t, int ndim, const int64_t* dims, void* host_ptr,
                    int device);
/* Free the array's device copy and any library-owned host copy.  Pending
 * work on the array's stream is synchronised first.  NULL is a no-op. */
int hpl_array_free(hpl_array a);
/* Make the copy at `where` valid, copying from the other copy only if stale.
 * mode WRITE or READWRITE additionally invalidates the other copy (the
 * caller announces it will modify this one).  HOST syncs block until the
 * data is on the host; DEVICE syncs are stream-ordered on the array stream. */
int hpl_array_sync(hpl_array a, hpl_where where, hpl_access mode);
/* Raw pointer to the copy at `where` (the paper's data());
 * no synchronisation and no validity change. */
int hpl_array_data(hpl_array a, hpl_where where, void** ptr);
/* Shape/state query; any output pointer may be NULL.  dims receives ndim
 * entries.  valid receives a bitmask of HPL_HOST | HPL_DEVICE. */
int hpl_array_info(hpl_array a, hpl_dtype* t, int* ndim, int64_t* dims, int64_t* nbytes,
                   int* valid);
/* Stream used for this array's transfers and for kernels that write it
 * (NULL = legacy default stream).  The stream must outlive its use. */
int hpl_array_set_stream(hpl_array a, void* stream);

/* ---- EP: the hot path ----------------------------------------------------
 * Result layout ("13 words", float64, as exchanged by the multi-GPU
 * allreduce): [0] sx, [1] sy, [2..11] q[0..9], [12] gc = sum q.  Counts are
 * exact integers (< 2^53).  If an annulus index l >= 10 occurred (P ~ 1e-22
 * per pair, never for classes S..E) word [0] is set to NaN and blocking calls
 * return HPL_ERANGE. */

/* eval(EP) over the 1-D index domain of pairs of shard `rank` of `nranks`
 * (pairs [rank*2^M/nranks, (rank+1)*2^M/nranks)) into `out13`, an HPL_F64
 * array with exactly 13 elements, which becomes device-valid/host-stale.
 * Asynchronous on out13's stream.  nranks must be a power of two <= 2^M. */
int hpl_ep_eval(int M, uint64_t seed, uint64_t a, int rank, int nranks, hpl_array out13);

/* Whole EP problem of 2^M pairs on the current device; blocking.
 * sx, sy, q[10] receive the result (gc = sum q). */
int hpl_ep_run(int M, uint64_t seed, uint64_t a, double* sx, double* sy, uint64_t q[10]);

/* One multi-GPU shard: writes the 13-word partial of pairs
 * [rank*2^M/nranks, (rank+1)*2^M/nranks) to the caller-owned device buffer
 * dev_out13 (13 doubles, e.g. a torch tensor), asynchronously on `stream`.
 * The caller combines shards with one allreduce(SUM). */
int hpl_ep_run_shard(int M, uint64_t seed, uint64_t a, int rank, int nranks, double* dev_out13,
                     void* stream);

/* EP over an arbitrary pair range [pair_begin, pair_begin + npairs) of the
 * stream (npairs may be 0; pair_begin + npairs <= 2^43).  Asynchronous on
 * `stream`; writes 13 doubles to dev_out13. */
int hpl_ep_run_range(uint64_t seed, uint64_t a, uint64_t pair_begin, uint64_t npairs,
                     double* dev_out13, void* stream);

/* Test hook: the LCG states x_{offset+1} .. x_{offset+n} (u64 < 2^46),
 * computed on the device by the same skip-ahead and step code the EP kernel
 * uses (its skip-ahead and the hot loop's step function), copied to
 * host_out[0..n-1].  Blocking.  n <= 2^28. */
int hpl_lcg_states(uint64_t seed, uint64_t a, uint64_t offset, uint64_t n, uint64_t* host_out);

/* ---- fused cross-GPU combine ----------------------------
 * EP's only exchange step is the sum of the ranks' 13-word partials
 * (PAPER.md:1264-1270 names multi-node/multi-GPU as the next step; SURVEY
 * §8(e)).  Instead of a separate allreduce, hpl_ep_run_fused's kernel does
 * it itself: its last block stores the shard's partial into slot [rank] of
 * every rank's inbox (device memory of that rank's GPU, mapped into this
 * process with CUDA IPC; peer stores over NVLink), then a tag word holding
 * the call's epoch with a system-scope release; it waits (acquire) until
 * every slot of its own inbox carries this call's epoch, sums the nranks
 * partials in rank order into dev_out13 and re-checks the tags (a peer that
 * gave up waiting and moved on would have changed them: the call then
 * reports failure instead of mixing calls).  Every rank therefore ends with
 * the same, bitwise reproducible result.
 * Setup, one process per GPU (or several processes sharing one GPU):
 *   1. hpl_comm_create(&c, rank, nranks, device, handle) on every rank;
 *   2. exchange the HPL_COMM_HANDLE_BYTES handles (e.g. an all_gather over
 *      torch.distributed) into `handles` (nranks * 64 bytes, rank order);
 *   3. hpl_comm_open(c, handles).
 * All ranks must then issue the same sequence of hpl_ep_run_fused calls
 * (same M, seed, a).  Ownership: the comm owns its inbox and mappings;
 * hpl_comm_free releases them (after the caller's streams are idle). */
#define HPL_COMM_HANDLE_BYTES 64
#define HPL_COMM_MAX_RANKS 8
typedef struct hpl_comm_s* hpl_comm;
/* nranks a power of two in [1, 8] (equal shards), 0 <= rank < nranks;
 * device -1 = current.  Writes the
 * 64-byte IPC handle of this rank's inbox to handle_out. */
int hpl_comm_create(hpl_comm* out, int rank, int nranks, int device, void* handle_out);
/* Map the peers' inboxes (handles in rank order; this rank's own entry is
 * ignored).  HPL_ESTATE if already open, HPL_ECUDA if a mapping fails. */
int hpl_comm_open(hpl_comm c, const void* handles);
/* Wait limit of the in-kernel combine (default 10 s).  A call that times out
 * writes NaN to word 0 and is counted in hpl_comm_status. */
int hpl_comm_set_timeout(hpl_comm c, double seconds);
int hpl_comm_free(hpl_comm c);
/* EP shard c.rank of c.nranks (pairs [rank 2^M/n, (rank+1) 2^M/n)) with the
 * in-kernel combine: dev_out13 (13 doubles on c's device) receives the WHOLE
 * problem's result on every rank.  Asynchronous on `stream`. */
int hpl_ep_run_fused(hpl_comm c, int M, uint64_t seed, uint64_t a, double* dev_out13, void* stream);
/* Synchronize `stream`; report the number of fused calls issued (epoch) and
 * of calls whose combine failed (timed out waiting for a peer, or saw a
 * peer's slot change during the fold; word 0 of those results is NaN).
 * Returns HPL_ECUDA if any failed. */
int hpl_comm_status(hpl_comm c, void* stream, uint64_t* epoch, uint64_t* timeouts);

/* ---- reduction -----------------------------------------
 * The paper's fifth benchmark, "the addition of 16M single-precision floating
 * point values" (SHOC): *dev_out =
 * sum(dev_in[0..n-1]) accumulated in FP64 (deterministic order), written as
 * one double into device memory, asynchronously on `stream`.  dev_in needs
 * only 4-byte alignment; n may be 0 (result 0).  Also registered for
 * hpl_eval as "sum_f32" (in:F32:r, out:F64:w). */
int hpl_reduce_sum_f32(const float* dev_in, int64_t n, double* dev_out, void* stream);

/* ---- matrix transpose -----------------------------------
 * The paper's transpose benchmark, "the transposition of a 16K x 16K matrix"
 * (AMD APP SDK; blocked through local
 * memory; Fig. 10(b) dest[idy][idx] = src[idx][idy],
 * PAPER.md:1132-1138): dev_dst[j*h + i] = dev_src[i*w + j] for i < h, j < w,
 * i.e. src is h x w and dst is w x h, both row-major float32 in device memory
 * of the current device; asynchronous on `stream`.  Both pointers 4-byte
 * aligned (16-byte aligned src with w % 4 == 0 takes the vector path); the
 * ranges must not overlap (EINVAL: no in-place transpose); h * w == 0 is a
 * no-op.  Bit-exact (data movement only).  Also registered for hpl_eval as
 * "transpose_f32" (dest:F32:w, src:F32:r) over dest's 2-D domain
 * (global = {w, h}); the local domain is not used (64 x 64 tiles). */
int hpl_transpose_f32(const float* dev_src, int64_t h, int64_t w, float* dev_dst, void* stream);

/* ---- generic eval over an index domain ----------------
 * The paper's eval(f).global(..).local(..)(args) for
 * hand-written CUDA kernels registered in the library (HPL captures C++
 * kernels at run time; here they are compiled ahead of time).
 * A global domain has 1..3 dimensions; a local domain must have the same
 * dimensionality and divide it in every dimension.  Each
 * point runs one kernel instance with global id (idx, idy, idz), local id
 * (lidx, ...) and group id (gidx, ...).  Scalars are passed
 * by value, arrays by reference. */
typedef enum { HPL_ARG_ARRAY = 0, HPL_ARG_F64 = 1, HPL_ARG_F32 = 2, HPL_ARG_I64 = 3, HPL_ARG_I32 = 4 } hpl_arg_kind;
typedef struct {
  int kind;         /* hpl_arg_kind */
  int access;       /* arrays: hpl_access the kernel needs (0 = the kernel's declared mode) */
  hpl_array array;  /* HPL_ARG_ARRAY */
  double f64;       /* HPL_ARG_F64 */
  float f32;        /* HPL_ARG_F32 */
  int64_t i64;      /* HPL_ARG_I64 */
  int32_t i32;      /* HPL_ARG_I32 */
} hpl_arg;

/* Evaluate registered kernel `name`.  global == NULL (or ndim == 0): the
 * global domain is the dimensions of the first argument, which must be an
 * array.  local == NULL or all zeros: the library chooses
 * (PAPER.md:436-437).  Before the launch every array argument read by the
 * kernel is made device-valid (copied only if stale); after it, every array
 * the kernel writes becomes device-valid / host-stale (the paper's automatic
 * transfers).  Launches on the first array argument's
 * stream and device; asynchronous.  Errors: EINVAL (unknown kernel, argument
 * count/kind/dtype mismatch, local not dividing global, domain too large),
 * ESTATE (an array read by the kernel has no valid copy), ECUDA. */
int hpl_eval(const char* name, int ndim, const int64_t* global, const int64_t* local, int nargs,
             const hpl_arg* args);
/* Registered kernels: count, and name/signature of kernel i (static strings).
 * Signature: comma-separated "name:TYPE:mode" for arrays (mode r, w, rw) and
 * "name:type" for scalars. */
int hpl_kernel_count(int* n);
int hpl_kernel_info(int i, const char** name, const char** signature);

/* Test hook: pairs [pair_begin, pair_begin + n) through the production lean
 * transform code (gen_stage / transform_stage), one pair per thread; writes
 * host_out[4i..4i+3] = {t, X, Y, l} with l = -1 for pairs taken by the rare
 * path (X, Y still filled) and -2 for rejected pairs.  Blocking; n <= 2^26. */
int hpl_ep_pairs_debug(uint64_t seed, uint64_t a, uint64_t pair_begin, uint64_t n, double* host_out);

/* ---- tuning / introspection ------------------------------------------- */
#define HPL_EP_LEAN 0      /* table log + rsqrt-Newton transform (default)   */
#define HPL_EP_LIBDEVICE 1 /* CUDA libdevice log / div / sqrt, as NPB writes it */
/* Select the kernel variant and launch shape for subsequent EP calls on this
 * thread (threads_per_block 0 / blocks_per_sm 0 = library default). */
int hpl_ep_set_config(int variant, int threads_per_block, int blocks_per_sm);
/* Launch shape the library would use for npairs pairs on the current device:
 * blocks, threads per block, dynamic shared-memory bytes. */
int hpl_ep_launch_shape(uint64_t npairs, int* blocks, int* threads, int* smem_bytes);
/* Number of EP kernel launches issued by this process so far (bench.py's
 * gpu_launches evidence). */
int hpl_ep_launch_count(uint64_t* count);

#ifdef __cplusplus
}
#endif
#endif /* HPL_H_ */
