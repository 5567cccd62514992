// hpl_runtime.cpp — the C ABI declared in include/hpl.h: error plumbing,
// devices, the Array coherence layer (PAPER.md:331-381, 1064-1069,
// 1174-1178) and the EP entry points (argument validation, sharding,
// result delivery).  All compute runs in ep_kernel.cu; nothing here computes
// any step of EP on the host.
#include <cuda_runtime.h>

#include <cstdarg>
#include <cstdio>
#include <cstddef>
#include <cstring>
#include <deque>
#include <mutex>
#include <new>
#include <vector>
#include <string>

#include "../../include/hpl.h"
#include "ep_launch.h"
#include "eval_launch.h"
#include "reduce_launch.h"

namespace hplep {

namespace {
thread_local std::string t_err;
thread_local EPConfig t_cfg;
}  // namespace

int set_error(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  t_err = buf;
  return code;
}

int set_cuda_error(cudaError_t e, const char* what) {
  cudaGetLastError();  // clear a non-sticky error
  if (e == cudaErrorNoDevice || e == cudaErrorInsufficientDriver)
    return set_error(HPL_ENODEV, "%s: %s", what, cudaGetErrorString(e));
  if (e == cudaErrorMemoryAllocation) return set_error(HPL_ENOMEM, "%s: %s", what, cudaGetErrorString(e));
  return set_error(HPL_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

static int current_device(int* dev) {
  cudaError_t e = cudaGetDevice(dev);
  if (e != cudaSuccess) return set_cuda_error(e, "cudaGetDevice");
  return 0;
}

// reading R9: odd a < 2^46, seed < 2^46, seed != 2^45 (the fixed point that
// would give t = 0); M <= 43 because the stream period is 2^44 uniforms.
static int validate(uint64_t seed, uint64_t a) {
  if (seed >> 46) return set_error(HPL_EINVAL, "seed must be < 2^46");
  if (seed == (uint64_t(1) << 45)) return set_error(HPL_EINVAL, "seed = 2^45 is a fixed point (x1 = x2 = 0, log 0)");
  if ((a >> 46) || (a & 1) == 0) return set_error(HPL_EINVAL, "a must be odd and < 2^46");
  return 0;
}

static int shard_range(int M, int rank, int nranks, uint64_t* begin, uint64_t* n) {
  if (M < 0 || M > 43) return set_error(HPL_EINVAL, "M must be in [0, 43] (period 2^44)");
  if (nranks < 1 || (nranks & (nranks - 1)) || uint64_t(nranks) > (uint64_t(1) << M))
    return set_error(HPL_EINVAL, "nranks must be a power of two <= 2^M");
  if (rank < 0 || rank >= nranks) return set_error(HPL_EINVAL, "rank out of range");
  *n = (uint64_t(1) << M) / uint64_t(nranks);
  *begin = uint64_t(rank) * (*n);
  return 0;
}

}  // namespace hplep

using namespace hplep;

// ---- device allocator (SURVEY §8(b) "memory ownership"): cudaMalloc unless a
// caller installs one, e.g. the Python binding installs torch's caching
// allocator (torch.cuda.caching_allocator_alloc/delete), so arrays draw from
// the same pool as the caller's tensors without a synchronous cudaMalloc.
namespace {
std::mutex g_alloc_mu;
hpl_alloc_fn g_alloc = nullptr;
hpl_free_fn g_free = nullptr;
void* g_alloc_ctx = nullptr;

struct DevAlloc {
  hpl_free_fn free = nullptr;  // nullptr: cudaFree
  void* ctx = nullptr;
};

int dev_alloc(void** p, size_t bytes, int device, DevAlloc* how) {
  hpl_alloc_fn a;
  {
    std::lock_guard<std::mutex> lk(g_alloc_mu);
    a = g_alloc;
    how->free = g_free;
    how->ctx = g_alloc_ctx;
  }
  if (a) {
    *p = a(bytes, device, how->ctx);
    if (!*p) return set_error(HPL_ENOMEM, "device allocator returned NULL for %zu bytes", bytes);
    return 0;
  }
  how->free = nullptr;
  cudaError_t e = cudaMalloc(p, bytes);
  if (e != cudaSuccess) return set_cuda_error(e, "cudaMalloc");
  return 0;
}

cudaError_t dev_free(void* p, size_t bytes, int device, const DevAlloc& how) {
  if (!p) return cudaSuccess;
  if (how.free) {
    how.free(p, bytes, device, how.ctx);
    return cudaSuccess;
  }
  return cudaFree(p);
}
}  // namespace

struct hpl_array_s {
  hpl_dtype t;
  int ndim;
  int64_t dims[3];
  int64_t count;
  size_t nbytes;
  void* host;
  bool host_owned;
  void* dev;
  int device;
  cudaStream_t stream;
  int valid;
  DevAlloc how;  // how the device copy was allocated (freed the same way)
};

static size_t dtype_size(int t) {
  switch (t) {
    case HPL_F64: case HPL_U64: case HPL_I64: return 8;
    case HPL_F32: case HPL_I32: case HPL_U32: return 4;
    default: return 0;
  }
}

namespace {
struct DeviceGuard {  // make `dev` current for the scope, restore afterwards
  int prev = -1;
  int rc = 0;
  explicit DeviceGuard(int dev) {
    cudaError_t e = cudaGetDevice(&prev);
    if (e == cudaSuccess && prev != dev) e = cudaSetDevice(dev);
    if (e != cudaSuccess) rc = set_cuda_error(e, "cudaSetDevice");
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};
}  // namespace

extern "C" {

const char* hpl_strerror(int code) {
  switch (code) {
    case HPL_OK: return "success";
    case HPL_EINVAL: return "invalid argument";
    case HPL_ENOMEM: return "out of memory";
    case HPL_ECUDA: return "CUDA error";
    case HPL_ENODEV: return "no suitable CUDA device";
    case HPL_ERANGE: return "annulus index out of range (l >= 10)";
    case HPL_ESTATE: return "array coherence misuse";
    default: return "unknown status";
  }
}

const char* hpl_last_error(void) { return t_err.c_str(); }

int hpl_version(void) { return (1 << 16) | 0; }

int hpl_device_count(int* n) {
  if (!n) return set_error(HPL_EINVAL, "n is NULL");
  int c = 0;
  cudaError_t e = cudaGetDeviceCount(&c);
  if (e != cudaSuccess) return set_cuda_error(e, "cudaGetDeviceCount");
  *n = c;
  return HPL_OK;
}

int hpl_set_device(int device) {
  int n = 0;
  int rc = hpl_device_count(&n);
  if (rc) return rc;
  if (device < 0 || device >= n) return set_error(HPL_EINVAL, "device %d out of range [0, %d)", device, n);
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) return set_cuda_error(e, "cudaSetDevice");
  return HPL_OK;
}

int hpl_get_device(int* device) {
  if (!device) return set_error(HPL_EINVAL, "device is NULL");
  return current_device(device);
}

// ------------------------------------------------------------------ arrays
int hpl_array_alloc(hpl_array* out, hpl_dtype t, int ndim, const int64_t* dims, void* host_ptr,
                    int device) {
  if (!out) return set_error(HPL_EINVAL, "out is NULL");
  const size_t es = dtype_size(t);
  if (es == 0) return set_error(HPL_EINVAL, "bad dtype %d", (int)t);
  if (ndim < 0 || ndim > 3) return set_error(HPL_EINVAL, "ndim must be in [0, 3]");
  if (ndim > 0 && !dims) return set_error(HPL_EINVAL, "dims is NULL");
  int64_t count = 1;
  for (int i = 0; i < ndim; ++i) {
    if (dims[i] <= 0) return set_error(HPL_EINVAL, "dims[%d] = %lld must be > 0", i, (long long)dims[i]);
    if (count > (int64_t(1) << 50) / dims[i]) return set_error(HPL_EINVAL, "array too large");
    count *= dims[i];
  }
  if (device < 0) {
    int rc = current_device(&device);
    if (rc) return rc;
  }
  int ndev = 0;
  int rc = hpl_device_count(&ndev);
  if (rc) return rc;
  if (device >= ndev) return set_error(HPL_EINVAL, "device %d out of range", device);
  DeviceGuard g(device);
  if (g.rc) return g.rc;
  hpl_array a = new (std::nothrow) hpl_array_s();
  if (!a) return set_error(HPL_ENOMEM, "host allocation of the descriptor");
  a->t = t;
  a->ndim = ndim;
  for (int i = 0; i < 3; ++i) a->dims[i] = i < ndim ? dims[i] : 1;
  a->count = count;
  a->nbytes = size_t(count) * es;
  a->device = device;
  a->stream = nullptr;
  int arc = dev_alloc(&a->dev, a->nbytes, device, &a->how);
  if (arc) { delete a; return arc; }
  cudaError_t e;
  if (host_ptr) {
    a->host = host_ptr;
    a->host_owned = false;
    a->valid = HPL_HOST;
  } else {
    e = cudaMallocHost(&a->host, a->nbytes);
    if (e != cudaSuccess) { dev_free(a->dev, a->nbytes, device, a->how); delete a; return set_cuda_error(e, "cudaMallocHost(array)"); }
    a->host_owned = true;
    a->valid = HPL_HOST | HPL_DEVICE;
  }
  *out = a;
  return HPL_OK;
}

int hpl_array_free(hpl_array a) {
  if (!a) return HPL_OK;
  DeviceGuard g(a->device);
  cudaError_t e1 = a->stream ? cudaStreamSynchronize(a->stream) : cudaDeviceSynchronize();
  cudaError_t e2 = dev_free(a->dev, a->nbytes, a->device, a->how);
  cudaError_t e3 = a->host_owned ? cudaFreeHost(a->host) : cudaSuccess;
  delete a;
  if (e1 != cudaSuccess) return set_cuda_error(e1, "hpl_array_free: synchronize");
  if (e2 != cudaSuccess) return set_cuda_error(e2, "cudaFree");
  if (e3 != cudaSuccess) return set_cuda_error(e3, "cudaFreeHost");
  return HPL_OK;
}

int hpl_array_sync(hpl_array a, hpl_where where, hpl_access mode) {
  if (!a) return set_error(HPL_EINVAL, "array is NULL");
  if (where != HPL_HOST && where != HPL_DEVICE) return set_error(HPL_EINVAL, "bad where");
  if (mode < HPL_READ || mode > HPL_READWRITE) return set_error(HPL_EINVAL, "bad access mode");
  DeviceGuard g(a->device);
  if (g.rc) return g.rc;
  if (!(a->valid & where)) {
    if (!(a->valid & (where == HPL_HOST ? HPL_DEVICE : HPL_HOST)))
      return set_error(HPL_ESTATE, "neither copy is valid");
    cudaError_t e;
    if (where == HPL_HOST) {
      e = cudaMemcpyAsync(a->host, a->dev, a->nbytes, cudaMemcpyDeviceToHost, a->stream);
      if (e == cudaSuccess) e = cudaStreamSynchronize(a->stream);
    } else {
      e = cudaMemcpyAsync(a->dev, a->host, a->nbytes, cudaMemcpyHostToDevice, a->stream);
    }
    if (e != cudaSuccess) return set_cuda_error(e, "hpl_array_sync copy");
    a->valid |= where;
  } else if (where == HPL_HOST && (mode & HPL_WRITE) && (a->valid & HPL_DEVICE)) {
    // the host is about to be modified while device work may still read it
    cudaError_t e = cudaStreamSynchronize(a->stream);
    if (e != cudaSuccess) return set_cuda_error(e, "hpl_array_sync synchronize");
  }
  if (mode & HPL_WRITE) a->valid = where;
  return HPL_OK;
}

int hpl_array_data(hpl_array a, hpl_where where, void** ptr) {
  if (!a || !ptr) return set_error(HPL_EINVAL, "NULL argument");
  if (where == HPL_HOST) *ptr = a->host;
  else if (where == HPL_DEVICE) *ptr = a->dev;
  else return set_error(HPL_EINVAL, "bad where");
  return HPL_OK;
}

int hpl_array_info(hpl_array a, hpl_dtype* t, int* ndim, int64_t* dims, int64_t* nbytes, int* valid) {
  if (!a) return set_error(HPL_EINVAL, "array is NULL");
  if (t) *t = a->t;
  if (ndim) *ndim = a->ndim;
  if (dims) for (int i = 0; i < a->ndim; ++i) dims[i] = a->dims[i];
  if (nbytes) *nbytes = int64_t(a->nbytes);
  if (valid) *valid = a->valid;
  return HPL_OK;
}

int hpl_array_set_stream(hpl_array a, void* stream) {
  if (!a) return set_error(HPL_EINVAL, "array is NULL");
  a->stream = static_cast<cudaStream_t>(stream);
  return HPL_OK;
}

// --------------------------------------------------------------------- EP
int hpl_ep_run_range(uint64_t seed, uint64_t a, uint64_t pair_begin, uint64_t npairs,
                     double* dev_out13, void* stream) {
  int rc = validate(seed, a);
  if (rc) return rc;
  if (!dev_out13) return set_error(HPL_EINVAL, "dev_out13 is NULL");
  if (pair_begin > (uint64_t(1) << 43) || npairs > (uint64_t(1) << 43) - pair_begin)
    return set_error(HPL_EINVAL, "pair range beyond 2^43 (period 2^44 uniforms)");
  int dev;
  rc = current_device(&dev);
  if (rc) return rc;
  return launch_ep(dev, seed, a, pair_begin, npairs, t_cfg, dev_out13, static_cast<cudaStream_t>(stream));
}

int hpl_ep_run_shard(int M, uint64_t seed, uint64_t a, int rank, int nranks, double* dev_out13,
                     void* stream) {
  uint64_t begin, n;
  int rc = shard_range(M, rank, nranks, &begin, &n);
  if (rc) return rc;
  return hpl_ep_run_range(seed, a, begin, n, dev_out13, stream);
}

// ---- fused cross-GPU combine ------------------------------
struct hpl_comm_s {
  int rank = 0, nranks = 0, device = -1;
  hplep::CommInbox* own = nullptr;                  // cudaMalloc'd on `device`
  hplep::CommInbox* peer[hplep::COMM_MAX_RANKS] = {};  // mapped (own at [rank])
  bool opened = false;
  unsigned long long epoch = 0;
  unsigned long long timeout_ns = 10ull * 1000000000ull;
};

int hpl_comm_create(hpl_comm* out, int rank, int nranks, int device, void* handle_out) {
  if (!out || !handle_out) return set_error(HPL_EINVAL, "NULL argument");
  if (nranks < 1 || nranks > hplep::COMM_MAX_RANKS || (nranks & (nranks - 1)))
    return set_error(HPL_EINVAL, "nranks must be a power of two in [1, %d] (equal EP shards)", hplep::COMM_MAX_RANKS);
  if (rank < 0 || rank >= nranks) return set_error(HPL_EINVAL, "rank out of range");
  if (device < 0) {
    int rc = current_device(&device);
    if (rc) return rc;
  }
  DeviceGuard g(device);
  if (g.rc) return g.rc;
  hpl_comm c = new (std::nothrow) hpl_comm_s;
  if (!c) return set_error(HPL_ENOMEM, "comm");
  c->rank = rank;
  c->nranks = nranks;
  c->device = device;
  cudaError_t e = cudaMalloc(&c->own, sizeof(hplep::CommInbox));
  if (e == cudaSuccess) e = cudaMemset(c->own, 0, sizeof(hplep::CommInbox));
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  cudaIpcMemHandle_t h;
  if (e == cudaSuccess) e = cudaIpcGetMemHandle(&h, c->own);
  if (e != cudaSuccess) {
    if (c->own) cudaFree(c->own);
    delete c;
    return set_cuda_error(e, "comm inbox");
  }
  static_assert(sizeof(cudaIpcMemHandle_t) == HPL_COMM_HANDLE_BYTES, "IPC handle size");
  std::memcpy(handle_out, &h, sizeof(h));
  c->peer[rank] = c->own;
  *out = c;
  return HPL_OK;
}

int hpl_comm_open(hpl_comm c, const void* handles) {
  if (!c || !handles) return set_error(HPL_EINVAL, "NULL argument");
  if (c->opened) return set_error(HPL_ESTATE, "comm already open");
  DeviceGuard g(c->device);
  if (g.rc) return g.rc;
  const unsigned char* hb = static_cast<const unsigned char*>(handles);
  for (int r = 0; r < c->nranks; ++r) {
    if (r == c->rank) continue;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, hb + size_t(r) * HPL_COMM_HANDLE_BYTES, sizeof(h));
    void* p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      for (int q = 0; q < r; ++q)
        if (q != c->rank && c->peer[q]) { cudaIpcCloseMemHandle(c->peer[q]); c->peer[q] = nullptr; }
      return set_cuda_error(e, "cudaIpcOpenMemHandle (peer inbox)");
    }
    c->peer[r] = static_cast<hplep::CommInbox*>(p);
  }
  c->opened = true;
  return HPL_OK;
}

int hpl_comm_set_timeout(hpl_comm c, double seconds) {
  if (!c || !(seconds > 0.0) || seconds > 3600.0) return set_error(HPL_EINVAL, "timeout must be in (0, 3600] s");
  c->timeout_ns = static_cast<unsigned long long>(seconds * 1e9);
  return HPL_OK;
}

int hpl_comm_free(hpl_comm c) {
  if (!c) return HPL_OK;
  DeviceGuard g(c->device);
  for (int r = 0; r < c->nranks; ++r)
    if (r != c->rank && c->peer[r]) cudaIpcCloseMemHandle(c->peer[r]);
  if (c->own) cudaFree(c->own);
  delete c;
  return HPL_OK;
}

int hpl_ep_run_fused(hpl_comm c, int M, uint64_t seed, uint64_t a, double* dev_out13, void* stream) {
  if (!c || !dev_out13) return set_error(HPL_EINVAL, "NULL argument");
  if (!c->opened) return set_error(HPL_ESTATE, "comm not opened (hpl_comm_open)");
  uint64_t begin, n;
  int rc = shard_range(M, c->rank, c->nranks, &begin, &n);
  if (!rc) rc = validate(seed, a);
  if (rc) return rc;
  DeviceGuard g(c->device);
  if (g.rc) return g.rc;
  hplep::CommParams cp;
  std::memset(&cp, 0, sizeof(cp));
  for (int r = 0; r < c->nranks; ++r) cp.inbox[r] = c->peer[r];
  cp.rank = c->rank;
  cp.nranks = c->nranks;
  cp.epoch = c->epoch + 1;
  cp.timeout_ns = c->timeout_ns;
  rc = launch_ep(c->device, seed, a, begin, n, t_cfg, dev_out13, static_cast<cudaStream_t>(stream), &cp);
  if (rc) return rc;
  c->epoch += 1;  // only launched calls advance the epoch
  return HPL_OK;
}

int hpl_comm_status(hpl_comm c, void* stream, uint64_t* epoch, uint64_t* timeouts) {
  if (!c || !epoch || !timeouts) return set_error(HPL_EINVAL, "NULL argument");
  DeviceGuard g(c->device);
  if (g.rc) return g.rc;
  cudaError_t e = cudaStreamSynchronize(static_cast<cudaStream_t>(stream));
  unsigned long long w[2] = {0, 0};  // {stale, timeouts}
  static_assert(offsetof(hplep::CommInbox, timeouts) == offsetof(hplep::CommInbox, stale) + 8, "layout");
  if (e == cudaSuccess) e = cudaMemcpy(w, &c->own->stale, sizeof(w), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return set_cuda_error(e, "comm status");
  *epoch = c->epoch;
  *timeouts = w[0] + w[1];
  if (w[1]) return set_error(HPL_ECUDA, "fused combine: %llu call(s) timed out waiting for a peer", w[1]);
  if (w[0]) return set_error(HPL_ECUDA, "fused combine: %llu call(s) saw a peer's slot change during the fold", w[0]);
  return HPL_OK;
}

int hpl_ep_eval(int M, uint64_t seed, uint64_t a, int rank, int nranks, hpl_array out13) {
  if (!out13) return set_error(HPL_EINVAL, "out13 is NULL");
  if (out13->t != HPL_F64 || out13->count != 13) return set_error(HPL_EINVAL, "out13 must be an HPL_F64 array of 13 elements");
  uint64_t begin, n;
  int rc = shard_range(M, rank, nranks, &begin, &n);
  if (rc) return rc;
  rc = validate(seed, a);
  if (rc) return rc;
  DeviceGuard g(out13->device);
  if (g.rc) return g.rc;
  rc = launch_ep(out13->device, seed, a, begin, n, t_cfg, static_cast<double*>(out13->dev), out13->stream);
  if (rc) return rc;
  out13->valid = HPL_DEVICE;  // the kernel wrote the device copy
  return HPL_OK;
}

}  // extern "C"
namespace {
struct RunCache {
  static constexpr int N = 64;
  hpl_array a[N] = {nullptr};
  void release() {
    for (auto& x : a)
      if (x) { hpl_array_free(x); x = nullptr; }
  }
  ~RunCache() { release(); }
};
thread_local RunCache t_run;
}  // namespace
extern "C" {

int hpl_ep_run(int M, uint64_t seed, uint64_t a, double* sx, double* sy, uint64_t q[10]) {
  if (!sx || !sy || !q) return set_error(HPL_EINVAL, "NULL output pointer");
  uint64_t b0, n0;
  int rc = shard_range(M, 0, 1, &b0, &n0);  // argument errors before any CUDA call
  if (!rc) rc = validate(seed, a);
  if (rc) return rc;
  int dev;
  rc = current_device(&dev);
  if (rc) return rc;
  // one cached 13-word Array per thread and device (the paper's Array with
  // a library-owned host copy); freed at thread exit or by
  // hpl_shutdown()
  if (dev >= RunCache::N) return set_error(HPL_EINVAL, "device index too large");
  hpl_array& slot = t_run.a[dev];
  if (!slot) {
    int64_t d = 13;
    rc = hpl_array_alloc(&slot, HPL_F64, 1, &d, nullptr, dev);
    if (rc) return rc;
  }
  hpl_array out = slot;
  rc = hpl_ep_eval(M, seed, a, 0, 1, out);
  if (rc) return rc;
  rc = hpl_array_sync(out, HPL_HOST, HPL_READ);  // 104-byte D2H, blocking
  if (rc) return rc;
  const double* h = static_cast<const double*>(out->host);
  if (h[0] != h[0]) return set_error(HPL_ERANGE, "an annulus index l >= 10 occurred");
  *sx = h[0];
  *sy = h[1];
  for (int k = 0; k < 10; ++k) q[k] = static_cast<uint64_t>(h[2 + k]);
  return HPL_OK;
}

int hpl_lcg_states(uint64_t seed, uint64_t a, uint64_t offset, uint64_t n, uint64_t* host_out) {
  int rc = validate(seed, a);
  if (rc) return rc;
  if (n > (uint64_t(1) << 28)) return set_error(HPL_EINVAL, "n must be <= 2^28");
  if (n == 0) return HPL_OK;
  if (!host_out) return set_error(HPL_EINVAL, "host_out is NULL");
  int dev;
  rc = current_device(&dev);
  if (rc) return rc;
  void* d = nullptr;
  DevAlloc how;
  rc = dev_alloc(&d, n * sizeof(uint64_t), dev, &how);
  if (rc) return rc;
  rc = launch_lcg_states(seed, a, offset, n, static_cast<uint64_t*>(d), nullptr);
  if (!rc) {
    cudaError_t e = cudaMemcpy(host_out, d, n * sizeof(uint64_t), cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) rc = set_cuda_error(e, "cudaMemcpy(states)");
  }
  cudaDeviceSynchronize();
  dev_free(d, n * sizeof(uint64_t), dev, how);
  return rc;
}

int hpl_ep_set_config(int variant, int threads_per_block, int blocks_per_sm) {
  if (variant != HPL_EP_LEAN && variant != HPL_EP_LIBDEVICE) return set_error(HPL_EINVAL, "unknown variant");
  if (threads_per_block < 0 || threads_per_block > 1024 || threads_per_block % 32)
    return set_error(HPL_EINVAL, "threads_per_block must be 0 or a multiple of 32 <= 1024");
  if (blocks_per_sm < 0 || blocks_per_sm > 32) return set_error(HPL_EINVAL, "blocks_per_sm must be in [0, 32]");
  t_cfg.variant = variant;
  t_cfg.threads_per_block = threads_per_block;
  t_cfg.blocks_per_sm = blocks_per_sm;
  return HPL_OK;
}

int hpl_ep_launch_shape(uint64_t npairs, int* blocks, int* threads, int* smem_bytes) {
  if (!blocks || !threads || !smem_bytes) return set_error(HPL_EINVAL, "NULL output pointer");
  int dev;
  int rc = current_device(&dev);
  if (rc) return rc;
  return launch_shape(dev, npairs, t_cfg, blocks, threads, smem_bytes);
}

int hpl_ep_launch_count(uint64_t* count) {
  if (!count) return set_error(HPL_EINVAL, "count is NULL");
  *count = launch_count();
  return HPL_OK;
}


// ------------------------------------------------------- generic eval (F1)
namespace {
struct SigArg {
  bool array;
  int dtype;  // arrays: hpl_dtype; scalars: hpl_arg_kind
  int mode;   // arrays: hpl_access
};

int parse_sig(const char* sig, SigArg* out, int maxn) {
  int n = 0;
  const char* p = sig;
  while (*p && n < maxn) {
    const char* e = p;
    while (*e && *e != ',') ++e;
    std::string item(p, e - p);
    size_t c1 = item.find(':');
    size_t c2 = item.find(':', c1 + 1);
    std::string type = item.substr(c1 + 1, c2 == std::string::npos ? std::string::npos : c2 - c1 - 1);
    SigArg a{false, 0, 0};
    if (c2 != std::string::npos) {  // array
      a.array = true;
      std::string m = item.substr(c2 + 1);
      a.mode = m == "r" ? HPL_READ : (m == "w" ? HPL_WRITE : HPL_READWRITE);
      a.dtype = type == "F64" ? HPL_F64 : type == "F32" ? HPL_F32 : type == "U64" ? HPL_U64
              : type == "I64" ? HPL_I64 : type == "I32" ? HPL_I32 : HPL_U32;
    } else {
      a.dtype = type == "f64" ? HPL_ARG_F64 : type == "f32" ? HPL_ARG_F32 : type == "i64" ? HPL_ARG_I64
              : HPL_ARG_I32;
    }
    out[n++] = a;
    p = *e ? e + 1 : e;
  }
  return n;
}

int64_t pow2_divisor(int64_t v, int64_t cap) {
  int64_t d = v & -v;
  return d < cap ? d : cap;
}
}  // namespace

int hpl_kernel_count(int* n) {
  if (!n) return set_error(HPL_EINVAL, "n is NULL");
  *n = kernel_count();
  return HPL_OK;
}

int hpl_kernel_info(int i, const char** name, const char** signature) {
  const KernelDesc* k = kernel_at(i);
  if (!k) return set_error(HPL_EINVAL, "kernel index %d out of range", i);
  if (name) *name = k->name;
  if (signature) *signature = k->signature;
  return HPL_OK;
}

int hpl_eval(const char* name, int ndim, const int64_t* global, const int64_t* local, int nargs,
             const hpl_arg* args) {
  if (!name) return set_error(HPL_EINVAL, "kernel name is NULL");
  const KernelDesc* K = kernel_find(name);
  if (!K) return set_error(HPL_EINVAL, "no kernel named '%s'", name);
  SigArg sig[16];
  const int ns = parse_sig(K->signature, sig, 16);
  if (nargs != ns) return set_error(HPL_EINVAL, "%s takes %d arguments (%s), got %d", name, ns, K->signature, nargs);
  if (nargs > 0 && !args) return set_error(HPL_EINVAL, "args is NULL");
  for (int i = 0; i < nargs; ++i) {
    if (sig[i].array) {
      if (args[i].kind != HPL_ARG_ARRAY || !args[i].array)
        return set_error(HPL_EINVAL, "%s argument %d must be an array", name, i);
      if (args[i].array->t != sig[i].dtype)
        return set_error(HPL_EINVAL, "%s argument %d has the wrong element type", name, i);
      if (args[i].access != 0 && args[i].access != sig[i].mode)
        return set_error(HPL_EINVAL, "%s argument %d: access mode differs from the kernel's", name, i);
    } else if (args[i].kind != sig[i].dtype) {
      return set_error(HPL_EINVAL, "%s argument %d must be a scalar of kind %d", name, i, sig[i].dtype);
    }
  }
  // ---- global domain: given, or the first argument's dims
  EvalDomain D;
  D.ndim = 0;
  for (int i = 0; i < 3; ++i) D.global[i] = D.local[i] = 1;
  if (global == nullptr || ndim == 0) {
    if (nargs == 0 || !sig[0].array) return set_error(HPL_EINVAL, "no global domain and no array first argument");
    const hpl_array a0 = args[0].array;
    if (a0->ndim < 1) return set_error(HPL_EINVAL, "the first argument is a scalar array");
    D.ndim = a0->ndim;
    for (int i = 0; i < D.ndim; ++i) D.global[i] = a0->dims[i];
  } else {
    if (ndim < 1 || ndim > 3) return set_error(HPL_EINVAL, "domains have 1..3 dimensions");
    D.ndim = ndim;
    for (int i = 0; i < ndim; ++i) {
      if (global[i] <= 0) return set_error(HPL_EINVAL, "global[%d] must be > 0", i);
      D.global[i] = global[i];
    }
  }
  // ---- local domain: given (must divide the global one) or chosen
  bool chosen = true;
  if (local) for (int i = 0; i < D.ndim; ++i) if (local[i] != 0) chosen = false;
  if (chosen) {
    int64_t budget = 256;
    for (int i = 0; i < D.ndim; ++i) {
      D.local[i] = pow2_divisor(D.global[i], budget);
      budget /= D.local[i];
    }
  } else {
    int64_t prod = 1;
    for (int i = 0; i < D.ndim; ++i) {
      if (local[i] <= 0 || D.global[i] % local[i] != 0)
        return set_error(HPL_EINVAL, "local[%d] = %lld must divide global[%d] = %lld", i, (long long)local[i], i,
                         (long long)D.global[i]);
      D.local[i] = local[i];
      prod *= local[i];
    }
    if (prod > 1024 || D.local[2] > 64) return set_error(HPL_EINVAL, "local domain too large for one group (<= 1024 threads)");
  }
  if (D.global[0] / D.local[0] > 0x7FFFFFFFll || D.global[1] / D.local[1] > 65535 || D.global[2] / D.local[2] > 65535)
    return set_error(HPL_EINVAL, "global domain too large");
  // ---- arrays: same device, large enough, coherence before the launch
  void* ptrs[16] = {nullptr};
  int device = -1;
  cudaStream_t stream = nullptr;
  for (int i = 0; i < nargs; ++i) {
    if (!sig[i].array) continue;
    hpl_array a = args[i].array;
    if (device < 0) {
      device = a->device;
      stream = a->stream;
    } else if (a->device != device) {
      return set_error(HPL_EINVAL, "array arguments live on different devices");
    }
    const int64_t need = K->need(D, i);
    if (need > a->count) return set_error(HPL_EINVAL, "%s argument %d holds %lld elements, needs %lld", name, i,
                                          (long long)a->count, (long long)need);
  }
  if (device < 0) {
    int rc = current_device(&device);
    if (rc) return rc;
  }
  DeviceGuard g(device);
  if (g.rc) return g.rc;
  for (int i = 0; i < nargs; ++i) {
    if (!sig[i].array) continue;
    hpl_array a = args[i].array;
    if (sig[i].mode & HPL_READ) {
      int rc = hpl_array_sync(a, HPL_DEVICE, HPL_READ);  // copies only if stale
      if (rc) return rc;
    }
    if (a->stream != stream) {  // order this array's pending work before the launch
      cudaError_t e = cudaStreamSynchronize(a->stream);
      if (e != cudaSuccess) return set_cuda_error(e, "cudaStreamSynchronize");
    }
    ptrs[i] = a->dev;
  }
  int rc = K->launch(D, ptrs, args, stream);
  if (rc) return rc;
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_cuda_error(e, name);
  // a written array whose own stream differs from the launch stream: order its
  // stream after the kernel, so a later hpl_array_sync(HOST) on that stream
  // (or any work the caller queues there) sees the kernel's output
  cudaEvent_t done = nullptr;
  for (int i = 0; i < nargs; ++i) {
    if (!sig[i].array || !(sig[i].mode & HPL_WRITE)) continue;
    hpl_array a = args[i].array;
    if (a->stream != stream) {
      if (!done) {
        e = cudaEventCreateWithFlags(&done, cudaEventDisableTiming);
        if (e == cudaSuccess) e = cudaEventRecord(done, stream);
        if (e != cudaSuccess) return set_cuda_error(e, "hpl_eval: completion event");
      }
      e = cudaStreamWaitEvent(a->stream, done, 0);
      if (e != cudaSuccess) { cudaEventDestroy(done); return set_cuda_error(e, "cudaStreamWaitEvent"); }
    }
    a->valid = HPL_DEVICE;
  }
  if (done) cudaEventDestroy(done);  // released once the recorded work completes
  return HPL_OK;
}


// ------------------------------------------------------------ reduction (F2)
namespace {
struct RedWs {
  int device;
  cudaStream_t stream;
  hplep::ReduceWorkspace ws;
  int sms;
};
std::mutex g_red_mu;
std::deque<RedWs> g_red;  // deque: references stay valid across push_back

int reduce_workspace(int device, cudaStream_t stream, hplep::ReduceWorkspace** ws, int* sms) {
  std::lock_guard<std::mutex> lk(g_red_mu);
  for (auto& w : g_red)
    if (w.device == device && w.stream == stream) {
      *ws = &w.ws;
      *sms = w.sms;
      return 0;
    }
  RedWs w{device, stream, {}, 0};
  cudaError_t e = cudaDeviceGetAttribute(&w.sms, cudaDevAttrMultiProcessorCount, device);
  if (e != cudaSuccess) return set_cuda_error(e, "cudaDeviceGetAttribute");
  w.ws.capacity = w.sms * 16;  // >= blocks of any launch configuration
  e = cudaMalloc(&w.ws.partials, sizeof(double) * w.ws.capacity);
  if (e == cudaSuccess) e = cudaMalloc(&w.ws.counter, sizeof(unsigned));
  if (e == cudaSuccess) e = cudaMemset(w.ws.counter, 0, sizeof(unsigned));
  if (e != cudaSuccess) return set_cuda_error(e, "reduce workspace");
  g_red.push_back(w);
  *ws = &g_red.back().ws;
  *sms = w.sms;
  return 0;
}
}  // namespace

int hpl_reduce_sum_f32(const float* dev_in, int64_t n, double* dev_out, void* stream) {
  if (n < 0) return set_error(HPL_EINVAL, "n must be >= 0");
  if (!dev_out || (n > 0 && !dev_in)) return set_error(HPL_EINVAL, "NULL pointer");
  if (reinterpret_cast<uintptr_t>(dev_in) & 3) return set_error(HPL_EINVAL, "dev_in must be 4-byte aligned");
  int dev;
  int rc = current_device(&dev);
  if (rc) return rc;
  hplep::ReduceWorkspace* ws;
  int sms;
  rc = reduce_workspace(dev, static_cast<cudaStream_t>(stream), &ws, &sms);
  if (rc) return rc;
  return hplep::launch_reduce_sum_f32(dev_in, n, dev_out, *ws, sms, static_cast<cudaStream_t>(stream));
}


int hpl_transpose_f32(const float* dev_src, int64_t h, int64_t w, float* dev_dst, void* stream) {
  if (h < 0 || w < 0) return set_error(HPL_EINVAL, "h and w must be >= 0");
  if (h > 0 && w > 0 && h > INT64_MAX / 4 / w) return set_error(HPL_EINVAL, "h * w too large");
  const int64_t n = h * w;
  if (n == 0) return HPL_OK;
  if (!dev_src || !dev_dst) return set_error(HPL_EINVAL, "NULL pointer");
  if ((reinterpret_cast<uintptr_t>(dev_src) | reinterpret_cast<uintptr_t>(dev_dst)) & 3)
    return set_error(HPL_EINVAL, "dev_src and dev_dst must be 4-byte aligned");
  const uintptr_t s0 = reinterpret_cast<uintptr_t>(dev_src), d0 = reinterpret_cast<uintptr_t>(dev_dst);
  const uintptr_t bytes = uintptr_t(n) * sizeof(float);
  if (s0 < d0 + bytes && d0 < s0 + bytes) return set_error(HPL_EINVAL, "dev_src and dev_dst overlap (no in-place transpose)");
  int dev;
  int rc = current_device(&dev);
  if (rc) return rc;
  int sms = 0;
  cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) return set_cuda_error(e, "cudaDeviceGetAttribute");
  return hplep::launch_transpose_f32(dev_src, dev_dst, h, w, sms, static_cast<cudaStream_t>(stream));
}

int hpl_ep_pairs_debug(uint64_t seed, uint64_t a, uint64_t pair_begin, uint64_t n, double* host_out) {
  int rc = validate(seed, a);
  if (rc) return rc;
  if (n > (uint64_t(1) << 26)) return set_error(HPL_EINVAL, "n must be <= 2^26");
  if (n == 0) return HPL_OK;
  if (!host_out) return set_error(HPL_EINVAL, "host_out is NULL");
  int dev;
  rc = current_device(&dev);
  if (rc) return rc;
  void* d = nullptr;
  DevAlloc how;
  rc = dev_alloc(&d, n * 4 * sizeof(double), dev, &how);
  if (rc) return rc;
  rc = launch_pairs_debug(dev, seed, a, pair_begin, n, static_cast<double*>(d), nullptr);
  if (!rc) {
    cudaError_t e = cudaMemcpy(host_out, d, n * 4 * sizeof(double), cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) rc = set_cuda_error(e, "cudaMemcpy(debug)");
  }
  cudaDeviceSynchronize();
  dev_free(d, n * 4 * sizeof(double), dev, how);
  return rc;
}

int hpl_set_device_allocator(hpl_alloc_fn alloc, hpl_free_fn free_fn, void* ctx) {
  if ((alloc == nullptr) != (free_fn == nullptr)) return set_error(HPL_EINVAL, "alloc and free must both be set or both be NULL");
  std::lock_guard<std::mutex> lk(g_alloc_mu);
  g_alloc = alloc;
  g_free = free_fn;
  g_alloc_ctx = alloc ? ctx : nullptr;
  return HPL_OK;
}

int hpl_shutdown(void) {
  t_run.release();
  int rc = release_ep_state();
  {
    std::lock_guard<std::mutex> lk(g_red_mu);
    for (auto& w : g_red) {
      DeviceGuard g(w.device);
      cudaStreamSynchronize(w.stream);
      cudaFree(w.ws.partials);
      cudaFree(w.ws.counter);
    }
    g_red.clear();
  }
  std::lock_guard<std::mutex> lk(g_alloc_mu);
  g_alloc = nullptr;
  g_free = nullptr;
  g_alloc_ctx = nullptr;
  return rc;
}

}  // extern "C"
