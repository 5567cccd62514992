/* A plain C client of the C ABI (include/hpl.h) — no Python, no torch.
 *   cpu  : library loads, status strings, argument validation (no GPU needed)
 *   gpu  : NPB class S through hpl_ep_run and the Array/eval path, checked
 *          against NPB's published verification sums (tests/golden); the
 *          transpose through eval on Arrays and the reduction on an Array's
 *          device copy, checked against their definitions; a caller-installed
 *          device allocator (counting, over cudart) and hpl_shutdown */
#include <cuda_runtime_api.h>
#include <math.h>
#include <stdio.h>
#include <string.h>

#include "hpl.h"

static int fails = 0;
#define CHECK(c) do { if (!(c)) { printf("FAIL %s:%d %s\n", __FILE__, __LINE__, #c); ++fails; } } while (0)

/* counting allocator over the CUDA runtime (caller-side, for the test) */
static int g_allocs = 0, g_frees = 0, g_ctx_tag = 0;
static size_t g_alloc_bytes = 0;
static void* g_ctx_seen = NULL;
static void* counting_alloc(size_t bytes, int device, void* ctx) {
  void* p = NULL;
  (void)device;
  ++g_allocs;
  g_alloc_bytes = bytes;
  g_ctx_seen = ctx;
  return cudaMalloc(&p, bytes) == cudaSuccess ? p : NULL;
}
static void counting_free(void* p, size_t bytes, int device, void* ctx) {
  (void)bytes; (void)device; (void)ctx;
  ++g_frees;
  cudaFree(p);
}

int main(int argc, char** argv) {
  const int gpu = argc > 1 && strcmp(argv[1], "gpu") == 0;
  CHECK(hpl_version() >> 16 == 1);
  CHECK(strcmp(hpl_strerror(HPL_OK), "success") == 0);
  CHECK(hpl_strerror(-42) != NULL);
  double sx, sy;
  uint64_t q[10];
  CHECK(hpl_ep_run(44, 271828183ull, 1220703125ull, &sx, &sy, q) == HPL_EINVAL);   /* M > 43 */
  CHECK(hpl_ep_run(24, 271828183ull, 1220703124ull, &sx, &sy, q) == HPL_EINVAL);   /* even a */
  CHECK(hpl_ep_run(24, 1ull << 45, 1220703125ull, &sx, &sy, q) == HPL_EINVAL);     /* fixed point */
  CHECK(hpl_ep_run(24, 271828183ull, 1220703125ull, NULL, &sy, q) == HPL_EINVAL);
  CHECK(strlen(hpl_last_error()) > 0);
  CHECK(hpl_ep_run_shard(24, 271828183ull, 1220703125ull, 3, 2, (double*)0x1000, NULL) == HPL_EINVAL);
  CHECK(hpl_eval("no_such_kernel", 0, NULL, NULL, 0, NULL) == HPL_EINVAL);
  CHECK(hpl_transpose_f32(NULL, 0, 7, NULL, NULL) == HPL_OK);                       /* empty */
  CHECK(hpl_transpose_f32((const float*)0x1000, 3, 4, (float*)0x1008, NULL) == HPL_EINVAL);  /* overlap */
  CHECK(hpl_reduce_sum_f32(NULL, -1, (double*)0x1000, NULL) == HPL_EINVAL);
  if (gpu) {
    /* NPB class S (M = 24); verification values: NPB ep.f (BASELINE.json) */
    CHECK(hpl_ep_run(24, 271828183ull, 1220703125ull, &sx, &sy, q) == HPL_OK);
    CHECK(fabs((sx - -3.247834652034740e3) / -3.247834652034740e3) <= 1e-8);
    CHECK(fabs((sy - -6.958407078382297e3) / -6.958407078382297e3) <= 1e-8);
    uint64_t gc = 0;
    for (int i = 0; i < 10; ++i) gc += q[i];
    CHECK(gc == 13176389ull && q[0] == 6140517ull && q[5] == 17ull);
    /* the same through eval(EP) into an Array and a host sync */
    hpl_array out;
    int64_t d = 13;
    CHECK(hpl_array_alloc(&out, HPL_F64, 1, &d, NULL, -1) == HPL_OK);
    CHECK(hpl_ep_eval(24, 271828183ull, 1220703125ull, 0, 1, out) == HPL_OK);
    int valid = 0;
    CHECK(hpl_array_info(out, NULL, NULL, NULL, NULL, &valid) == HPL_OK && valid == HPL_DEVICE);
    CHECK(hpl_array_sync(out, HPL_HOST, HPL_READ) == HPL_OK);
    double* h;
    CHECK(hpl_array_data(out, HPL_HOST, (void**)&h) == HPL_OK);
    CHECK(h[0] == sx && h[1] == sy && (uint64_t)h[12] == gc);
    CHECK(hpl_array_free(out) == HPL_OK);

    /* transpose (Fig. 10(b)) through eval on two Arrays: dest (w x h) = src (h x w) */
    enum { H = 70, W = 131 };
    hpl_array src, dst;
    int64_t ds[2] = {H, W}, dd[2] = {W, H};
    CHECK(hpl_array_alloc(&src, HPL_F32, 2, ds, NULL, -1) == HPL_OK);
    CHECK(hpl_array_alloc(&dst, HPL_F32, 2, dd, NULL, -1) == HPL_OK);
    float* hs;
    CHECK(hpl_array_data(src, HPL_HOST, (void**)&hs) == HPL_OK);
    for (int i = 0; i < H * W; ++i) hs[i] = (float)i * 0.5f - 100.0f;
    CHECK(hpl_array_sync(src, HPL_HOST, HPL_WRITE) == HPL_OK);
    hpl_arg args[2];
    memset(args, 0, sizeof(args));
    args[0].kind = HPL_ARG_ARRAY; args[0].array = dst;
    args[1].kind = HPL_ARG_ARRAY; args[1].array = src;
    CHECK(hpl_eval("transpose_f32", 0, NULL, NULL, 2, args) == HPL_OK);
    CHECK(hpl_array_sync(dst, HPL_HOST, HPL_READ) == HPL_OK);
    float* hd;
    CHECK(hpl_array_data(dst, HPL_HOST, (void**)&hd) == HPL_OK);
    int bad = 0;
    for (int i = 0; i < H; ++i)
      for (int j = 0; j < W; ++j) bad += hd[j * H + i] != hs[i * W + j];
    CHECK(bad == 0);
    /* reduction of src's device copy: sum of (i/2 - 100), exact in double */
    void* dsrc;
    double* dsum;
    hpl_array sum;
    int64_t one = 1;
    CHECK(hpl_array_alloc(&sum, HPL_F64, 1, &one, NULL, -1) == HPL_OK);
    CHECK(hpl_array_data(src, HPL_DEVICE, &dsrc) == HPL_OK);
    CHECK(hpl_array_data(sum, HPL_DEVICE, (void**)&dsum) == HPL_OK);
    CHECK(hpl_reduce_sum_f32((const float*)dsrc, H * W, dsum, NULL) == HPL_OK);
    CHECK(hpl_array_sync(sum, HPL_DEVICE, HPL_WRITE) == HPL_OK);  /* the kernel wrote the device copy */
    CHECK(hpl_array_sync(sum, HPL_HOST, HPL_READ) == HPL_OK);
    double* hsum;
    CHECK(hpl_array_data(sum, HPL_HOST, (void**)&hsum) == HPL_OK);
    const double n = (double)(H * W), want = 0.5 * n * (n - 1) / 2.0 - 100.0 * n;
    CHECK(*hsum == want);
    CHECK(hpl_array_free(src) == HPL_OK && hpl_array_free(dst) == HPL_OK && hpl_array_free(sum) == HPL_OK);

    /* a caller-installed device allocator (include/hpl.h): Arrays draw from it
       and return to it; after hpl_shutdown the library re-creates its state */
    CHECK(hpl_set_device_allocator(counting_alloc, counting_free, &g_ctx_tag) == HPL_OK);
    hpl_array c13;
    CHECK(hpl_array_alloc(&c13, HPL_F64, 1, &d, NULL, -1) == HPL_OK);
    CHECK(g_allocs == 1 && g_alloc_bytes == 104 && g_ctx_seen == &g_ctx_tag);
    CHECK(hpl_ep_eval(20, 271828183ull, 1220703125ull, 0, 1, c13) == HPL_OK);
    CHECK(hpl_array_sync(c13, HPL_HOST, HPL_READ) == HPL_OK);
    CHECK(hpl_array_free(c13) == HPL_OK);
    CHECK(g_frees == 1);
    CHECK(hpl_shutdown() == HPL_OK);  /* frees the library's own buffers, resets the allocator */
    CHECK(hpl_ep_run(20, 271828183ull, 1220703125ull, &sx, &sy, q) == HPL_OK);
    CHECK(g_allocs == 1);             /* cudaMalloc again after hpl_shutdown */
    gc = 0;
    for (int i = 0; i < 10; ++i) gc += q[i];
    CHECK(gc == 823561ull);           /* M = 20 (smoke value) */
  }
  printf("%s: %d failures\n", gpu ? "gpu" : "cpu", fails);
  return fails != 0;
}
