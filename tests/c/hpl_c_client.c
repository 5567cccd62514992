/* A plain C client of the C ABI (include/hpl.h) — no Python, no torch.
 *   cpu  : library loads, status strings, argument validation (no GPU needed)
 *   gpu  : NPB class S through hpl_ep_run and the Array/eval path, checked
 *          against NPB's published verification sums (tests/golden) */
#include <math.h>
#include <stdio.h>
#include <string.h>

#include "hpl.h"

static int fails = 0;
#define CHECK(c) do { if (!(c)) { printf("FAIL %s:%d %s\n", __FILE__, __LINE__, #c); ++fails; } } while (0)

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
  }
  printf("%s: %d failures\n", gpu ? "gpu" : "cpu", fails);
  return fails != 0;
}
