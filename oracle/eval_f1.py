"""F1 oracle — TEST INFRASTRUCTURE, NOT PRODUCT CODE.

Plain CPU definitions of the paper's own example kernels that run through
``hpl_eval``, written out step by step in the paper's order:

  domain_ids  Fig. 2: for every point of a 1-3-D
              global domain with local domain ``local``, the global id, the
              local id (``gid % local``) and the group id (``gid // local``),
              as 9 int32 words per point in x-fastest order.
  saxpy       Fig. 3: ``y[idx] = a * x[idx] + y[idx]`` in
              float64 with two roundings (a product, then a sum; the paper's
              expression is not an fma).
  dotp        Fig. 4: each group of M lanes writes its
              products ``v1[i] * v2[i]`` (rounded to float32) to Local memory;
              lane 0 sums the M products in lane order into ``pSums[gidx]``,
              one float32 rounding per add.

Pinned in tests/test_eval.py (``-m "not gpu"``): the Fig. 2 example ids the
paper prints, the coverage/partition identities of the id triples, saxpy
against exact rational arithmetic, dotp against float64 dot products and a
brute-force Fraction sum of the float32 chain.
Shares nothing with the CUDA tree; numpy is used only as an array container.
"""
import numpy as np


def domain_ids(global_dims, local_dims):
    """[n, 9] int32: (gx, gy, gz, lx, ly, lz, grx, gry, grz) for every point,
    x fastest (Fig. 2: idx/idy/idz, lidx/lidy/lidz, gidx/gidy/gidz)."""
    g = list(global_dims) + [1] * (3 - len(global_dims))
    lo = list(local_dims) + [1] * (3 - len(local_dims))
    out = np.zeros((g[0] * g[1] * g[2], 9), dtype=np.int32)
    k = 0
    for z in range(g[2]):
        for y in range(g[1]):
            for x in range(g[0]):
                p = (x, y, z)
                out[k, 0:3] = p
                out[k, 3:6] = [p[d] % lo[d] for d in range(3)]
                out[k, 6:9] = [p[d] // lo[d] for d in range(3)]
                k += 1
    return out


def saxpy(y, x, a):
    """Fig. 3 body ``y[idx] = a * x[idx] + y[idx]`` for every idx (float64;
    numpy rounds the product and the sum separately)."""
    y = np.asarray(y, dtype=np.float64)
    x = np.asarray(x, dtype=np.float64)
    prod = np.float64(a) * x        # a * x[idx], rounded
    return prod + y                 # + y[idx], rounded


def dotp(v1, v2, M):
    """Fig. 4: pSums[g] = lane 0's in-order float32 sum of the group's M
    float32 products (sharedM[lidx] = v1[idx] * v2[idx]; then for i in 0..M-1:
    pSums[gidx] += sharedM[i])."""
    v1 = np.asarray(v1, dtype=np.float32)
    v2 = np.asarray(v2, dtype=np.float32)
    ng = len(v1) // M
    shared = (v1 * v2).astype(np.float32).reshape(ng, M)  # one rounding per product
    psums = np.zeros(ng, dtype=np.float32)
    for i in range(M):                                     # lane 0's loop, in order
        psums = (psums + shared[:, i]).astype(np.float32)
    return psums
