#!/usr/bin/env python
"""Probe the sm_100a stochastic-rounding conversion cvt.rs.f16x2.f32 (F2FP...RS): which random
bits round which element, and how.  GPU only; writes gpurun_out/cvt_rs_probe.npz for analysis."""
import os
import subprocess
import sys
import tempfile

import numpy as np

SRC = r'''
#include <cstdint>
extern "C" __global__ void probe(const float* a, const float* b, const unsigned* r, unsigned* out, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  unsigned d;
  asm volatile("cvt.rs.f16x2.f32 %0, %1, %2, %3;" : "=r"(d) : "f"(a[i]), "f"(b[i]), "r"(r[i]));
  out[i] = d;
}
'''


def main():
    import torch
    from torch.utils.cpp_extension import load_inline  # noqa: F401  (torch only for memory)
    tmp = tempfile.mkdtemp()
    cu = os.path.join(tmp, "p.cu")
    open(cu, "w").write(SRC)
    cubin = os.path.join(tmp, "p.cubin")
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-cubin", "-o", cubin, cu])
    from cuda.bindings import driver as drv
    drv.cuInit(0)
    torch.cuda.init()
    torch.zeros(1, device="cuda")
    err, mod = drv.cuModuleLoad(cubin.encode())
    err, fn = drv.cuModuleGetFunction(mod, b"probe")
    rng = np.random.default_rng(1)
    n = 1 << 20
    a = np.concatenate([rng.uniform(-2, 2, n // 4), rng.uniform(-1e-4, 1e-4, n // 4),
                        rng.normal(0, 0.3, n // 4), rng.uniform(-70000, 70000, n // 4)]).astype(np.float32)
    b = rng.permutation(a).astype(np.float32)
    r = rng.integers(0, 2 ** 32, n, dtype=np.uint64).astype(np.uint32)
    # single-bit patterns on a fixed pair
    m = 33 * 64
    a2 = np.repeat(rng.uniform(0.1, 1.9, 64).astype(np.float32), 33)
    b2 = np.repeat(rng.uniform(0.1, 1.9, 64).astype(np.float32), 33)
    r2 = np.tile(np.array([0] + [1 << k for k in range(32)], dtype=np.uint32), 64)
    A, B, R = (np.concatenate([x, y]) for x, y in ((a, a2), (b, b2), (r, r2)))
    N = len(A)
    ta, tb, tr = (torch.from_numpy(x).cuda() for x in (A, B, R.view(np.int32)))
    to = torch.empty(N, dtype=torch.int32, device="cuda")
    import ctypes
    args = [ctypes.c_void_p(t.data_ptr()) for t in (ta, tb, tr, to)] + [ctypes.c_int(N)]
    ptrs = (ctypes.c_void_p * len(args))(*[ctypes.cast(ctypes.pointer(x), ctypes.c_void_p) for x in args])
    drv.cuLaunchKernel(fn, (N + 255) // 256, 1, 1, 256, 1, 1, 0, 0, ptrs, 0)
    torch.cuda.synchronize()
    os.makedirs("gpurun_out", exist_ok=True)
    np.savez("gpurun_out/cvt_rs_probe.npz", a=A, b=B, r=R, out=to.cpu().numpy().view(np.uint32))
    print("ok", N)


if __name__ == "__main__":
    sys.exit(main())
