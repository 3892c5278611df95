#!/usr/bin/env python
"""Check per-row counts of the GPU partition against the input for large nnz (GPU only)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_huangylhbl21_b200 as hc  # noqa: E402

nnz = int(float(sys.argv[1]))
m = int(float(sys.argv[2])) if len(sys.argv) > 2 else 50_082_603
n = int(float(sys.argv[3])) if len(sys.argv) > 3 else 39_780
dev = "cuda:0"
(du, dv, dr), _ = synth.powerlaw_device(m, n, nnz, 5, n_test=1, device=dev)
mdl = hc.Model(m, n, 128)
torch.cuda.synchronize()
mdl.load(du, dv, dr)
del dv, dr
torch.cuda.empty_cache()
mdl.partition(1, (1, 1), seed=5)
b, off, pr, pc = mdl.get_partition()
prt = torch.from_numpy(pr).to(dev)
want = torch.zeros(m, dtype=torch.int64, device=dev)
for lo in range(0, nnz, 1 << 29):
    want += torch.bincount(prt[du[lo:lo + (1 << 29)].long()].long(), minlength=m)
del du
torch.cuda.empty_cache()
su = torch.empty(nnz, dtype=torch.int32, device=dev)
mdl._check(hc.lib().hccmf_get_records(mdl._h, su.data_ptr(), None, None))
got = torch.zeros(m, dtype=torch.int64, device=dev)
for lo in range(0, nnz, 1 << 29):
    got += torch.bincount(su[lo:lo + (1 << 29)].long(), minlength=m)
sorted_ok = bool((su[1:] >= su[:-1]).all())
diff = (got != want).nonzero().flatten()
print(f"nnz={nnz} sum got {int(got.sum())} want {int(want.sum())} sorted {sorted_ok} rows differing {diff.numel()}",
      flush=True)
if diff.numel():
    i = int(diff[0])
    print("first row", i, int(got[i]), int(want[i]))
    # where do the rows start in su?
    print("boundary positions of the first differing row", int((su < i).sum()), int((su <= i).sum()))
