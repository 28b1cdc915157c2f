#!/usr/bin/env python3
"""PCIe probe for the e2e path: pinned H2D / D2H of 1 GiB, alone and together,
contiguous and as the interior box (504 of 512 columns, 504 of 512 rows) of a
512^3 grid via cudaMemcpy3DAsync (torch strided copy to a pinned view)."""
import json
import time

import torch

n = 512
N = n * n * n
h_in = torch.empty(N, dtype=torch.float64).pin_memory()
h_out = torch.empty(N, dtype=torch.float64).pin_memory()
d_a = torch.empty(N, dtype=torch.float64, device="cuda")
d_b = torch.empty(N, dtype=torch.float64, device="cuda")
s_up, s_dn = torch.cuda.Stream(), torch.cuda.Stream()
B = N * 8


def t(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


res = {}
res["h2d_GBs"] = B / t(lambda: d_a.copy_(h_in, non_blocking=True)) / 1e9
res["d2h_GBs"] = B / t(lambda: h_out.copy_(d_b, non_blocking=True)) / 1e9


def both():
    with torch.cuda.stream(s_up):
        d_a.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s_dn):
        h_out.copy_(d_b, non_blocking=True)


res["bidir_GBs_each"] = B / t(both) / 1e9
hv = h_out.view(n, n, n)[:, 4:-4, 4:-4]
dv = d_b.view(n, n, n)[:, 4:-4, 4:-4]
res["d2h_box_GBs"] = dv.numel() * 8 / t(lambda: hv.copy_(dv, non_blocking=True)) / 1e9
# chunked (16 chunks) h2d
ch = N // 16
def chunked():
    for c in range(16):
        d_a[c * ch:(c + 1) * ch].copy_(h_in[c * ch:(c + 1) * ch], non_blocking=True)
res["h2d_16chunks_GBs"] = B / t(chunked) / 1e9
print(json.dumps(res))
