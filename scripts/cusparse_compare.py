#!/usr/bin/env python
"""The paper's Table 6 on B200 (MemXCT vs the vendor sparse library): the same
memoized matrices, exported from the plan (memxct_export_coo), as 32-bit-index CSR handed to
cuSPARSE through torch (torch.mv on a sparse CSR tensor -> cusparseSpMV), against our staged
SpMV (memxct_spmv_time).  Rows and columns in natural order (what a library user would build)
and in the plan's two-level Hilbert order (the paper's "+Hilbert" column).  Also checks that
cuSPARSE computes the same products (relative L2 vs our kernel).

    python scripts/cusparse_compare.py --configs 2,3 [--reps 10]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def csr_from_coo(r, c, v, nrows):
    import torch
    keep = r >= 0
    r, c, v = r[keep], c[keep], v[keep]
    key = r.long() * (1 << 31) + c.long()
    del keep
    order = torch.argsort(key)
    del key
    r, c, v = r[order], c[order], v[order]
    del order
    counts = torch.bincount(r.long(), minlength=nrows)
    crow = torch.zeros(nrows + 1, dtype=torch.int64, device=r.device)
    crow[1:] = torch.cumsum(counts, 0)
    del r, counts
    return crow.int(), c, v


def timed(fn, reps):
    import torch
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="2,3")
    ap.add_argument("--orders", default="natural,plan")
    ap.add_argument("--reps", type=int, default=10)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_hidayetoglubgrg19_b200 import MemXCT, inputs
    for cfg in map(int, a.configs.split(",")):
        n, m, c = inputs.CONFIGS[cfg]
        for vo in a.orders.split(","):
            plan = MemXCT(n, m, c, vector_order=vo).build()
            ours = plan.spmv_time(a.reps)
            nnz = plan.stats()["nnz"]
            res = {"config": cfg, "order": vo, "nnz": nnz, "ours_fwd_ms": ours["fwd_us"] / 1e3,
                   "ours_back_ms": ours["back_us"] / 1e3}
            for d, (nr, nc) in ((0, (m * c, n * n)), (1, (n * n, m * c))):
                crow, col, val = csr_from_coo(*plan.export_coo(d), nr)
                A = torch.sparse_csr_tensor(crow, col, val, size=(nr, nc))
                x = torch.rand(nc, device="cuda")
                t = timed(lambda: torch.mv(A, x), a.reps)
                y = torch.mv(A, x)
                ref = plan.forward(x) if d == 0 else plan.back(x)
                err = float(torch.linalg.vector_norm((y - ref).double()) / torch.linalg.vector_norm(ref.double()))
                name = "fwd" if d == 0 else "back"
                res[f"cusparse_{name}_ms"] = t
                res[f"cusparse_{name}_rel_l2_vs_ours"] = err
                res[f"speedup_{name}"] = t / res[f"ours_{name}_ms"]
                res[f"cusparse_{name}_gflops"] = 2 * nnz / (t * 1e6)
                res[f"cusparse_{name}_csr_gbs"] = (8 * nnz + 4 * (nr + 1) + 4 * nr) / (t * 1e6)
                del A, crow, col, val, x, y, ref
                torch.cuda.empty_cache()
            print(json.dumps(res), flush=True)
            plan.close()
            del plan
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
