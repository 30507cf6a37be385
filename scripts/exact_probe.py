"""Diagnostic: where (if anywhere) the fp32-accumulating mxf4 tensor kernels stop being
exact.  Compares the tensor variant with the CUDA-core POPC variant (integer adds) at
growing K on dense random rows and prints mismatch statistics per kernel."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ipps_binderlp19_b200 as snp  # noqa: E402

torch.cuda.set_device(0)
g = torch.Generator(device="cuda").manual_seed(5)


def rows(r, k, p):
    bits = (torch.rand((r, k), generator=g, device="cuda") < p).to(torch.uint8)
    return snp.snp_pack(bits, nbits=k)


for nbits in [4096, 8193, 16385, 32769, 65537, 131073, 262145, 524289, 1048577, 4194305, 8388607]:
    for shape, (m, n) in (("fastid", (8, 600)), ("ld", (256, 256)), ("many", (80, 600))):
        A = rows(m, nbits, 0.97)
        B = A if shape == "ld" else rows(n, nbits, 0.98)
        res = {}
        for v in ("tc", "popc"):
            snp.snp_set_variant(v)
            out = snp.snp_fastid(A, B, nbits, "and")
            res[v] = out.view(torch.int32).cpu().numpy().astype(np.int64)
            res[v + "_k"] = snp.snp_last_kernel()
        snp.snp_set_variant("auto")
        d = res["tc"] - res["popc"]
        print(f"nbits={nbits:8d} {shape:6s} kern={res['tc_k']:12s} max={res['popc'].max():8d} "
              f"mismatch={int((d != 0).sum()):7d}/{d.size} maxabs={int(np.abs(d).max())}", flush=True)
