"""GPU: every SPADEN_TILE_CFG in argv gives bitwise the same y (and matches the
fp64 oracle) on a few matrices; prints one line per cfg.  Experiment harness."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import workloads as W  # noqa: E402

cfgs = [int(c) for c in sys.argv[1].split(",")]
mats = [("fem62k", W.make("fem62k")), ("pl14", W.powerlaw(14, 6, seed=1)), ("rand", W.random_sparse(3000, 2900, 0.01, 3)),
        ("fem_small", W.fem(6, 7, 8, seed=2))]
dev = torch.device("cuda:0")
ref = {}
for cfg in cfgs:
    os.environ["SPADEN_TILE_CFG"] = str(cfg)
    import paper_conf_icpp_cheny24_b200 as sp
    out = []
    for name, A in mats:
        for storage in ("fp32", "fp16"):
            M = sp.convert(torch.from_numpy(A.rowptr).to(dev), torch.from_numpy(A.colidx).to(dev),
                           torch.from_numpy(A.values).to(dev), A.n, storage=storage)
            x = W.vector(A.n, 2)
            y = M.spmv(torch.from_numpy(x).to(dev)).cpu().numpy()
            vals = A.values if storage == "fp32" else oracle.f32_to_f16(A.values)
            ys, s = oracle.spmv(A.rowptr, A.colidx, vals, x)
            err = oracle.componentwise_error(y, ys, s)
            key = (name, storage)
            same = None
            if key in ref:
                same = bool(np.array_equal(ref[key].view(np.uint32), y.view(np.uint32)))
            else:
                ref[key] = y
            out.append(f"{name}/{storage}: err={err:.2e} same={same} tiles={M.info.n_tiles} long={M.info.n_long}")
            assert err <= 1e-5, (cfg, key, err)
            assert same in (None, True), (cfg, key)
            M.free()
    print(cfg, " | ".join(out), flush=True)
print("cfg_check ok")
