"""Probe: time tsg_spgemm under several option sets on one config and check they give the same C.

usage: python scripts/variant_probe.py C2 '{"med_warp": false}' '{"med_warp": true}' ...
Per option set: median of 10 production calls (CUDA events, no stats) and the step times of an
instrumented call; every option set's C is compared array by array with the first one's."""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg  # noqa: E402
from workloads import gen  # noqa: E402

cfg = sys.argv[1]
variants = [json.loads(a) for a in sys.argv[2:]] or [{}]
A = gen.config(cfg)
T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(),
                     torch.from_numpy(A.val).cuda(), (A.m, A.n))
ARR = ("tile_ptr", "tile_col", "tile_nnz", "row_ptr", "mask", "idx", "val")


def arrays(C):
    return {k: getattr(C, k).clone() for k in ARR}


base = None
out = []
for opts in variants:
    for _ in range(3):
        C = tsg.spgemm(T, T, **opts)
        del C
    ts = []
    for _ in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        C = tsg.spgemm(T, T, **opts)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        del C
    Ci = tsg.spgemm(T, T, stats=True, timing=True, **opts)
    st = Ci.stats
    same = None
    try:
        cur = arrays(Ci)
        if base is None:
            base = cur
        else:
            same = all(torch.equal(base[k], cur[k]) for k in ARR)
    except Exception as e:  # noqa: BLE001
        same = f"compare failed: {e}"
    out.append({"opts": opts, "ms": round(float(np.median(ts)), 4),
                "step_ms": {k: round(v, 4) for k, v in st.items() if isinstance(v, float)},
                "same_as_first": same})
    del Ci
print(json.dumps({"config": cfg, "results": out}))
