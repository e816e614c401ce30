"""usage: python scripts/shard_probe.py CONFIG [N1,N2,...]

Predict strong scaling of the sharded C = A^2 on one GPU: time tsg_spgemm(slice_rows(A, I_g,
I_g+1), A) for every shard g of an N-way product-balanced tile-row partition and report the
max over g (what the N-GPU step would take with B resident, C left sharded)."""
import sys, json
import numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg
from paper_conf_ppopp_niuljs0022_b200 import dist as tdist
from workloads import gen

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
NS = [int(x) for x in sys.argv[2].split(',')] if len(sys.argv) > 2 else [1, 2, 4, 8]
A = gen.config(cfg)
T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(),
                     torch.from_numpy(A.val).cuda(), (A.m, A.n))
s = torch.cuda.current_stream()
out = {}
for N in NS:
    cuts = tdist.partition_device(T, T, N)
    per = []
    for g in range(N):
        Ag = tsg.slice_rows(T, int(cuts[g]), int(cuts[g + 1])) if N > 1 else T
        for _ in range(2):
            C = tsg.spgemm(Ag, T); del C
        ts = []
        for _ in range(5):
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(s); C = tsg.spgemm(Ag, T); e1.record(s); e1.synchronize(); ts.append(e0.elapsed_time(e1)); del C
        per.append(float(np.median(ts)))
    out[N] = {"max_ms": max(per), "min_ms": min(per), "sum_ms": sum(per), "speedup_vs_1": None,
              "per_shard_ms": [round(x, 3) for x in per]}
# one GPU = every shard of the first partition computed in turn (C5 needs >= 4 blocks on one GPU)
base = out[NS[0]]["sum_ms"]
for N in out:
    out[N]["speedup_vs_1"] = base / out[N]["max_ms"]
print(json.dumps(out, indent=1))
