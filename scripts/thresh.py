"""Time tsg_spgemm (C = A^2) for several dense thresholds t_nnz (results are identical; only the
accumulator class split changes).  Usage: python scripts/thresh.py C3 64 128 192 257"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_niuljs0022_b200 as tsg
from workloads import gen

cfg = sys.argv[1]
A = gen.config(cfg)
dev = torch.device("cuda")
T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).to(dev), torch.from_numpy(A.col).to(dev),
                     torch.from_numpy(A.val).to(dev), (A.m, A.n))
for th in [int(x) for x in sys.argv[2:]]:
    for _ in range(3):
        C = tsg.spgemm(T, T, dense_threshold=th); del C
    ms = []
    for _ in range(5):
        C = tsg.spgemm(T, T, stats=True, timing=True, dense_threshold=th)
        ms.append((C.stats["ms_total"], C.stats["ms_step2"], C.stats["ms_step3"], C.stats["tiles_dense"]))
        del C
    ms.sort()
    print(cfg, "t_nnz", th, "total/step2/step3 ms, dense tiles", ms[len(ms) // 2], flush=True)
