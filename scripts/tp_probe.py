import sys, time, torch; sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg
from workloads import gen
for cfg in ("C4", "C2"):
    A = gen.config(cfg)
    T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(), torch.from_numpy(A.val).cuda(), (A.m, A.n))
    for _ in range(2): TT = tsg.transpose(T)
    torch.cuda.synchronize(); t0 = time.perf_counter(); TT = tsg.transpose(T); torch.cuda.synchronize(); print(cfg, "transpose ms", round((time.perf_counter() - t0) * 1e3, 3), TT.num_tiles)
