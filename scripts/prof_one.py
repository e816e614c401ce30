"""One warm tsg_spgemm call inside a cudaProfilerStart/Stop region (for ncu --profile-from-start off).
usage: python scripts/prof_one.py C2 '{"med_warp": true}'"""
import json
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg  # noqa: E402
from workloads import gen  # noqa: E402

cfg = sys.argv[1]
opts = json.loads(sys.argv[2]) if len(sys.argv) > 2 else {}
A = gen.config(cfg)
T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(),
                     torch.from_numpy(A.val).cuda(), (A.m, A.n))
for _ in range(2):
    C = tsg.spgemm(T, T, **opts)
    del C
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
C = tsg.spgemm(T, T, **opts)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print("ok", C.num_tiles)
