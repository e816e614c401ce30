"""Break the bench's end-to-end step (C2) into H2D, conversion, SpGEMM and D2H, and measure raw
pinned-copy bandwidth both ways (diagnostic for the e2e leg of bench.py)."""
import sys, time, json
import numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg
from workloads import gen

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
A = gen.config(cfg)
s = torch.cuda.current_stream()
def ev():
    e = torch.cuda.Event(enable_timing=True); e.record(s); return e
out = {}
for nbytes in (256 << 20, 1 << 30):
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True); d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    for _ in range(2): d.copy_(h, non_blocking=True); h.copy_(d, non_blocking=True)
    torch.cuda.synchronize()
    e0 = ev(); d.copy_(h, non_blocking=True); e1 = ev(); h.copy_(d, non_blocking=True); e2 = ev(); e2.synchronize()
    out[f"h2d_GBs_{nbytes>>20}MB"] = nbytes / e0.elapsed_time(e1) / 1e6
    out[f"d2h_GBs_{nbytes>>20}MB"] = nbytes / e1.elapsed_time(e2) / 1e6
h_rp = torch.from_numpy(A.rowptr).pin_memory(); h_ci = torch.from_numpy(A.col).pin_memory(); h_v = torch.from_numpy(A.val).pin_memory()
T = tsg.csr_to_tiles(h_rp, h_ci, h_v, (A.m, A.n))
C = tsg.spgemm(T, T)
bufs = {k: torch.empty(v.numel(), dtype={torch.uint16: torch.int16}.get(v.dtype, v.dtype), pin_memory=True) for k, v in C.arrays().items()}
del C
for it in range(3):
    torch.cuda.synchronize()
    e0 = ev(); T = tsg.csr_to_tiles(h_rp, h_ci, h_v, (A.m, A.n)); e1 = ev()
    C = tsg.spgemm(T, T); e2 = ev()
    C.copy_to_host(bufs); e3 = ev(); e3.synchronize()
    out[f"it{it}"] = {"convert_incl_h2d_ms": e0.elapsed_time(e1), "spgemm_ms": e1.elapsed_time(e2), "d2h_ms": e2.elapsed_time(e3)}
    del C, T
print(json.dumps(out, indent=1))
