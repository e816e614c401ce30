"""C1 per-call latency: CUDA-event time of one tsg_spgemm call (median of 200) and the CUDA API
calls it makes (torch.profiler with CUPTI), to see where a small call's time goes."""
import sys, json, time
import numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg
from workloads import gen

cfg = sys.argv[1] if len(sys.argv) > 1 else "C1"
opts = {"rows": dict(path_rows=True), "tiles": dict(path_general=True), "auto": {}}[sys.argv[2] if len(sys.argv) > 2 else "auto"]
A = gen.config(cfg)
T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(), torch.from_numpy(A.val).cuda(), (A.m, A.n))
s = torch.cuda.current_stream()
for _ in range(20):
    C = tsg.spgemm(T, T, **opts)
torch.cuda.synchronize()
ts, ws = [], []
for _ in range(200):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record(s); C = tsg.spgemm(T, T, **opts); e1.record(s); e1.synchronize()
    ws.append((time.perf_counter() - t0) * 1e3)
    ts.append(e0.elapsed_time(e1)); del C
st = tsg.spgemm(T, T, stats=True, **opts).stats
res = {"config": cfg, "event_ms_median": float(np.median(ts)), "wall_ms_median": float(np.median(ws)),
       "launches": st["kernel_launches"], "host_syncs": st["host_syncs"], "path": st["path"]}
from torch.profiler import profile, ProfilerActivity
with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
    for _ in range(20):
        C = tsg.spgemm(T, T, **opts); del C
    torch.cuda.synchronize()
print(json.dumps(res))
print(prof.key_averages().table(sort_by="self_cpu_time_total", row_limit=25))
