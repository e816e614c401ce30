"""Warm per-kernel GPU times of tsg_spgemm on one config (torch.profiler / CUPTI, back-to-back
production calls): where the time of a call goes, kernel by kernel.
usage: python scripts/kernel_times.py C2 [opts-json] [shards]
shards = N: the first shard of the N-way device partition times the full matrix (a rank's call in
the N-GPU run)."""
import json
import sys

import torch
from torch.profiler import ProfilerActivity, profile

sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg  # noqa: E402
from workloads import gen  # noqa: E402

cfg = sys.argv[1]
opts = json.loads(sys.argv[2]) if len(sys.argv) > 2 else {}
A = gen.config(cfg)
T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(),
                     torch.from_numpy(A.val).cuda(), (A.m, A.n))
L = T
if len(sys.argv) > 3 and int(sys.argv[3]) > 1:
    from paper_conf_ppopp_niuljs0022_b200 import dist as tdist
    cuts = tdist.partition_device(T, T, int(sys.argv[3]))
    L = tsg.slice_rows(T, int(cuts[0]), int(cuts[1]))
for _ in range(3):
    C = tsg.spgemm(L, T, **opts)
    del C
torch.cuda.synchronize()
N = 5
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for _ in range(N):
        C = tsg.spgemm(L, T, **opts)
        del C
    torch.cuda.synchronize()
rows = []
for e in prof.key_averages():
    if e.device_type is not None and "k_" in e.key and e.self_device_time_total > 0:
        import re
        m = re.search(r"(k_\w+(<[^>]*>)?)", e.key)
        rows.append((e.self_device_time_total / N, e.count / N, (m.group(1) if m else e.key)[:60]))
rows.sort(reverse=True)
tot = sum(r[0] for r in rows)
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
ts = []
for _ in range(10):
    ev0.record(); C = tsg.spgemm(L, T, **opts); ev1.record(); ev1.synchronize(); ts.append(ev0.elapsed_time(ev1)); del C
ts.sort()
print(f"{cfg} shards={sys.argv[3] if len(sys.argv) > 3 else 1}: call {ts[len(ts) // 2]:.3f} ms, kernel time per call {tot / 1000:.3f} ms")
for us, cnt, name in rows:
    print(f"{us:10.1f} us  x{cnt:4.1f}  {100 * us / tot:5.1f}%  {name}")
