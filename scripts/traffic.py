"""DRAM traffic per step of one tsg_spgemm call (the roofline's `traffic` field, bench.py).

Run under ncu with the capture limited to one warm call:
    ncu --profile-from-start off --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
        --csv --log-file gpurun_out/traffic_C2.csv python scripts/traffic.py C2
then `python scripts/traffic.py --summarize gpurun_out/traffic_C2.csv C2` writes
profiles/traffic_r02_C2.json: bytes per step (launches up to the scan that exports the first
blocking read = step 1 (a0 + a1), up to the second = step 2 (a2 + a3), after it = step 3 (a4))."""
import csv, json, os, sys

if len(sys.argv) > 1 and sys.argv[1] == "--summarize":
    path, cfg = sys.argv[2], sys.argv[3]
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    ii = h.index("ID")
    per = {}
    for r in rows[hi + 1:]:
        if len(r) < len(h):
            continue
        d = per.setdefault(int(r[ii]), {"name": r[ki]})
        d[r[mi]] = float(r[vi].replace(",", ""))
    # a step ends with the scan that exports its blocking read: the first k_scan_1pass after the
    # step's own kernels (step 1: the row kernels; step 2: the symbolic kernels)
    ends = {1: ("k_row_merge", "k_row_small", "k_row_rank", "k_row_big"), 2: ("k_s2", "k_s2_light", "k_sym_rows")}
    step, seen, out, kern = 1, False, {"step1": 0.0, "step2": 0.0, "step3": 0.0}, {}
    for i in sorted(per):
        d = per[i]
        b = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
        out[f"step{step}"] += b
        name = d["name"].split("(")[0].split("::")[-1].split("<")[0].strip()
        kern.setdefault(f"step{step}", {}).setdefault(d["name"].split("(")[0].split("::")[-1], 0.0)
        kern[f"step{step}"][d["name"].split("(")[0].split("::")[-1]] += b
        if step < 3 and name in ends[step]:
            seen = True
        elif step < 3 and seen and name == "k_scan_1pass":
            step, seen = step + 1, False
    out = {k: int(v) for k, v in out.items()}
    out["unit"] = "bytes (dram__bytes_read.sum + dram__bytes_write.sum) per call, one warm call, ncu"
    out["per_kernel"] = {s: {k: int(v) for k, v in m.items()} for s, m in kern.items()}
    dst = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles",
                       f"traffic_r02_{cfg}.json")
    json.dump(out, open(dst, "w"), indent=1)
    print(json.dumps(out))
    sys.exit(0)

import numpy as np
import torch
sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg
from workloads import gen

A = gen.config(sys.argv[1] if len(sys.argv) > 1 else "C2")
T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(),
                     torch.from_numpy(A.val).cuda(), (A.m, A.n))
for _ in range(3):
    C = tsg.spgemm(T, T)
    del C
torch.cuda.synchronize()
torch.cuda.profiler.start()
C = tsg.spgemm(T, T)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("calls done", C.num_tiles, C.nnz)
