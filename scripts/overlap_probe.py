"""Probe: do two row blocks of one product overlap on the GPU when issued from two host threads
on two streams (each tsg_spgemm call on its own stream)?  Prints sequential vs concurrent time."""
import sys, threading, time, json
import numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg
from paper_conf_ppopp_niuljs0022_b200 import dist as tdist
from workloads import gen

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
K = int(sys.argv[2]) if len(sys.argv) > 2 else 2
A = gen.config(cfg)
T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(), torch.from_numpy(A.val).cuda(), (A.m, A.n))
cuts = tdist.partition_device(T, T, K)
blocks = [tsg.slice_rows(T, int(cuts[b]), int(cuts[b + 1])) for b in range(K)]
streams = [torch.cuda.Stream() for _ in range(K)]

def one(b, out):
    with torch.cuda.stream(streams[b]):
        out[b] = tsg.spgemm(blocks[b], T, stream=streams[b])

def seq():
    out = [None] * K
    for b in range(K):
        one(b, out)
    torch.cuda.synchronize()
    return out

from concurrent.futures import ThreadPoolExecutor
pool = ThreadPoolExecutor(max_workers=K)  # long-lived threads: each keeps its scratch arena

def conc():
    out = [None] * K
    futs = [pool.submit(one, b, out) for b in range(K)]
    for f in futs: f.result()
    torch.cuda.synchronize()
    return out

for f in (seq, conc):
    for _ in range(3): f()
res = {}
for name, f in (("seq", seq), ("conc", conc), ("seq2", seq), ("conc2", conc)):
    ts = []
    for _ in range(10):
        torch.cuda.synchronize(); t0 = time.perf_counter(); o = f(); ts.append((time.perf_counter() - t0) * 1e3); del o
    res[name] = round(float(np.median(ts)), 3)
full = []
for _ in range(10):
    torch.cuda.synchronize(); t0 = time.perf_counter(); C = tsg.spgemm(T, T); torch.cuda.synchronize(); full.append((time.perf_counter() - t0) * 1e3); del C
res["one_call"] = round(float(np.median(full)), 3)
print(json.dumps({"config": cfg, "blocks": K, "wall_ms": res}))
