#!/usr/bin/env python
"""Benchmark of the TileSpGEMM hot path: fp64 C = A^2 GFLOPS (2 x products / time) on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl tsg|reference]

One step = one tsg_spgemm call (steps 1-3 of Section 3.3 plus all allocation, the paper's timed
region P:2969-2986), inputs resident in HBM, timed with CUDA events on the launching stream,
max over ranks.  The default workload is C2 stencil27-128 (BASELINE.json configs[1]); its
inputs (A: ~0.7 GB in tile form) are larger than the 126 MB L2, so no flush is needed; smaller
configs flush L2 with a 512 MB write between timed steps (outside the events).

Prints ONE JSON line (rank 0).  ``--impl reference`` times the CPU oracle (the reference arm of
this tier) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "fp64 C=A^2 GFLOPS (2×products/time) at 1/2/4/8 B200; % HBM roofline"
UNIT = "GFLOPS"
L2_BYTES = 126 * 2 ** 20
ROW_BLOCKS = {"C5": 4}
E2E_BLOCKS = int(os.environ.get("TSG_E2E_BLOCKS", "4"))  # tile-row blocks of the e2e leg when C fits the pinned host buffer
E2E_PINNED_MAX = 24 * 2 ** 30  # bytes of pinned host memory the e2e leg may use for C
VDT = {"f64": np.float64, "f32": np.float32, "f16": np.float16}  # tile-row blocks per step on one GPU (C5's C is ~144 GB in tile form)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def tile_bytes(tm, ntiles, nnz, vbytes=8):
    """S(M) = 8(tm+1) + 60*tiles + (1 + value bytes)*nnz  (9*nnz for fp64)."""
    return 8 * (tm + 1) + 60 * ntiles + (1 + vbytes) * nnz


class ClockSampler:
    """nvidia-smi sampled every 200 ms while the timed region runs (B200_PROFILING.md clocks line)."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None
        time.sleep(0.3)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx = max(mx, float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


def oracle_baseline(A, budget_s: float = 12.0, max_rows=None, B=None, prec: str = "f64", with_omp: bool = False):
    """The oracle as it stands (single thread) on a bounded row sample of A*B (B = A by default)."""
    import oracle

    oracle.build()
    B = A if B is None else B
    m = A.m
    # calibrate on a small row block, then size the sample to ~budget_s seconds
    probe = np.arange(0, min(m, 256), dtype=np.int64)
    t0 = time.perf_counter()
    oracle.spgemm(A, B, rows=probe, prec=prec)
    dt = max(time.perf_counter() - t0, 1e-4)
    rows_per_s = len(probe) / dt
    R = int(min(m, max(len(probe), rows_per_s * budget_s)))
    if max_rows:
        R = min(R, max_rows)
    rows = np.arange(0, R, dtype=np.int64)
    sub = gen_row_block(A, R)
    prods = oracle.products(sub, B)
    t0 = time.perf_counter()
    C = oracle.spgemm(A, B, rows=rows, prec=prec)
    el = time.perf_counter() - t0
    omp = None
    if with_omp and prec == "f64":  # SURVEY 8(d) oracle_omp: the same code over row chunks, all host cores
        nt = os.cpu_count() or 1
        t0 = time.perf_counter()
        oracle.spgemm(A, B, rows=rows, prec=prec, threads=nt)
        eo = time.perf_counter() - t0
        omp = {"value": 2.0 * prods / eo / 1e9, "unit": UNIT, "threads": nt, "seconds": round(eo, 3)}
    return {"value": 2.0 * prods / el / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle", "oracle_omp": omp,
            "sample": f"rows [0,{R}) of {m} ({prods} products, nnz {C.nnz}), single-threaded C Gustavson "
                      f"(oracle/tsg_oracle.c), {el:.2f} s", "seconds": el, "products": int(prods),
            "host_cores": os.cpu_count(), "cpu_model": _cpu_model(), "_C": C}


def sample_parity(tsg, T, Bt, C_ref, tol: float = 1e-12):
    """The GPU result on the oracle's row sample (rows [0, R) of C = A*B, the tile rows covering them
    multiplied by the same kernels): CSR structure bit for bit, values within tol * sum|a*b|."""
    R = C_ref.m
    tr = (R + 15) // 16
    Ab = tsg.slice_rows(T, 0, tr) if tr != T.tile_m else T
    Cg = tsg.spgemm(Ab, Bt)
    rp, ci, v = (x.cpu().numpy() for x in tsg.tiles_to_csr(Cg))
    del Cg, Ab
    rp = rp[:R + 1]
    nz = int(rp[-1])
    structure_ok = bool(np.array_equal(rp, C_ref.rowptr) and np.array_equal(ci[:nz], C_ref.col))
    err = None
    ok = False
    if structure_ok:
        d = np.abs(v[:nz].astype(np.float64) - C_ref.val.astype(np.float64))
        bound = tol * C_ref.abs
        ok = bool(np.all(d <= bound))
        err = float(np.max(d / np.where(C_ref.abs > 0, C_ref.abs, 1.0))) if nz else 0.0
    return {"rows": int(R), "nnz": nz, "structure_ok": structure_ok, "max_rel_err": err,
            "within_tolerance": ok,
            "tolerance": f"|c - c_ref| <= {tol:g} * sum|a*b| per entry" +
                         (" (north_star)" if tol <= 1e-12 else " (fp32 accumulation, reading D1)")}


def gen_row_block(A, R):
    from workloads import gen

    return gen.row_block(A, 0, R)


def run_reference(args):
    """--impl reference: the CPU oracle timed as it stands on bounded samples of the workload."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    from workloads import gen

    A = gen.config(args.config)
    if args.dtype != "f64":
        A = gen.CSR(A.m, A.n, A.rowptr, A.col, A.val.astype(VDT[args.dtype]), A.name)
    prec = "f64" if args.dtype == "f64" else "f32"
    B = _csr_transpose(A) if args.aat else A
    for _ in range(args.warmup):
        oracle_baseline(A, budget_s=2.0, B=B, prec=prec)
    vals, secs, prods = [], 0.0, 0
    last = None
    for _ in range(args.steps):
        last = oracle_baseline(A, budget_s=args.ref_step_s, B=B, prec=prec)
        vals.append(last["value"])
        secs += last["seconds"]
        prods += last["products"]
    value = 2.0 * prods / secs / 1e9
    line = {"impl": "reference", "metric": _metric(args), "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / max(args.steps, 1),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": {"f64": "f64", "f32": "f32", "f16": "f16 in, f32 accumulate/out"}[args.dtype], "data": "synthetic",
            "config": {"workload": f"{args.config} {gen.CONFIGS[args.config][0]}" + (", C = A*A^T" if args.aat else ""),
                       "n": A.m, "nnz_a": A.nnz},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": last["sample"]},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def _non_json(o, path="line"):
    """Paths of values json cannot encode (a stray tensor in the bench line)."""
    if isinstance(o, dict):
        return [p for k, v in o.items() for p in _non_json(v, f"{path}.{k}")]
    if isinstance(o, (list, tuple)):
        return [p for i, v in enumerate(o) for p in _non_json(v, f"{path}[{i}]")]
    return [] if o is None or isinstance(o, (str, int, float, bool)) else [f"{path}: {type(o).__name__}"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--impl", default="tsg", choices=["tsg", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget-s", type=float, default=12.0)
    ap.add_argument("--ref-step-s", type=float, default=6.0)
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no clocks/baseline/e2e)")
    ap.add_argument("--path", default="auto", choices=["auto", "rows", "tiles"],
                    help="pipeline: the library's dispatch (auto), the fused per-tile-row path wherever every "
                         "tile row is narrow (rows), or the per-C-tile path (tiles); same C either way")
    ap.add_argument("--aat", action="store_true",
                    help="C = A * A^T (the paper's second workload, SURVEY f1); A^T is formed once with "
                         "tsg_tiles_transpose outside the timed region, like the CSR->tile conversion")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32", "f16"],
                    help="value type (SURVEY f3): f64 (BASELINE's metric), f32, or f16 inputs with f32 "
                         "accumulation/output (the paper's Section 4.7 setup, P:3143-3152)")
    ap.add_argument("--row-blocks", type=int, default=0,
                    help="compute each rank's C in this many tile-row blocks, one after the other (0 = "
                         "config default: C5 needs 4 on one GPU, its C alone is ~144 GB in tile form)")
    args = ap.parse_args()
    if args.warmup < 3 and not args.profile:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)

    import torch

    import paper_conf_ppopp_niuljs0022_b200 as tsg
    from workloads import gen

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    # one process per GPU; ranks beyond the visible GPUs share them (functional checks of the
    # multi-rank path on a 1-GPU box with TSG_DIST_BACKEND=gloo -- not a measurement)
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist = None
    if world > 1:
        import torch.distributed as dist

        backend = os.environ.get("TSG_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)

    A = gen.config(args.config)
    if args.dtype != "f64":
        A = gen.CSR(A.m, A.n, A.rowptr, A.col, A.val.astype(VDT[args.dtype]), A.name)
    vb = np.dtype(VDT[args.dtype]).itemsize  # value bytes of A and B
    cb = 8 if args.dtype == "f64" else 4     # value bytes of C
    stream = torch.cuda.current_stream()
    T = tsg.csr_to_tiles(torch.from_numpy(A.rowptr).to(dev), torch.from_numpy(A.col).to(dev),
                         torch.from_numpy(A.val).to(dev), (A.m, A.n))
    # the right operand: A itself (C = A^2, BASELINE's metric) or A^T (C = A A^T)
    Bt = tsg.transpose(T) if args.aat else T
    Bcsr = _csr_transpose(A) if args.aat else A
    # shard C tile rows across ranks (strong scaling of one matrix), and within a
    # rank optionally into row blocks computed one after the other (C does not fit otherwise)
    # row blocks per rank: a config whose C does not fit one GPU in one call (C5) is computed in
    # blocks; ranks sharing a GPU (functional multi-rank runs on one box) share its memory too
    ranks_per_gpu = -(-world // max(1, torch.cuda.device_count()))
    K = args.row_blocks or max(1, -(-ROW_BLOCKS.get(args.config, 1) * ranks_per_gpu // world))
    from paper_conf_ppopp_niuljs0022_b200 import dist as tdist

    # product-balanced cuts computed by the library on the device (tsg_partition_tile_rows)
    cuts = tdist.partition_device(T, Bt, world * K)
    blocks = [(int(cuts[rank * K + b]), int(cuts[rank * K + b + 1])) for b in range(K)]
    I0, I1 = blocks[0][0], blocks[-1][1]
    shards = [tsg.slice_rows(T, b0, b1) if (b0, b1) != (0, T.tile_m) else T for b0, b1 in blocks]
    Ashard = tsg.slice_rows(T, I0, I1) if (I0, I1) != (0, T.tile_m) else T

    popts = {"auto": {}, "rows": dict(path_rows=True), "tiles": dict(path_general=True)}[args.path]

    def run_blocks(stats=False, timing=False, products=False):
        """One step: C = A_shard * B block by block (the production call: no stats unless asked);
        returns the summed stats of the blocks (None without stats)."""
        tot = None
        for Ab in shards:
            C = tsg.spgemm(Ab, Bt, stats=stats or timing or products, timing=timing, products=products,
                           structural=products, **popts)
            if C.stats is not None:
                tot = tot or {}
                for k, v in C.stats.items():
                    tot[k] = tot.get(k, 0) + v
            del C
        return tot

    # one instrumented call for the exact counts (products and |C'| are properties of the input)
    st0 = run_blocks(products=True)
    small_inputs = tile_bytes(T.tile_m, T.num_tiles, T.nnz) < 2 * L2_BYTES
    flush = torch.empty(512 * 2 ** 20, dtype=torch.uint8, device=dev) if small_inputs else None

    for _ in range(args.warmup):
        run_blocks()
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    launches0 = tsg.kernel_launch_count()
    step_ms = []
    with ClockSampler(local) if not args.profile else _Null() as clk:
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
        for _ in range(args.steps):
            if flush is not None:
                flush.fill_(1)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            run_blocks()  # the production call: no stats, no per-step events
            e1.record(stream)
            e1.synchronize()
            step_ms.append(e0.elapsed_time(e1))
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
    launches = tsg.kernel_launch_count() - launches0
    # per-step times (library-recorded CUDA events on the launching stream) from instrumented calls
    # after the timed loop, medians
    s1_ms, s2_ms, s3_ms, sa_ms, host_ms = [], [], [], [], []
    stats_last = None
    for _ in range(max(3, min(args.steps, 10))):
        if flush is not None:
            flush.fill_(1)
        st = run_blocks(timing=True)
        s1_ms.append(st["ms_step1"] + st["ms_index"])
        s2_ms.append(st["ms_step2"])
        s3_ms.append(st["ms_step3"])
        sa_ms.append(st["ms_alloc"])
        host_ms.append((st["ms_host_sync"], st["ms_host_alloc"]))
        stats_last = st
    local_ms = float(np.median(step_ms))
    ms = local_ms
    prods_local = st0["products"]
    prods = prods_local
    if dist:
        t = torch.tensor([local_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        p = torch.tensor([prods_local], dtype=torch.int64, device=dev)
        dist.all_reduce(p)
        prods = int(p.item())
    value = 2.0 * prods / (ms / 1e3) / 1e9

    # the collectives around the sharded step, measured next to it (not in the
    # metric: B is resident and C stays sharded): broadcast of B's seven arrays from rank 0 and the
    # uneven all-gather + rebasing of the C shards into the full C on every rank
    multi = None
    if dist:
        def timed(fn, reps=3):
            ts = []
            for _ in range(reps):
                dist.barrier()
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                fn()
                e1.record(stream)
                e1.synchronize()
                t = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                ts.append(float(t.item()))
            return float(np.median(ts))

        meta = (Bt.m, Bt.n, Bt.num_tiles, Bt.nnz, Bt.val.dtype)
        t_b = timed(lambda: tdist.broadcast_tiles(Bt.arrays() if rank == 0 else None, meta if rank == 0 else None,
                                                  0, dev))
        # reassembly: count-exact gatherv of the C shards to rank 0 when the full C fits there
        # (next to the step, not in the metric); otherwise C stays distributed (C5: ~144 GB)
        t_r, where = None, "left distributed (each rank owns its tile rows)"
        if K == 1:
            Cl = tsg.spgemm(shards[0], Bt)
            c_bytes = torch.tensor([sum(v.numel() * v.element_size() for v in Cl.arrays().values())],
                                   dtype=torch.int64, device=dev)
            dist.all_reduce(c_bytes)
            free = torch.tensor([torch.cuda.mem_get_info(dev)[0] // ranks_per_gpu], dtype=torch.int64, device=dev)
            dist.all_reduce(free, op=dist.ReduceOp.MIN)
            if int(c_bytes.item()) < 0.6 * int(free.item()):
                t_r = timed(lambda: tdist.gatherv_tiles(Cl, 0), reps=2)
                where = f"gatherv to rank 0 ({int(c_bytes.item()) / 1e9:.2f} GB, count-exact point-to-point)"
            else:
                where = (f"left distributed: C is {int(c_bytes.item()) / 1e9:.1f} GB, more than 60% of a rank's free "
                         "device memory")
            del Cl
        multi = {"t_bcast_ms": t_b, "bcast_bytes": int(sum(v.numel() * v.element_size() for v in Bt.arrays().values())),
                 "t_reassemble_ms": t_r, "reassembly": where, "partition": "device (tsg_partition_tile_rows)",
                 "row_blocks_per_rank": K, "ranks_per_gpu": ranks_per_gpu,
                 "backend": os.environ.get("TSG_DIST_BACKEND", "nccl"),
                 "note": "not in the metric: B resident, C left sharded (SURVEY 8(e))"}

    # roofline of the dominant kernel (step 3 numeric unless another step is longer)
    bw, bw_src = peaks()
    nnzC, ntC = stats_last["nnz_c"], stats_last["tiles_c"]
    steps_ms = {"step1": float(np.median(s1_ms)), "step2": float(np.median(s2_ms)), "step3": float(np.median(s3_ms))}
    alloc_ms = float(np.median(sa_ms))
    alg = {  # algorithmic bytes per launch of each step's kernels
        # (B is read once per row block; value bytes vb for A and B, cb for C)
        "step1": 4 * Ashard.num_tiles + 8 * (Ashard.tile_m + 1) + K * (6 * Bt.num_tiles + 8 * (Bt.tile_m + 1)) + 12 * ntC,
        "step2": 32 * (Ashard.num_tiles + K * Bt.num_tiles) + 60 * ntC,
        "step3": (1 + vb) * (Ashard.nnz + K * Bt.nnz) + (1 + cb) * nnzC + 48 * (Ashard.num_tiles + K * Bt.num_tiles)
                 + 56 * ntC,
    }
    if int(stats_last["path"]) == len(shards):  # the row path: "step2" is the fused step-1 merge + step-2 masks
        alg["step2"] += alg["step1"]
        alg["step1"] = 12 * Ashard.num_tiles + 8 * (Ashard.tile_m + 1)  # the plan: tile columns, costs, offsets
    dom = max(steps_ms, key=steps_ms.get)
    achieved = alg[dom] / (steps_ms[dom] / 1e3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", f"traffic_r02_{args.config}.json")
    if os.path.exists(tp) and world == 1 and K == 1 and args.dtype == "f64" and not args.aat and args.path == "auto":
        traffic = json.load(open(tp)).get(dom)  # captured for the default single-GPU fp64 call only
    bytes_alg = tile_bytes(Ashard.tile_m, Ashard.num_tiles, Ashard.nnz, vb) + \
        K * tile_bytes(Bt.tile_m, Bt.num_tiles, Bt.nnz, vb) + tile_bytes(Ashard.tile_m, ntC, nnzC, cb)
    roof = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": bw, "unit": "GB/s",
            "frac": achieved / bw, "traffic": traffic, "algorithmic_bytes": alg[dom], "peak_source": bw_src,
            "kernel_ms": steps_ms[dom]}

    # end to end through the public API with host buffers (H2D of A's CSR, D2H of C's tile arrays).
    # C is computed in tile-row blocks; when the whole C fits a pinned host buffer the copy of block
    # b (tsg_tiles_copy_to_host_async on a second stream) overlaps the computation of block b+1.
    e2e = None
    if not args.profile and args.e2e_steps > 0:
        h_rp = torch.from_numpy(A.rowptr).pin_memory()
        h_ci = torch.from_numpy(A.col).pin_memory()
        h_v = torch.from_numpy(A.val).pin_memory()
        Ke = K if K > 1 else E2E_BLOCKS
        ecuts = tdist.partition_device(T, Bt, world * Ke)
        eblocks = [(int(ecuts[rank * Ke + b]), int(ecuts[rank * Ke + b + 1])) for b in range(Ke)]
        bsizes, bo = [], 0
        for b0, b1 in eblocks:
            Ab = tsg.slice_rows(T, b0, b1) if (b0, b1) != (0, T.tile_m) else T
            Cx = tsg.spgemm(Ab, Bt)
            bsizes.append({k: (v.numel(), _host_dtype(v)) for k, v in Cx.arrays().items()})
            bo += sum(v.numel() * v.element_size() for v in Cx.arrays().values())
            del Cx, Ab
        pipeline = 2 * bo <= E2E_PINNED_MAX  # two sets of pinned host buffers (consecutive steps)
        if pipeline:  # one pinned host destination per block, two sets (consecutive steps alternate)
            bufs2 = [[{k: torch.empty(n, dtype=dt, pin_memory=True) for k, (n, dt) in sz.items()} for sz in bsizes]
                     for _ in range(2)]
            bufs = bufs2[0]
        else:  # blocks copied one after the other into one buffer sized for the largest block
            mx = {k: max(sz[k][0] for sz in bsizes) for k in bsizes[0]}
            bufs = [{k: torch.empty(mx[k], dtype=bsizes[0][k][1], pin_memory=True) for k in mx}]
        bi = h_rp.numel() * 8 + h_ci.numel() * 4 + h_v.numel() * vb
        s_copy = torch.cuda.Stream()
        s_in = torch.cuda.Stream()  # one stream for all steps' inputs (the caching allocator pools per stream)

        def e2e_step():
            e0, ec, e1 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            e0.record(stream)
            Th = tsg.csr_to_tiles(h_rp, h_ci, h_v, (A.m, A.n))
            Bh = tsg.transpose(Th) if args.aat else Th
            ec.record(stream)
            live = []
            for i, (b0, b1) in enumerate(eblocks):
                Ah = tsg.slice_rows(Th, b0, b1) if (b0, b1) != (0, Th.tile_m) else Th
                Cx = tsg.spgemm(Ah, Bh, **popts)
                if pipeline:
                    done = torch.cuda.Event()
                    done.record(stream)
                    s_copy.wait_event(done)
                    Cx.copy_to_host(bufs[i], stream=s_copy, blocking=False)
                    live.append((Cx, Ah))  # alive until the copy stream has passed
                else:
                    Cx.copy_to_host(bufs[0])
                    del Cx, Ah
            if pipeline:
                done = torch.cuda.Event()
                done.record(s_copy)
                stream.wait_event(done)
            e1.record(stream)
            e1.synchronize()
            del live, Th, Bh
            return e0.elapsed_time(e1), e0.elapsed_time(ec)

        def e2e_stream(nsteps):
            """Steps back to back as a pipeline would run them: step s+1's H2D + conversion (on
            their own stream) overlap step s's D2H (PCIe is full duplex); every step still copies
            its own inputs in and its whole C out.  Returns the wall time of the nsteps on the device."""
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s_in)
            live, done = [None] * nsteps, [None] * nsteps
            for st in range(nsteps):
                Th = tsg.csr_to_tiles(h_rp, h_ci, h_v, (A.m, A.n), stream=s_in)
                Bh = tsg.transpose(Th, stream=s_in) if args.aat else Th
                conv = torch.cuda.Event()
                conv.record(s_in)
                stream.wait_event(conv)
                keep = [Th, Bh]
                for i, (b0, b1) in enumerate(eblocks):
                    Ah = tsg.slice_rows(Th, b0, b1) if (b0, b1) != (0, Th.tile_m) else Th
                    Cx = tsg.spgemm(Ah, Bh, **popts)
                    ev = torch.cuda.Event()
                    ev.record(stream)
                    s_copy.wait_event(ev)
                    Cx.copy_to_host(bufs2[st % 2][i], stream=s_copy, blocking=False)
                    keep += [Cx, Ah]
                done[st] = torch.cuda.Event()
                done[st].record(s_copy)
                live[st] = keep
                del Th, Bh, keep
                if st >= 1:  # step st-1's copies are done before step st's start (one copy stream)
                    done[st - 1].synchronize()
                    live[st - 1] = None
            e1.record(s_copy)
            e1.synchronize()
            live.clear()
            return e0.elapsed_time(e1)

        e2e_step()  # warm-up (allocator growth, first touch of the pinned buffers)
        e2e_ms, conv_ms = [], []
        for _ in range(args.e2e_steps):
            t_all, t_conv = e2e_step()
            e2e_ms.append(t_all)
            conv_ms.append(t_conv)
        lat = float(np.mean(e2e_ms))  # one step alone: its latency
        if pipeline:
            e2e_stream(2)  # warm-up of the pipelined form (second set of host buffers)
            em = e2e_stream(args.e2e_steps) / args.e2e_steps
        else:
            em = lat
        if dist:
            t = torch.tensor([em], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            em = float(t.item())
        e2e = {"value": 2.0 * prods / (em / 1e3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": int(bi),
               "d2h_bytes_per_step": int(bo), "ms_per_step": em,
               "h2d_convert_ms": round(float(np.mean(conv_ms)), 3),
               "latency_ms_one_step": round(lat, 3),
               "step_ms_all": [round(x, 3) for x in e2e_ms],
               "blocks": Ke, "copy_overlapped": pipeline,
               "includes": "every step: H2D of A's CSR + tsg_csr_to_tiles + tsg_spgemm per tile-row block + D2H of C's "
                           "tile arrays; block b's copy overlaps block b+1's SpGEMM and, when C fits two pinned host "
                           "buffers, step s+1's H2D + conversion overlap step s's D2H (steps back to back, "
                           "ms_per_step = total / steps; latency_ms_one_step = one step alone); warm-up steps first"}

    if rank != 0:
        if dist:
            dist.destroy_process_group()
        return 0
    cpu = None
    parity = None
    if not args.no_cpu_baseline and not args.profile and world == 1:
        cpu = oracle_baseline(A, budget_s=args.cpu_budget_s, B=Bcsr, prec="f64" if args.dtype == "f64" else "f32",
                              with_omp=True)
        cpu.pop("seconds", None)
        cpu.pop("products", None)
        C_ref = cpu.pop("_C")
        parity = sample_parity(tsg, T, Bt, C_ref, tol=1e-12 if args.dtype == "f64" else 1e-5)
        del C_ref
    clocks = clk.summary() if not args.profile else None
    line = {
        "metric": _metric(args), "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": {"f64": "f64", "f32": "f32", "f16": "f16 in, f32 accumulate/out"}[args.dtype],
        "data": "synthetic",
        "config": {"workload": f"{args.config} {gen.CONFIGS[args.config][0]}" + (", C = A*A^T" if args.aat else ""),
                   "n": A.m, "nnz_a": A.nnz,
                   "products": prods, "nnz_c": nnzC if world == 1 else None, "tiles_c": ntC if world == 1 else None,
                   "parallelism": (f"tile-row shards x{world}" if world > 1 else "single GPU") +
                                  (f", {K} tile-row blocks per rank computed in turn" if K > 1 else ""),
                   "l2": ("512 MB flush between timed steps" if flush is not None else
                          f"inputs larger than L2 (A tiles {tile_bytes(T.tile_m, T.num_tiles, T.nnz) / 1e6:.0f} MB > 126 MB)"),
                   "timing": "ms_per_step = median of the timed steps (CUDA events around the production "
                             "tsg_spgemm call, no stats); step_ms = medians of separate instrumented calls",
                   "t_ms_median": round(float(np.median(step_ms)), 4), "t_ms_mean": round(float(np.mean(step_ms)), 4),
                   "step_ms": {k: round(v, 4) for k, v in steps_ms.items()}, "alloc_sync_ms": round(alloc_ms, 4),
                   "step_ms_all": [round(x, 3) for x in step_ms],
                   "path": {0: "per-C-tile pipeline", 1: "fused per-tile-row pipeline"}.get(
                       int(stats_last["path"]) if K == 1 else -1, "mixed (row blocks)"),
                   "step1_mode": _step1_mode(stats_last),
                   "tiles_structural": int(st0["tiles_structural"]) if st0["tiles_structural"] >= 0 else None,
                   "host_sync_alloc_ms": [round(float(np.mean([h[0] for h in host_ms])), 3),
                                          round(float(np.mean([h[1] for h in host_ms])), 3)],
                   "bytes_alg": bytes_alg, "hbm_frac_path": bytes_alg / (ms / 1e3) / 1e9 / bw,
                   # per-call counts of the last timed call(s) (tsg_stats; summed over row blocks)
                   "call_stats": {k: stats_last.get(k) for k in
                                  ("candidates", "pairs", "tiles_c", "tiles_dense", "step1_merge_rows",
                                   "step1_big_rows", "step1_list_tiles", "host_syncs", "kernel_launches",
                                   "bytes_scratch", "bytes_out")}},
        "roofline": roof,
        "cpu_baseline": cpu,
        "parity": parity,
        "e2e": e2e,
        "gpu_launches": int(launches),
        "multi_gpu": multi,
        "clocks": clocks,
    }
    bad = _non_json(line)
    if bad:
        raise TypeError(f"bench line holds non-JSON values at {bad}")
    print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()
    return 0


def _step1_mode(st):
    """Step-1 formulation used (tsg_stats): warp merge of <= 32 sorted candidate lists per tile row,
    and/or bitmap rank / sort for wide rows; A tiles expanded through B row lists (mode ii)."""
    parts = []
    if st.get("step1_merge_rows"):
        parts.append(f"warp merge ({int(st['step1_merge_rows'])} tile rows)")
    if st.get("step1_big_rows"):
        parts.append(f"global-memory rank/sort ({int(st['step1_big_rows'])} tile rows)")
    if st.get("step1_list_tiles"):
        parts.append(f"B-row lists for {int(st['step1_list_tiles'])} A tiles")
    return "; ".join(parts) or "shared-memory sort"


def _cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def _metric(args):
    m = METRIC.replace("C=A^2", "C=A*A^T") if args.aat else METRIC
    return m.replace("fp64", {"f64": "fp64", "f32": "fp32", "f16": "fp16-in/fp32-out"}[args.dtype])


def _csr_transpose(A):
    """Host CSR of A^T (only for the row-partition weights of C = A A^T; the product uses the
    library's tile transpose)."""
    from workloads.gen import CSR

    rows = np.repeat(np.arange(A.m, dtype=np.int64), np.diff(A.rowptr))
    order = np.lexsort((rows, A.col))
    rp = np.zeros(A.n + 1, np.int64)
    np.add.at(rp, A.col.astype(np.int64) + 1, 1)
    return CSR(A.n, A.m, np.cumsum(rp), rows[order].astype(np.int32), A.val[order])


def _host_dtype(t):
    import torch

    return torch.int16 if t.dtype == torch.uint16 else t.dtype


class _Null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


if __name__ == "__main__":
    sys.exit(main())
