"""Multi-GPU sharding of the TileSpGEMM hot path (no counterpart in the paper,
which runs on one GPU -- P:3760-3766 calls distributed blocking SpGEMM related work).

C tile rows are independent: tile row I of C needs tile row I of A and all of B.  So

1. ``partition_device`` (tsg_partition_tile_rows in the library): contiguous tile-row ranges
   [I_g, I_{g+1}) cut on the device at equal shares of the prefix sum of per-tile-row
   intermediate products (load balance by work, not rows); ``partition_tile_rows`` is the same
   rule from host CSR (used to check the device cuts);
2. ``broadcast_tiles``: rank ``src`` holds B; its seven Section-3.2 arrays go to every rank with
   ``torch.distributed.broadcast`` (NCCL over NVLink on the B200 box);
3. each rank runs the local ``tsg.spgemm(slice_rows(A, I_g, I_{g+1}), B)``;
4. reassembly, count-exact (no padding): ``gatherv_tiles`` sends every shard to one rank with
   point-to-point transfers of exactly its bytes; ``allgatherv_tiles`` gives every rank the full C
   with one exact-size broadcast per source.  ``assemble`` rebases ``tile_ptr`` / ``tile_nnz`` by
   the exclusive scan of the per-rank tile and nonzero counts.  When the full C does not fit one
   GPU (C5: ~144 GB in tile form) it is left distributed -- every rank owns its tile rows.

Only collectives and host bookkeeping live here; every arithmetic step of the method runs in
libtsg's kernels.  The collectives are device-agnostic (torch tensors), so the world_size-2 gloo
tests in tests/test_dist_gloo.py cover them on CPU.
"""
from __future__ import annotations

import numpy as np

TILE = 16
ARRAYS = ("tile_ptr", "tile_col", "tile_nnz", "row_ptr", "mask", "idx", "val")
_CODES = ("float64", "float32", "float16")


def tile_row_products(A, B) -> np.ndarray:
    """Intermediate products per tile row of A*B from host CSR (the partition weights)."""
    rn = np.diff(B.rowptr).astype(np.int64)
    w = rn[A.col.astype(np.int64)] if A.col.size else np.zeros(0, np.int64)
    cs = np.concatenate(([0], np.cumsum(w)))
    row = cs[A.rowptr[1:]] - cs[A.rowptr[:-1]]
    tm = (A.m + TILE - 1) // TILE
    pad = np.zeros(tm * TILE, np.int64)
    pad[:A.m] = row
    return pad.reshape(tm, TILE).sum(axis=1)


def cuts_from_weights(w: np.ndarray, world: int) -> np.ndarray:
    """cuts[g] = first tile row whose product prefix reaches g * total / world (monotone)."""
    tm = w.size
    if world <= 1 or tm == 0:
        return np.array([0, tm] if world <= 1 else [0] * world + [tm], dtype=np.int64)
    pre = np.concatenate(([0], np.cumsum(w))).astype(np.int64)
    total = int(pre[-1])
    # exact integer form of searchsorted-left of g*total/world: first i with pre[i]*world >= g*total
    cuts = [0]
    for g in range(1, world):
        cuts.append(int(np.searchsorted(pre * world, g * total, side="left")))
    cuts.append(tm)
    return np.maximum.accumulate(np.clip(np.array(cuts, dtype=np.int64), 0, tm))


def partition_tile_rows(A, B, world: int) -> np.ndarray:
    """Host-CSR form of the partition (cuts[g] .. cuts[g+1] = tile rows of rank g)."""
    return cuts_from_weights(tile_row_products(A, B), world)


def partition_device(A_tiles, B_tiles, world: int, stream=None) -> np.ndarray:
    """The partition computed by the library on the device from the tile handles (no host CSR
    needed, e.g. for a chained C = (A^2) A whose left operand only exists in tile form)."""
    from . import partition_tile_rows as _dev

    if world <= 1:
        return np.array([0, A_tiles.tile_m], dtype=np.int64)
    return _dev(A_tiles, B_tiles, world, stream)[0]


def _wire(t):
    """Byte view of 16-bit masks for the wire (neither NCCL nor gloo carries 16-bit integers)."""
    import torch

    return t.view(torch.uint8) if t.dtype in (torch.uint16, torch.int16) else t


def _unwire(t, k):
    import torch

    return t.view(torch.uint16) if k == "mask" else t


def _wire_dev(dev, group=None):
    """Device the collectives move bytes on: the tensors' own device, except CUDA tensors under
    gloo (gloo's point-to-point and all-gather take host tensors only), which stage via host."""
    import torch
    import torch.distributed as dist

    if dev.type == "cuda" and dist.get_backend(group) == "gloo":
        return torch.device("cpu")
    return dev


def _shapes(m, nt, nnz, vdt):
    import torch

    tm = (m + TILE - 1) // TILE
    return {"tile_ptr": (tm + 1, torch.int64), "tile_col": (nt, torch.int32), "tile_nnz": (nt + 1, torch.int64),
            "row_ptr": (16 * nt, torch.uint8), "mask": (32 * nt, torch.uint8), "idx": (nnz, torch.uint8),
            "val": (nnz, vdt)}


def broadcast_tiles(arrays: dict | None, meta: tuple | None, src: int, device, group=None):
    """Broadcast the seven arrays of a tile matrix from ``src``; returns (meta, arrays) everywhere.

    meta = (m, n, num_tiles, nnz, dtype) with dtype a torch value type (a 4-tuple means fp64).  On
    non-src ranks pass arrays=None, meta=None; every rank gets the 5-tuple back.
    """
    import torch
    import torch.distributed as dist

    codes = [getattr(torch, c) for c in _CODES]
    if meta is not None:
        vals = list(meta[:4]) + [codes.index(meta[4]) if len(meta) > 4 else 0]
    else:
        vals = [0, 0, 0, 0, 0]
    device = torch.device(device)
    wdev = _wire_dev(device, group)
    mt = torch.tensor(vals, dtype=torch.int64, device=wdev)
    dist.broadcast(mt, src, group=group)
    m, n, nt, nnz, dc = (int(x) for x in mt.tolist())
    shapes = _shapes(m, nt, nnz, codes[dc])
    out = {}
    for k in ARRAYS:
        if arrays is not None:
            t = _wire(arrays[k].contiguous()).to(wdev)
        else:
            t = torch.empty(shapes[k][0], dtype=shapes[k][1], device=wdev)
        if t.numel():
            dist.broadcast(t, src, group=group)
        out[k] = _unwire(t.to(device), k)
    return (m, n, nt, nnz, codes[dc]), out


def _local(C):
    arrays = C.arrays() if hasattr(C, "arrays") else {k: C[k] for k in ARRAYS}
    m_local = C.m if hasattr(C, "m") else C["m"]
    n = C.n if hasattr(C, "n") else C["n"]
    return arrays, int(m_local), int(n)


def _counts(arrays, m_local, group):
    """(m, num_tiles, nnz, value dtype code) of every rank: one all_gather of 4 int64."""
    import torch
    import torch.distributed as dist

    dev = _wire_dev(arrays["tile_ptr"].device, group)
    vdt = str(arrays["val"].dtype).replace("torch.", "")
    mine = torch.tensor([m_local, arrays["tile_col"].numel(), arrays["val"].numel(), _CODES.index(vdt)],
                        dtype=torch.int64, device=dev)
    world = dist.get_world_size(group)
    allc = [torch.zeros_like(mine) for _ in range(world)]
    dist.all_gather(allc, mine, group=group)
    return [tuple(int(x) for x in c.tolist()) for c in allc]


def allgatherv(t, group=None):
    """Count-exact all-gather of a 1-D tensor: one broadcast per source of exactly its elements."""
    import torch
    import torch.distributed as dist

    world, rank = dist.get_world_size(group), dist.get_rank(group)
    wdev = _wire_dev(t.device, group)
    src = _wire(t.contiguous()).to(wdev)
    n = torch.tensor([src.numel()], dtype=torch.int64, device=wdev)
    sizes = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(sizes, n, group=group)
    out = []
    for g in range(world):
        sz = int(sizes[g].item())
        buf = src if g == rank else torch.empty(sz, dtype=src.dtype, device=wdev)
        if sz:
            dist.broadcast(buf, dist.get_global_rank(group, g) if group is not None else g, group=group)
        buf = buf.to(t.device)
        out.append(buf.view(t.dtype) if t.dtype != src.dtype else buf)
    return out


def assemble(pieces: list, n: int):
    """Concatenate per-rank C shards (contiguous tile-row ranges, in rank order) into one matrix.

    pieces[g] = dict(m=rows, arrays...) with rank-local offsets.  tile_ptr and tile_nnz are
    rebased by the exclusive scan of the per-rank tile and nonzero counts.
    Returns (m, n, arrays) with torch tensors.
    """
    import torch

    tile_base, nnz_base = 0, 0
    out = {k: [] for k in ARRAYS}
    m = 0
    for g, p in enumerate(pieces):
        tp, tz = p["tile_ptr"], p["tile_nnz"]
        nt, nz = int(tp[-1].item()), int(tz[-1].item())
        out["tile_ptr"].append((tp[:-1] if g < len(pieces) - 1 else tp) + tile_base)
        out["tile_nnz"].append((tz[:-1] if g < len(pieces) - 1 else tz) + nnz_base)
        for k in ("tile_col", "row_ptr", "mask", "idx", "val"):
            out[k].append(_wire(p[k]))
        tile_base += nt
        nnz_base += nz
        m += int(p["m"])
    res = {k: torch.cat(v) for k, v in out.items()}
    res["mask"] = res["mask"].view(torch.uint16)
    return m, n, res


def allgatherv_tiles(C, group=None):
    """Every rank's C shard (a Tiles object or an arrays dict with keys m, n) on every rank,
    count-exact; returns (m, n, arrays)."""
    arrays, m_local, n = _local(C)
    gathered = {k: allgatherv(arrays[k], group) for k in ARRAYS}
    counts = _counts(arrays, m_local, group)
    pieces = [dict(m=counts[g][0], **{k: gathered[k][g] for k in ARRAYS}) for g in range(len(counts))]
    return assemble(pieces, n)


def gatherv_tiles(C, dst: int = 0, group=None, out_device=None):
    """Every rank's C shard sent to rank ``dst`` only, count-exact (point-to-point transfers of
    exactly each shard's bytes).  ``out_device`` ("cpu" with pinned buffers, or the default: the
    shard's device) receives them.  Returns (m, n, arrays) on ``dst`` and None elsewhere."""
    import torch
    import torch.distributed as dist

    arrays, m_local, n = _local(C)
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    counts = _counts(arrays, m_local, group)
    glob = (lambda g: dist.get_global_rank(group, g)) if group is not None else (lambda g: g)
    wdev = _wire_dev(arrays["tile_ptr"].device, group)
    if rank != dst:
        ops = [dist.P2POp(dist.isend, _wire(arrays[k].contiguous()).to(wdev), glob(dst), group=group)
               for k in ARRAYS if arrays[k].numel()]
        for r in dist.batch_isend_irecv(ops) if ops else []:
            r.wait()
        return None
    dev = torch.device(out_device) if out_device is not None else arrays["tile_ptr"].device
    pin = dev.type == "cpu" and torch.cuda.is_available()
    pieces, ops = [], []
    for g in range(world):
        m_g, nt_g, nnz_g, dc = counts[g]
        if g == rank:
            pieces.append(dict(m=m_g, **{k: (arrays[k].to(dev) if dev != arrays[k].device else arrays[k])
                                         for k in ARRAYS}))
            continue
        shapes = _shapes(m_g, nt_g, nnz_g, getattr(torch, _CODES[dc]))
        bufs = {}
        for k in ARRAYS:
            nel, dt = shapes[k]
            # receive on the wire device (the shard's device under NCCL), staged to `dev`
            # afterwards if that differs
            bufs[k] = torch.empty(nel, dtype=dt, device=wdev)
            if nel:
                ops.append(dist.P2POp(dist.irecv, bufs[k], glob(g), group=group))
        pieces.append(dict(m=m_g, **bufs))
    for r in dist.batch_isend_irecv(ops) if ops else []:
        r.wait()
    if dev != wdev or dev != arrays["tile_ptr"].device:
        for p in pieces:
            for k in ARRAYS:
                if p[k].device != dev:
                    h = torch.empty(p[k].shape, dtype=p[k].dtype, device=dev, pin_memory=pin)
                    h.copy_(p[k])
                    p[k] = h
    for p in pieces:
        p["mask"] = _unwire(_wire(p["mask"]), "mask")
    return assemble(pieces, n)


def spgemm_sharded(A_tiles, B_tiles, group=None, reassemble: str = "gather"):
    """C = A*B with C tile rows sharded over the process group (cuts computed on the device).

    reassemble: "gather" -> full C on rank 0 (None elsewhere), "all" -> full C on every rank,
    "none" -> C stays distributed.  Returns (local C shard, cuts, reassembled or None)."""
    import torch.distributed as dist

    from . import slice_rows, spgemm

    world, rank = dist.get_world_size(group), dist.get_rank(group)
    cuts = partition_device(A_tiles, B_tiles, world)
    shard = slice_rows(A_tiles, int(cuts[rank]), int(cuts[rank + 1]))
    Cl = spgemm(shard, B_tiles)
    full = None
    if reassemble == "gather":
        full = gatherv_tiles(Cl, 0, group)
    elif reassemble == "all":
        full = allgatherv_tiles(Cl, group)
    return Cl, cuts, full
