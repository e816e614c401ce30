"""Small C = A*B cases through every kernel class, for compute-sanitizer (memcheck / racecheck /
synccheck): stencil, FEM strip (dense tiles), R-MAT (hub rows, staged small tiles), row slices,
transpose, precision variants, tiles -> CSR; both pipelines, the scratch retry, the tile records of
hypersparse operands, the structural diagnostic and the device partition (round 2); the row-path
dense class per tile row (fp64, fp32, fp16 inputs) and the 2^32-biased offsets (round 2 closing)."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import paper_conf_ppopp_niuljs0022_b200 as tsg
from workloads import gen


def tiles(A, dt=np.float64):
    return tsg.csr_to_tiles(torch.from_numpy(A.rowptr).cuda(), torch.from_numpy(A.col).cuda(),
                            torch.from_numpy(A.val.astype(dt)).cuda(), (A.m, A.n))


for A in (gen.config("C1"), gen.stencil27(8), gen.strip_fem(6, 12, 6), gen.rmat(10),
          gen.hub(4096, hub_rows=(0, 3000), hub_cols=(0, 5), density=0.002)):
    T = tiles(A)
    tsg.workspace_release()  # the first call overflows the arena and is redone (the retry path)
    C = tsg.spgemm(T, T, stats=True)
    for opts in (dict(path_rows=True), dict(path_general=True), dict(dense_threshold=1, path_rows=True),
                 dict(structural=True, products=True, stats=True), dict(small_stage=True), dict(sort_only=True),
                 dict(debug_high_offsets=True), dict(debug_high_offsets=True, path_rows=True, dense_threshold=1)):
        tsg.spgemm(T, T, **opts)
    S = tsg.spgemm(tsg.slice_rows(T, 1, max(2, T.tile_m // 2)), T)
    tsg.partition_tile_rows(T, T, 3)
    D = tsg.spgemm(T, tsg.transpose(T))
    rp, ci, v = tsg.tiles_to_csr(C)
    C32 = tsg.spgemm(tiles(A, np.float32), tiles(A, np.float32))
    H = tiles(A, np.float16)
    C16 = tsg.spgemm(H, H, dense_threshold=1, path_rows=True)  # the dense class from half inputs
    torch.cuda.synchronize()
    print(A.name if hasattr(A, "name") else "A", C.num_tiles, C.nnz, S.nnz, D.nnz, C32.nnz, flush=True)
print("sanitize cases done")
