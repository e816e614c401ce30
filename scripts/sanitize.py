"""Small C = A*B cases through every kernel class, for compute-sanitizer (memcheck / racecheck /
synccheck): stencil, FEM strip (dense tiles), R-MAT (hub rows, staged small tiles), row slices,
transpose, precision variants, tiles -> CSR."""
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
    C = tsg.spgemm(T, T, stats=True)
    S = tsg.spgemm(tsg.slice_rows(T, 1, max(2, T.tile_m // 2)), T)
    D = tsg.spgemm(T, tsg.transpose(T))
    rp, ci, v = tsg.tiles_to_csr(C)
    C32 = tsg.spgemm(tiles(A, np.float32), tiles(A, np.float32))
    torch.cuda.synchronize()
    print(A.name if hasattr(A, "name") else "A", C.num_tiles, C.nnz, S.nnz, D.nnz, C32.nnz, flush=True)
print("sanitize cases done")
