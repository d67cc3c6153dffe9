"""Worker of test_gpu_p2p.test_p2p_two_processes_ipc_same_gpu (launched by torchrun):
2 ranks on cuda:0, gloo for the one-time handle exchange, CUDA IPC + stream flags for
the fused halo exchange; rank 0 saves the gathered field to $P2P_OUT."""
import os
import tempfile

import numpy as np
import torch
import torch.distributed as dist

import synthetic
from paper_conf_cgo_georgakoudispb25_b200 import halo
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W

rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)
dev = torch.device("cuda", 0)
torch.zeros(1, device=dev)
dist.init_process_group("gloo")
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(prefix=f"p2p-r{rank}-"), mode="all")
k = W.register("stencil4_p2p")
nx, ny, nz, T = 48, 40, 32, 5
nzl = nz // world
u0 = synthetic.stencil_inputs(nx, ny, nz)
parts = halo.p2p_arena(nx, ny, nzl, dev)
arena, u, w, flags = parts
lo, hi = max(0, rank * nzl - 2), min(nz, (rank + 1) * nzl + 2)
u[lo - (rank * nzl - 2):hi - (rank * nzl - 2)] = torch.from_numpy(u0[lo:hi]).to(dev)
w.copy_(u)
left, right, opened = halo.connect_ipc(arena, rank, world)
torch.cuda.synchronize()
dist.barrier()
st = halo.P2PZSlabStencil(k, parts, nx=nx, ny=ny, nzl=nzl, nzg=nz, rank=rank, world=world,
                          coeffs=synthetic.STENCIL_COEFFS, left=left, right=right)
for _ in range(T):
    st.sweep()
torch.cuda.synchronize()
dist.barrier()                      # neighbours done with our arena before unmapping
mine = st.current[2:nzl + 2].cpu().numpy()
allp = [None] * world
dist.all_gather_object(allp, mine)
for b in opened:
    P.proteus_ipc_close_handle(b)
if rank == 0:
    np.save(os.environ["P2P_OUT"], np.concatenate(allp))
P.proteus_finalize()
dist.destroy_process_group()
