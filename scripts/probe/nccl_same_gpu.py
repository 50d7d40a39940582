"""Probe: can two NCCL ranks share one GPU (for an on-box multi-rank check)?"""
import os, torch, torch.distributed as dist
dist.init_process_group("nccl")
r = dist.get_rank()
torch.cuda.set_device(0)
x = torch.full((4,), float(r + 1), device="cuda")
try:
    dist.all_reduce(x)
    torch.cuda.synchronize()
    print("rank", r, "allreduce ok", x.tolist(), flush=True)
except Exception as e:
    print("rank", r, "allreduce failed", repr(e)[:300], flush=True)
if r == 0:
    f, t = torch.cuda.mem_get_info()
    print("mem free/total GB", f / 1e9, t / 1e9, flush=True)
dist.destroy_process_group()
