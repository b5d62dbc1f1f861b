"""Probe: can two NCCL ranks share one GPU on this box?  (torchrun --nproc-per-node 2)

Each rank binds cuda:0, initialises an NCCL process group and runs one
all_to_all_single with uneven splits.  Prints one JSON line per rank with the outcome.
"""
import json
import os
import sys

import torch
import torch.distributed as dist

rank = int(os.environ.get("RANK", "0"))
world = int(os.environ.get("WORLD_SIZE", "1"))
torch.cuda.set_device(0)
res = {"rank": rank, "world": world}
try:
    dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
    send = torch.arange(10, dtype=torch.float32, device="cuda") + 100 * rank
    ins = [3, 7] if rank == 0 else [4, 6]
    outs = [3, 4] if rank == 0 else [7, 6]
    recv = torch.empty(sum(outs), device="cuda")
    dist.all_to_all_single(recv, send, output_split_sizes=outs, input_split_sizes=ins)
    torch.cuda.synchronize()
    res["ok"] = True
    res["recv"] = recv.tolist()
    dist.destroy_process_group()
except Exception as e:  # report, do not hang
    res["ok"] = False
    res["error"] = repr(e)[:400]
print(json.dumps(res), flush=True)
sys.exit(0)
