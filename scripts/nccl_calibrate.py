#!/usr/bin/env python
"""NCCL calibration at the exchange sizes of SURVEY §8e (the planning model's X(P)).

  python -m torch.distributed.run --nproc-per-node P --master-addr 127.0.0.1 scripts/nccl_calibrate.py

Per size: allgather (the receive size = the whole replicated vector: PageRank's
contributions at scale 25 are 134 MB, ~67 MB compacted; SpMV's y at scale 22 is
16.8 MB) and in-place allreduce (SSSP's min over uint32 dist: 33.6 MB at scale 23;
BFS's max over an n-byte map: 67 MB at scale 26).  CUDA events, 5 warm-ups + 20
timed calls, max over ranks; rank 0 prints one JSON line per (op, size).  With one
GPU (P = 1) the numbers are the local copy cost only.
"""
import json
import os

import torch
import torch.distributed as dist

SIZES_MB = [8.4, 16.8, 33.6, 67.1, 134.2]


def main():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local),
                            init_method=None if "MASTER_ADDR" in os.environ else "tcp://127.0.0.1:29533",
                            rank=rank, world_size=world)
    for op in ("allgather_f32", "allreduce_min_u32", "allreduce_max_u8"):
        for mb in SIZES_MB:
            total = int(mb * 1e6)
            if op == "allgather_f32":
                per = total // 4 // world
                send = torch.ones(per, dtype=torch.float32, device="cuda")
                recv = torch.empty(per * world, dtype=torch.float32, device="cuda")
                fn = lambda: dist.all_gather_into_tensor(recv, send)  # noqa: E731
            elif op == "allreduce_min_u32":
                buf = torch.ones(total // 4, dtype=torch.int32, device="cuda")
                fn = lambda: dist.all_reduce(buf, op=dist.ReduceOp.MIN)  # noqa: E731
            else:
                buf = torch.ones(total, dtype=torch.uint8, device="cuda")
                fn = lambda: dist.all_reduce(buf, op=dist.ReduceOp.MAX)  # noqa: E731
            for _ in range(5):
                fn()
            torch.cuda.synchronize()
            dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(20):
                fn()
            e1.record()
            torch.cuda.synchronize()
            t = torch.tensor([e0.elapsed_time(e1) / 20], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
            if rank == 0:
                # algorithm bandwidth = bytes of the result / time; NCCL's bus bandwidth scales it by
                # (P-1)/P (allgather) or 2(P-1)/P (allreduce)
                fac = (world - 1) / world if op.startswith("allgather") else 2 * (world - 1) / world
                print(json.dumps({"op": op, "mb": mb, "P": world, "ms": round(ms, 4),
                                  "algbw_gbs": round(total / (ms * 1e-3) / 1e9, 1),
                                  "busbw_gbs": round(total * fac / (ms * 1e-3) / 1e9, 1)}), flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
