"""Worker for tests/test_gpu_join.py::test_torchrun_parity_all_gpus (run under
torch.distributed.run, one rank per GPU): M1 split N ways over the real
symmetric-memory path (mgj.symmetric_join), every rank's global (count,
checksum, pair digest) against the CPU oracle, and the materialised shards of
all ranks together against the oracle's sorted triples (rank 0 checks)."""
import json
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_sigmod_paullhl21_b200 import datagen, mgj  # noqa: E402


def main():
    rank, world, local = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"]), int(os.environ["LOCAL_RANK"])
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    w = datagen.M1()
    d = w.rank_inputs(rank, world)
    cfg = mgj.make_config(rank=rank, world_size=world, r_capacity=d["r_keys"].size, s_capacity=d["s_keys"].size,
                          recv_capacity_r=w.n_r, recv_capacity_s=w.n_s, materialize=True, out_capacity=w.n_s)
    j = mgj.symmetric_join(cfg)
    t = [torch.from_numpy(d[k].view(np.int32)).cuda() for k in ("r_keys", "r_pays", "s_keys", "s_pays")]
    s = torch.cuda.Stream()
    torch.cuda.synchronize()
    res = j.run(*t, stream=s)
    k, a, b = j.materialized(res)
    parts = [None] * world
    dist.all_gather_object(parts, (res["match_count"], res["checksum"], res["pair_digest"], k, a, b))
    ok = True
    if rank == 0:
        full = w.rank_inputs()
        ref = oracle.join(full["r_keys"], full["r_pays"], full["s_keys"], full["s_pays"], materialize=True)
        ok = all((p[0], p[1], p[2]) == (ref["count"], ref["checksum"], ref["pair_digest"]) for p in parts)
        K = np.concatenate([p[3] for p in parts])
        A = np.concatenate([p[4] for p in parts])
        B = np.concatenate([p[5] for p in parts])
        o = np.lexsort((B, A, K))
        ok = ok and np.array_equal(K[o], ref["key"]) and np.array_equal(A[o], ref["pay_r"]) and \
            np.array_equal(B[o], ref["pay_s"])
        print(json.dumps({"ok": bool(ok), "world": world, "count": parts[0][0]}))
    j.close()
    dist.barrier()
    dist.destroy_process_group()
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main()
