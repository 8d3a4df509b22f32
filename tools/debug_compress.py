"""Small compressed-shuffle join at one rank, with status and a few internal arrays (debugging aid)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
from paper_conf_sigmod_paullhl21_b200 import datagen, mgj

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 16
d = datagen.Workload("unique", n, n).rank_inputs()
t = [torch.from_numpy(d[k].view(np.int32)).cuda() for k in ("r_keys", "r_pays", "s_keys", "s_pays")]
j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n, compress=True))
j.partition(*t); j.shuffle(); j.join()
r = j.result(check=False)
ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
print("status", r["status"], "count", r["match_count"], ref["count"], "chk", hex(r["checksum"]), hex(ref["checksum"]),
      "dig ok", r["pair_digest"] == ref["pair_digest"], "recv units", r["recv_r"], r["recv_s"])
meta = j.debug("META", np.int32)
print("meta", meta[:16].tolist())
