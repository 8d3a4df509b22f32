"""Run one M2 join with a SCAT_PROF library (prints per-phase clock64 totals of CTA 0)."""
import os, sys
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import torch
from paper_conf_sigmod_paullhl21_b200 import mgj
n = 1 << 29
cols = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(4)]
mgj.gen_relation("unique", 0, n, n, 0.0, 0, n, cols[0], cols[1])
mgj.gen_relation("unique", 1, n, n, 0.0, 0, n, cols[2], cols[3])
j = mgj.Join(mgj.make_config(r_capacity=n, s_capacity=n))
for _ in range(2):
    r = j.run(*cols)
torch.cuda.synchronize()
print("ms", r["phase_ms"])
