import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import torch
from paper_conf_sigmod_paullhl21_b200 import mgj
import numpy as np
for z in (0.5, 1.0):
    n_r, n_s = 1 << 27, 1 << 29
    cols = [torch.empty(x, dtype=torch.int32, device="cuda") for x in (n_r, n_r, n_s, n_s)]
    mgj.gen_relation("zipf", 0, n_r, n_s, z, 0, n_r, cols[0], cols[1])
    mgj.gen_relation("zipf", 1, n_r, n_s, z, 0, n_s, cols[2], cols[3])
    j = mgj.Join(mgj.make_config(r_capacity=n_r, s_capacity=n_s))
    for _ in range(3):
        res = j.run(*cols)
    # co-partition size distribution of S: keys with the same low B1+B2 bits
    B1, B2 = res["radix_bits_global"], res["radix_bits_local"]
    m = (1 << (B1 + B2)) - 1
    hs = torch.bincount((cols[2] & m).long(), minlength=m + 1)
    hr = torch.bincount((cols[0] & m).long(), minlength=m + 1)
    print(f"z={z} items={res['n_items']} B2={B2} ms={res['phase_ms']} copart S max={int(hs.max())} mean={float(hs.float().mean()):.0f} "
          f">8448: {int((hs > 8448).sum())} R max={int(hr.max())} slices~{int((hs // 7400 + 1).sum())}")
    j.close()
    del cols
