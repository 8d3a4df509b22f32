"""Debug: chunk streaming at N virtual ranks; prints status, counts and each
rank's S round counters (epoch << 32 | tiles) and non-empty tiles per round."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_sigmod_paullhl21_b200 import mgj, datagen
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import oracle

def al(x, a): return (x + a - 1) // a * a
def layout(P):
    off = 0; L = {}
    L["sig"] = off; off = al(off + 4 * 8 * 8, 4096)
    L["mail"] = off; off = al(off + 8 * 2 * P * 4, 4096)
    L["resmail"] = off; off = al(off + 8 * 8 * 8, 4096)
    L["umail"] = off; off = al(off + 8 * 2 * P * 4, 4096)
    L["cfgmail"] = off; off = al(off + 8 * 4 * 8, 4096)
    L["rbmail"] = off; off = al(off + 16 * (P + 1) * 4, 4096)
    L["rdone"] = off
    return L

N = int(sys.argv[1]) if len(sys.argv) > 1 else 2
ov = int(sys.argv[2]) if len(sys.argv) > 2 else 2
w = datagen.Workload("unique", 300007, 400009)
parts = [w.rank_inputs(g, N) for g in range(N)]
cap_r = max(p["r_keys"].size for p in parts); cap_s = max(p["s_keys"].size for p in parts)
cfgs = [mgj.make_config(rank=g, world_size=N, r_capacity=cap_r, s_capacity=cap_s, recv_capacity_r=w.n_r,
                        recv_capacity_s=w.n_s, shuffle_overlap=ov, peer_timeout_ms=3000, trace=True) for g in range(N)]
nb = mgj.arena_bytes(cfgs[0])
arenas = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(N)]
joins = [mgj.Join(cfgs[g], [a.data_ptr() for a in arenas], nb) for g in range(N)]
tens = [[torch.from_numpy(p[k]).cuda() for k in ("r_keys", "r_pays", "s_keys", "s_pays")] for p in parts]
streams = [torch.cuda.Stream() for _ in range(N)]
torch.cuda.synchronize()
for g in range(N): joins[g].partition(*tens[g], stream=streams[g])
for g in range(N): joins[g].shuffle(streams[g])
for g in range(N): joins[g].join(streams[g])
res = []
for g in range(N):
    try:
        res.append(joins[g].result())
    except Exception as e:
        print("rank", g, "result error", e)
        res.append({"status": "err", "match_count": -1, "recv_r": -1, "recv_s": -1})
torch.cuda.synchronize()
d = w.rank_inputs()
ref = oracle.join(d["r_keys"], d["r_pays"], d["s_keys"], d["s_pays"])
L = layout(1024)
for g in range(N):
    a = arenas[g].cpu().numpy()
    rd = a[L["rdone"]: L["rdone"] + 16 * 8].view(np.uint64)
    nt = a[L["rbmail"]: L["rbmail"] + 16 * 4].view(np.uint32)
    rb1 = a[L["rbmail"] + 16 * 4: L["rbmail"] + 16 * 4 + 3 * 1024 * 4].view(np.uint32).reshape(3, 1024)
    print("rank", g, "status", res[g]["status"], "count", res[g]["match_count"], "ref", ref["count"],
          "rdone", [(int(x) >> 32, int(x) & 0xffffffff) for x in rd[:8]], "ntile", nt[:8].tolist(),
          "rb[1][:4]", rb1[1][:4].tolist(), "rb[2][:4]", rb1[2][:4].tolist(), "recv", res[g]["recv_r"], res[g]["recv_s"])
    try:
        print("  trace", {k: [round(x, 1) for x in v] for k, v in joins[g].trace().items()})
    except Exception as e:
        print("  trace error", e)
