"""Short C5 driver for ncu launch lists: create the DTDG, run one warm-up sequence
and then `--seqs` sequences of S timesteps (Algorithm 1), nothing else."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--S", type=int, default=4)
ap.add_argument("--seqs", type=int, default=1)
ap.add_argument("--strategy", type=int, default=-1)
a = ap.parse_args()
if a.strategy >= 0:
    stg.stg_aggregate_set_strategy(a.strategy)
cfg = gen.CONFIGS[a.config]
d = gen.dtdg(cfg)
V, F, H, S = cfg.V, cfg.F, cfg.H, a.S
g = stg.stg_dtdg_create(V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
X = torch.from_numpy(gen.features(cfg, 0)).cuda()
Ys = [torch.from_numpy(gen.labels(cfg, t)).cuda() for t in range(S)]
p = {k: torch.from_numpy(v).cuda() for k, v in gen.tgcn_params(F, H, 1).items()}
grads = {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
         "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}
dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
Hs = torch.empty(S, V, H, device="cuda")
H0 = torch.zeros(V, H, device="cuda")
Gw = torch.empty(2, V, H, device="cuda")
st = stg.stg_state_stack_create(S * V * 3 * H * 4 + (64 << 20))
for k in range(1 + a.seqs):
    t0 = (k * S) % (d.T - S)
    stg.stg_tgcn_train_sequence(g, t0, S, p, p["w_o"], p["b_o"], [X] * S, Ys, H0, Hs, Gw, grads, dw, db, loss, st)
    torch.cuda.synchronize()
    if k == 0:
        print("warm-up launches:", stg.kernel_launch_count(), flush=True)
print("total launches:", stg.kernel_launch_count(), flush=True)
