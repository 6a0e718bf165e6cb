"""One Algorithm-1 epoch of the original T-GCN cell (NEXT-2) on a DTDG config with
the per-step library calls (Python loop, one stream): CUDA-event epoch time and
the per-phase split.  Prints one JSON line."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--seq", type=int, default=16)
ap.add_argument("--epochs", type=int, default=2)
a = ap.parse_args()
cfg = gen.CONFIGS[a.config]
d = gen.dtdg(cfg)
V, F, H, T, S = cfg.V, cfg.F, cfg.H, d.T, a.seq
g = stg.stg_dtdg_create(V, T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
p = {k: torch.from_numpy(v).cuda() for k, v in gen.tgcn2_params(F, H, cfg.seed).items()}
Xs = [torch.from_numpy(gen.features(cfg, i)).cuda() for i in range(2)]
Ys = [torch.from_numpy(gen.labels(cfg, t)).cuda() for t in range(T)]
grads = {"Wg": torch.zeros(F + H, 2 * H, device="cuda"), "bg": torch.zeros(2 * H, device="cuda"),
         "Wc": torch.zeros(F + H, H, device="cuda"), "bc": torch.zeros(H, device="cuda")}
dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
st = stg.stg_state_stack_create(S * V * 3 * H * 4 + (64 << 20))
Hb = [torch.zeros(V, H, device="cuda") for _ in range(S + 1)]
G = [torch.zeros(V, H, device="cuda") for _ in range(2)]


def epoch():
    H0 = torch.zeros(V, H, device="cuda")
    for t0 in range(0, T, S):
        n = min(S, T - t0)
        Hb[0].copy_(H0)
        for i in range(n):
            v = stg.stg_dtdg_get_snapshot(g, t0 + i)
            stg.stg_tgcn2_step(v, p, Xs[(t0 + i) % 2], Hb[i], Hb[i + 1], st)
            stg.stg_mse_head(Hb[i + 1], Ys[t0 + i], p["w_o"], p["b_o"], loss_accum=loss)
        G[0].zero_()
        k = 0
        for i in range(n - 1, -1, -1):
            v = stg.stg_dtdg_get_backward_snapshot(g, t0 + i)
            stg.stg_mse_head(Hb[i + 1], Ys[t0 + i], p["w_o"], p["b_o"], dH=G[k], accumulate=True, dw_o=dw, db_o=db)
            stg.stg_tgcn2_step_backward(v, p, Xs[(t0 + i) % 2], G[k], grads, st, dH_prev=G[1 - k])
            k = 1 - k
        for name in grads:
            stg.stg_sgd_update(p[name], grads[name], 1e-3)
        H0 = Hb[n].clone()


epoch()
torch.cuda.synchronize()
stg.stg_profile_enable(True)
stg.stg_profile_read(reset=True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(a.epochs):
    epoch()
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / max(1, a.epochs)
prof = stg.stg_profile_read(reset=True)
E = sum(g.num_edges(t) for t in range(T))
print(json.dumps({"model": "original T-GCN (NEXT-2), per-step library calls, one stream", "config": a.config,
                  "ms_per_epoch": ms, "timesteps_per_s": T / (ms / 1e3),
                  "aggregated_edges_per_s": 4 * E / (ms / 1e3),
                  "note": "4 aggregations per timestep (2 fwd: widths 2H, H; 2 bwd)",
                  "phases_ms_per_epoch": {k: v[0] / max(1, a.epochs) for k, v in prof.items()}}), flush=True)
