"""CUDA-graph replay of whole DTDG epochs vs eager epochs (C5s or C5): the same
parameters / loss bit for bit after K epochs, and the epoch time both ways.
Epoch = Algorithm 1 over all T timestamps in sequences of S, SGD after each sequence."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5s")
ap.add_argument("--S", type=int, default=16)
ap.add_argument("--epochs", type=int, default=4)
a = ap.parse_args()
cfg = gen.CONFIGS[a.config]
d = gen.dtdg(cfg)
V, F, H, S, T = cfg.V, cfg.F, cfg.H, a.S, d.T
seqs = [(t0, min(S, T - t0)) for t0 in range(0, T, S)]
Xs = [torch.from_numpy(gen.features(cfg, t % 2)).cuda() for t in range(2)]
Ys = [torch.from_numpy(gen.labels(cfg, t)).cuda() for t in range(T)]


def run(use_graph):
    g = stg.stg_dtdg_create(V, T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                            d.del_dst, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    p = {k: torch.from_numpy(v).cuda() for k, v in gen.tgcn_params(F, H, cfg.seed).items()}
    grads = {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
             "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}
    dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    Hbuf = [torch.empty(S, V, H, device="cuda") for _ in range(2)]
    H0 = torch.zeros(V, H, device="cuda")
    Gw = torch.empty(2, V, H, device="cuda")
    st = stg.stg_state_stack_create(S * V * 3 * H * 4 + (64 << 20))

    def epoch():
        Hp = H0
        for k, (t0, n) in enumerate(seqs):
            Hs = Hbuf[k % 2]
            stg.stg_tgcn_train_sequence(g, t0, n, p, p["w_o"], p["b_o"], [Xs[t % 2] for t in range(t0, t0 + n)],
                                        Ys[t0:t0 + n], Hp, Hs, Gw, grads, dw, db, loss, st)
            for kk in ("W", "b", "L", "l"):
                stg.stg_sgd_update(p[kk], grads[kk], 0.01)
            stg.stg_sgd_update(p["w_o"], dw, 0.01)
            stg.stg_sgd_update(p["b_o"], db, 0.01)
            Hp = Hs[n - 1]

    epoch()
    epoch()                                            # warm-up: cache / workspace state settles
    torch.cuda.synchronize()
    run_epoch = epoch
    if use_graph:
        cg = torch.cuda.CUDAGraph()
        with torch.cuda.graph(cg, capture_error_mode="relaxed"):
            epoch()
        run_epoch = cg.replay                          # (capturing ran nothing: epoch 3 is the first replay)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(a.epochs):
        run_epoch()
    e1.record()
    torch.cuda.synchronize()
    return {k: v.clone() for k, v in p.items()}, loss.item(), e0.elapsed_time(e1) / a.epochs


pe, le, te = run(False)
pg, lg, tg = run(True)
same = all(torch.equal(pe[k], pg[k]) for k in pe)
print(json.dumps({"config": a.config, "epochs": a.epochs, "eager_ms": te, "graph_ms": tg, "params_bit_identical": same,
                  "loss_eager": le, "loss_graph": lg}))
