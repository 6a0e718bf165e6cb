import sys, numpy as np, torch
sys.path.insert(0, "/root/repo"); sys.path.insert(0, ".")
import gen, oracle
import paper_conf_ipps_cherianmcc24_b200 as stg
for name in ("C3", "C2"):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    ref = oracle.static_graph(cfg.V, s, d, self_loops=True)
    for W in (132, 200, 256):
        x = gen.features(cfg, 3, width=W).astype(np.float64)
        y = stg.stg_gcn_aggregate_fwd(g.view(), torch.from_numpy(x).float().cuda()).cpu().numpy()
        r = oracle.aggregate_fwd(ref, x)
        err = np.abs(y - r)
        bad = np.argwhere(err > 1e-4)
        print(name, W, "maxerr", err.max(), "nbad", len(bad), "bad cols", np.unique(bad[:, 1])[:20] if len(bad) else None,
              "bad rows", np.unique(bad[:, 0])[:10] if len(bad) else None, flush=True)
