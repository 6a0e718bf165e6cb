"""Debug: one TGCN step + backward in linear-first vs aggregate-first order (C2)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

cfg = gen.CONFIGS["C2"]
s, d = gen.static_edges(cfg)
g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
V, F, H = cfg.V, cfg.F, 32
p = {k: torch.from_numpy(v).cuda() for k, v in gen.tgcn_params(F, H, 11).items()}
X = torch.from_numpy(gen.features(cfg, 5)).cuda()
Hp = torch.from_numpy(gen.uniform_pm1(3, 3, V * H).reshape(V, H)).cuda()
G = torch.from_numpy(gen.uniform_pm1(4, 4, V * H).reshape(V, H)).cuda()
out = {}
for order in (0, 1):
    stg.stg_set_conv_order(order)
    stack = stg.stg_state_stack_create(64 << 20)
    Hn = stg.stg_tgcn_step(g.view(), p, X, Hp, stack=stack)
    grads = {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
             "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}
    dHp = stg.stg_tgcn_step_backward(g.view(), p, X, G, grads, stack)
    torch.cuda.synchronize()
    out[order] = (Hn.cpu().numpy(), dHp.cpu().numpy(), {k: v.cpu().numpy() for k, v in grads.items()})
stg.stg_set_conv_order(0)
a, b = out[0], out[1]
print("H' maxdiff", np.abs(a[0] - b[0]).max())
dd = np.abs(a[1] - b[1])
print("dH maxdiff", dd.max(), "rows with diff > 1e-4:", np.nonzero(dd.max(1) > 1e-4)[0][:20], (dd.max(1) > 1e-4).sum(),
      "cols:", np.nonzero(dd.max(0) > 1e-4)[0])
for k in a[2]:
    print(k, "maxdiff", np.abs(a[2][k] - b[2][k]).max(), "max", np.abs(a[2][k]).max())
