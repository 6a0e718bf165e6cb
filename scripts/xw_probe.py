"""Time the TGCN forward phases on C5 (one static snapshot) with STG_XW_DEBUG
variants (bit0 no stores, bit1 no MMA, bit2 no loads, bit3 no smem staging)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

V, F, H = 1 << 20, 64, 32
rng = np.random.default_rng(0)
s = rng.integers(0, V, 8_000_000)
d = rng.integers(0, V, 8_000_000)
g = stg.stg_static_graph_create(V, s, d, stg.STG_SELF_LOOPS)
p = {k: torch.from_numpy(v).cuda() for k, v in gen.tgcn_params(F, H, 1).items()}
X = torch.rand(V, F, device="cuda")
Hp = torch.rand(V, H, device="cuda")
for dbg in [0, 1, 2, 4, 8, 12, 13, 15]:
    os.environ["STG_XW_DEBUG"] = str(dbg)
    for _ in range(2):
        stg.stg_tgcn_step(g.view(), p, X, Hp)
    torch.cuda.synchronize()
    stg.stg_profile_enable(True)
    stg.stg_profile_read(reset=True)
    for _ in range(10):
        stg.stg_tgcn_step(g.view(), p, X, Hp)
    torch.cuda.synchronize()
    prof = stg.stg_profile_read(reset=True)
    stg.stg_profile_enable(False)
    print(json.dumps({"dbg": dbg, **{k: round(v[0] / max(v[1], 1), 4) for k, v in prof.items() if v[1]}}), flush=True)
