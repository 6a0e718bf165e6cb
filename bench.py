#!/usr/bin/env python
"""bench.py — STGraph hot path on B200: one step = one Algorithm-1 TGCN training
epoch over the C5 DTDG (wiki-talk-temporal-shaped, 2^20 nodes,
~8M edges + self-loops, T=41 on-demand snapshots, F=64, H=32, sequences of 16).

Every step runs, per timestamp t: Get-Graph(t) (delta-apply snapshot build),
P' = X_t·W, forward aggregation over the in-CSR, GRU; then per sequence in LIFO
order: Get-Backward-Graph(t), head gradient, GRU backward, backward aggregation
over the out-CSR, dW; and one SGD step per sequence.

metric: aggregated edges/s (fwd+bwd) = Σ_t 2·|E_t| per epoch ÷ epoch time
(plus timesteps/s).  `--impl reference` times the fp64 oracle on the host.
Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "aggregated edges/s (fwd+bwd)"
UNIT = "edges/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5")
    ap.add_argument("--seq", type=int, default=16, help="sequence length S (reading C16)")
    ap.add_argument("--lr", type=float, default=1e-3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--mode", default="sharded", choices=["sharded", "peer", "replicas"],
                    help="N>1: row-block shards of one graph with X_t resident on every rank (SURVEY §8(e) "
                         "resident mode, default), row-block shards with X_t row-sharded and P' rows gathered "
                         "from their owners over NVLink peer memory (sharded mode; also runs at N=1), or "
                         "independent replicas")
    ap.add_argument("--graphs", type=int, default=-1,
                    help="replay each epoch as one CUDA graph (1/0; default: on for static-temporal configs, "
                         "whose tiny per-timestamp work is launch-bound, off for DTDGs)")
    ap.add_argument("--schedule", default="auto", choices=["auto", "batched", "per-step"],
                    help="static graphs: sequence-batched (NEXT-1, default) or per-timestamp Algorithm-1 driver")
    ap.add_argument("--naive", action="store_true",
                    help="DTDG configs: NaiveGraph mode (every snapshot materialised at create, P:L202-204; "
                         "Table III's time/memory trade-off against the default on-demand snapshots)")
    ap.add_argument("--order", default="linear-first", choices=["linear-first", "aggregate-first"],
                    help="graph-convolution order (reading C14): linear-first Â(XW)+b, the headline (forward over "
                         "the in-CSR at width 3H, backward over the out-CSR), or aggregate-first (ÂX)W+b (SURVEY "
                         "§8(f) NEXT-1: forward at width F, no backward aggregation or backward snapshots)")
    ap.add_argument("--shard-sim", default=None, metavar="K/N",
                    help="(testing on one GPU) run rank K's row block of an N-way sharding, no process group")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks and throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.Q,
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for n, v in zip(names, f[3:7]):
                if v.lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def workload_name(cfg) -> str:
    """The config.workload string both arms print (the BASELINE.json config it is shaped on)."""
    names = ["C1", "C2", "C3", "C4", "C5"]
    return cfg.desc + (" (BASELINE.json configs[%d])" % names.index(cfg.name) if cfg.name in names else "")


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs (STREAM-style copy, burst)"
    return 6650.0, "fallback 6.65 TB/s (B200_PROFILING.md)"


# ------------------------------------------------------------------ oracle (CPU baseline / reference arm)
def oracle_timestep(cfg, d, t: int, S_prev):
    """The fp64 oracle on one C5 timestep: Get-Graph (fold S_{t-1} -> S_t), CSR pair
    build, TGCN forward, MSE head, TGCN backward.  Returns (edges aggregated, seconds, S_t)."""
    import gen
    import oracle
    X = gen.features(cfg, t % 2)
    Y = gen.labels(cfg, t)
    p = gen.tgcn_params(cfg.F, cfg.H, cfg.seed)
    Hp = np.zeros((cfg.V, cfg.H))
    t0 = time.perf_counter()
    A, D = oracle.batch(d, t)
    s_, d_ = oracle.unkey(D)
    D = D[s_ != d_]
    S = oracle.set_apply(S_prev, D, np.concatenate([A, oracle.keys(np.arange(cfg.V), np.arange(cfg.V))]))
    g = oracle.csr(cfg.V, S)
    f = oracle.tgcn_fwd(g, p, X, Hp)
    grads = oracle.zero_grads(cfg.F, cfg.H)
    _, dH = oracle.mse_head(f["Hn"], Y, p["w_o"], p["b_o"], grads)
    oracle.tgcn_bwd(g, p, X, Hp, f, dH, grads)
    dt = time.perf_counter() - t0
    return 2 * g["E"], dt, S


def oracle_timestep_static(cfg, g, t: int, reps: int = 1):
    """The fp64 oracle on `reps` timesteps of a static-temporal config (the graph is
    built once, outside the timing): TGCN forward, MSE head, TGCN backward."""
    import gen
    import oracle
    X = gen.features(cfg, t % 2)
    Y = gen.labels(cfg, t)
    p = gen.tgcn_params(cfg.F, cfg.H, cfg.seed)
    Hp = np.zeros((cfg.V, cfg.H))
    t0 = time.perf_counter()
    for _ in range(reps):
        f = oracle.tgcn_fwd(g, p, X, Hp)
        grads = oracle.zero_grads(cfg.F, cfg.H)
        _, dH = oracle.mse_head(f["Hn"], Y, p["w_o"], p["b_o"], grads)
        oracle.tgcn_bwd(g, p, X, Hp, f, dH, grads)
    return 2 * g["E"] * reps, time.perf_counter() - t0


def static_reps(cfg) -> int:
    """Timesteps per oracle sample: about 20 M edge-visits of work (seconds of CPU)."""
    return max(1, int(2e7 // max(1, 2 * cfg.E)))


def host_info() -> dict:
    """nproc and the CPU model of the box the oracle baseline ran on."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.startswith("Model name:"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


def run_reference(args):
    import gen
    import oracle
    cfg = gen.CONFIGS[args.config]
    oracle.build()
    threads = oracle.use_openmp(True)          # the oracle on ALL host cores (its OpenMP build)
    edges, secs = 0, 0.0
    if cfg.kind == "static":
        s_, d_ = gen.static_edges(cfg)
        g = oracle.static_graph(cfg.V, s_, d_, self_loops=True)
        reps = static_reps(cfg)
        for i in range(args.warmup + args.steps):
            e, dt = oracle_timestep_static(cfg, g, i, reps)
            if i >= args.warmup:
                edges += e
                secs += dt
        value = edges / secs
        sample = ("per step: %d %s timesteps (TGCN fwd + MSE head + bwd on the static CSR) in the fp64 oracle"
                  % (reps, cfg.name))
        T = cfg.T
    else:
        d = gen.dtdg(cfg)
        S = next(oracle.snapshot_sets_fold(d, self_loops=True))
        t = 1
        for i in range(args.warmup + args.steps):
            e, dt, S = oracle_timestep(cfg, d, t, S)
            if i >= args.warmup:
                edges += e
                secs += dt
            t = t + 1 if t + 1 < d.T else 1
            if t == 1:
                S = next(oracle.snapshot_sets_fold(d, self_loops=True))
        value = edges / secs
        sample = ("per step: one %s timestep (fold S_{t-1}->S_t, CSR pair, TGCN fwd + MSE head + bwd) in the fp64 "
                  "oracle" % cfg.name)
        T = d.T
    out = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / args.steps,
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": workload_name(cfg), "config": cfg.name, "V": cfg.V, "F": cfg.F, "H": cfg.H, "T": T,
                      "sample": sample},
           "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                            "sample": sample + " (OpenMP build of the same oracle source, %d threads)" % threads,
                            "host": host_info()},
           "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# ------------------------------------------------------------------ our arm
def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        if rank == 0:
            run_reference(args)
        return

    import torch
    import torch.distributed as dist

    import gen
    import paper_conf_ipps_cherianmcc24_b200 as stg

    sim = args.shard_sim is not None
    if sim:
        rank, world = (int(x) for x in args.shard_sim.split("/"))
    # STG_BENCH_BACKEND=gloo: functional check of the N > 1 flow with every rank on the
    # GPUs that exist (ranks share a device when there are fewer GPUs than ranks)
    backend = os.environ.get("STG_BENCH_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    pg = world > 1 and not sim                  # a real process group (torchrun)
    peer = args.mode == "peer" and not sim
    if pg:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    elif peer:                                  # N=1 sharded mode: a one-rank group for the peer plumbing
        import socket
        with socket.socket() as sk:
            sk.bind(("127.0.0.1", 0))
            port = sk.getsockname()[1]
        dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=0, world_size=1)
    dev = torch.device("cuda", local)
    cfg = gen.CONFIGS[args.config]
    static = cfg.kind == "static"
    if static:
        s_e, d_e = gen.static_edges(cfg)
        d = None
        T = cfg.T
    else:
        d = gen.dtdg(cfg)
        s_e, d_e = d.src0, d.dst0
        T = d.T
    V, F, H = cfg.V, cfg.F, cfg.H
    S = args.seq
    seqs = [(t0, min(S, T - t0)) for t0 in range(0, T, S)]
    # N > 1, sharded (default): destination row blocks with ~E/N in-edges of S_0 each
    # (SURVEY §8(e)); each rank's DTDG holds the edges into its block, X_t is resident
    # on every rank, and the per-sequence gradients are summed by one NCCL all-reduce.
    sharded = (world > 1 and args.mode == "sharded") or peer
    lo, hi = 0, V
    bounds = [0, V]
    if sharded:
        from paper_conf_ipps_cherianmcc24_b200 import parallel
        bounds = parallel.base_row_blocks(V, s_e, d_e, world, self_loops=True)
        lo, hi = bounds[rank], bounds[rank + 1]
    R = hi - lo
    batched = static and not sharded and (args.schedule in ("auto", "batched"))
    peer_drv = None
    if peer:
        from paper_conf_ipps_cherianmcc24_b200 import parallel
        peer_drv = parallel.PeerTGCN(stg, bounds, V, F, H, S)
    dist_arg = (rank, world, lo, hi) if sharded else None
    if static:
        g = stg.stg_static_graph_create(V, s_e, d_e, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS, dist=dist_arg)
        E_t = [g.view().num_edges] * T
    else:
        g = stg.stg_dtdg_create(V, T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                                d.del_dst, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS |
                                (stg.STG_NAIVE if args.naive else 0), dist=dist_arg)
        E_t = [g.num_edges(t) for t in range(T)]
    agg_first = args.order == "aggregate-first"
    stg.stg_set_conv_order(1 if agg_first else 0)
    # aggregated edges per epoch: every snapshot forward and backward (linear-first), forward only
    # (aggregate-first: the backward needs no aggregation)
    edges_per_step = (1 if agg_first else 2) * sum(E_t)   # this rank's edges (whole graph unless sharded)
    edges_all = edges_per_step
    if pg:
        te = torch.tensor([float(edges_per_step)], dtype=torch.float64, device=torch.device("cuda", local))
        dist.all_reduce(te)
        edges_all = int(te.item())

    # inputs: 2 distinct seeded X_t matrices cycled over t (each 256 MB > L2), labels per t
    NX = 2
    # (sharded mode: every rank holds only its rows of X_t)
    Xh = [torch.from_numpy(gen.features(cfg, i)[lo:hi].copy() if peer else gen.features(cfg, i))
          for i in range(NX)]
    Yh = [torch.from_numpy(gen.labels(cfg, t)[lo:hi].copy()) for t in range(T)]
    Xd = [x.to(dev) for x in Xh]
    Yd = [y.to(dev) for y in Yh]
    p = {k: torch.from_numpy(v).to(dev) for k, v in gen.tgcn_params(F, H, cfg.seed).items()}
    # all gradients live in one flat buffer: one all-reduce per sequence when sharded
    gshapes = {"W": (F, 3 * H), "b": (3 * H,), "L": (3, 2 * H, H), "l": (3, H), "w_o": (H,), "b_o": (1,)}
    gflat = torch.zeros(sum(int(np.prod(v)) for v in gshapes.values()), device=dev)
    gv, off = {}, 0
    for k, shp in gshapes.items():
        n = int(np.prod(shp))
        gv[k] = gflat[off:off + n].view(shp)
        off += n
    grads = {k: gv[k] for k in ("W", "b", "L", "l")}
    dw_o, db_o = gv["w_o"], gv["b_o"]
    loss = torch.zeros(1, device=dev)
    Hbuf = [torch.empty(S, R, H, device=dev) for _ in range(2)]
    H0 = torch.zeros(R, H, device=dev)
    Gw = torch.empty(2, R, H, device=dev)
    stack = stg.stg_state_stack_create(S * max(R, 1) * (3 * H + (F if agg_first else 0)) * 4 + (64 << 20))
    stream = torch.cuda.current_stream()

    def sgd():
        if sharded and pg:
            dist.all_reduce(gflat)               # whole-graph gradient = Σ_ranks (NCCL, ~51 KB)
        for k in ("W", "b", "L", "l"):
            stg.stg_sgd_update(p[k], grads[k], args.lr)
        stg.stg_sgd_update(p["w_o"], dw_o, args.lr)
        stg.stg_sgd_update(p["b_o"], db_o, args.lr)

    def epoch(Xsrc, Ysrc):
        Hprev = H0
        for k, (t0, n) in enumerate(seqs):
            Hs = Hbuf[k % 2]
            if peer:
                peer_drv.train_sequence(g, t0, p, p["w_o"], p["b_o"], [Xsrc(t) for t in range(t0, t0 + n)],
                                        [Ysrc(t) for t in range(t0, t0 + n)], Hprev, Hs, grads, dw_o, db_o, loss)
            elif batched:
                stg.stg_tgcn_train_sequence_batched(g, n, p, p["w_o"], p["b_o"], [Xsrc(t) for t in range(t0, t0 + n)],
                                                    [Ysrc(t) for t in range(t0, t0 + n)], Hprev, Hs, grads, dw_o,
                                                    db_o, loss, stack)
            else:
                stg.stg_tgcn_train_sequence(g, t0, n, p, p["w_o"], p["b_o"], [Xsrc(t) for t in range(t0, t0 + n)],
                                            [Ysrc(t) for t in range(t0, t0 + n)], Hprev, Hs, Gw, grads, dw_o, db_o,
                                            loss, stack)
            sgd()
            Hprev = Hs[n - 1]

    Xdev = lambda t: Xd[t % NX]
    Ydev = lambda t: Yd[t]
    for _ in range(args.warmup):
        epoch(Xdev, Ydev)
    torch.cuda.synchronize()
    # CUDA graph of one whole epoch (static graphs: no host-side snapshot state), replayed
    # (DTDGs too when the epoch is launch-bound — its features fit in L2, e.g. C4: the
    # snapshot cache walk is the same every epoch, and the row scan's tile claims and
    # status tags are device-side, so replays are exact; tests/test_gpu_tgcn.py)
    small = V * 3 * H * 4 <= 64 * (1 << 20)
    use_graphs = (args.graphs == 1) or (args.graphs < 0 and (static or small) and not pg and not peer)
    cg = None
    run_epoch = lambda: epoch(Xdev, Ydev)
    launches_per_epoch = None
    if use_graphs:
        # capture on a stream that has already run an epoch: the library's per-stream
        # scratch (aggregation work queues, partials) exists before the capture, so
        # nothing is allocated while capturing
        cap_s = torch.cuda.Stream(device=dev)
        cap_s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(cap_s):
            epoch(Xdev, Ydev)
        torch.cuda.current_stream().wait_stream(cap_s)
        torch.cuda.synchronize()
        cg = torch.cuda.CUDAGraph()
        l0 = stg.kernel_launch_count()
        with torch.cuda.graph(cg, stream=cap_s, capture_error_mode="relaxed"):
            epoch(Xdev, Ydev)
        launches_per_epoch = stg.kernel_launch_count() - l0
        cg.replay()
        torch.cuda.synchronize()
        run_epoch = cg.replay

    # ---------------- timed region (device-resident inputs)
    clocks = ClockSampler(local)
    # per-phase CUDA events are recorded during the timed region itself (on the stream
    # each phase is launched on): they give the aggregation's average launch time for
    # the roofline; the pipelined phases overlap, so the phase SPLIT comes from a
    # single-stream pass below
    stg.stg_profile_read(reset=True)
    stg.stg_profile_enable(True)
    if pg:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    time.sleep(0.3)
    launches0 = stg.kernel_launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for _ in range(args.steps):
        run_epoch()
    ev1.record(stream)
    torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1)
    launches = stg.kernel_launch_count() - launches0
    prof_timed = stg.stg_profile_read(reset=True)
    stg.stg_profile_enable(False)
    if cg is not None:
        launches = launches_per_epoch * args.steps       # graph replays launch the captured kernels
    clk = clocks.stop()
    if pg:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = t.item()
        dist.barrier()
    value = edges_all * args.steps / (ms / 1e3)
    # sharded: the ranks advance the same T timestamps together; replicas: N epochs
    tsps = (1 if sharded else world) * T * args.steps / (ms / 1e3)

    # ---------------- per-phase device times: single-stream pass (same work, one kernel after another)
    nprof = max(1, min(args.steps, 2))
    stg.stg_set_pipeline(False)
    stg.stg_profile_read(reset=True)
    stg.stg_profile_enable(True)
    e0s, e1s = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0s.record(stream)
    for _ in range(nprof):
        epoch(Xdev, Ydev)
    e1s.record(stream)
    torch.cuda.synchronize()
    ms_single = e0s.elapsed_time(e1s) / nprof
    prof = stg.stg_profile_read(reset=True)
    stg.stg_profile_enable(False)
    stg.stg_set_pipeline(True)
    sub = {k: prof.pop(k) for k in ("snap_step", "snap_transpose")}

    # roofline of the dominant kernel: the aggregation (fwd + bwd, W = 3H), timed in the timed region
    Wagg = F if agg_first else 3 * H
    E_mean = sum(E_t) / T                       # this rank's edges per snapshot
    # compulsory bytes per launch: col 4E + rowptr 4(V+1) + node_ids 4V + row scale 4V
    # + read each source row once 4VW + write each output row 4VW
    # (sharded rank, mean of fwd and bwd: the fwd reads all V source rows and writes R rows, the bwd the
    # reverse; R = V unsharded gives 4E + 4(V+1) + 8V + 8VW)
    alg_bytes = 4 * E_mean + 2 * (V + 1) + 2 * (R + 1) + 4 * (V + R) + 4 * Wagg * (V + R)
    f_ms, f_n = prof_timed["agg_fwd"]
    b_ms, b_n = prof_timed["agg_bwd"]
    agg_timing = "CUDA events around every aggregation launch on its stream, over the timed region"
    if f_n + b_n == 0:                  # graph replay: no per-launch events, take the single-stream pass
        f_ms, f_n = prof["agg_fwd"]
        b_ms, b_n = prof["agg_bwd"]
        agg_timing = ("CUDA events around every aggregation launch in the single-stream pass (the timed "
                      "region replays a CUDA graph: no per-launch events)")
    agg_avg_s = ((f_ms + b_ms) / (f_n + b_n)) / 1e3 if (f_n + b_n) else float("nan")
    agg_fwd_s = (f_ms / f_n) / 1e3 if f_n else float("nan")
    agg_bwd_s = (b_ms / b_n) / 1e3 if b_n else float("nan")
    peak, peak_src = measured_peaks()
    achieved = alg_bytes / agg_avg_s / 1e9
    traffic, traffic_src = None, None
    tp = os.path.join(ROOT, "profiles", "agg_traffic.json")
    if os.path.exists(tp):
        try:
            tj = json.load(open(tp))
            traffic, traffic_src = tj.get("bytes_per_launch"), tj.get("source")
        except Exception:
            traffic = None
    step_ms_prof = sum(v[0] for v in prof.values()) / nprof
    # snapshot builder roofline: compulsory bytes of ONE delta step of ONE CSR
    # direction, unsharded: read/write col (4E each), rowptr (4(V+1) each), the whole-graph
    # in/out degrees (read + write 4V each), node_ids (read deg 4V, write ids 4V), norms (8V),
    # schedule items (16 B per row) and the sorted deltas (8 B per key, read by the merge and
    # by the degree histogram: 16 B per delta)
    snap_rl = None
    if not static and sub["snap_step"][1]:
        nd = [g.num_deltas(t, False) + g.num_deltas(t, True) for t in range(1, T)]
        d_mean = sum(nd) / max(1, len(nd))
        sbytes = 8 * E_mean + 8 * (V + 1) + 16 * V + 8 * V + 8 * V + 16 * V + 16 * d_mean
        st_s = sub["snap_step"][0] / sub["snap_step"][1] / 1e3
        snap_rl = {"bound": "hbm", "achieved": sbytes / st_s / 1e9, "peak": peak, "unit": "GB/s",
                   "frac": sbytes / st_s / 1e9 / peak, "alg_bytes_per_step": sbytes,
                   "avg_step_us": st_s * 1e6, "steps_per_epoch": sub["snap_step"][1] / nprof,
                   "transposes_per_epoch": sub["snap_transpose"][1] / nprof,
                   "avg_transpose_us": (1e3 * sub["snap_transpose"][0] / sub["snap_transpose"][1]
                                        if sub["snap_transpose"][1] else None),
                   "bytes_model": "one delta step of one CSR direction: 8E col + 8(V+1) rowptr + 16V degrees "
                                  "+ 8V node_ids + 8V norms + 16V schedule items + 16|delta|",
                   "timing": "CUDA events around each delta step in the single-stream pass"}
    tensor_pipe = None
    tpp = os.path.join(ROOT, "profiles", "tensor_pipe.json")
    if os.path.exists(tpp):
        try:
            tensor_pipe = json.load(open(tpp))
        except Exception:
            tensor_pipe = None

    # ---------------- end-to-end through the public API with host buffers
    e2e = None
    if not args.no_e2e:
        Xpin = [x.pin_memory() for x in Xh]
        Ypin = [y.pin_memory() for y in Yh]
        # a copy stream (STG_E2E_COPY_STREAMS > 1 alternates timestamps over several: measured
        # slower, 208 vs 205 ms per C5 epoch) and three staging buffer sets, so the copies of
        # the next sequence — across epoch boundaries too — run while the current one
        # computes; a sequence's set is refilled once the sequence three back is done
        ncs = max(1, int(os.environ.get("STG_E2E_COPY_STREAMS", "1")))
        copies = [torch.cuda.Stream(device=dev) for _ in range(ncs)]
        NB = 3
        stage = [[torch.empty(R if peer else V, F, device=dev) for _ in range(S)] for _ in range(NB)]
        ystage = [[torch.empty(R, device=dev) for _ in range(S)] for _ in range(NB)]
        loss_h = [torch.empty(1, pin_memory=True) for _ in range(2)]
        vals = []
        h2d = 0
        nseq = len(seqs)
        done = [None] * NB

        def issue(gk):
            """H2D copies of global sequence gk (sequence gk % nseq of its epoch) into set gk % NB."""
            nonlocal h2d
            t0, n = seqs[gk % nseq]
            buf = gk % NB
            evs = []
            for i in range(n):
                cs = copies[(t0 + i) % ncs]
                with torch.cuda.stream(cs):
                    if done[buf] is not None:
                        cs.wait_event(done[buf])
                    stage[buf][i].copy_(Xpin[(t0 + i) % NX], non_blocking=True)
                    ystage[buf][i].copy_(Ypin[t0 + i], non_blocking=True)
                    h2d += Xpin[0].numel() * 4 + Ypin[0].numel() * 4
                    ev = torch.cuda.Event()              # per timestamp: its step starts when X_t landed
                    ev.record(cs)
                    evs.append(ev)
            return evs

        def e2e_run(nepochs):
            """nepochs epochs back to back; every epoch reads its loss back (D2H) before the
            next one's result is needed; returns the last loss."""
            nonlocal done
            done = [None] * NB
            total = nepochs * nseq
            ready = issue(0)
            Hprev = H0
            last = None
            vals.clear()
            for gk in range(total):
                k = gk % nseq
                t0, n = seqs[k]
                buf = gk % NB
                if k == 0:
                    Hprev = H0
                per_step = (not peer) and (not batched)
                if not per_step:
                    stream.wait_event(ready[-1])
                nxt = issue(gk + 1) if gk + 1 < total else None
                Hs = Hbuf[k % 2]
                if peer:
                    peer_drv.train_sequence(g, t0, p, p["w_o"], p["b_o"], stage[buf][:n], ystage[buf][:n],
                                            Hprev, Hs, grads, dw_o, db_o, loss)
                elif batched:
                    stg.stg_tgcn_train_sequence_batched(g, n, p, p["w_o"], p["b_o"], stage[buf][:n],
                                                        ystage[buf][:n], Hprev, Hs, grads, dw_o, db_o, loss, stack)
                else:
                    stg.stg_tgcn_train_sequence(g, t0, n, p, p["w_o"], p["b_o"], stage[buf][:n], ystage[buf][:n],
                                                Hprev, Hs, Gw, grads, dw_o, db_o, loss, stack, xy_ready=ready)
                sgd()
                ev = torch.cuda.Event()
                ev.record(stream)
                done[buf] = ev
                Hprev = Hs[n - 1]
                if k == nseq - 1:                        # the epoch's result: D2H now, read one epoch later
                    lb = loss_h[(gk // nseq) % 2]
                    lb.copy_(loss, non_blocking=True)
                    lev = torch.cuda.Event()
                    lev.record(stream)
                    if last is not None:
                        last[1].synchronize()
                        vals.append(float(last[0].item()))
                    last = (lb, lev)
                ready = nxt
            torch.cuda.synchronize()
            vals.append(float(last[0].item()))
            return vals[-1]

        e2e_run(1)
        h2d = 0
        torch.cuda.synchronize()
        if pg:
            dist.barrier()
        t0w = time.perf_counter()
        e2e_run(args.steps)
        e2e_s = time.perf_counter() - t0w
        if pg:
            tt = torch.tensor([e2e_s], device=dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            e2e_s = tt.item()
        e2e = {"value": edges_all * args.steps / e2e_s, "unit": UNIT,
               "h2d_bytes_per_step": int(h2d / args.steps), "d2h_bytes_per_step": 4,
               "ms_per_step": 1e3 * e2e_s / args.steps,
               "note": "X_t (this rank's rows in sharded mode) and y_t copied H2D per timestamp from pinned host "
                       "memory on %d copy stream(s), timestamps alternating; three staging sets so the next "
                       "sequence's copies (across epoch boundaries too) overlap the current one; every "
                       "epoch's loss read back D2H; wall clock over the K epochs" % ncs}

    # ---------------- CPU baseline: the oracle on one C5 timestep, 1 core and all cores (rank 0, N=1 only)
    cpu = None
    if rank == 0 and world == 1 and not sim and not args.no_cpu_baseline:
        import oracle
        oracle.build()
        res = {}
        for omp in (False, True):
            thr = oracle.use_openmp(omp)
            if static:
                reps = static_reps(cfg)
                e_c, dt_c = oracle_timestep_static(cfg, oracle.static_graph(V, s_e, d_e, self_loops=True), 1, reps)
                smp = "%d %s timesteps: TGCN fwd + MSE head + bwd on the static CSR" % (reps, cfg.name)
            else:
                S0 = next(oracle.snapshot_sets_fold(d, self_loops=True))
                e_c, dt_c, _ = oracle_timestep(cfg, d, 1, S0)
                smp = "one %s timestep (t=1): fold S_0->S_1, CSR pair, TGCN fwd + MSE head + bwd" % cfg.name
            res[omp] = (e_c / dt_c, thr, dt_c)
        oracle.use_openmp(False)
        cpu = {"value": res[True][0], "unit": UNIT, "cores": res[True][1], "kind": "oracle",
               "sample": smp + ", fp64; all cores: the OpenMP build of the same oracle source (row loops "
                               "split over %d threads), %.1f s" % (res[True][1], res[True][2]),
               "single_core": {"value": res[False][0], "unit": UNIT, "cores": 1, "seconds": res[False][2]},
               "host": host_info()}

    if rank == 0 or sim:
        out = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 1 if sim else world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": "strong" if sharded else "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": workload_name(cfg), "config": cfg.name,
                       "V": V,
                       "E_mean": int(E_mean), "T": T, "F": F, "H": H, "seq_len": S, "sequences": len(seqs),
                       "step": "one Algorithm-1 training epoch over all T timestamps",
                       "l2": ("inputs larger than L2 (X_t 256 MB, graph ~0.3 GB, state 8 GB)" if cfg.name == "C5"
                              else "working set fits in L2 (not flushed between epochs)"),
                       "cuda_graph": cg is not None,
                       "conv_order": args.order + (" (Â(XW)+b, headline)" if not agg_first else
                                                   " ((ÂX)W+b, NEXT-1: value counts forward aggregations only)"),
                       "schedule": "sequence-batched (NEXT-1)" if batched else "per-timestamp Algorithm 1",
                       "parallelism": ("row-block shards x%d, sharded mode: X_t row-sharded, P' gathered from "
                                       "its owners over CUDA-IPC peer memory inside the aggregation, partial dP "
                                       "reduce-scattered over peer loads" % world) if peer else
                                      (("row-block shards x%d (resident X_t, NCCL gradient all-reduce per "
                                        "sequence)" % world) if sharded else ("replicas" if world > 1 else "single")),
                       "E_local_mean_rank0": int(E_mean)},
            "timesteps_per_s": tsps,
            "graph_memory_bytes": None if static else g.memory(),
            "snapshots": None if static else ("materialised (NaiveGraph, STG_NAIVE)" if args.naive
                                              else "on demand from base + deltas (Algorithm 2 cache)"),
            "shard_sim": args.shard_sim,
            "gpu_launches": int(launches),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "dram_GBps_at_traffic": (traffic / agg_avg_s / 1e9) if traffic else None,
                         "dram_frac_at_traffic": (traffic / agg_avg_s / 1e9 / peak) if traffic else None,
                         "alg_bytes_model": "compulsory: 4E col + 4(V+1) rowptr + 4V node_ids + 4V row scale "
                                            "+ 4VW (each source row once) + 4VW (output)",
                         "kernel": "k_agg_stream + k_agg_hubs (fwd in-CSR + bwd out-CSR, W=%d)" % Wagg,
                         "alg_bytes_per_launch": alg_bytes, "avg_launch_ms": agg_avg_s * 1e3,
                         "avg_fwd_ms": agg_fwd_s * 1e3, "avg_bwd_ms": agg_bwd_s * 1e3,
                         "launches_timed": f_n + b_n,
                         "timing": agg_timing,
                         "traffic_source": traffic_src, "peak_source": peak_src},
            "aggregation_edges_per_s": (2 * E_mean / (agg_fwd_s + agg_bwd_s)) if f_n and b_n else None,
            "aggregation_metric": "SURVEY §8(d): 2E / (t_fwd + t_bwd) at W = 3H for one snapshot (mean E_t), "
                                  "launch times from the timed region",
            "snapshot_roofline": snap_rl,
            "tensor_pipe": tensor_pipe,
            "single_stream_ms_per_step": ms_single,
            "phases_ms_per_step": {k: v[0] / nprof for k, v in prof.items()},
            "phase_share": {k: (v[0] / nprof) / step_ms_prof for k, v in prof.items()} if step_ms_prof else None,
            "fig9_split": ({"gnn": 1.0 - (prof["snapshot"][0] / nprof) / step_ms_prof,
                            "graph_update": (prof["snapshot"][0] / nprof) / step_ms_prof}
                           if step_ms_prof and not static else None),
            "phases_note": "phases from a single-stream pass of the same epoch (stg_set_pipeline(0)): no overlap, "
                           "so the shares are the exact Fig. 9 split (P:L316, L345); the timed region runs the "
                           "three-stream pipeline",
            "clocks": clk,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        print(json.dumps(out), flush=True)
    if peer_drv is not None:
        torch.cuda.synchronize()
        if pg:
            dist.barrier()
        peer_drv.close()
    if pg or peer:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
