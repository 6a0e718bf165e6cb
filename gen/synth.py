"""Seeded synthetic inputs shaped like the paper's datasets.

This module is shared by the oracle tests, the CUDA parity tests and bench.py.
It holds NO arithmetic of the method (no CSR build, no normalisation, no
aggregation, no GRU): it only draws numbers and turns an event stream into the
per-timestamp add/delete batches that the paper's preprocessing describes
(§VII.B: "The first half of the dataset is the first snapshot.
Then the window is moved ... In the case of STGraph-GPMA, the data is further
processed to contain changes between consecutive snapshots").

Every random number is a counter hash h(seed, stream, i) built from splitmix64,
so any language can reproduce the same bits.  Feature values are
(h>>40)/2^24 scaled to [-1,1) or [0,1): multiples of 2^-23 / 2^-24, exact in
fp32 (reading C18).
"""
from __future__ import annotations

import dataclasses
import numpy as np

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser over uint64 (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = (np.asarray(x, dtype=np.uint64) + _GOLDEN)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def counter_hash(seed: int, stream: int, n: int, start: int = 0) -> np.ndarray:
    """h(seed, stream, i) for i in [start, start+n): splitmix64(key + i*golden)."""
    with np.errstate(over="ignore"):
        key = splitmix64(np.array([(seed & 0xFFFFFFFF) << 32 | (stream & 0xFFFFFFFF)], dtype=np.uint64))[0]
        i = np.arange(start, start + n, dtype=np.uint64)
        return splitmix64(key + i * _GOLDEN)


def uniform_pm1(seed: int, stream: int, n: int) -> np.ndarray:
    """fp32 values in [-1, 1), multiples of 2^-23 (exact in fp32)."""
    h = counter_hash(seed, stream, n)
    return ((h >> np.uint64(40)).astype(np.float64) / float(1 << 24) * 2.0 - 1.0).astype(np.float32)


def uniform_01(seed: int, stream: int, n: int) -> np.ndarray:
    """fp32 values in [0, 1), multiples of 2^-24 (exact in fp32)."""
    h = counter_hash(seed, stream, n)
    return ((h >> np.uint64(40)).astype(np.float64) / float(1 << 24)).astype(np.float32)


def unit_f64(seed: int, stream: int, n: int) -> np.ndarray:
    """float64 in [0,1) with 53 random bits (for sampling decisions only)."""
    h = counter_hash(seed, stream, n)
    return (h >> np.uint64(11)).astype(np.float64) * (1.0 / float(1 << 53))


def permutation(seed: int, stream: int, n: int) -> np.ndarray:
    """A seeded permutation of [0, n) (argsort of counter hashes)."""
    return np.argsort(counter_hash(seed, stream, n), kind="stable").astype(np.int64)


def zipf_ids(seed: int, stream: int, n: int, V: int, alpha: float, perm: np.ndarray) -> np.ndarray:
    """n ids drawn with P(rank k) ∝ (k+1)^-alpha, ranks mapped through perm."""
    w = np.arange(1, V + 1, dtype=np.float64) ** (-alpha)
    cdf = np.cumsum(w)
    u = unit_f64(seed, stream, n) * cdf[-1]
    r = np.searchsorted(cdf, u, side="right")
    np.minimum(r, V - 1, out=r)
    return perm[r]


# --------------------------------------------------------------------------
# Workload table (SURVEY §8 "Config sizes", BASELINE.json configs[0..4])
# --------------------------------------------------------------------------
@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    kind: str          # "static" | "dtdg"
    V: int
    F: int
    H: int
    T: int             # timestamps (static); for dtdg filled from the window
    seed: int
    E: int = 0         # static: directed edges incl. loops as generated
    M: int = 0         # dtdg: events
    rho: float = 0.0   # dtdg: probability an event repeats an earlier pair
    slide: int = 0     # dtdg: events the window moves per timestamp
    alpha: float = 0.8
    desc: str = ""


CONFIGS = {
    # BASELINE.json configs[0]: Hungary-Chickenpox-shaped (Table II row 3)
    "C1": Config("C1", "static", V=20, F=4, H=16, T=520, seed=1, E=102,
                 desc="hungary-chickenpox-shaped static-temporal"),
    # configs[1]: Wikimath-shaped (Table II row 1), density 0.024
    "C2": Config("C2", "static", V=1068, F=8, H=32, T=731, seed=2, E=27079,
                 desc="wikimath-shaped static-temporal"),
    # configs[2]: Windmill-large-shaped: 319^2 = 101,761 ("102K", complete incl. loops)
    "C3": Config("C3", "static", V=319, F=8, H=32, T=17472, seed=3, E=319 * 319,
                 desc="windmill-large-shaped static-temporal"),
    # configs[3]: sx-mathoverflow-shaped DTDG (Table II row 9: 24K nodes, 506K temporal edges)
    "C4": Config("C4", "dtdg", V=24818, F=8, H=32, T=0, seed=4, M=506550, rho=0.5,
                 slide=9400, desc="sx-mathoverflow-shaped DTDG"),
    # configs[4]: wiki-talk-temporal-shaped DTDG scaled to ~1M nodes / ~8M edges
    "C5": Config("C5", "dtdg", V=1 << 20, F=64, H=32, T=0, seed=5, M=16_500_000, rho=0.0,
                 slide=206_000, desc="wiki-talk-temporal-shaped DTDG, scaled to 2^20 nodes"),
    # scaled-down C5 for element-by-element parity (same recipe, smaller V and M)
    "C5s": Config("C5s", "dtdg", V=1 << 14, F=64, H=32, T=0, seed=6, M=240_000, rho=0.0,
                  slide=3000, desc="C5 recipe at V=2^14 (parity size)"),
    # C6 (optional, Montevideo-bus-shaped, Table II row 4)
    "C6": Config("C6", "static", V=675, F=4, H=16, T=740, seed=7, E=690,
                 desc="montevideo-bus-shaped static-temporal"),
}


# --------------------------------------------------------------------------
# Static graphs (edge lists only)
# --------------------------------------------------------------------------
def _c1_edges(cfg: Config):
    V = cfg.V
    iu, ju = np.triu_indices(V, k=1)                  # 190 undirected candidate pairs
    order = np.argsort(counter_hash(cfg.seed, 10, iu.size), kind="stable")
    npairs = (cfg.E - V) // 2                         # 41 pairs -> 82 directed + 20 loops
    a, b = iu[order[:npairs]], ju[order[:npairs]]
    loops = np.arange(V)
    src = np.concatenate([a, b, loops])
    dst = np.concatenate([b, a, loops])
    return src.astype(np.int32), dst.astype(np.int32)


def _chung_lu_edges(cfg: Config, n_target: int, loops: bool):
    """Distinct directed pairs, src/dst Zipf(alpha) over permuted ids, kept in draw order."""
    V = cfg.V
    perm_s = permutation(cfg.seed, 11, V)
    perm_d = permutation(cfg.seed, 12, V)
    keys_seen = np.zeros(0, dtype=np.int64)
    out_s, out_d = [], []
    have = 0
    batch = max(4 * n_target, 1024)
    start = 0
    while have < n_target:
        s = zipf_ids(cfg.seed, 13 + 2 * start, batch, V, cfg.alpha, perm_s)
        d = zipf_ids(cfg.seed, 14 + 2 * start, batch, V, cfg.alpha, perm_d)
        if not loops:
            keep = s != d
            s, d = s[keep], d[keep]
        k = s.astype(np.int64) * V + d
        allk = np.concatenate([keys_seen, k])
        _, first = np.unique(allk, return_index=True)
        first = np.sort(first)
        new = first[first >= keys_seen.size] - keys_seen.size
        new = new[: n_target - have]
        out_s.append(s[new]); out_d.append(d[new])
        keys_seen = np.concatenate([keys_seen, k[new]])
        have += new.size
        start += 1
    return np.concatenate(out_s).astype(np.int32), np.concatenate(out_d).astype(np.int32)


def _c6_edges(cfg: Config):
    """Montevideo-bus-like: random successor links (bus routes), 690 distinct non-loop pairs."""
    V = cfg.V
    perm = permutation(cfg.seed, 20, V)
    src = perm
    dst = np.roll(perm, -1)
    extra = cfg.E - V
    h = counter_hash(cfg.seed, 21, 4 * extra)
    cand_s = (h[: 2 * extra] % np.uint64(V)).astype(np.int64)
    cand_d = (h[2 * extra:] % np.uint64(V)).astype(np.int64)
    keep = cand_s != cand_d
    k = np.concatenate([src * V + dst, cand_s[keep] * V + cand_d[keep]])
    _, first = np.unique(k, return_index=True)
    first = np.sort(first)[: cfg.E]
    k = k[first]
    return (k // V).astype(np.int32), (k % V).astype(np.int32)


def static_edges(cfg: Config):
    """(src, dst) int32 edge list of a static config (no normalisation applied)."""
    if cfg.name == "C1":
        return _c1_edges(cfg)
    if cfg.name == "C2":
        return _chung_lu_edges(cfg, cfg.E, loops=False)
    if cfg.name == "C3":
        i, j = np.meshgrid(np.arange(cfg.V), np.arange(cfg.V), indexing="ij")
        return i.ravel().astype(np.int32), j.ravel().astype(np.int32)
    if cfg.name == "C6":
        return _c6_edges(cfg)
    raise ValueError(cfg.name)


def random_edges(seed: int, V: int, E: int, loops: bool = True, stream: int = 30):
    """Uniform random (possibly duplicated) directed edges for small tests."""
    h = counter_hash(seed, stream, 2 * E)
    s = (h[:E] % np.uint64(max(V, 1))).astype(np.int32)
    d = (h[E:] % np.uint64(max(V, 1))).astype(np.int32)
    if not loops:
        keep = s != d
        s, d = s[keep], d[keep]
    return s, d


# --------------------------------------------------------------------------
# DTDG: event stream -> sliding window -> base + add/delete batches
# --------------------------------------------------------------------------
@dataclasses.dataclass
class DTDG:
    V: int
    T: int
    W: int                # window length in events
    slide: int            # window step in events
    ev_src: np.ndarray    # int32 [M] events in time order
    ev_dst: np.ndarray
    src0: np.ndarray      # base snapshot S_0 (distinct pairs of window 0)
    dst0: np.ndarray
    add_off: np.ndarray   # int64 [T+1], batch 0 empty
    add_src: np.ndarray
    add_dst: np.ndarray
    del_off: np.ndarray
    del_src: np.ndarray
    del_dst: np.ndarray

    def window(self, t: int):
        """Event index range [lo, hi) that defines snapshot t."""
        lo = t * self.slide
        return lo, lo + self.W


def events(cfg: Config):
    """Temporal edge stream (src, dst) int32 of length cfg.M, in time order."""
    V, M = cfg.V, cfg.M
    perm_s = permutation(cfg.seed, 40, V)
    perm_d = permutation(cfg.seed, 41, V)
    s = zipf_ids(cfg.seed, 42, M, V, cfg.alpha, perm_s)
    d = zipf_ids(cfg.seed, 43, M, V, cfg.alpha, perm_d)
    # self-loops are not part of the interaction streams: re-draw dst uniformly
    loop = np.nonzero(s == d)[0]
    if loop.size:
        h = counter_hash(cfg.seed, 44, loop.size)
        d[loop] = (s[loop] + 1 + (h % np.uint64(V - 1)).astype(np.int64)) % V
    if cfg.rho > 0.0:
        # with probability rho an event repeats the pair of a uniformly chosen earlier event
        r = unit_f64(cfg.seed, 45, M)
        j = np.floor(unit_f64(cfg.seed, 46, M) * np.arange(M)).astype(np.int64)
        orig = np.arange(M, dtype=np.int64)
        rep = (r < cfg.rho) & (np.arange(M) > 0)
        orig[rep] = j[rep]
        while True:                       # resolve chains to a fresh event
            nxt = orig[orig]
            if np.array_equal(nxt, orig):
                break
            orig = nxt
        s, d = s[orig], d[orig]
    return s.astype(np.int32), d.astype(np.int32)


def dtdg_from_events(V: int, ev_src: np.ndarray, ev_dst: np.ndarray, W: int, slide: int) -> DTDG:
    """Sliding-window DTDG: snapshot t = distinct pairs of events [t*slide, t*slide+W).

    Each event e is visible for timestamps t with t*slide <= e < t*slide + W.  Per pair
    the visibility intervals are merged; a merged run [lo, hi] contributes an add at lo
    (lo > 0), a delete at hi+1 (hi < T-1), and membership of S_0 when lo == 0.
    """
    M = ev_src.size
    T = (M - W) // slide + 1
    e = np.arange(M, dtype=np.int64)
    lo = np.maximum(0, (e - W) // slide + 1)
    hi = np.minimum(T - 1, e // slide)
    ok = lo <= hi
    key = ev_src.astype(np.int64) * V + ev_dst.astype(np.int64)
    idx = np.nonzero(ok)[0]
    order = idx[np.argsort(key[idx], kind="stable")]
    k, l, h = key[order], lo[order], hi[order]
    newrun = np.ones(k.size, dtype=bool)
    newrun[1:] = (k[1:] != k[:-1]) | (l[1:] > h[:-1] + 1)
    starts = np.nonzero(newrun)[0]
    ends = np.append(starts[1:], k.size) - 1
    run_key, run_lo = k[starts], l[starts]
    # hi is nondecreasing within a pair, so the run end is the hi of its last event
    run_hi = np.maximum.reduceat(h, starts) if k.size else h
    base = run_key[run_lo == 0]
    a_sel = run_lo > 0
    d_sel = run_hi < T - 1
    a_t, a_k = run_lo[a_sel], run_key[a_sel]
    d_t, d_k = run_hi[d_sel] + 1, run_key[d_sel]
    ao = np.lexsort((a_k, a_t)); a_t, a_k = a_t[ao], a_k[ao]
    do = np.lexsort((d_k, d_t)); d_t, d_k = d_t[do], d_k[do]
    add_off = np.searchsorted(a_t, np.arange(T + 1), side="left").astype(np.int64)
    del_off = np.searchsorted(d_t, np.arange(T + 1), side="left").astype(np.int64)
    base = np.sort(base)
    return DTDG(V=V, T=T, W=W, slide=slide, ev_src=ev_src, ev_dst=ev_dst,
                src0=(base // V).astype(np.int32), dst0=(base % V).astype(np.int32),
                add_off=add_off, add_src=(a_k // V).astype(np.int32), add_dst=(a_k % V).astype(np.int32),
                del_off=del_off, del_src=(d_k // V).astype(np.int32), del_dst=(d_k % V).astype(np.int32))


def dtdg(cfg: Config) -> DTDG:
    ev_s, ev_d = events(cfg)
    return dtdg_from_events(cfg.V, ev_s, ev_d, cfg.M // 2, cfg.slide)


# --------------------------------------------------------------------------
# Per-timestamp features, labels and model parameters
# --------------------------------------------------------------------------
def features(cfg: Config, t: int, width: int | None = None, nonneg: bool = False) -> np.ndarray:
    w = cfg.F if width is None else width
    f = uniform_01 if nonneg else uniform_pm1
    return f(cfg.seed, 1000 + t, cfg.V * w).reshape(cfg.V, w)


def labels(cfg: Config, t: int) -> np.ndarray:
    return uniform_pm1(cfg.seed, 500_000 + t, cfg.V)


def tgcn_params(F: int, H: int, seed: int, scale: float = 1.0):
    """TGCN parameters, U[±1/sqrt(fan_in)]; layout as in include/stg.h.

    W [F,3H] (z|r|h), b [3H], L [3][2H,H], l [3][H], head w_o [H], b_o [1].
    """
    def u(stream, n, fan_in):
        return (uniform_pm1(seed, stream, n).astype(np.float64) * scale / np.sqrt(fan_in)).astype(np.float32)
    return {
        "W": u(900, F * 3 * H, F).reshape(F, 3 * H),
        "b": u(901, 3 * H, F),
        "L": u(902, 3 * 2 * H * H, 2 * H).reshape(3, 2 * H, H),
        "l": u(903, 3 * H, 2 * H).reshape(3, H),
        "w_o": u(904, H, H),
        "b_o": u(905, 1, H),
    }


def edge_weights(seed: int, n: int, lo: float = 0.5, hi: float = 2.0, stream: int = 40) -> np.ndarray:
    """n seeded positive edge weights in [lo, hi) (NEXT-4 inputs), multiples of 2^-24 scaled."""
    return (lo + (hi - lo) * uniform_01(seed, stream, n)).astype(np.float32)


def tgcn2_params(F: int, H: int, seed: int, scale: float = 1.0):
    """Original T-GCN cell parameters (NEXT-2): Wg [F+H, 2H] (r | u), bg [2H], Wc [F+H, H],
    bc [H], U[±1/sqrt(fan_in)], plus the surrogate head w_o [H], b_o [1]."""
    K = F + H
    a = scale / np.sqrt(K)

    def u(stream, n, bound):
        return (uniform_pm1(seed, stream, n) * np.float32(bound)).astype(np.float32)
    return {"Wg": u(81, K * 2 * H, a).reshape(K, 2 * H), "bg": u(82, 2 * H, a),
            "Wc": u(83, K * H, a).reshape(K, H), "bc": u(84, H, a),
            "w_o": u(85, H, scale / np.sqrt(H)), "b_o": u(86, 1, scale / np.sqrt(H))}
