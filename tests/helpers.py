"""Shared helpers for the GPU parity tests: comparisons against the oracle."""
import numpy as np
import torch

import oracle

GRAPH_KEYS = ("in_rowptr", "in_col", "out_rowptr", "out_col", "in_deg", "out_deg", "in_ids", "out_ids")


def assert_graph_equal(gpu: dict, ref: dict, edge_ids: bool = True, tag=""):
    """Bit-exact for every integer array; norms within one fp32 rounding of fp64."""
    for k in GRAPH_KEYS:
        a = gpu[k].cpu().numpy()
        b = np.asarray(ref[k])
        assert a.shape == b.shape, (tag, k, a.shape, b.shape)
        if not np.array_equal(a, b):
            bad = np.nonzero(a != b)[0][:10]
            raise AssertionError("%s %s differs at %s: gpu %s ref %s" % (tag, k, bad, a[bad], b[bad]))
    if edge_ids:
        assert np.array_equal(gpu["out_eid"].cpu().numpy(), ref["out_eid"]), (tag, "out_eid")
    # in_row / out_row are the COO row ids implied by the rowptrs
    V = ref["V"]
    assert np.array_equal(gpu["in_row"].cpu().numpy(), np.repeat(np.arange(V), np.diff(ref["in_rowptr"])))
    assert np.array_equal(gpu["out_row"].cpu().numpy(), np.repeat(np.arange(V), np.diff(ref["out_rowptr"])))
    for k in ("norm_src", "norm_dst"):
        a = gpu[k].cpu().numpy().astype(np.float64)
        np.testing.assert_allclose(a, ref[k], rtol=2.5e-7, atol=0, err_msg=k)


def cond_err(y_gpu, y_ref, scale) -> float:
    """Reading C19: max_i |y_gpu - y_ref| / s_i with s_i the oracle over |x|;
    rows/entries with s_i = 0 must be exactly 0 on the GPU."""
    y = np.asarray(y_gpu, np.float64)
    r = np.asarray(y_ref, np.float64)
    s = np.asarray(scale, np.float64)
    zero = s == 0
    assert np.all(y[zero] == 0.0), "nonzero output where the condition scale is 0"
    d = np.abs(y - r)[~zero] / s[~zero]
    return float(d.max()) if d.size else 0.0


def to_gpu(a, dtype=torch.float32):
    return torch.from_numpy(np.ascontiguousarray(a)).to(device="cuda", dtype=dtype)


def oracle_graph_from_set(V, S, dgl_both=False):
    return oracle.csr(V, S, dgl_both)
