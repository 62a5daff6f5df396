"""Rodinia-shaped workloads (BASELINE.json configs[1]):
array specs, seeded inputs, and the CPU twin of each instrumented program as an
event trace for the oracle.

The CUDA programs are csrc/work_rodinia.cu (xplw_hotspot, xplw_backprop); this
module re-states what they access, independently, from the same program
description.  Nothing here computes a shadow record or a diagnosis.

Sizes: backprop 640K inputs (Table III, "Backprop 640K"), hid 16;
hotspot 1024 x 1024 x 20 iterations (Rodinia default, not from the paper).
"""
from __future__ import annotations

import numpy as np

from .trace import D2H, DEVICE, H2D, HOST, R, RW, W, batch

ALIGN = 256


def layout(spec, dev_base, host_base):
    """Place the arrays of `spec` [(name, nbytes, kind, where)] in two arenas;
    returns (addrs, total_dev_bytes, total_host_bytes)."""
    off = {"dev": 0, "host": 0}
    addrs = []
    for name, nbytes, kind, where in spec:
        base = dev_base if where == "dev" else host_base
        addrs.append(base + off[where])
        off[where] += (nbytes + ALIGN - 1) // ALIGN * ALIGN + ALIGN
    return addrs, off["dev"], off["host"]


def arena_sizes(spec):
    _, d, h = layout(spec, 0, 0)
    return d, h


# ---------------------------------------------------------------------------
# hotspot
def hotspot_spec(rows, cols):
    n = rows * cols * 4
    return [("temp_host", n, HOST, "host"), ("power_host", n, HOST, "host"),
            ("result_host", n, HOST, "host"), ("d_power", n, DEVICE, "dev"),
            ("d_temp0", n, DEVICE, "dev"), ("d_temp1", n, DEVICE, "dev")]


def hotspot_accesses(rows, cols):
    return 7 * rows * cols


def hotspot_trace(addrs, spec, rows, cols, iters, diag_each, params):
    temp_h, power_h, result_h, d_power, d_t0, d_t1 = addrs
    n = rows * cols
    ops = [("REG", a, s[1], s[2]) for a, s in zip(addrs, spec)]
    ar = np.arange(n, dtype=np.uint64)
    ops.append(batch("HB", temp_h + 4 * ar, 4, W))
    ops.append(batch("HB", power_h + 4 * ar, 4, W))
    ops.append(("X", H2D, d_power, power_h, 4 * n))
    ops.append(("X", H2D, d_t0, temp_h, 4 * n))
    i = np.repeat(np.arange(rows, dtype=np.int64), cols)
    j = np.tile(np.arange(cols, dtype=np.int64), rows)
    idx = i * cols + j
    nb = [idx, np.maximum(i - 1, 0) * cols + j, np.minimum(i + 1, rows - 1) * cols + j,
          i * cols + np.maximum(j - 1, 0), i * cols + np.minimum(j + 1, cols - 1)]
    t = [d_t0, d_t1]
    src = 0
    for _ in range(iters):
        a = np.concatenate([t[src] + 4 * x.astype(np.uint64) for x in nb] +
                           [d_power + 4 * idx.astype(np.uint64), t[1 - src] + 4 * idx.astype(np.uint64)])
        acc = np.concatenate([np.full(6 * n, R, np.uint8), np.full(n, W, np.uint8)])
        ops += [("KB",), batch("DB", a, 4, acc), ("KE",)]
        src = 1 - src
        if diag_each:
            ops.append(("DIAG",) + params + (1, ()))
    ops.append(("X", D2H, result_h, t[src], 4 * n))
    ops.append(batch("HB", result_h + 4 * ar, 4, R))
    ops += [("FREE", a) for a in addrs]
    ops.append(("DIAG",) + params + (1, ()))
    return ops


# ---------------------------------------------------------------------------
# backprop
BP = 16


def backprop_spec(n_in, hid):
    nw = (n_in + 1) * (hid + 1) * 4
    nblk = n_in // BP
    return [("input_units", (n_in + 1) * 4, HOST, "host"), ("input_weights", nw, HOST, "host"),
            ("partial_sum", nblk * hid * 4, HOST, "host"), ("hidden_delta", (hid + 1) * 4, HOST, "host"),
            ("prev_weights", nw, HOST, "host"),
            ("input_cuda", (n_in + 1) * 4, DEVICE, "dev"), ("output_hidden_cuda", (hid + 1) * 4, DEVICE, "dev"),
            ("input_hidden_cuda", nw, DEVICE, "dev"), ("hidden_partial_sum", nblk * hid * 4, DEVICE, "dev"),
            ("hidden_delta_cuda", (hid + 1) * 4, DEVICE, "dev"),
            ("input_prev_weights_cuda", nw, DEVICE, "dev")]


def backprop_accesses(n_in, hid):
    nblk = n_in // BP
    return nblk * BP * BP * 2 + nblk * BP * 2 + nblk * BP * BP * 5 + BP * 4


def backprop_trace(addrs, spec, n_in, hid, params):
    (input_units, input_weights, partial_sum, hidden_delta, prev_weights, input_cuda,
     _output_hidden_cuda, input_hidden_cuda, hidden_partial_sum, hidden_delta_cuda,
     input_prev_weights_cuda) = addrs
    nblk = n_in // BP
    nw = (n_in + 1) * (hid + 1)
    ops = [("REG", a, s[1], s[2]) for a, s in zip(addrs, spec)]
    u64 = lambda x: np.asarray(x, dtype=np.uint64)
    ops.append(batch("HB", input_units + 4 * u64(np.arange(n_in + 1)), 4, W))
    ops.append(batch("HB", input_weights + 4 * u64(np.arange(nw)), 4, W))
    ops.append(batch("HB", prev_weights + 4 * u64(np.arange(nw)), 4, W))
    ops.append(("X", H2D, input_cuda, input_units, (n_in + 1) * 4))
    ops.append(("X", H2D, input_hidden_cuda, input_weights, nw * 4))
    # thread grid: block by, threads (ty, tx) in 16 x 16
    by = np.repeat(np.arange(nblk, dtype=np.int64), BP * BP)
    ty = np.tile(np.repeat(np.arange(BP, dtype=np.int64), BP), nblk)
    tx = np.tile(np.arange(BP, dtype=np.int64), nblk * BP)
    index = (hid + 1) * BP * by + (hid + 1) * ty + tx + 1 + (hid + 1)
    index_in = BP * by + ty + 1
    # layerforward: tx==0 reads the input unit; every thread reads and rewrites its
    # weight; ty==0 writes the tile's partial sum of column tx
    a = np.concatenate([input_cuda + 4 * u64(index_in[tx == 0]), input_hidden_cuda + 4 * u64(index),
                        input_hidden_cuda + 4 * u64(index), hidden_partial_sum + 4 * u64((by * hid + tx)[ty == 0])])
    k = np.concatenate([np.full((tx == 0).sum(), R), np.full(index.size, R), np.full(index.size, W),
                        np.full((ty == 0).sum(), W)]).astype(np.uint8)
    ops += [("KB",), batch("DB", a, 4, k), ("KE",)]
    ops.append(("X", D2H, partial_sum, hidden_partial_sum, nblk * hid * 4))
    jj = np.repeat(np.arange(hid, dtype=np.int64), nblk)
    kk = np.tile(np.arange(nblk, dtype=np.int64), hid)
    ops.append(batch("HB", partial_sum + 4 * u64(kk * hid + jj), 4, R))
    ops.append(batch("HB", hidden_delta + 4 * u64(np.arange(hid + 1)), 4, W))
    ops.append(("X", H2D, hidden_delta_cuda, hidden_delta, (hid + 1) * 4))
    ops.append(("X", H2D, input_prev_weights_cuda, prev_weights, nw * 4))
    # adjust_weights
    index_y = BP * by + ty + 1
    index_x = tx + 1
    bias = (ty == 0) & (by == 0)
    a = np.concatenate([hidden_delta_cuda + 4 * u64(index_x), input_cuda + 4 * u64(index_y),
                        input_prev_weights_cuda + 4 * u64(index), input_hidden_cuda + 4 * u64(index),
                        hidden_delta_cuda + 4 * u64(index_x[bias]), input_prev_weights_cuda + 4 * u64(index_x[bias]),
                        input_hidden_cuda + 4 * u64(index_x[bias])])
    k = np.concatenate([np.full(2 * index.size, R), np.full(2 * index.size, RW),
                        np.full(bias.sum(), R), np.full(2 * bias.sum(), RW)]).astype(np.uint8)
    ops += [("KB",), batch("DB", a, 4, k), ("KE",)]
    ops.append(("X", D2H, input_weights, input_hidden_cuda, nw * 4))
    ops.append(("X", D2H, input_units, input_cuda, (n_in + 1) * 4))
    ops += [("FREE", a) for a in addrs]
    ops.append(("DIAG",) + params + (1, ()))
    return ops


def fill_inputs(name, host_arrays, seed):
    """Seeded input values for the apps' host arrays (torch pinned tensors or numpy).
    The access pattern of hotspot and backprop does not depend on them."""
    rng = np.random.default_rng(seed)
    for t in host_arrays:
        a = t.numpy() if hasattr(t, "numpy") else t
        a.view(np.float32)[:] = rng.random(a.size // 4, dtype=np.float32)
