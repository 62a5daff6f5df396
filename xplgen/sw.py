"""Smith-Waterman workload (the paper's SW study, Fig. 7/8 P:L341-349; SURVEY §8(d)
cfg1 SW-128 and cfg3 SW-16K): seeded sequences, the exact DP the kernels compute,
and the CPU twin of csrc/work_sw.cu (xplw_sw) as an event trace for the oracle.
No shadow arithmetic here."""
from __future__ import annotations

import numpy as np

from .trace import MANAGED, R, W, batch

MATCH, MISMATCH, GAP = 3, -3, 2


def sw_spec(n, m):
    return [("a", 4 * n, MANAGED, "managed"), ("b", 4 * m, MANAGED, "managed"),
            ("H", 4 * (n + 1) * (m + 1), MANAGED, "managed")]


def sw_inputs(n, m, seed):
    rng = np.random.default_rng(seed)
    return {"a": rng.integers(0, 4, size=n).astype(np.int32), "b": rng.integers(0, 4, size=m).astype(np.int32)}


def sw_dp(a, b):
    """H of Smith-Waterman (floor 0), by anti-diagonals."""
    n, m = len(a), len(b)
    H = np.zeros((n + 1, m + 1), np.int32)
    for d in range(2, n + m + 1):
        i = np.arange(max(1, d - m), min(n, d - 1) + 1)
        j = d - i
        s = np.where(a[i - 1] == b[j - 1], MATCH, MISMATCH)
        h = np.maximum(np.maximum(H[i - 1, j - 1] + s, H[i - 1, j] - GAP), H[i, j - 1] - GAP)
        H[i, j] = np.maximum(h, 0)
    return H


def sw_traceback(H, a, b):
    """The host traceback of xplw_sw: start cell and the cells/elements it reads."""
    n, m = H.shape[0] - 1, H.shape[1] - 1
    flat = H.reshape(-1)
    at = int(np.argmax(flat))  # first maximum, row-major
    ld = m + 1
    i, j = at // ld, at % ld
    reads_h, reads_a, reads_b, length = [], [], [], 0
    while i > 0 and j > 0:
        h = H[i, j]
        reads_h.append(i * ld + j)
        if h == 0:
            break
        length += 1
        reads_a.append(i - 1)
        reads_b.append(j - 1)
        sc = MATCH if a[i - 1] == b[j - 1] else MISMATCH
        reads_h.append((i - 1) * ld + j - 1)
        if H[i - 1, j - 1] + sc == h:
            i, j = i - 1, j - 1
            continue
        reads_h.append((i - 1) * ld + j)
        if H[i - 1, j] - GAP == h:
            i -= 1
        else:
            j -= 1
    return reads_h, reads_a, reads_b, length


def _diag_cells(n, m, d):
    i = np.arange(max(1, d - m), min(n, d - 1) + 1, dtype=np.int64)
    return i, d - i


def sw_trace(addrs, spec, n, m, per_diagonal, tb_every, diag_every, inp, params):
    return list(sw_trace_iter(addrs, spec, n, m, per_diagonal, tb_every, diag_every, inp, params))


def sw_trace_iter(addrs, spec, n, m, per_diagonal, tb_every, diag_every, inp, params):
    """The CPU twin of xplw_sw, op by op (a generator: cfg3's full trace, ~2e9
    events, never has to exist at once)."""
    A, B, Hh = addrs
    ld = m + 1
    u64 = lambda x: np.asarray(x, dtype=np.uint64)
    for x, s in zip(addrs, spec):
        yield ("REG", x, s[1], s[2])
    yield batch("HB", A + 4 * u64(np.arange(n)), 4, W)
    yield batch("HB", B + 4 * u64(np.arange(m)), 4, W)
    yield batch("HB", Hh + 4 * u64(np.arange((n + 1) * (m + 1))), 4, W)

    def cell_events(i, j):
        rd = np.concatenate([A + 4 * u64(i - 1), B + 4 * u64(j - 1), Hh + 4 * u64((i - 1) * ld + j - 1),
                             Hh + 4 * u64((i - 1) * ld + j), Hh + 4 * u64(i * ld + j - 1)])
        wr = Hh + 4 * u64(i * ld + j)
        return ("DB", np.concatenate([rd, wr]).astype(np.uint64), np.full(rd.size + wr.size, 4, np.uint32),
                np.concatenate([np.full(rd.size, R, np.uint8), np.full(wr.size, W, np.uint8)]))

    if not per_diagonal:
        ii = np.repeat(np.arange(1, n + 1, dtype=np.int64), m)
        jj = np.tile(np.arange(1, m + 1, dtype=np.int64), n)
        yield ("KB",)
        yield cell_events(ii, jj)
        yield ("KE",)
    elif per_diagonal == 2:
        # one launch with a device-side epoch split after every anti-diagonal:
        # the same event sequence as one launch per diagonal (KE KB at a split)
        for d in range(2, n + m + 1):
            i, j = _diag_cells(n, m, d)
            yield ("KB",)
            yield cell_events(i, j)
            yield ("KE",)
    else:
        for d in range(2, n + m + 1):
            i, j = _diag_cells(n, m, d)
            yield ("KB",)
            yield cell_events(i, j)
            yield ("KE",)
            if tb_every > 0 and (d - 1) % tb_every == 0:
                yield batch("HB", Hh + 4 * u64(i * ld + j), 4, R)
            if diag_every > 0 and (d - 1) % diag_every == 0:
                yield ("DIAG",) + params + (1, ())
    H = sw_dp(inp["a"], inp["b"])
    yield batch("HB", Hh + 4 * u64(np.arange((n + 1) * (m + 1))), 4, R)
    rh, ra, rb, _ = sw_traceback(H, inp["a"], inp["b"])
    yield batch("HB", np.concatenate([Hh + 4 * u64(rh), A + 4 * u64(ra), B + 4 * u64(rb)]), 4, R)
    if per_diagonal != 1:
        ii = np.repeat(np.arange(1, n + 1, dtype=np.int64), m)
        jj = np.tile(np.arange(1, m + 1, dtype=np.int64), n)
        yield ("KB",)
        yield batch("DB", Hh + 4 * u64(ii * ld + jj), 4, W)
        yield ("KE",)
    for x in addrs:
        yield ("FREE", x)
    yield ("DIAG",) + params + (1, ())


def sw_accesses(n, m, per_diagonal):
    """per_diagonal: 0 = one launch, 1 = one launch per anti-diagonal, 2 = one
    launch with a device-side epoch split per anti-diagonal."""
    return 6 * n * m + (0 if per_diagonal == 1 else n * m)
