"""Independent HISTORY-based evaluator: the pin for the oracle's state machine.

The oracle (oracle/xpl_oracle.cpp) keeps one record per word and updates it
event by event.  This module never keeps a record: it stores every write and
read of every word with a timestamp and answers each question of the paper
from the history directly (SURVEY.md §8(c) "pins"):

  * wC / wG  = some CPU / GPU write fell in the interval
  * rXY      = some read by Y in the interval whose *visible* last write
               was made by X (CPU if there was none, reading D3)
               - a host read at time t sees the latest write before t;
               - a GPU read in epoch e sees the latest write before e
                 began (snapshot, D5); GPU writes of e land when e ends.
  * host events issued while a GPU epoch is open happen after it     (D20)

Report fields are then recomputed here from those per-word facts, with runs
found by a regular expression and blocks by slicing, i.e. by different code
from the oracle's loops.  Pure Python: for tiny traces only.
"""
from __future__ import annotations

import re

R, W = 1, 2


class _Row:
    def __init__(self, rid, base, nbytes, kind):
        self.id, self.base, self.bytes, self.kind = rid, base, nbytes, kind
        self.words = (nbytes + 3) // 4
        self.live = True
        self.ever = False
        self.writes = {}  # word -> [(time, side)]
        self.reads = {}   # word -> [(time, reader_side, origin_side)]


def _words(rows_live, addr, size):
    if size == 0:
        return None, []
    cands = [r for r in rows_live if r.base <= addr < r.base + r.bytes]
    if not cands:
        return None, []
    r = cands[0]
    w0 = (addr - r.base) // 4
    w1 = min(r.words - 1, (addr + size - 1 - r.base) // 4)
    return r, list(range(w0, w1 + 1))


def _origin(row, w, t):
    best = None
    for tw, side in row.writes.get(w, []):
        if tw < t and (best is None or tw > best[0]):
            best = (tw, side)
    return "C" if best is None else best[1]


def evaluate(ops):
    rows = []
    live = lambda: [r for r in rows if r.live]
    clock = [0]
    interval_start = [0]
    depth = [0]
    epoch = {"start": None, "events": [], "deferred": []}
    results = []

    def tick():
        clock[0] += 2
        return clock[0]

    def host(addr, size, acc):
        r, ws = _words(live(), addr, size)
        if r is None:
            return
        r.ever = True
        t = tick()
        for w in ws:
            if acc & R:
                r.reads.setdefault(w, []).append((t, "C", _origin(r, w, t)))
            if acc & W:
                r.writes.setdefault(w, []).append((t + 1, "C"))

    def dev(addr, size, acc):
        r, ws = _words(live(), addr, size)
        if r is None:
            return
        r.ever = True
        epoch["events"].append((r, ws, acc))

    def kb():
        if depth[0] == 0:
            epoch["start"] = tick()
            epoch["events"] = []
            epoch["deferred"] = []
        depth[0] += 1

    def ke():
        depth[0] -= 1
        if depth[0]:
            return
        t0 = epoch["start"]
        t1 = tick()
        for r, ws, acc in epoch["events"]:
            for w in ws:
                if acc & R:
                    r.reads.setdefault(w, []).append((t0, "G", _origin(r, w, t0)))
        for r, ws, acc in epoch["events"]:
            for w in ws:
                if acc & W:
                    r.writes.setdefault(w, []).append((t1, "G"))
        for f, args in epoch["deferred"]:
            f(*args)

    def copy(d, dst, src, nbytes):
        if d == 0:
            host(dst, nbytes, W)
        elif d == 1:
            host(src, nbytes, R)
        elif d == 2:
            host(src, nbytes, R)
            host(dst, nbytes, W)
        else:
            own = depth[0] == 0
            if own:
                kb()
            if d == 3:
                dev(src, nbytes, R)
            dev(dst, nbytes, W)
            if own:
                ke()

    def diag(thr, block_words, min_run, reset, names):
        t_now = tick()
        lo = interval_start[0]
        min_run = max(min_run, 1)
        out = []
        for r in rows:
            if not r.live and getattr(r, "dropped", False):
                continue
            bits = []
            for w in range(r.words):
                wr = [(t, s) for t, s in r.writes.get(w, []) if lo <= t <= t_now]
                rd = [(t, y, x) for t, y, x in r.reads.get(w, []) if lo <= t <= t_now]
                b = {
                    "wC": any(s == "C" for _, s in wr),
                    "wG": any(s == "G" for _, s in wr),
                    "rCC": any(y == "C" and x == "C" for _, y, x in rd),
                    "rGC": any(y == "C" and x == "G" for _, y, x in rd),
                    "rCG": any(y == "G" and x == "C" for _, y, x in rd),
                    "rGG": any(y == "G" and x == "G" for _, y, x in rd),
                }
                bits.append(b)
            cpu = [b["wC"] or b["rCC"] or b["rGC"] for b in bits]
            gpu = [b["wG"] or b["rCG"] or b["rGG"] for b in bits]
            rep = {
                "id": r.id, "base": r.base, "bytes": r.bytes, "words": r.words,
                "kind": r.kind, "live": int(r.live),
                "w_c": sum(b["wC"] for b in bits), "w_g": sum(b["wG"] for b in bits),
                "r_cc": sum(b["rCC"] for b in bits), "r_cg": sum(b["rCG"] for b in bits),
                "r_gc": sum(b["rGC"] for b in bits), "r_gg": sum(b["rGG"] for b in bits),
                "any_acc": sum(c or g for c, g in zip(cpu, gpu)),
                "gpu_acc": sum(gpu),
                "alternating": sum(c and g and (b["wC"] or b["wG"]) for c, g, b in zip(cpu, gpu, bits)),
            }
            rep["density_pct_any"] = (100 * rep["any_acc"]) // r.words
            rep["density_pct_gpu"] = (100 * rep["gpu_acc"]) // r.words
            B = block_words or r.words
            nb = nw = 0
            for k in range(0, r.words, B):
                blk = gpu[k:k + B]
                g = sum(blk)
                if g >= 1 and 100 * g <= thr * len(blk):
                    nb += 1
                    nw += len(blk)
            rep["low_density_blocks"], rep["low_density_words"] = nb, nw
            for key, pred in (("h2d_unused", lambda b: b["wC"] and not b["rCG"]),
                              ("d2h_unneeded", lambda b: b["rCC"])):
                s = "".join("1" if pred(b) else "0" for b in bits)
                lens = [len(m) for m in re.findall("1+", s) if len(m) >= min_run]
                rep[key + "_runs"] = len(lens)
                rep[key + "_words"] = sum(lens)
            rep["ever_accessed"] = int(r.ever)
            f = 0
            if r.kind == 1 and rep["alternating"]:
                f |= 1
            if r.kind in (0, 1) and rep["low_density_blocks"]:
                f |= 2
            if r.kind == 0 and rep["h2d_unused_runs"]:
                f |= 4
            if r.kind == 0 and rep["d2h_unneeded_runs"]:
                f |= 8
            if rep["any_acc"] == 0:
                f |= 16
            rep["flags"] = f
            rep["name_idx"] = 0xFFFFFFFF
            if r.live:
                for j, a in enumerate(names):
                    if r.base <= a < r.base + r.bytes:
                        rep["name_idx"] = j
                        break
            out.append(rep)
        if reset:
            interval_start[0] = tick()
            for r in rows:
                if not r.live:
                    r.dropped = True
        return out

    for op in ops:
        t = op[0]
        if t == "REG":
            rows.append(_Row(len(rows), op[1], op[2], op[3]))
        elif t == "FREE":
            for r in rows:
                if r.live and r.base == op[1]:
                    r.live = False
                    break
        elif t == "KB":
            kb()
        elif t == "KE":
            ke()
        elif t in ("H", "HB"):
            items = [(op[1], op[2], op[3])] if t == "H" else list(zip(op[1].tolist(), op[2].tolist(), op[3].tolist()))
            for a, s, k in items:
                if depth[0]:
                    epoch["deferred"].append((host, (a, s, k)))
                else:
                    host(a, s, k)
        elif t in ("D", "DB"):
            items = [(op[1], op[2], op[3])] if t == "D" else list(zip(op[1].tolist(), op[2].tolist(), op[3].tolist()))
            for a, s, k in items:
                dev(a, s, k)
        elif t == "X":
            if depth[0] and op[1] <= 2:
                epoch["deferred"].append((copy, (op[1], op[2], op[3], op[4])))
            else:
                copy(op[1], op[2], op[3], op[4])
        elif t == "DIAG":
            results.append(diag(*op[1:6]))
    return results
