"""Event traces: the common input language of the oracle and the CUDA path.

A trace is a list of tuples (SURVEY.md §8(c) trace language):

    ('REG', ptr, bytes, kind)            kind: DEVICE=0, MANAGED=1, HOST=2
    ('FREE', ptr)
    ('KB',) / ('KE',)                    GPU epoch begin / end (kernel launch wrapper)
    ('H', addr, size, acc)               host access; acc: R=1, W=2, RW=3
    ('D', addr, size, acc)               device access (only between KB and KE)
    ('HB', addrs, sizes, accs)           a batch of host accesses (numpy arrays)
    ('DB', addrs, sizes, accs)           a batch of device accesses (numpy arrays)
    ('X', dir, dst, src, bytes)          transfer; dir: H2D=0 D2H=1 H2H=2 D2D=3 MEMSET=4
    ('DIAG', thr_pct, block_words, min_run, reset, names)

Nothing here knows what a shadow record is.
"""
from __future__ import annotations

import itertools

import numpy as np

DEVICE, MANAGED, HOST = 0, 1, 2
R, W, RW = 1, 2, 3
H2D, D2H, H2H, D2D, MEMSET = 0, 1, 2, 3, 4

KIND_CHAR = {DEVICE: "D", MANAGED: "M", HOST: "H"}
ACC_STR = {R: "R", W: "W", RW: "RW"}


def to_text(ops) -> str:
    """Render a trace in the oracle CLI's text format."""
    out = []
    for op in ops:
        t = op[0]
        if t == "REG":
            out.append(f"REG {op[1]:#x} {op[2]} {KIND_CHAR[op[3]]}")
        elif t == "FREE":
            out.append(f"FREE {op[1]:#x}")
        elif t in ("KB", "KE"):
            out.append(t)
        elif t in ("H", "D"):
            out.append(f"{t} {op[1]:#x} {op[2]} {ACC_STR[op[3]]}")
        elif t in ("HB", "DB"):
            c = t[0]
            for a, s, k in zip(op[1].tolist(), op[2].tolist(), op[3].tolist()):
                out.append(f"{c} {a:#x} {s} {ACC_STR[k]}")
        elif t == "X":
            out.append(f"X {op[1]} {op[2]:#x} {op[3]:#x} {op[4]}")
        elif t == "DIAG":
            names = " ".join(f"{a:#x}" for a in op[5])
            out.append(f"DIAG {op[1]} {op[2]} {op[3]} {op[4]} {names}".rstrip())
        elif t == "PAGES":
            out.append(f"PAGES {op[1]}")
        elif t == "ADVISE":
            out.append(f"ADVISE {op[1]:#x} {op[2]} {op[3]} {op[4]}")
        else:
            raise ValueError(op)
    return "\n".join(out) + "\n"


def parse_text(text: str):
    """Parse the text format back into trace tuples (for the golden fixtures)."""
    kinds = {"D": DEVICE, "M": MANAGED, "H": HOST}
    accs = {"R": R, "W": W, "RW": RW}
    ops = []
    for line in text.splitlines():
        line = line.split("#", 1)[0].strip()
        if not line:
            continue
        t = line.split()
        n = lambda s: int(s, 0)
        if t[0] == "REG":
            ops.append(("REG", n(t[1]), n(t[2]), kinds.get(t[3], None) if t[3] in kinds else n(t[3])))
        elif t[0] == "FREE":
            ops.append(("FREE", n(t[1])))
        elif t[0] in ("KB", "KE"):
            ops.append((t[0],))
        elif t[0] in ("H", "D"):
            ops.append((t[0], n(t[1]), n(t[2]), accs[t[3]] if t[3] in accs else n(t[3])))
        elif t[0] == "X":
            ops.append(("X", n(t[1]), n(t[2]), n(t[3]), n(t[4])))
        elif t[0] == "DIAG":
            ops.append(("DIAG", n(t[1]), n(t[2]), n(t[3]), n(t[4]), tuple(n(x) for x in t[5:])))
        elif t[0] == "PAGES":  # the UM page view of the live rows (NEXT-3)
            ops.append(("PAGES", n(t[1])))
        elif t[0] == "ADVISE":  # cudaMemAdvise: ptr bytes advice(1..6) device(-1 = CPU)
            ops.append(("ADVISE", n(t[1]), n(t[2]), n(t[3]), n(t[4])))
        else:
            raise ValueError(line)
    return ops


def batch(kind: str, addrs, sizes, accs):
    """A ('HB'|'DB', ...) op from array-likes."""
    a = np.asarray(addrs, dtype=np.uint64)
    s = np.broadcast_to(np.asarray(sizes, dtype=np.uint32), a.shape).copy()
    k = np.broadcast_to(np.asarray(accs, dtype=np.uint8), a.shape).copy()
    return (kind, a, s, k)


# ---------------------------------------------------------------------------
# Brute-force enumeration (SURVEY.md §8(c) "pins"): one allocation of 2 words,
# up to 3 segments (host or GPU), up to 2 ops per segment from {R,W,RW}x{w0,w1},
# optional reset-diagnose between segments.

SEG_OPS = [()] + [(o,) for o in itertools.product((R, W, RW), (0, 1))] + [
    (a, b) for a in itertools.product((R, W, RW), (0, 1)) for b in itertools.product((R, W, RW), (0, 1))
]


def schedules(max_segments=3):
    """(sides, diag_after) patterns: sides alternate host/GPU, diag_after[i]
    says whether a reset-diagnose follows segment i (the last always has one)."""
    out = []
    for nseg in range(1, max_segments + 1):
        for first in ("H", "G"):
            sides = tuple(first if i % 2 == 0 else ("G" if first == "H" else "H") for i in range(nseg))
            for mask in itertools.product((False, True), repeat=nseg - 1):
                out.append((sides, tuple(mask) + (True,)))
    return out


def enumerated_trace(schedule, assignments, base=0x10000, stride=64, kind=MANAGED):
    """One session: every assignment (a tuple of per-segment op tuples) gets its
    own 8-byte allocation; all share the schedule's epoch/diagnose structure."""
    sides, diag_after = schedule
    ops = []
    bases = []
    for j in range(len(assignments)):
        b = base + j * stride
        bases.append(b)
        ops.append(("REG", b, 8, kind))
    for i, side in enumerate(sides):
        addrs, accs = [], []
        for j, asg in enumerate(assignments):
            for acc, w in asg[i]:
                addrs.append(bases[j] + 4 * w)
                accs.append(acc)
        if side == "H":
            if addrs:
                ops.append(batch("HB", addrs, 4, accs))
        else:
            ops.append(("KB",))
            if addrs:
                ops.append(batch("DB", addrs, 4, accs))
            ops.append(("KE",))
        if diag_after[i]:
            ops.append(("DIAG", 50, 0, 1, 1, ()))
    return ops


def random_trace(seed, n_allocs=6, n_steps=60, max_words=300, p_device=0.5):
    """A seeded random trace over a handful of allocations: host and GPU
    segments, multi-word and unaligned accesses, transfers, frees and
    re-registrations, diagnoses with random parameters.  Always valid."""
    rng = np.random.default_rng(seed)
    ops = []
    live = {}  # base -> bytes
    next_base = [0x100000]

    def new_alloc():
        nbytes = int(rng.integers(1, max_words * 4))
        kind = int(rng.integers(0, 3))
        b = next_base[0]
        next_base[0] += ((nbytes + 4095) // 4096 + 1) * 4096
        live[b] = nbytes
        ops.append(("REG", b, nbytes, kind))

    def rand_access():
        b = list(live)[int(rng.integers(0, len(live)))]
        nb = live[b]
        off = int(rng.integers(0, nb + 8))  # sometimes beyond the end (clipped or missed)
        size = int(rng.choice([1, 2, 4, 8, 16]))
        return b + off, size, int(rng.integers(1, 4))

    for _ in range(n_allocs):
        new_alloc()
    for _ in range(n_steps):
        r = rng.random()
        if r < 0.35:  # host segment
            n = int(rng.integers(1, 40))
            acc = [rand_access() for _ in range(n)]
            ops.append(batch("HB", [a for a, _, _ in acc], [s for _, s, _ in acc], [k for _, _, k in acc]))
        elif r < 0.35 + 0.3 * p_device * 2:  # GPU epoch
            ops.append(("KB",))
            n = int(rng.integers(1, 80))
            acc = [rand_access() for _ in range(n)]
            ops.append(batch("DB", [a for a, _, _ in acc], [s for _, s, _ in acc], [k for _, _, k in acc]))
            if rng.random() < 0.3:  # host accesses while the epoch is open (deferred, D20)
                a, s, k = rand_access()
                ops.append(("H", a, s, k))
            if rng.random() < 0.2:
                b = list(live)[int(rng.integers(0, len(live)))]
                ops.append(("X", MEMSET, b, 0, int(rng.integers(1, live[b] + 1))))
            ops.append(("KE",))
        elif r < 0.80:  # transfer
            b = list(live)[int(rng.integers(0, len(live)))]
            nb = live[b]
            off = int(rng.integers(0, nb))
            nbytes = int(rng.integers(1, nb - off + 1))
            d = int(rng.integers(0, 5))
            b2 = list(live)[int(rng.integers(0, len(live)))]
            off2 = int(rng.integers(0, live[b2]))
            nbytes = min(nbytes, live[b2] - off2)
            nbytes = max(nbytes, 1)
            if d in (H2D, MEMSET):
                ops.append(("X", d, b + off, 0x7000_0000, nbytes))
            elif d == D2H:
                ops.append(("X", d, 0x7000_0000, b + off, nbytes))
            else:
                ops.append(("X", d, b + off, b2 + off2, min(nbytes, nb - off)))
        elif r < 0.88:  # free + re-register (possibly at the same base)
            if len(live) > 1:
                b = list(live)[int(rng.integers(0, len(live)))]
                ops.append(("FREE", b))
                nb = live.pop(b)
                if rng.random() < 0.5:
                    nbytes = int(rng.integers(1, nb + 1))
                    live[b] = nbytes
                    ops.append(("REG", b, nbytes, int(rng.integers(0, 3))))
                else:
                    new_alloc()
        else:
            thr = int(rng.choice([0, 10, 50, 100]))
            blk = int(rng.choice([0, 1, 3, 16, 64, 1000]))
            mr = int(rng.choice([1, 2, 4, 32, 256]))
            names = tuple(list(live)[: int(rng.integers(0, len(live) + 1))])
            ops.append(("DIAG", thr, blk, mr, int(rng.random() < 0.8), names))
    ops.append(("DIAG", 50, 0, 4, 1, ()))
    return ops


def epoch_chain_trace(seed, n_allocs=4, n_chains=3, chain_len=6, max_words=20000, n_ev=3000):
    """Chains of back-to-back GPU epochs (nothing between them: the shape a
    single-launch wavefront with device-side epoch splits produces, NEXT-2),
    each chain preceded by a host segment and followed by a diagnose.  Device
    events hit a few hot words often (so reads of earlier segments' writes
    recur) and random words of every allocation, multi-word and unaligned."""
    rng = np.random.default_rng(seed)
    ops, allocs, base = [], [], 0x200000
    for _ in range(n_allocs):
        nb = int(rng.integers(4, max_words * 4))
        ops.append(("REG", base, nb, int(rng.integers(0, 3))))
        allocs.append((base, nb))
        base += ((nb + 4095) // 4096 + 1) * 4096

    def accesses(n):
        k = rng.integers(0, len(allocs), size=n)
        b = np.array([allocs[i][0] for i in k], np.uint64)
        nb = np.array([allocs[i][1] for i in k], np.int64)
        hot = rng.random(n) < 0.3
        off = np.where(hot, 4 * rng.integers(0, 64, size=n), rng.integers(0, nb))
        size = rng.choice(np.array([1, 2, 4, 8, 16], np.uint32), size=n, p=[0.05, 0.05, 0.6, 0.2, 0.1])
        return b + off.astype(np.uint64), size.astype(np.uint32), rng.integers(1, 4, size=n).astype(np.uint8)

    for _ in range(n_chains):
        ops.append(("HB",) + accesses(int(rng.integers(1, 500))))
        for _ in range(chain_len):
            ops += [("KB",), ("DB",) + accesses(int(rng.integers(1, n_ev))), ("KE",)]
        ops.append(("DIAG", int(rng.choice([10, 50, 100])), int(rng.choice([0, 64, 1000])),
                    int(rng.choice([1, 4, 256])), int(rng.random() < 0.7), ()))
    ops.append(("DIAG", 50, 0, 4, 1, ()))
    return ops


def with_pages(ops, sizes, seed):
    """Insert the UM page view before every diagnose (several page sizes) and
    random cudaMemAdvise calls after registrations."""
    import numpy as np
    rng = np.random.default_rng(seed)
    out = []
    for op in ops:
        if op[0] == "DIAG":
            out += [("PAGES", int(P)) for P in sizes]
        out.append(op)
        if op[0] == "REG" and rng.random() < 0.6:
            out.append(("ADVISE", op[1] + int(rng.integers(0, op[2])), 4, int(rng.integers(1, 7)),
                        int(rng.choice([-1, 0]))))
    return out
