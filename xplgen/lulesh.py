"""LULESH-shaped workload (the paper's main study, §II-C, §III-D
P:L261-311, Fig. 4/5): the mesh topology (input) and the
CPU twin of csrc/work_lulesh.cu (xplw_lulesh) as an event trace for the oracle.

The domain object (3736 bytes) is laid out here independently of the
CUDA program (tests/test_gpu_workloads.py checks the offsets against it).
Nothing here computes a shadow record or a diagnosis.
"""
from __future__ import annotations

import numpy as np

from .trace import MANAGED, R, RW, W

# domain layout (bytes)
DOM_BYTES = 3736
NSLOT = 50
OFF_NUMELEM, OFF_NUMNODE, OFF_DT, OFF_TIME, OFF_CYCLE, OFF_PAD = 400, 404, 408, 416, 424, 428
OFF_DTC, OFF_DTH, OFF_MISC, OFF_PARAMS = 432, 440, 448, 504
(X, Y, Z, XD, YD, ZD, XDD, YDD, ZDD, FX, FY, FZ, NODALMASS,
 E, P, Q, V, VOLO, VNEW, DELV, VDOV, AREALG, SS, ELEMMASS, QL, QQ,
 NODELIST, LXIM, LXIP, NODEELEMSTART, CORNERLIST, SYMMX, ELEMBC) = range(33)
TMP_FORCE, TMP_DVDX = 48, 49
NAMES = ["x", "y", "z", "xd", "yd", "zd", "xdd", "ydd", "zdd", "fx", "fy", "fz", "nodalMass",
         "e", "p", "q", "v", "volo", "vnew", "delv", "vdov", "arealg", "ss", "elemMass", "ql", "qq",
         "nodelist", "lxim", "lxip", "nodeElemStart", "nodeElemCornerList", "symmX", "elemBC",
         "letam", "letap", "lzetam", "lzetap", "symmY", "symmZ",
         "delv_xi", "delv_eta", "delv_zeta", "delx_xi", "delx_eta", "delx_zeta", "dxx", "dyy", "dzz"]


def sizes(s):
    ne, nn, nsym = s ** 3, (s + 1) ** 3, (s + 1) ** 2
    return ne, nn, nsym, (ne + 255) // 256


def slot_bytes(s, k):
    ne, nn, nsym, _ = sizes(s)
    if k <= NODALMASS:
        return 8 * nn
    if k <= QQ:
        return 8 * ne
    return {NODELIST: 32 * ne, LXIM: 4 * ne, LXIP: 4 * ne, NODEELEMSTART: 4 * (nn + 1),
            CORNERLIST: 32 * ne, SYMMX: 4 * nsym, ELEMBC: 4 * ne, 33: 4 * ne, 34: 4 * ne, 35: 4 * ne,
            36: 4 * ne, 37: 4 * nsym, 38: 4 * nsym}.get(k, 8 * ne)


def lulesh_spec(s):
    _, _, _, nblk = sizes(s)
    return ([("dom", DOM_BYTES, MANAGED, "managed"), ("dt_block", 16 * nblk, MANAGED, "managed")] +
            [(NAMES[k], slot_bytes(s, k), MANAGED, "managed") for k in range(48)])


def topology(s, seed):
    """nodelist, lxim, lxip, node->corner CSR, symmetry plane, elemBC (int32)."""
    ne, nn, nsym, _ = sizes(s)
    e = np.arange(ne)
    ex, ey, ez = e % s, (e // s) % s, e // (s * s)
    s1 = s + 1
    corners = []
    for dz in (0, 1):
        for dy in (0, 1):
            for dx in (0, 1):
                corners.append((ex + dx) + s1 * ((ey + dy) + s1 * (ez + dz)))
    nodelist = np.stack(corners, axis=1).astype(np.int32)          # ne x 8
    lxim = np.where(ex > 0, e - 1, e).astype(np.int32)
    lxip = np.where(ex < s - 1, e + 1, e).astype(np.int32)
    flat = nodelist.reshape(-1)                                      # corner id = 8e + k
    order = np.argsort(flat, kind="stable")
    start = np.zeros(nn + 1, np.int32)
    np.cumsum(np.bincount(flat, minlength=nn), out=start[1:])
    corner_list = order.astype(np.int32)
    n = np.arange(nn)
    symm = n[(n % s1) == 0].astype(np.int32)
    elem_bc = np.random.default_rng(seed).integers(0, 8, size=ne).astype(np.int32)
    return {NODELIST: nodelist.reshape(-1), LXIM: lxim, LXIP: lxip, NODEELEMSTART: start,
            CORNERLIST: corner_list, SYMMX: symm, ELEMBC: elem_bc}


class _Ev:
    """Collects (addr, size, kind) events of one epoch."""

    def __init__(self):
        self.a, self.s, self.k = [], [], []

    def add(self, addr, size, kind):
        addr = np.asarray(addr, dtype=np.uint64).reshape(-1)
        self.a.append(addr)
        self.s.append(np.full(addr.size, size, np.uint32))
        self.k.append(np.full(addr.size, kind, np.uint8))

    def op(self, t):
        return (t, np.concatenate(self.a), np.concatenate(self.s), np.concatenate(self.k))


def lulesh_trace(addrs, spec, s, steps, topo, params, tmp_addrs, windows=None, reset=1, final=True):
    """The CPU twin of xplw_lulesh: returns (ops, device hook calls).
    tmp_addrs[step] = (force temporary, gradient temporary) base addresses, as
    the program's cudaMallocManaged returned them.

    Sampled form (the cfg5 full-size parity, where the whole trace does not fit):
    windows = {k: [(w0, w1), ...]} word windows of array slot k (0..47); then
    only the events of those words are emitted, plus every event of `dom` and
    `dt_block` -- a word's record depends only on the events that touch it --
    and events of one address repeated inside one GPU epoch are emitted once
    (their multiplicity does not matter, D5/D21).  The temporaries are left out
    (their REG/FREE stay, so ids match); hooks is then None.  reset: the
    diagnoses' reset flag; final=False: no final frees + diagnose (the
    program's keep_allocs)."""
    ops = list(lulesh_trace_iter(addrs, spec, s, steps, topo, params, tmp_addrs, windows, reset, final))
    hooks = None if windows is not None else sum(op[1].size for op in ops if op[0] == "DB")
    return ops, hooks


def lulesh_trace_iter(addrs, spec, s, steps, topo, params, tmp_addrs, windows=None, reset=1, final=True,
                      tmp_windows=None):
    """lulesh_trace op by op (a generator: the full cfg4 trace, ~4e8 events per
    timestep, never has to exist at once).  Sampled form only: tmp_windows =
    {0: [(w0, w1), ...], 1: [...]} keeps the events of those word windows of the
    force (0) / gradient (1) temporaries too (else temporaries have none)."""
    ne, nn, nsym, nblk = sizes(s)
    dom, dtb = addrs[0], addrs[1]
    A = [addrs[2 + k] for k in range(48)]
    u = lambda x: np.asarray(x, dtype=np.uint64)
    for a, sp in zip(addrs, spec):
        yield ("REG", a, sp[1], sp[2])
    sampled = windows is not None
    if sampled:
        tab = {}
        for k in range(48):
            es = 8 if k <= QQ else 4
            t = np.zeros(slot_bytes(s, k) // es, bool)
            for w0, w1 in windows.get(k, ()):
                t[(4 * w0) // es:-(-(4 * w1) // es)] = True
            tab[k] = t

    def D(k, idx):  # a double of slot k
        idx = np.asarray(idx).reshape(-1)
        return A[k] + 8 * u(idx[tab[k][idx]] if sampled else idx)

    def I4(k, idx):  # an int of slot k
        idx = np.asarray(idx).reshape(-1)
        return A[k] + 4 * u(idx[tab[k][idx]] if sampled else idx)

    def rep(addr, n):  # one address read by n threads of a kernel
        return addr * np.ones(min(n, 1) if sampled else n, np.uint64)

    def TMP(fn, which=None, base=None):  # events of a temporary
        if not sampled:
            return fn()
        if not tmp_windows or which not in tmp_windows:
            return np.zeros(0, np.uint64)
        a = np.asarray(fn(), np.uint64).reshape(-1)
        w = (a - np.uint64(base)) >> np.uint64(2)  # first word of each (8-byte) event
        keep = np.zeros(a.size, bool)
        for w0, w1 in tmp_windows[which]:
            keep |= (w + np.uint64(1) >= np.uint64(w0)) & (w < np.uint64(w1))
        return a[keep]

    # ---- host initialisation ----
    h = _Ev()
    h.add(dom + 8 * u(np.arange(NSLOT)), 8, W)
    for off, sz in ((OFF_NUMELEM, 4), (OFF_NUMNODE, 4), (OFF_DT, 8), (OFF_TIME, 8), (OFF_CYCLE, 4),
                    (OFF_PAD, 4), (OFF_DTC, 8), (OFF_DTH, 8)):
        h.add([dom + off], sz, W)
    h.add(dom + OFF_MISC + 4 * u(np.arange(14)), 4, W)
    h.add(dom + OFF_PARAMS + 4 * u(np.arange(808)), 4, W)
    for k in range(48):
        nb = slot_bytes(s, k)
        if k <= QQ:
            h.add(D(k, np.arange(nb // 8)), 8, W)
        else:  # int arrays, and the never-used ones zero-filled as 4-byte words
            h.add(I4(k, np.arange(nb // 4)), 4, W)
    h.add(dtb + 8 * u(np.arange(2 * nblk)), 8, W)
    yield h.op("HB")

    ptr = lambda k, n: rep(dom + 8 * k, n)
    e = np.arange(ne)
    nidx = np.arange(nn)
    nl = topo[NODELIST].reshape(ne, 8).astype(np.int64)
    st, cl = topo[NODEELEMSTART].astype(np.int64), topo[CORNERLIST].astype(np.int64)
    cnt = st[1:] - st[:-1]
    node_of_corner = np.repeat(nidx, cnt)
    symm = topo[SYMMX].astype(np.int64)
    grid_e = nblk * 256
    grid_n = (nn + 255) // 256 * 256
    grid_s = (nsym + 255) // 256 * 256
    numelem = lambda g: rep(dom + OFF_NUMELEM, g)

    for step in range(steps):
        tf, tg = tmp_addrs[step]
        yield ("REG", tf, 8 * 24 * ne, MANAGED)
        yield ("H", dom + 8 * TMP_FORCE, 8, W)
        kernels = []
        # 1 zero forces
        ev = _Ev()
        for k in (FX, FY, FZ):
            ev.add(ptr(k, nn), 8, R)
            ev.add(D(k, nidx), 8, W)
        kernels.append(ev)
        # 2 integrate stress
        ev = _Ev()
        ev.add(numelem(grid_e), 4, R)
        for k in (NODELIST, X, Y, Z):
            ev.add(ptr(k, ne), 8, R)
        for k in (P, Q):
            ev.add(ptr(k, ne), 8, R)
            ev.add(D(k, e), 8, R)
        ev.add(ptr(TMP_FORCE, ne), 8, R)
        ev.add(I4(NODELIST, 8 * e[:, None] + np.arange(8)), 4, R)
        for k in (X, Y, Z):
            ev.add(D(k, nl), 8, R)
        ev.add(TMP(lambda: tf + 8 * u(np.arange(24 * ne)), 0, tf), 8, W)
        kernels.append(ev)
        # 3 hourglass
        ev = _Ev()
        ev.add(numelem(grid_e), 4, R)
        for k in (NODELIST, XD, YD, ZD):
            ev.add(ptr(k, ne), 8, R)
        for k in (SS, ELEMMASS, VOLO, V):
            ev.add(ptr(k, ne), 8, R)
            ev.add(D(k, e), 8, R)
        ev.add(ptr(TMP_FORCE, ne), 8, R)
        ev.add(I4(NODELIST, 8 * e[:, None] + np.arange(8)), 4, R)
        for k in (XD, YD, ZD):
            ev.add(D(k, nl), 8, R)
        ev.add(TMP(lambda: tf + 8 * u(np.arange(24 * ne)), 0, tf), 8, RW)
        kernels.append(ev)
        # 4 corner sums
        ev = _Ev()
        for k in (NODEELEMSTART, CORNERLIST, TMP_FORCE, FX, FY, FZ):
            ev.add(ptr(k, nn), 8, R)
        ev.add(I4(NODEELEMSTART, nidx), 4, R)
        ev.add(I4(NODEELEMSTART, nidx + 1), 4, R)
        ev.add(I4(CORNERLIST, np.arange(len(cl))), 4, R)
        ev.add(TMP(lambda: tf + 8 * u(3 * cl[:, None] + np.arange(3)), 0, tf), 8, R)
        for k in (FX, FY, FZ):
            ev.add(D(k, nidx), 8, W)
        kernels.append(ev)
        for ev in kernels:
            yield ("KB",)
            yield ev.op("DB")
            yield ("KE",)
        yield ("H", dom + 8 * TMP_FORCE, 8, W)
        yield ("FREE", tf)
        kernels = []
        # 5 accel
        ev = _Ev()
        for k in (NODALMASS, FX, FY, FZ):
            ev.add(ptr(k, nn), 8, R)
            ev.add(D(k, nidx), 8, R)
        for k in (XDD, YDD, ZDD):
            ev.add(ptr(k, nn), 8, R)
            ev.add(D(k, nidx), 8, W)
        kernels.append(ev)
        # 6 symmetry
        ev = _Ev()
        ev.add(ptr(SYMMX, nsym), 8, R)
        ev.add(I4(SYMMX, np.arange(nsym)), 4, R)
        for k in (XDD, YDD, ZDD):
            ev.add(ptr(k, nsym), 8, R)
            ev.add(D(k, symm), 8, W)
        kernels.append(ev)
        # 7 velocity, 8 position
        for src, dst in (((XDD, YDD, ZDD), (XD, YD, ZD)), ((XD, YD, ZD), (X, Y, Z))):
            ev = _Ev()
            ev.add(rep(dom + OFF_DT, nn), 8, R)
            for k in src:
                ev.add(ptr(k, nn), 8, R)
                ev.add(D(k, nidx), 8, R)
            for k in dst:
                ev.add(ptr(k, nn), 8, R)
                ev.add(D(k, nidx), 8, RW)
            kernels.append(ev)
        for ev in kernels:
            yield ("KB",)
            yield ev.op("DB")
            yield ("KE",)
        yield ("REG", tg, 8 * 3 * ne, MANAGED)
        yield ("H", dom + 8 * TMP_DVDX, 8, W)
        kernels = []
        # 9 kinematics
        ev = _Ev()
        ev.add(numelem(grid_e), 4, R)
        for k in (NODELIST, X, Y, Z, XD, YD, ZD):
            ev.add(ptr(k, ne), 8, R)
        ev.add(I4(NODELIST, 8 * e[:, None] + np.arange(8)), 4, R)
        for k in (X, Y, Z, XD, YD, ZD):
            ev.add(D(k, nl), 8, R)
        for k in (VOLO, V):
            ev.add(ptr(k, ne), 8, R)
            ev.add(D(k, e), 8, R)
        for k in (VNEW, DELV, AREALG):
            ev.add(ptr(k, ne), 8, R)
            ev.add(D(k, e), 8, W)
        ev.add(ptr(TMP_DVDX, ne), 8, R)
        ev.add(TMP(lambda: tg + 8 * u(np.arange(3 * ne)), 1, tg), 8, W)
        kernels.append(ev)
        # 10 lagrange
        ev = _Ev()
        ev.add(numelem(grid_e), 4, R)
        ev.add(ptr(TMP_DVDX, ne), 8, R)
        ev.add(TMP(lambda: tg + 8 * u(np.arange(3 * ne)), 1, tg), 8, R)
        ev.add(ptr(VNEW, ne), 8, R)
        ev.add(D(VNEW, e), 8, R)
        ev.add(ptr(VDOV, ne), 8, R)
        ev.add(D(VDOV, e), 8, W)
        kernels.append(ev)
        for ev in kernels:
            yield ("KB",)
            yield ev.op("DB")
            yield ("KE",)
        yield ("H", dom + 8 * TMP_DVDX, 8, W)
        yield ("FREE", tg)
        kernels = []
        lxim, lxip = topo[LXIM].astype(np.int64), topo[LXIP].astype(np.int64)
        # 11 monoq gradient
        ev = _Ev()
        ev.add(numelem(grid_e), 4, R)
        for k in (VDOV, LXIM, LXIP, VNEW, QL):
            ev.add(ptr(k, ne), 8, R)
        ev.add(I4(LXIM, e), 4, R)
        ev.add(I4(LXIP, e), 4, R)
        ev.add(D(VDOV, lxip), 8, R)
        ev.add(D(VDOV, lxim), 8, R)
        ev.add(D(VNEW, e), 8, R)
        ev.add(D(QL, e), 8, W)
        kernels.append(ev)
        # 12 monoq region
        ev = _Ev()
        ev.add(numelem(grid_e), 4, R)
        for k in (ELEMBC, QL, VDOV, QQ):
            ev.add(ptr(k, ne), 8, R)
        ev.add(I4(ELEMBC, e), 4, R)
        ev.add(D(QL, e), 8, R)
        ev.add(D(VDOV, e), 8, R)
        ev.add(D(QQ, e), 8, W)
        kernels.append(ev)
        # 13 EOS stages
        misc = lambda i: rep(dom + OFF_MISC + 4 * i, ne)
        stages = [((0, 1, 2), (DELV, P, Q, QQ, QL), (E,), RW), ((3, 4), (E, VNEW), (P,), W),
                  ((5, 6), (P, E, VNEW), (SS,), W), ((7, 8, 9), (QL, QQ, P), (Q,), W)]
        for ms, ins, outs, kind in stages:
            ev = _Ev()
            ev.add(numelem(grid_e), 4, R)
            ev.add(rep(dom + OFF_TIME, ne), 8, R)
            for i in ms:
                ev.add(misc(i), 4, R)
            for k in ins:
                ev.add(ptr(k, ne), 8, R)
                ev.add(D(k, e), 8, R)
            for k in outs:
                ev.add(ptr(k, ne), 8, R)
                ev.add(D(k, e), 8, kind)
            kernels.append(ev)
        # 14 volumes
        ev = _Ev()
        ev.add(numelem(grid_e), 4, R)
        ev.add(ptr(VNEW, ne), 8, R)
        ev.add(D(VNEW, e), 8, R)
        ev.add(ptr(V, ne), 8, R)
        ev.add(D(V, e), 8, W)
        kernels.append(ev)
        # 15 courant, 16 hydro
        for courant in (True, False):
            ev = _Ev()
            ev.add(numelem(grid_e), 4, R)
            for k in ((SS, VDOV, AREALG) if courant else (VDOV,)):
                ev.add(ptr(k, ne), 8, R)
                ev.add(D(k, e), 8, R)
            ev.add(dtb + 8 * u((0 if courant else nblk) + np.arange(nblk)), 8, W)
            kernels.append(ev)
        for ev in kernels:
            yield ("KB",)
            yield ev.op("DB")
            yield ("KE",)
        # TimeIncrement (host)
        h = _Ev()
        h.add(dtb + 8 * u(np.arange(2 * nblk)), 8, R)
        h.add([dom + OFF_DTC], 8, W)
        h.add([dom + OFF_DTH], 8, W)
        h.add(dom + 4 * u(np.arange(100, 780)), 4, R)
        h.add([dom + OFF_DT], 8, W)
        h.add([dom + OFF_TIME], 8, W)
        h.add([dom + OFF_CYCLE], 4, W)
        h.add(dom + OFF_MISC + 4 * u(np.arange(14)), 4, W)
        yield h.op("HB")
        yield ("DIAG",) + params + (reset, ())
    if final:
        for a in addrs:
            yield ("FREE", a)
        yield ("DIAG",) + params + (reset, ())
