"""Virtual shards on one GPU (SURVEY §4 "multi-GPU without a cluster"): R
contexts, each holding one contiguous piece of every logical allocation; host
records, transfers and device events go to the context that owns their address
(the instrumented replay kernel is re-bound per context); every context
diagnoses into partials; xpl_combine_partials must reproduce the oracle's
report of the unsharded allocations exactly, for R = 1, 2, 3, 5."""
import numpy as np
import pytest
import torch

from oracle import run_trace as oracle_run
from tests.test_sharding_cpu import make_trace

pytestmark = pytest.mark.gpu


def split_pieces(allocs, R):
    pieces = []  # (rank, rid, piece_base, piece_bytes, goff, logical_bytes)
    for rid, (base, nb) in enumerate(allocs):
        lw = (nb + 3) // 4
        chunk = -(-lw // R)
        for r in range(R):
            goff = r * chunk
            n = min(lw, goff + chunk) - goff
            if n <= 0:
                continue
            pb = min(nb, 4 * (goff + n)) - 4 * goff
            pieces.append((r, rid, base + 4 * goff, pb, goff, nb))
    return pieces


def owner_of(pieces):
    lo = np.array([p[2] for p in pieces], np.uint64)
    hi = lo + np.array([p[3] for p in pieces], np.uint64)
    rank = np.array([p[0] for p in pieces])
    order = np.argsort(lo)
    lo, hi, rank = lo[order], hi[order], rank[order]

    def f(addr):
        addr = np.asarray(addr, np.uint64)
        k = np.clip(np.searchsorted(lo, addr, side="right") - 1, 0, len(lo) - 1)
        inside = (addr >= lo[k]) & (addr < hi[k])
        return np.where(inside, rank[k], -1)
    return f, lo, hi


@pytest.mark.parametrize("R", [1, 2, 3, 5])
@pytest.mark.parametrize("seed,params", [(11, (50, 0, 256)), (12, (30, 64, 8)), (13, (50, 7, 3))])
def test_virtual_shards(R, seed, params):
    from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
    thr, B, min_run = params
    ops, allocs = make_trace(seed)
    exp = oracle_run(ops + [("DIAG", thr, B, min_run, 1, ())])[-1]
    pieces = split_pieces(allocs, R)
    own, lo, hi = owner_of(pieces)
    ctxs = [xpl.Context(pool_words=1 << 20) for _ in range(R)]
    s = torch.cuda.current_stream().cuda_stream
    try:
        kinds = {rid: op[3] for rid, op in enumerate(o for o in ops if o[0] == "REG")}
        for r, rid, pb, pbytes, goff, nb in pieces:
            ctxs[r].register_piece(pb, pbytes, kinds[rid], rid, goff, nb)
        for op in ops:
            if op[0] == "REG":
                continue
            if op[0] == "HB":
                ow = own(op[1])
                for r in range(R):
                    m = ow == r
                    if m.any():
                        rec = np.zeros(int(m.sum()), dtype=xpl.HOST_ACCESS_DTYPE)
                        rec["addr"], rec["size"], rec["kind"] = op[1][m], op[2][m], op[3][m]
                        ctxs[r].record_host(rec)
            elif op[0] == "DB":
                ow = own(op[1])
                for r in range(R):
                    ctxs[r].kernel_begin(s)
                for r in range(R):
                    m = ow == r
                    if m.any():
                        ctxs[r].bind()
                        ta = torch.from_numpy(op[1][m].astype(np.uint64).view(np.int64)).cuda()
                        ts = torch.from_numpy(op[2][m].astype(np.uint32).view(np.int32)).cuda()
                        tk = torch.from_numpy(op[3][m].astype(np.uint8)).cuda()
                        ctxs[r].replay(ta.data_ptr(), ts.data_ptr(), tk.data_ptr(), int(m.sum()), stream=s)
                        torch.cuda.current_stream().synchronize()
                for r in range(R):
                    ctxs[r].kernel_end(s)
            elif op[0] in ("KB", "KE"):
                continue
            elif op[0] == "X":  # H2D of a byte range: every owner gets its part
                d0, nbytes = op[2], op[4]
                for k in range(len(lo)):
                    a, b = max(int(lo[k]), d0), min(int(hi[k]), d0 + nbytes)
                    if a < b:
                        r = int(own([a])[0])
                        ctxs[r].record_copy(a, op[3] + (a - d0), b - a, op[1])
            else:
                raise AssertionError(op)
        blobs = [c.diagnose_partials(thr, B, min_run, True) for c in ctxs]
        got = xpl.combine_partials(blobs, thr, B, min_run)
    finally:
        for c in ctxs:
            c.close()
    assert len(got) == len(exp)
    for g, e in zip(got, exp):
        diff = {f: (g[f], e[f]) for f in e if g[f] != e[f]}
        assert not diff, (R, e["id"], diff)
