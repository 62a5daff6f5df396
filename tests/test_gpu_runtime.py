"""Runtime rules of the C-ABI around streams and device-side epoch splits
(include/xpl.h): a split inside an epoch that has several streams is reported
(XPL_ERR_STATE) instead of silently racing the fold; a stream the runtime
adopted can be released and destroyed; D2D copies and memsets of any length are
recorded in full (one range per side)."""
import numpy as np
import pytest

from oracle import run_trace as oracle_run
from xplgen.trace import DEVICE, MANAGED

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
    return torch, xpl


def _dev(torch, a):
    return torch.from_numpy(a).cuda()


def test_split_in_multistream_epoch_is_reported(env):
    torch, xpl = env
    base = 0x4000_0000
    n = 4096
    addr = _dev(torch, (base + 4 * np.arange(n, dtype=np.uint64)).view(np.int64))
    size = _dev(torch, np.full(n, 4, np.int32))
    acc = _dev(torch, np.full(n, 3, np.uint8))
    seg = _dev(torch, np.array([0, n // 2, n], np.int64))
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    with xpl.Context(pool_words=1 << 20) as ctx:
        ctx.register(base, 4 * n, DEVICE)
        # allowed: one stream
        ctx.kernel_begin(s1.cuda_stream)
        ctx.replay_split(addr.data_ptr(), size.data_ptr(), acc.data_ptr(), seg.data_ptr(), 2, stream=s1.cuda_stream)
        ctx.kernel_end(s1.cuda_stream)
        ctx.sync()
        # forbidden: a second stream joined the epoch
        ctx.kernel_begin(s1.cuda_stream)
        ctx.kernel_begin(s2.cuda_stream)
        ctx.replay_split(addr.data_ptr(), size.data_ptr(), acc.data_ptr(), seg.data_ptr(), 2, stream=s1.cuda_stream)
        ctx.kernel_end(s2.cuda_stream)
        ctx.kernel_end(s1.cuda_stream)
        with pytest.raises(xpl.XplError) as ei:
            ctx.sync()
        assert ei.value.status == 5  # XPL_ERR_STATE
        ctx.sync()  # reported once


def test_release_stream_then_destroy(env):
    torch, xpl = env
    base = 0x5000_0000
    n = 1000
    addr = _dev(torch, (base + 4 * np.arange(n, dtype=np.uint64)).view(np.int64))
    size = _dev(torch, np.full(n, 4, np.int32))
    acc = _dev(torch, np.full(n, 1, np.uint8))
    with xpl.Context(pool_words=1 << 20) as ctx:
        ctx.register(base, 4 * n, MANAGED)
        s = torch.cuda.Stream()
        ctx.kernel_begin(s.cuda_stream)
        ctx.replay(addr.data_ptr(), size.data_ptr(), acc.data_ptr(), n, stream=s.cuda_stream)
        ctx.kernel_end(s.cuda_stream)
        ctx.release_stream(s.cuda_stream)
        s.synchronize()
        del s
        torch.cuda.synchronize()
        rep = ctx.diagnose(50, 0, 256, reset=True)
        assert rep[0]["r_cg"] == n
        # the default stream is never adopted
        ctx.kernel_begin(0)
        ctx.replay(addr.data_ptr(), size.data_ptr(), acc.data_ptr(), n, stream=0)
        ctx.kernel_end(0)
        assert ctx.diagnose(50, 0, 256, reset=True)[0]["r_cg"] == n


def test_long_d2d_and_memset_recorded_in_full(env):
    torch, xpl = env
    # small: every field against the oracle
    words = (1 << 20) + 123
    a, b = 1 << 42, (1 << 42) + (1 << 30)
    ops = [("REG", a, 4 * words, DEVICE), ("REG", b, 4 * words, DEVICE),
           ("X", 3, b, a, 4 * words), ("DIAG", 50, 0, 256, 1, ()),
           ("X", 4, a, 0, 4 * words - 2), ("DIAG", 50, 0, 256, 1, ())]
    with xpl.Context(pool_words=2 * words + (1 << 20)) as ctx:
        ctx.register(a, 4 * words, DEVICE)
        ctx.register(b, 4 * words, DEVICE)
        ctx.record_copy(b, a, 4 * words, 3)
        got = [ctx.diagnose(50, 0, 256, reset=True)]
        ctx.record_copy(a, 0, 4 * words - 2, 4)
        got.append(ctx.diagnose(50, 0, 256, reset=True))
    assert got == oracle_run(ops)
    # > 2^30 words per side (round 1 cut each side into 2^24-word pieces, at most
    # 64 of them: a 4 GiB+ copy lost words): the closed form, every word once
    words = (1 << 30) + 77
    a, b = 1 << 44, (1 << 44) + (1 << 33)
    with xpl.Context(pool_words=2 * words + (1 << 20), max_rows=8) as ctx:
        ctx.register(a, 4 * words, DEVICE)
        ctx.register(b, 4 * words, DEVICE)
        ctx.record_copy(b, a, 4 * words, 3)  # D2D: GPU reads src, writes dst (D7)
        r = ctx.diagnose(50, 0, 256, reset=True)
        assert (r[0]["r_cg"], r[0]["any_acc"], r[1]["w_g"], r[1]["any_acc"]) == (words, words, words, words)
        ctx.record_copy(a, 0, 4 * words, 4)  # memset: GPU writes dst
        r = ctx.diagnose(50, 0, 256, reset=True)
        assert (r[0]["w_g"], r[0]["any_acc"], r[1]["any_acc"]) == (words, words, 0)
