"""Host logic of the replay driver (no GPU): the grouping of back-to-back GPU
epochs into one cooperative launch with device-side epoch splits (NEXT-2) must
keep every event, in order, in the epoch it belongs to -- flattening the SPLIT
ops back gives the original trace -- and must leave everything else alone."""
from xplgen.trace import epoch_chain_trace, random_trace


def _flatten(ops):
    out = []
    for op in ops:
        if op[0] == "SPLIT":
            for seg in op[1]:
                out += [("KB",)] + list(seg) + [("KE",)]
        else:
            out.append(op)
    return out


def _same(a, b):
    assert len(a) == len(b)
    for x, y in zip(a, b):
        assert x[0] == y[0]
        for u, v in zip(x[1:], y[1:]):
            assert (u == v).all() if hasattr(u, "all") else u == v


def test_group_splits_roundtrip():
    from paper_conf_ipps_pirkelbauerlvl20_b200.replay import _group_splits
    for seed in range(5):
        ops = epoch_chain_trace(seed, chain_len=4)
        g = _group_splits(ops)
        splits = [op for op in g if op[0] == "SPLIT"]
        assert len(splits) == 3 and all(len(op[1]) == 4 for op in splits)
        _same(_flatten(g), ops)
        ops = random_trace(seed, n_steps=60, p_device=0.9)
        g = _group_splits(ops)
        assert all(len(op[1]) >= 2 for op in g if op[0] == "SPLIT")
        _same(_flatten(g), ops)


def test_group_splits_leaves_nested_and_interrupted_epochs():
    from paper_conf_ipps_pirkelbauerlvl20_b200.replay import _group_splits
    ops = [("KB",), ("KB",), ("D", 1, 4, 1), ("KE",), ("KE",), ("KB",), ("D", 2, 4, 2), ("KE",)]
    assert _group_splits(ops) == ops  # the nested epoch is not a plain segment
    ops = [("KB",), ("D", 1, 4, 1), ("H", 1, 4, 1), ("KE",), ("KB",), ("KE",)]
    assert _group_splits(ops) == ops  # a deferred host access inside the first epoch
