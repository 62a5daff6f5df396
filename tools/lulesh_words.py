#!/usr/bin/env python
"""Distinct shadow words the LULESH-shaped program touches per GPU epoch, summed
over one steady-state timestep (timestep 2), from its CPU twin (xplgen.lulesh):
the unit count behind the hook path's algorithmic bytes in bench.py (DESIGN.md
§5: 1 B shadow read + <= 1 B written per distinct word per epoch).
  python tools/lulesh_words.py [s]"""
import json
import sys

import numpy as np

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
from xplgen import lulesh as L  # noqa: E402
from xplgen.rodinia import layout  # noqa: E402

s = int(sys.argv[1]) if len(sys.argv) > 1 else 100
spec = L.lulesh_spec(s)
addrs, _, _ = layout(spec, 0, 0, 1 << 40)
topo = L.topology(s, 0x58504C05)
tmps = [((1 << 44) + t * (1 << 34), (1 << 44) + t * (1 << 34) + (1 << 33)) for t in range(2)]
step, epochs, words, events = 0, 0, 0, 0
for op in L.lulesh_trace_iter(addrs, spec, s, 2, topo, (50, 0, 256), tmps, final=False):
    if op[0] == "DIAG":
        step += 1
    if op[0] == "DB" and step == 1:
        a = np.asarray(op[1], np.uint64)
        z = np.asarray(op[2], np.uint64)
        w = np.unique(np.concatenate([a >> np.uint64(2), (a + z - np.uint64(1)) >> np.uint64(2)]))
        words += int(w.size)
        events += int(a.size)
        epochs += 1
print(json.dumps({"s": s, "epochs_per_timestep": epochs, "hooked_accesses_per_timestep": events,
                  "distinct_words_per_epoch_summed": words}))
