"""Exact oracle parity of a tuning variant of the library (DC_LIB=<variant.so>)
at sizes that cross its tile shapes, both schedules (diagnostic; the shipped
library is covered by tests/)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import dcgen
import oracle
import paper_conf_ipps_lopez_ortizss13_b200 as dc

oracle.build()
ok = True
for n in [(1 << 23) + 7, 3 * (1 << 22) + 5, (1 << 24) + 3 * 25088 + 11, (1 << 25) - 5]:
    for dist in ("uniform", "few", "reverse"):
        keys = dcgen.sort_keys(n, dist, seed=13, device="cuda")
        k_in = keys.cpu().numpy().view(np.uint32).copy()
        for two in (True, False):
            k = keys.clone()
            p = dc.Plan(n)
            p.set_two_level(two)
            p.sort_(k, key_type="u32")
            good = np.array_equal(k.cpu().numpy().view(np.uint32), oracle.mergesort(k_in))
            ok &= good
            print(f"n={n} dist={dist} two_level={two} sched={p.schedule('u32')} exact={good}",
                  flush=True)
print("VARIANT_OK" if ok else "VARIANT_MISMATCH")
sys.exit(0 if ok else 1)
