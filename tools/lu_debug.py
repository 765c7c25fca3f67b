"""Development: where a vbatched_dgetrf factor departs from the oracle (python tools/lu_debug.py m n)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from harness import LUBatch  # noqa: E402

m, n = int(sys.argv[1]), int(sys.argv[2])
lb = LUBatch(np.array([m], np.int32), np.array([n], np.int32), seed=41).fill()
lb.getrf()
torch.cuda.synchronize()
A = lb.inputs[0]
Fo, ipo, info_o = oracle.dgetrf(A)
Fg = lb.block(0)[:m, :n]
ipg = np.asarray(lb.ipiv_of(0))
print("info", info_o, lb.info()[0], "ipiv first diff", np.nonzero(ipg != ipo)[0][:10])
d = np.abs(Fg - Fo) > 1e-9 * (1 + np.abs(Fo))
rows, cols = np.nonzero(d)
print("bad entries", d.sum(), "rows", np.unique(rows)[:20], "cols", np.unique(cols)[:40])
