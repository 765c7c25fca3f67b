"""One vbatched_dgeqrf call (3000 x U{1..512}) for profilers."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
from harness import QRBatch  # noqa: E402
cnt, nmax = (int(x) for x in (sys.argv[1:] or ["3000", "512"]))
n = np.random.default_rng(nmax).integers(1, nmax + 1, cnt).astype(np.int32)
qb = QRBatch(n, n, seed=13).fill()
qb.geqrf()
torch.cuda.synchronize()
