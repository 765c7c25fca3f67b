"""Debug helper: which matrices of a config fail parity (sizes, errors)."""
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch, vbgen
from harness import DeviceBatch, compare_with_oracle
cfgs = sys.argv[1:] or ["C3"]
for cfg in cfgs:
    if cfg.startswith("u"):
        nn, cnt = (int(x) for x in cfg[1:].split("x"))
        n = np.full(cnt, nn, dtype=np.int32); seed = 3
    else:
        c = vbgen.CONFIGS[cfg]; n = vbgen.sizes(c); seed = c.seed
    db = DeviceBatch(n, seed=seed).fill()
    db.dpotrf(max_n=int(n.max()))
    torch.cuda.synchronize()
    info = db.info()
    bad = []
    lo = int(os.environ.get('NLO', '0')); idx = [i for i in range(db.B) if n[i] > lo]
    for i in idx[:int(os.environ.get('NCHK', '100000'))]:
        r = compare_with_oracle(db.host_matrix_input(i), db.block(i), info[i])
        if not r["ok"]:
            bad.append((i, int(n[i]), {k: (float(r[k]) if k != "info" else r[k]) for k in r if k in ("bwd", "rowdiff", "info")}))
    print(cfg, "checked", len(idx[:int(os.environ.get('NCHK', '100000'))]), "bad", len(bad), bad[:8], flush=True)
    if bad:
        i = bad[0][0]; nn = int(n[i])
        L = np.tril(db.block(i)); A = db.host_matrix_input(i)
        import oracle
        Lo = np.tril(oracle.dpotrf(A)[0]) if hasattr(oracle, "dpotrf") else None
        if Lo is not None:
            d = np.abs(L - Lo) > 1e-8 * np.abs(Lo).max()
            rows, cols = np.nonzero(d)
            print("first bad entries (row,col):", list(zip(rows[:10].tolist(), cols[:10].tolist())), "count", d.sum(), flush=True)
