import sys, numpy as np, torch
sys.path.insert(0, '.')
from paper_conf_icpp_koppehelggp21_b200.dist import CudaOps, compute_splitters, owners, prefix8
DEV = torch.device('cuda:0')
for nparts in (1, 2, 3, 4, 5, 7, 8, 9, 16, 64):
  for n in (1, 4095, 4097, 300001):
    rng = np.random.default_rng(n + nparts)
    keys = rng.integers(0, 2**64, n, dtype=np.uint64)
    sp = compute_splitters(prefix8(keys), nparts)
    ops = CudaOps(DEV)
    k = torch.from_numpy(keys.view(np.int64)).to(DEV)
    perm_fill = None
    sk, sl, sv, perm, counts = ops.route(k, None, None, torch.from_numpy(sp.view(np.int64)).to(DEV) if nparts > 1 else None, nparts)
    torch.cuda.synchronize()
    own = owners(prefix8(keys), sp)
    order = np.argsort(own, kind='stable'); eperm = np.empty(n, np.int64); eperm[order] = np.arange(n)
    p = perm.cpu().numpy().astype(np.int64)
    bad = np.nonzero(p != eperm)[0]
    print(nparts, n, 'counts ok' if counts.cpu().tolist() == np.bincount(own, minlength=nparts).tolist() else 'COUNTS BAD', 'bad', len(bad), bad[:5], p[bad[:5]], eperm[bad[:5]], own[bad[:5]], flush=True)
