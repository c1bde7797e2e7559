"""Debug repro (SPECK_ESC_CHECK builds): one small config, then the ESC check record."""
import ctypes
import sys

import torch

sys.path.insert(0, '.')
import workloads as W  # noqa: E402
import paper_conf_ppopp_pargerwms20_b200 as sp  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else 'c3'
opts = dict(kv.split('=') for kv in sys.argv[2:])
opts = {k: int(v) for k, v in opts.items()}
(label, A, B), = W.config(cfg, small=True)
print(label, A.rows, A.nnz, opts, flush=True)
h = sp.Handle(0, **opts)
try:
    C = h.spgemm(A.to('cuda'), B.to('cuda'))
    torch.cuda.synchronize()
    print('ok', C.nnz)
except Exception as ex:
    print('failed', ex)
L = sp.load()
out = (ctypes.c_int * 9)()
if hasattr(L, 'speck_debug_esc'):
    print('dbg rc', L.speck_debug_esc(out), list(out))
