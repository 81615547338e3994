"""Time ag_graph_load_csr from pinned host memory (the e2e step's dominant part)."""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import aggen
from paper_conf_ipps_lib13_b200 import agraph as A

g = aggen.config(sys.argv[1] if len(sys.argv) > 1 else "C2")
rp = torch.from_numpy(g.row_ptr.view(np.int64)).pin_memory()
col = torch.from_numpy(g.col.view(np.int32)).pin_memory()
w = torch.from_numpy(g.w.view(np.int32)).pin_memory()
for layout in (A.LAYOUT_AUTO, A.LAYOUT_IDENTITY):
    for it in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        G = A.Graph(g.V, rp, col, w, layout=layout)
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        G.free()
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        print(f"layout={layout} load {1e3*(t1-t0):.1f} ms free {1e3*(t2-t1):.1f} ms")
t0 = time.perf_counter()
d = torch.empty(g.E, dtype=torch.int32, device="cuda")
torch.cuda.synchronize()
t1 = time.perf_counter()
d.copy_(col, non_blocking=True)
torch.cuda.synchronize()
t2 = time.perf_counter()
print(f"pure H2D of col ({g.E*4/1e6:.0f} MB): {1e3*(t2-t1):.1f} ms = {g.E*4/(t2-t1)/1e9:.1f} GB/s")
