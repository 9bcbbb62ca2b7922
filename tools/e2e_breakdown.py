"""Host-side breakdown of one end-to-end generation through the public API (fresh space per step)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space  # noqa: E402

spec = A.config_spec(sys.argv[1] if len(sys.argv) > 1 else "C5")
torch_alloc = (sys.argv[2] != "native") if len(sys.argv) > 2 else True
torch.cuda.synchronize()
for it in range(5):
    t0 = time.perf_counter()
    sp = Space(spec, torch_alloc=torch_alloc)
    t1 = time.perf_counter()
    sp.plan()
    t2 = time.perf_counter()
    sp.generate()
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    S = sp.size()
    gs = sp.group_sizes()
    t4 = time.perf_counter()
    sp.generate()
    torch.cuda.synchronize()
    t5 = time.perf_counter()
    sp.close()
    torch.cuda.synchronize()
    t6 = time.perf_counter()
    print(f"create {1e3*(t1-t0):.2f} plan {1e3*(t2-t1):.2f} generate(fresh) {1e3*(t3-t2):.2f} "
          f"size {1e3*(t4-t3):.2f} generate(again) {1e3*(t5-t4):.2f} close {1e3*(t6-t5):.2f} ms", flush=True)
