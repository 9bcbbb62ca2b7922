"""Fresh-space generations with the host-phase build (atfgen.cpp compiled with -DATF_HOST_PROF into
build/hostprof/libatfgen.so): per level
round, host time to queue it and time waiting for the device.  ATF_LIB_PATH=... python tools/host_rounds.py C3-IS2"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import time  # noqa: E402

import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space, _lib as L  # noqa: E402

spec = A.config_spec(sys.argv[1] if len(sys.argv) > 1 else "C3-IS2")
flags = L.ATF_FLAG_NO_SEG_BOUNDS if spec.name.startswith("C5") else 0
for it in range(4):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    with Space(spec, flags=flags) as sp:
        t1 = time.perf_counter()
        sp.generate()
        torch.cuda.synchronize()
        t2 = time.perf_counter()
    print(f"--- fresh #{it}: create {1e3 * (t1 - t0):.2f} ms, generate {1e3 * (t2 - t1):.2f} ms", file=sys.stderr, flush=True)
