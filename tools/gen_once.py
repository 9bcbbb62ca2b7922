"""Generate one config's search space `--reps` times on cuda:0 (profiling driver for ncu).

    python tools/gen_once.py C5 [--reps N] [--decode N_IDX]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import atfspec as A  # noqa: E402
from paper_conf_hpdc_raschg18_b200 import Space  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--reps", type=int, default=1)
    ap.add_argument("--decode", type=int, default=0)
    ap.add_argument("--legacy", action="store_true")
    ap.add_argument("--flags", type=int, default=None, help="atf_space_opts.flags (default: the bench headline's)")
    ap.add_argument("--profile-last", action="store_true",
                    help="cudaProfilerStart/Stop around the last rep (ncu --profile-from-start off)")
    a = ap.parse_args()
    spec = A.config_spec(a.config)
    torch.cuda.set_device(0)
    from paper_conf_hpdc_raschg18_b200 import _lib as L
    flags = a.flags if a.flags is not None else L.ATF_FLAG_NO_SEG_BOUNDS
    with Space(spec, device=0, flags=flags | (L.ATF_FLAG_LEGACY_WIDE if a.legacy else 0)) as sp:
        for i in range(a.reps):
            last = i == a.reps - 1
            if last and a.profile_last:
                torch.cuda.synchronize()
                torch.cuda.profiler.start()
            sp.generate()
            if last and a.profile_last:
                torch.cuda.synchronize()
                torch.cuda.profiler.stop()
        print(a.config, "S =", sp.size(), "groups =", sp.group_sizes(), flush=True)
        if a.decode:
            from atfspec.fuzz import splitmix64_indices
            import numpy as np
            idx = torch.from_numpy(splitmix64_indices(a.decode, sp.size(), A.c4_indices_seed())
                                   .view(np.int64)).cuda()
            out = sp.decode(idx)
            torch.cuda.synchronize()
            print("decoded", out.shape)


if __name__ == "__main__":
    main()
