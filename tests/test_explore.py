"""Search techniques on top of decode / encode / neighbours."""
import numpy as np
import pytest
import torch

import atfspec as A
from oracle import run as orc


def test_annealing_acceptance_formula():
    """P = exp(-(t' - t)/T) if t' >= t, else 1 (T = 4)."""
    from paper_conf_hpdc_raschg18_b200.explore import annealing_accept
    g = torch.Generator().manual_seed(0)
    n = 200_000
    t = torch.full((n,), 10.0, dtype=torch.float64)
    assert annealing_accept(t, t - 1.0, 4.0, g).all()                      # downhill: always
    for d in (0.0, 1.0, 4.0, 12.0):
        acc = annealing_accept(t, t + d, 4.0, g).double().mean().item()
        assert abs(acc - np.exp(-d / 4.0)) < 0.01, d


@pytest.fixture(scope="module")
def Space():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpdc_raschg18_b200 import Space as S
    return S


@pytest.mark.gpu
def test_exhaustive_visits_the_space_in_order(Space):
    from paper_conf_hpdc_raschg18_b200 import explore as X
    spec = A.c3_xgemm((12, 30, 8))
    with Space(spec) as sp:
        sp.generate()
        S = sp.size()
        ex = X.ExhaustiveSearch()
        ex.initialize(sp)
        got = torch.cat([ex.get_next_configs(1000) for _ in range((S + 999) // 1000)], dim=1)
        assert ex.get_next_configs(10).shape[1] == 0
        _, want = orc.decode(spec, np.arange(S, dtype=np.uint64))
        assert np.array_equal(got.cpu().numpy(), want)


@pytest.mark.gpu
@pytest.mark.parametrize("name", ["C3", "C5", "C2"])
def test_neighbors_are_valid_single_parameter_moves(Space, name):
    spec = {"C3": lambda: A.c3_xgemm((12, 30, 8)), "C5": lambda: A.c5_chains(300, 4),
            "C2": lambda: A.c2_xgemm_direct(64)}[name]()
    from paper_conf_hpdc_raschg18_b200 import explore as X
    with Space(spec) as sp:
        sp.generate()
        rs = X.RandomSearch(seed=3)
        rs.initialize(sp)
        cur = rs.get_next_configs(20_000)
        nb, moved = sp.neighbors(cur, seed=11)
        c, b, m = cur.cpu().numpy(), nb.cpu().numpy(), moved.cpu().numpy()
        diff = c != b
        assert (diff.sum(axis=0) == (m >= 0)).all()                  # exactly one parameter changes
        rows = np.nonzero(m >= 0)[0]
        assert (diff[m[rows], rows]).all()                           # ... the reported one
        assert len(rows) > 0.2 * len(m)   # chained divisibility leaves few valid one-parameter moves
        chk = orc.check(spec, b.T.copy())                            # every neighbour is valid
        assert chk["valid"] == chk["rows"]
        chk0 = orc.check(spec, c.T.copy())                           # random-search samples too
        assert chk0["valid"] == chk0["rows"]
        # deterministic in the seed
        nb2, moved2 = sp.neighbors(cur, seed=11)
        assert torch.equal(nb2, nb) and torch.equal(moved2, moved)


@pytest.mark.gpu
def test_annealing_and_random_search_find_the_optimum(Space):
    """A smooth synthetic cost over C3 at a small GEMM shape; the global minimum by brute
    force over every configuration (decode of all indices)."""
    from paper_conf_hpdc_raschg18_b200 import explore as X
    spec = A.c3_xgemm((12, 30, 8))
    target = torch.tensor([6, 10, 4, 3, 5, 2, 5, 2, 2, 2, 1, 0, 1, 0], dtype=torch.float64, device="cuda")

    def cost(cfg):
        v = cfg.to(torch.float64)
        return ((torch.log2(v + 1.0) - torch.log2(target + 1.0).unsqueeze(1)) ** 2).sum(dim=0)

    with Space(spec) as sp:
        sp.generate()
        allc = sp.decode(torch.arange(sp.size(), dtype=torch.int64, device="cuda"))
        all_cost = cost(allc)
        opt = float(all_cost.min())
        # T = 4 is for runtimes; this cost is O(1), so anneal at a matching scale
        best_sa, cfg_sa = X.tune(sp, X.SimulatedAnnealing(chains=256, seed=1, temperature=0.02), cost,
                                 evaluations=256 * 200, batch=256)
        assert best_sa >= opt - 1e-9
        assert best_sa <= float(torch.quantile(all_cost, 0.001)) + 1e-9   # within the best 0.1 %
        assert sp.encode(cfg_sa.unsqueeze(1)).item() >= 0
        assert abs(float(cost(cfg_sa.unsqueeze(1))[0]) - best_sa) < 1e-12
        best_rs, _ = X.tune(sp, X.RandomSearch(seed=2), cost, evaluations=4 * sp.size())
        assert best_rs >= opt - 1e-9
        best_tp, _ = X.tune(sp, X.IndexSearch(lambda n: torch.randint(1, sp.size() + 1, (n,))), cost, 1000)
        assert best_tp >= opt - 1e-9
