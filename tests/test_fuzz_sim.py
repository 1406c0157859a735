"""CPU fuzz of the planner: the same seeded random cases as tests/test_gpu_fuzz.py,
executed by the host emulation of each tile plan's tables (ll_plan_simulate) and
compared with the oracle, bit-exact."""
import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import gen
from tests._fuzz import fuzz_case

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


def _seeds(default):
    """Seeds of the fuzz cases: the default list, or LL_FUZZ_SEEDS="a-b" for an
    extended run (e.g. the round-end robustness pass)."""
    import os
    e = os.environ.get("LL_FUZZ_SEEDS")
    if not e:
        return default
    a, b = (int(x) for x in e.split("-"))
    return list(range(a, b + 1))


@pytest.mark.parametrize("seed", _seeds([1, 2, 3, 4]))
def test_fuzz_plans_simulated(seed):
    rng = np.random.default_rng(9000 + seed)
    tiles = 0
    for case in range(60):
        kind, la, lb, w, opts = fuzz_case(rng)
        OA, OB = O.Layout(*la), O.Layout(*lb)
        try:
            plan = ll.ll_plan_convert(ll.Layout(*la), ll.Layout(*lb), w, **opts)
        except ll.LLError as e:
            assert "UNSUPPORTED" in str(e), (case, kind, opts, str(e))
            continue
        d = plan.describe()
        assert d["class"] == O.classify(OA, OB) if OA.d_in <= 16 and OB.d_in <= 16 else True
        if d["exec"] != "tile":
            continue
        src = O.pack(OA, gen.random_bits(rng, 1 << OA.d_out, w))
        assert np.array_equal(plan.simulate(src, 1 << OB.d_in), O.convert(OA, OB, src)), (case, kind, w, opts)
        tiles += 1
    assert tiles >= 30
