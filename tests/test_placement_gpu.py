"""Residency ablations: the same SEPO table with its page
pool in pinned host memory (GPU threads access it over the host link, the paper's Fig. 7 experiment)
or in managed memory (hardware demand paging). The method is unchanged, so results must equal the
oracle's exactly, in one pass with a pool that holds the table and in several passes with a pool a
quarter of the footprint (postpone + evict still work when the pool is not in HBM)."""
import pytest

import gen
from tests.util import device_inputs, footprint_pages, oracle_expected, run_job

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("placement", [1, 2])
@pytest.mark.parametrize("cfg", ["C1", "C5z"])
def test_pool_placement_parity(cuda, placement, cfg):
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    s = gen.config(cfg, scale=0.25 if cfg == "C1" else 1e-4)
    inp = device_inputs(s)
    exp = oracle_expected(s)
    nb, pb = 1 << 14, 4096
    F = footprint_pages(s, nb, pb, inputs=inp)
    got, passes, st = run_job(s, sepo.budget_for(nb, pb, F + 512), nb, pb, inputs=inp, placement=placement)
    assert got == exp and passes == 1
    got, passes, st = run_job(s, sepo.budget_for(nb, pb, max(8, F // 4)), nb, pb, inputs=inp, placement=placement,
                              check_dups=True)
    assert got == exp
    assert passes >= 2 and st["cross_gen_dups"] == 0


def test_pool_placement_invalid(cuda):
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    with pytest.raises(sepo.SepoError):
        sepo.Table(sepo.budget_for(1 << 10, 4096, 16), 1 << 10, 4096, placement=7)
