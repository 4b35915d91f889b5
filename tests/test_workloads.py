"""Synthetic inputs are paper-shaped (SURVEY.md §8(d) structural targets; Table 1)."""
import numpy as np
import pytest

from workloads import configs, shaped

TARGETS = {  # generator: (n target (Table 1 row total), anchor row, min max-in-degree)
    "transformer": (19393, "transformer6", 7),
    "inception_v3": (16901, "nasnet4", 4),
    "nmt": (30060, "nmt2", 36),
}


@pytest.mark.parametrize("kind", sorted(TARGETS))
def test_shaped_generator_stats(kind):
    g = configs._base_graph(kind)
    st = shaped.stats(g)
    n_t, anchor, min_in = TARGETS[kind]
    assert abs(st["n"] - n_t) <= 0.05 * n_t
    assert 1.2 <= st["m_over_n"] <= 1.8
    assert st["max_in"] >= min_in
    counts = shaped.TABLE1[anchor]
    tot = sum(counts)
    for got, c in zip(st["mix_pct"], counts):
        assert abs(got - 100.0 * c / tot) <= 2.0
    # sum p near 1 s: 2-device makespans land in the paper's per-step range (L328, L355)
    assert 0.5e9 <= st["sum_p_ns"] <= 1.5e9


def test_generators_are_deterministic():
    a = shaped.transformer()
    b = shaped.transformer()
    assert (a.p == b.p).all() and (a.src == b.src).all() and (a.nbytes == b.nbytes).all()


def test_configs_cover_baseline():
    assert set(configs.CONFIGS) == {"tiny12", "inception_v3_2dev", "nmt4_2dev_commheavy",
                                    "transformer_2dev", "transformer_4dev_8gpu"}
    g = configs.graph_for(configs.CONFIGS["transformer_4dev_8gpu"])
    assert g.D == 4 and g.beta0.shape == (16,)
    assert all(g.beta0[d * 4 + d] == 0 for d in range(4))
