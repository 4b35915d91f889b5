"""Search state guards on the GPU path (pesto.h pesto_search_*: PESTO_ESTATE): a search keeps
the per-base layouts, transfer times and base makespans of the comm model it was created
under, so a pesto_comm_model call after pesto_search_create makes every later step, eval or
commit fail with ESTATE instead of walking records of the old model."""
import numpy as np
import pytest

from workloads import dag

pytestmark = pytest.mark.gpu


def test_comm_model_change_after_search_is_rejected():
    from paper_conf_middleware_hafeezsg021_b200 import pesto as P
    g = dag.random_dag(5, 300, 1.5, D=2, p_max=4000, max_bytes=300_000, beta0=700,
                       beta1_fs=30_000)
    G = P.Graph.from_arrays(g, device=0)
    order = G.seed_order(P.ORDER_CRITICAL_PATH)
    xs = dag.random_placements(g, 3, 2)
    S = P.Search(G, xs, np.stack([order, order]), 256, (50, 20, 20, 10), seed=1)
    S.step()                                          # fine under the model it was made with
    before = [S.get(b)[0] for b in range(2)]
    G.comm_model(0, 1, 900, 50_000)                   # change one link after creation
    for call in (S.step, S.eval, S.commit):
        with pytest.raises(P.PestoError) as e:
            call()
        assert e.value.status == P.ESTATE
    assert [S.get(b)[0] for b in range(2)] == before  # nothing was committed
