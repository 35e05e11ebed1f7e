"""Generator determinism and achieved shape (SURVEY 4 'Generator tests')."""
import numpy as np

from gmbe_inputs import make_config, graph_stats, SHAPES, chung_lu_bipartite, planted_blocks


def test_er40_matches_survey_recipe():
    nu, nv, e = make_config("er40")
    assert (nu, nv, len(e)) == (40, 40, 239)
    assert e[:5].tolist() == [[0, 2], [0, 3], [0, 11], [0, 13], [0, 20]]


def test_seeded_determinism_and_shape():
    a = make_config("gh")
    b = make_config("gh")
    assert np.array_equal(a[2], b[2])
    st = graph_stats(*a)
    # SURVEY Appendix A seed-0 probe: |E| 440,237, Delta(U) 3,384, Delta(V) 821
    assert (st["m"], st["delta_u"], st["delta_v"]) == (440237, 3384, 821)


def test_planted_blocks_keep_edge_budget():
    nu, nv, m, du, dv = 4000, 3000, 20000, 300, 200
    g = chung_lu_bipartite(nu, nv, m, du, dv, seed=5)
    p = planted_blocks(nu, nv, g[2], K=5, amin=10, amax=20, p_in=0.7, seed=5)
    st = graph_stats(*p)
    assert st["m"] == m == len(p[2])
    p2 = planted_blocks(nu, nv, g[2], K=5, amin=10, amax=20, p_in=0.7, seed=5)
    assert np.array_equal(p[2], p2[2])
