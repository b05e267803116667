"""The paper's CPU ECL-CC versions (baselines/) give the oracle's labels."""
import numpy as np
import pytest

import baselines
import graphgen as gg
import oracle


@pytest.mark.parametrize("name,sd", [("C1", 0), ("C2", 6), ("C3", 6), ("C4", 8), ("C5", 11)])
def test_omp_and_serial_match_oracle(name, sd):
    g = gg.make_config(name, seed=2, scale_down=sd)
    for gg_ in (g, gg.shuffle_rows(g, seed=3)):
        nidx, nl = gg_.numpy()
        expect, _ = oracle.bfs(nidx, nl)
        assert np.array_equal(baselines.ser(nidx, nl), expect)
        for t in (1, 4, 16):
            assert np.array_equal(baselines.omp(nidx, nl, t), expect)


def test_empty_and_edgeless():
    assert baselines.ser(np.zeros(1, np.int64), np.zeros(0, np.int32)).size == 0
    out = baselines.omp(np.zeros(6, np.int64), np.zeros(0, np.int32), 4)
    assert out.tolist() == [0, 1, 2, 3, 4]
