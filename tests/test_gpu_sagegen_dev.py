"""The per-rank device generator (sagegen/sagegen_dev.cu, bench infrastructure for multi-GPU
inputs such as C5) reproduces sagegen.rmat exactly: every rank's rows [v_begin, v_end) equal the
corresponding rows of the host generator, weights included, at scales <= 16."""
import numpy as np
import pytest

import sagegen as sg

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("scale,ef,sym,parts", [(10, 16, True, 1), (12, 8, False, 3), (14, 16, True, 4),
                                                (16, 16, True, 2)])
def test_device_rmat_equals_host(scale, ef, sym, parts):
    g = sg.rmat(scale, ef, 3, sym)
    w = sg.weights(g, 1)
    n = g.n
    for r in range(parts):
        vb, ve = n * r // parts, n * (r + 1) // parts
        off, col, wd = sg.rmat_device(scale, ef, 3, sym, vb, ve, weights_seed=1)
        b0 = int(g.off[vb])
        assert np.array_equal(off.cpu().numpy(), g.off[vb:ve + 1] - b0)
        assert np.array_equal(col.cpu().numpy(), g.col[b0:int(g.off[ve])])
        assert np.array_equal(wd.cpu().numpy().view(np.uint32), w[b0:int(g.off[ve])])
