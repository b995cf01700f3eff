"""Source injection at every position class the kernels resolve differently:
each component of a 4-wide (ISO, acoustic) or 2-wide (elastic) thread group, the first and
last plane of a z-slab and of a z-chunk, the grid corners -- bitwise equal under the z-slab
decomposition (P = 1, 2, 3; the source lands in different slabs and local planes) and within
the north-star tolerance of the fp64 oracle.  The ISO and acoustic P kernels resolve the
source node once per thread (common.cuh src_hit), the elastic S kernel per plane; both must
add the same amplitude at the same point as the oracle."""
import numpy as np
import pytest

import oracle
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
from gpu_common import TOL_FIELD, gpu_forward, grids, oracle_fields, rel_l2

pytestmark = pytest.mark.gpu

NX, NY, NZ = 37, 21, 48  # ragged x (not a multiple of 4); P = 2: slabs [0, 24) [24, 48); P = 3: 16-plane slabs
SOURCES = [
    (0, 0, 0),            # corner, component 0
    (13, 7, 23),          # component 1 (13 = 4 * 3 + 1), last plane of slab 0 (P = 2)
    (22, 10, 24),         # component 2, first plane of slab 1 (P = 2)
    (35, 20, 16),         # component 3, first plane of slab 1 (P = 3)
    (36, 20, 47),         # the ragged last x column, last plane of the grid
]


def _media(kind):
    return inputs.random_media((NZ, NY, NX), seed=71, elastic=(kind == "elastic"))


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_source_positions_decomposition_bitwise(monkeypatch, kind):
    monkeypatch.setenv("SEIS_NO_PERSIST", "1")  # (the z-march kernels, not the small-grid ones)
    m = _media(kind)
    h, dt, nt = 10.0, 5e-4, 24
    w = inputs.source_series(kind, nt, dt, 35.0)
    rec = np.asarray([[s[0], s[1], s[2]] for s in SOURCES], np.int32)
    for src in SOURCES:
        outs = []
        for P in (1, 2, 3):
            g, _ = grids(NX, NY, NZ, h, dt, nb=4, free_surface=int(kind == "elastic"), pml_f=35.0, slabs=P)
            outs.append(gpu_forward(kind, g, m, src, w, rec))
        assert np.abs(outs[0][0]).max() > 0, f"no signal for source {src}"
        for s, f in outs[1:]:
            assert np.array_equal(s, outs[0][0]), f"seismogram differs, source {src}"
            for a, b in zip(f, outs[0][1]):
                assert np.array_equal(a, b), f"field differs, source {src}"


@pytest.mark.parametrize("kind", ["iso", "acoustic", "elastic"])
def test_source_positions_against_oracle(monkeypatch, kind):
    monkeypatch.setenv("SEIS_NO_PERSIST", "1")
    m = _media(kind)
    h, dt, nt = 10.0, 5e-4, 24
    w = inputs.source_series(kind, nt, dt, 35.0)
    fs = int(kind == "elastic")
    for src in (SOURCES[1], SOURCES[3], SOURCES[4]):
        g, og = grids(NX, NY, NZ, h, dt, nb=4, free_surface=fs, pml_f=35.0, slabs=2)
        rec = np.asarray([src], np.int32)
        _, fields = gpu_forward(kind, g, m, src, w, rec)
        if kind == "iso":
            st = oracle.iso_state(og)
            oracle.iso_run(og, m["vp"], st, 0, nt, [src], w[:, None], rec)
        elif kind == "acoustic":
            st = oracle.ac_state(og)
            oracle.ac_run(og, m["vp"], m["rho"], st, 0, nt, [src], w[:, None], rec)
        else:
            st = oracle.el_state(og)
            oracle.el_run(og, m["vp"], m["vs"], m["rho"], st, 0, nt, [src], w[:, None], rec, component=2)
        for a, b in zip(fields, oracle_fields(kind, st)):
            if np.linalg.norm(b) > 0:
                assert rel_l2(a, b) <= TOL_FIELD, f"source {src}"
