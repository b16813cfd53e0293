"""CPU checks of the six-dataset inputs (synth.DATASETS, the bench's
`datasets` table): every field has the per-field shape of the paper's
Table 2, is finite fp32, and the RTM snapshots taken one at a
time are exactly the corresponding slices of the whole c5 set (so the table
measures snapshots of the set the parity tests cover).  Small-scale oracle
round trips check that each recipe compresses within the bound."""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle
import synth

SHAPE_ELEMS = {
    "Hurricane": 100 * 500 * 500,
    "NYX": 512 ** 3,
    "QMCPack": 288 * 115 * 69 * 69,
    "RTM": 449 * 449 * 235,
    "HACC": 280_953_867,
    "CESM-ATM": 1800 * 3600,
}


def test_table2_field_sizes_and_bounds():
    assert set(synth.DATASETS) == set(SHAPE_ELEMS)
    assert synth.DATASET_RELS == [1e-2, 1e-3, 1e-4]
    for name, spec in synth.DATASETS.items():
        assert spec["fields"], name
        dims = spec["dims"].split(" ")[0].replace(",", "")
        if "x" in dims:
            assert math.prod(int(d) for d in dims.split("x")) == SHAPE_ELEMS[name], name
        else:
            assert int(dims) == SHAPE_ELEMS[name], name


@pytest.mark.parametrize("name,field", [("CESM-ATM", "T"), ("Hurricane", "QCLOUD")])
def test_small_fields_finite_and_round_trip(name, field):
    x = synth.dataset_field(name, field).numpy()
    assert x.dtype == np.float32 and x.size == SHAPE_ELEMS[name] and np.isfinite(x).all()
    oracle.build()
    sl = x[: 1 << 18]
    for rel in synth.DATASET_RELS:
        st, s = oracle.compress(sl, rel, oracle.REL)
        assert st == oracle.OK
        st, y = oracle.decompress(s, sl.size)
        assert st == oracle.OK
        eb = float(np.frombuffer(s[16:20].tobytes(), np.float32)[0])
        assert np.abs(y.astype(np.float64) - sl).max() <= eb + np.spacing(np.abs(sl).max())


def test_rtm_single_snapshots_are_slices_of_the_set():
    shape = (24, 20, 12)
    whole = synth.rtm_like(6, shape, 7, "cpu")
    per = math.prod(shape)
    for s in (0, 3, 5):
        one = synth.rtm_like(6, shape, 7, "cpu", snaps=[s])
        assert np.array_equal(one.numpy(), whole[s * per:(s + 1) * per].numpy()), s
    two = synth.rtm_like(6, shape, 7, "cpu", snaps=[4, 1])
    assert np.array_equal(two[:per].numpy(), whole[4 * per:5 * per].numpy())
    assert np.array_equal(two[per:].numpy(), whole[per:2 * per].numpy())
