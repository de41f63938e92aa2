"""The unmodified torch GraphSAGE consumer (examples/train_sage.py) on the sample+extract
path, sequential and with the Trainer's Extract/Train pipelining (SURVEY
§8(f).4): both see the same batches and features, so the loss trajectories agree (up to the
float atomics of index_add_)."""
import os
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                "examples"))


def test_pipelined_extract_train_matches_sequential():
    import train_sage
    seq, t_seq = train_sage.train("tiny", steps=40, hidden=64, classes=7, pipeline=False, log=None)
    pip, t_pip = train_sage.train("tiny", steps=40, hidden=64, classes=7, pipeline=True, log=None)
    assert len(seq) == len(pip) == 40
    for a, b in zip(seq, pip):
        assert abs(a - b) <= 1e-3 * max(1.0, abs(a)), (a, b)
    assert all(x == x and x < 1e3 for x in seq)  # finite
