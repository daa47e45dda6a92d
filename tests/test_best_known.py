"""The best-known sequences of tests/golden/best_known.json (written by scripts/best_known_gpu.py
from long GPU searches) are permutations whose ORACLE penalty equals the stored value -- so every
% gap the bench reports is measured against a value the oracle itself confirms."""
import base64
import json
import os

import numpy as np
import pytest

import gen
import oracle

PATH = os.path.join(os.path.dirname(__file__), "golden", "best_known.json")


def _instance(e):
    if e["problem"] == "ucddcp":
        return gen.ucddcp_instance(e["n"], e["seed"])
    return gen.cdd_instance(e["n"], e["seed"], e["h"])


@pytest.mark.skipif(not os.path.exists(PATH), reason="best_known.json not generated yet")
def test_best_known_sequences_verify_with_the_oracle():
    data = json.load(open(PATH))
    assert len(data["instances"]) == 40 + 10 + 10 + 40
    for name, e in data["instances"].items():
        g = _instance(e)
        assert g.name() == name
        J = np.frombuffer(base64.b64decode(e["seq_b64"]), dtype="<i2")
        assert sorted(J.tolist()) == list(range(g.n)), name
        pr = oracle.Problem.from_instance(g)
        z = oracle.ucddcp_eval(pr, J) if e["problem"] == "ucddcp" else oracle.cdd_eval(pr, J)
        assert z == e["penalty"], name
