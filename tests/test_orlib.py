"""OR-library loader: parsing, due dates, and the paper's Table I written as an
sch file (which pins the column order p, a, b to the worked example: penalty 81 at d = 16, P:122;
UCDDCP 77 at d = 22)."""
import json

import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_awasthillw16_b200 import orlib

TABLE1_SCH = "1\n5\n6 7 9\n5 9 5\n2 6 4\n4 9 3\n4 3 2\n"        # p a b (Table I)
TABLE1_UCD = "1\n5\n6 5 7 9 5\n5 5 9 5 4\n2 2 6 4 3\n4 3 9 3 2\n4 3 3 2 1\n"  # P M a b gamma


def _prob(inst: orlib.OrInstance) -> oracle.Problem:
    g = gen.Instance(inst.n, inst.P, inst.alpha, inst.beta,
                     inst.M if inst.M is not None else inst.P.copy(),
                     inst.gamma if inst.gamma is not None else np.ones(inst.n, dtype=np.int32),
                     inst.d, 0, inst.h)
    return oracle.Problem.from_instance(g)


def test_table1_as_sch_file():
    (inst,) = orlib.parse_sch(TABLE1_SCH)
    assert inst.n == 5 and list(inst.P) == [6, 5, 2, 4, 4]
    t = orlib.OrInstance(**{**inst.__dict__, "d": 16})
    assert oracle.cdd_eval(_prob(t), np.arange(5, dtype=np.int16)) == 81


def test_table1_as_ucddcp_file(tmp_path):
    f = tmp_path / "ucd.txt"
    f.write_text(TABLE1_UCD)
    (inst,) = orlib.read_ucddcp(str(f))
    assert inst.d == 21 and list(inst.M) == [5, 5, 2, 3, 3] and list(inst.gamma) == [5, 4, 3, 2, 1]
    t = orlib.OrInstance(**{**inst.__dict__, "d": 22})
    assert oracle.ucddcp_eval(_prob(t), np.arange(5, dtype=np.int16)) == 77


def test_roundtrip_and_due_dates():
    gs = [gen.cdd_instance(n, 3, 0.4) for n in (10, 57, 100)]
    insts = [orlib.OrInstance(g.n, g.P, g.alpha, g.beta, k=i + 1) for i, g in enumerate(gs)]
    back = orlib.parse_sch(orlib.write_sch(insts))
    for g, b in zip(gs, back):
        assert np.array_equal(g.P, b.P) and np.array_equal(g.alpha, b.alpha) and np.array_equal(g.beta, b.beta)
        for h in (0.2, 0.4, 0.6, 0.8):
            assert b.with_h(h).d == gen.cdd_instance(g.n, 3, h).d
    assert orlib.deviation_pct(102, 100) == pytest.approx(2.0)


@pytest.mark.parametrize("bad", ["", "x", "0\n", "2\n2\n1 1 1\n1 1 1\n", "1\n2\n1 1 1\n1 1\n",
                                 "1\n1\n1 -1 1\n", "1\n1\n1 1 1\n7\n"])
def test_malformed_files(bad):
    with pytest.raises(ValueError):
        orlib.parse_sch(bad)


@pytest.mark.gpu
def test_cli_runs_sa_on_a_file(tmp_path, capsys):
    g = gen.cdd_instance(100, 2, 0.6)
    f = tmp_path / "sch100.txt"
    f.write_text(orlib.write_sch([orlib.OrInstance(g.n, g.P, g.alpha, g.beta)]))
    orlib.main([str(f), "--k", "1", "--h", "0.6", "--chains", "4096", "--steps", "500",
                "--best-known", "100000"])
    out = json.loads(capsys.readouterr().out.strip().splitlines()[-1])
    assert out["d"] == g.d
    pr = oracle.Problem.from_instance(g)
    assert oracle.cdd_eval(pr, np.array(out["sequence"], dtype=np.int16)) == out["best"]
    assert out["deviation_pct"] == pytest.approx(100.0 * (out["best"] - 100000) / 100000)
