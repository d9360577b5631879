"""Algorithm 1 (App. A): the oracle against hand-worked traces, and the library's host-side
state machine (sr_controller_update, no GPU needed) against both the traces and the oracle."""
import json
import math
import os
import random

import pytest

from oracle.controller import Algorithm1, epoch_report

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "alg1_traces.json")


def _traces():
    with open(GOLDEN) as f:
        return json.load(f)["traces"]


def _diff(d):
    return math.nan if d == "nan" else float(d)


@pytest.mark.parametrize("tr", _traces(), ids=lambda t: t["name"])
def test_oracle_replays_hand_traces(tr):
    a = Algorithm1(**tr["params"])
    assert a.state == "training" and a.patience == 0  # line 1
    for d, ev, st, pat in zip(tr["diffs"], tr["events"], tr["states"], tr["patience"]):
        assert a.step(_diff(d)) == ev
        assert a.state == st and a.patience == pat


def _lib_controller(params):
    from paper_conf_sigcomm_kimjyyh20_b200 import Controller
    return Controller(params["thresh_sat"], params["count_sat"], params["thresh_online"], params["count_online"])


@pytest.mark.parametrize("tr", _traces(), ids=lambda t: t["name"])
def test_library_controller_replays_hand_traces(tr):
    c = _lib_controller(tr["params"])
    assert c.state == "training" and c.patience == 0
    for d, ev, st, pat in zip(tr["diffs"], tr["events"], tr["states"], tr["patience"]):
        assert c.update(_diff(d)) == ev
        assert c.state == st and c.patience == pat


def test_library_controller_matches_oracle_random():
    rng = random.Random(5)
    for trial in range(200):
        params = {"thresh_sat": rng.choice([0.0, 0.02, 0.05]), "count_sat": rng.randint(0, 4),
                  "thresh_online": rng.choice([0.0, 0.1, 0.3]), "count_online": rng.randint(0, 4)}
        a, c = Algorithm1(**params), _lib_controller(params)
        for _ in range(60):
            # quantised diffs so ties with the thresholds occur
            d = rng.choice([-0.1, 0.0, 0.02, 0.05, 0.1, 0.2, 0.3, 0.5])
            assert c.update(d) == a.step(d)
            assert c.state == a.state and c.patience == a.patience


def test_library_controller_rejects_bad_params():
    from paper_conf_sigcomm_kimjyyh20_b200 import SRError
    with pytest.raises(SRError):
        _lib_controller({"thresh_sat": 0.1, "count_sat": -1, "thresh_online": 0.1, "count_online": 0})


def test_epoch_report_uses_prev_while_training_and_init_while_suspended():
    a = Algorithm1(0.05, 0, 0.1, 0)
    r = epoch_report(a, 30.0, 29.99, 28.0, 27.0)  # Training: diff vs PREV (line 6) = 0.01 < 0.05 -> suspend
    assert r["state_before"] == "training" and abs(r["diff"] - 0.01) < 1e-12 and r["event"] == "suspend"
    assert r["q_dnn"] == 3.0 and abs(r["q_dnn_prev"] - 2.99) < 1e-12
    r = epoch_report(a, 30.0, 30.0, 29.95, 27.0)  # Suspended: diff vs INIT (line 17) = 0.05 < 0.1 -> resume
    assert r["state_before"] == "suspended" and abs(r["diff"] - 0.05) < 1e-12 and r["event"] == "resume"
    assert r["state_after"] == "training"
