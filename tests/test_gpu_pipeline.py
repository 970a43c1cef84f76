"""NEXT-2 on the GPU: a replayed 1F1B exporter stage swaps every
micro-batch out after its forward and back in before its backward, on two
swap streams, at the points mpress_schedule_1f1b picks; every restored byte
must equal the generator (R18) and the swap must not deadlock the stage."""
import os
import sys

import pytest

pytestmark = pytest.mark.gpu
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))


@pytest.mark.parametrize("S", [4, 2, 1])
def test_replay_restores_every_byte(S):
    import replay_1f1b
    r = replay_1f1b.replay(S, 0, 4, scale=64, n_fwd_gemms=2, max_ctas=32)
    assert r["restored_bytes_wrong"] == 0
    # the schedule the native executor ran is the oracle's for the measured times
    from oracle import pipeline as P
    q = r["schedule_params_ns"]
    assert P.schedule(S, 0, 4, q["t_fwd"], q["t_bwd"], q["t_out"], q["t_in"], slack=q["slack"]) == \
        (r["schedule_slots"], r["schedule_summary"])
    assert r["peak_resident_sets_noswap"] == min(S, 4)
    assert r["measured_stage_ms_swap"] > 0


def test_replay_paced_to_live_interval():
    """The executor's swaps paced to the 1F1B period: every byte
    still restored, and the scheduler is fed the paced swap times."""
    import replay_1f1b
    r = replay_1f1b.replay(4, 0, 4, scale=64, n_fwd_gemms=2, max_ctas=32, pace_frac=0.7)
    assert r["restored_bytes_wrong"] == 0 and r["pace_mbps"] > 0
    assert r["t_out_ms"] >= r["micro_batch_bytes"] / (r["pace_mbps"] * 1e3) * 0.99
